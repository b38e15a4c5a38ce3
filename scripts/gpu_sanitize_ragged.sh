mkdir -p gpurun_out/san3
for fam in scan scan_mc; do
  for tool in memcheck synccheck initcheck; do
    timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool $tool --print-limit 20 --show-backtrace device \
      python scripts/sanitize_cases.py $fam > gpurun_out/san3/${fam}_${tool}.log 2>&1
    echo "rc=$?" >> gpurun_out/san3/${fam}_${tool}.log
  done
done
grep -H "ERROR SUMMARY\|rc=" gpurun_out/san3/*.log > gpurun_out/san3/summary.txt
