# compute-sanitizer over the two kernels added late in round 2 (k_scan_grid,
# k_scan_w512): memcheck, racecheck, synccheck, initcheck; one log per tool.
mkdir -p gpurun_out/san2
for fam in scan_w512 scan_grid; do
  for tool in memcheck synccheck initcheck racecheck; do
    extra=""; [ $tool = racecheck ] && extra="--racecheck-report hazard"
    timeout 600 /usr/local/cuda/bin/compute-sanitizer --tool $tool --print-limit 20 --show-backtrace device $extra \
      python scripts/sanitize_cases.py $fam > gpurun_out/san2/${fam}_${tool}.log 2>&1
    echo "rc=$?" >> gpurun_out/san2/${fam}_${tool}.log
    grep -q "rc=86\|not permitted\|disabled" gpurun_out/san2/${fam}_${tool}.log && break 2
  done
done
grep -H "ERROR SUMMARY\|RACECHECK SUMMARY\|rc=" gpurun_out/san2/*.log > gpurun_out/san2/summary.txt
