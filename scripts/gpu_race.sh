mkdir -p gpurun_out/san2
for fam in scan scan_il scan_mc_lb stream fused; do
  timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 20 python scripts/sanitize_cases.py $fam > gpurun_out/san2/${fam}_racecheck.log 2>&1
  echo "rc=$?" >> gpurun_out/san2/${fam}_racecheck.log
done
grep -H "RACECHECK SUMMARY\|rc=" gpurun_out/san2/*.log > gpurun_out/san2/summary.txt
