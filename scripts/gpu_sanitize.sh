# compute-sanitizer over small shapes of every kernel family:
# memcheck, racecheck, synccheck, initcheck; one log per tool and family.
mkdir -p gpurun_out/san
for fam in scan scan_r16 scan_il scan_mc scan_mc_lb stream fused warp onchip split strided; do
  for tool in memcheck racecheck synccheck initcheck; do
    extra=""; [ $tool = racecheck ] && extra="--racecheck-report hazard"
    timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool $tool --print-limit 20 --show-backtrace device $extra \
      python scripts/sanitize_cases.py $fam > gpurun_out/san/${fam}_${tool}.log 2>&1
    echo "rc=$?" >> gpurun_out/san/${fam}_${tool}.log
  done
done
grep -H "ERROR SUMMARY\|RACECHECK SUMMARY\|rc=" gpurun_out/san/*.log > gpurun_out/san/summary.txt
