# compute-sanitizer over the SPLIT families (register-tile passes and the sliding window)
mkdir -p gpurun_out/san2
for fam in split split_sw; do
  for tool in memcheck racecheck synccheck initcheck; do
    extra=""; [ $tool = racecheck ] && extra="--racecheck-report hazard"
    timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool $tool --print-limit 20 --show-backtrace device $extra \
      python scripts/sanitize_cases.py $fam > gpurun_out/san2/${fam}_${tool}.log 2>&1
    echo "rc=$?" >> gpurun_out/san2/${fam}_${tool}.log
  done
done
grep -H "ERROR SUMMARY\|RACECHECK SUMMARY\|rc=" gpurun_out/san2/*.log > gpurun_out/san2/summary.txt
