mkdir -p gpurun_out
( for dl in 1 8; do echo "== delta $dl"; for args in "1024 1 f64 0 0" "4096 1 f64 0 0" "1024 64 f64 0 0"; do TRI_SCAN_DELTA=$dl timeout 120 python scripts/prof_one.py $args - 2 | grep graph; done; done
for args in "1024 1 f64 0 3" "1024 1 f64 0 1" "1024 1 f64 0 4"; do timeout 120 python scripts/prof_one.py $args - 2 | grep "graph\|variant" | sed 's/ G=0.*//'; done ) > gpurun_out/scan_times.log 2>&1
