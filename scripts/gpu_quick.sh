# quick GPU loop: a pytest selection ($1, -k expression), then bench lines of the given configs ($2..)
mkdir -p gpurun_out
sel="$1"; shift
if [ -n "$sel" ]; then
timeout 1200 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 900 -k "$sel" > gpurun_out/pytest_quick.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_quick.log
fi
for c in "$@"; do timeout 600 python bench.py --config $c --no-e2e --no-cpu > gpurun_out/qbench_$c.json 2> gpurun_out/qbench_$c.err; done
