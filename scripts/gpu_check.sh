# One GPU round trip: smoke, the -m gpu suite, a Snort-like bench line.
# Usage (on the box): TAG=r2e bash scripts/gpu_check.sh
set -x
T=${TAG:-r2}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$T.log 2>&1; echo smoke=$?; tail -3 gpurun_out/smoke_$T.log
timeout ${PYTEST_TIMEOUT:-1500} python -m pytest tests -q -m gpu ${PYTEST_ARGS:-} > gpurun_out/pytest_$T.log 2>&1; echo pytest=$?
tail -30 gpurun_out/pytest_$T.log
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_$T.json 2>gpurun_out/bench_$T.err; echo bench=$?
tail -1 gpurun_out/bench_$T.json | cut -c1-2500; tail -5 gpurun_out/bench_$T.err
