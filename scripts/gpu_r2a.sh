# round 2, first mode-B build: parity (prefilter + mode B + parity suites), stats, bench
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r2d.log 2>&1; echo smoke=$?; tail -3 gpurun_out/smoke_r2d.log
timeout 900 python -m pytest tests/test_prefilter.py tests/test_gpu_parity.py -q -m gpu -x > gpurun_out/pytest_r2d.log 2>&1; echo pytest=$?
tail -30 gpurun_out/pytest_r2d.log
RX_INFO_OUT=gpurun_out/snort_info_r2d.txt timeout 600 python scripts/stats_run.py snort > gpurun_out/stats_r2d.log 2>&1; echo stats=$?
head -3 gpurun_out/stats_r2d.log; grep -v "group" gpurun_out/stats_r2d.log | tail -5
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_r2d.json 2>gpurun_out/bench_r2d.err; echo bench=$?
tail -1 gpurun_out/bench_r2d.json | cut -c1-1600; tail -5 gpurun_out/bench_r2d.err
