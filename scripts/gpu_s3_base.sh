# session-3 baseline: GPU tests, bench on every config (1 GPU), window stats, overhead modes, launch list
set -x
nproc; nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_snort.log 2>&1; echo bench=$?
tail -1 gpurun_out/bench_snort.log
RX_STATS=1 timeout 300 python bench.py --steps 1 --warmup 0 --no-cpu-baseline > gpurun_out/stats_snort.log 2>&1
grep "rx stats" gpurun_out/stats_snort.log | head -2
for d in 1 2; do RX_DBG=$d timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/dbg${d}_snort.log 2>&1; tail -1 gpurun_out/dbg${d}_snort.log | cut -c1-400; done
timeout 1500 python -m pytest tests -q -m gpu ${PYTEST_EXTRA} > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -5 gpurun_out/pytest_gpu.log
for c in dotstar clamav; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; echo bench_$c=$?
  tail -1 gpurun_out/bench_$c.log
  RX_STATS=1 timeout 300 python bench.py --config $c --steps 1 --warmup 0 --no-cpu-baseline 2>&1 | grep "rx stats" | head -1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 20 --csv --log-file gpurun_out/launches_snort.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
