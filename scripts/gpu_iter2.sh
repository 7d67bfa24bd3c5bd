# iteration: bench snort + window stats, GPU tests (all but the 10k config unless FULL=1), other configs
set -x
T=${TAG:-x}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 600 python bench.py --steps 10 --warmup 3 ${BENCH_EXTRA} > gpurun_out/bench_snort_$T.log 2>&1; echo bench=$?
tail -1 gpurun_out/bench_snort_$T.log | cut -c1-2500
RX_STATS=1 timeout 300 python bench.py --steps 1 --warmup 0 --no-cpu-baseline 2>&1 | grep "rx stats" | head -1
SEL="not config5"; [ -n "$FULL" ] && SEL=""
timeout 2400 python -m pytest tests -q -m gpu -x -k "$SEL" > gpurun_out/pytest_gpu_$T.log 2>&1; echo pytest=$?
tail -15 gpurun_out/pytest_gpu_$T.log
for c in ${CONFIGS:-dotstar clamav}; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${c}_$T.log 2>&1; echo bench_$c=$?
  tail -1 gpurun_out/bench_${c}_$T.log | cut -c1-1500
  RX_STATS=1 timeout 300 python bench.py --config $c --steps 1 --warmup 0 --no-cpu-baseline 2>&1 | grep "rx stats" | head -1
done
