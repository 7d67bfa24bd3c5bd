# RX_STATS accounting of the Snort-like bench step (per-group window activity) + a bench line
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
RX_STATS=1 RX_INFO_OUT=gpurun_out/snort_info.txt timeout 600 python scripts/stats_run.py snort > gpurun_out/stats_snort.log 2>&1; echo stats=$?
tail -40 gpurun_out/stats_snort.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_snort_r2a.json 2>gpurun_out/bench_snort_r2a.err; echo bench=$?
tail -1 gpurun_out/bench_snort_r2a.json | cut -c1-1500
