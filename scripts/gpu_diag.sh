# GPU diagnostics of the Snort-like bench step: the -m gpu suite (config 5
# apart), RX_F_STATS accounting, ncu launch list and one ncu --set full
# capture of rx_prefilter + rx_pass1.  Usage: TAG=r2f bash scripts/gpu_diag.sh
set -x
T=${TAG:-r2}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
if [ -z "$SKIP_TESTS" ]; then
timeout 1500 python -m pytest tests -q -m gpu ${PYTEST_ARGS:---deselect tests/test_gpu_configs.py::test_config5_multi_10k_prefix} > gpurun_out/pytest_$T.log 2>&1; echo pytest=$?
tail -30 gpurun_out/pytest_$T.log
fi
timeout 600 python scripts/stats_run.py snort > gpurun_out/stats_$T.log 2>&1; echo stats=$?
grep -v "group " gpurun_out/stats_$T.log | tail -5
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$T.json 2>gpurun_out/bench_$T.err; echo bench=$?
tail -1 gpurun_out/bench_$T.json | cut -c1-1500
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches_$T.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch_$T.log 2>&1; echo ncu_launch=$?
timeout 1500 ncu --set full --import-source on --clock-control none -k regex:"rx_pass1|rx_prefilter" -s 8 -c 2 \
  -o /tmp/prof_$T python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full_$T.log 2>&1; echo ncu=$?
tail -3 gpurun_out/ncu_full_$T.log
ncu -i /tmp/prof_$T.ncu-rep --page details --csv > gpurun_out/ncu_details_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page raw --csv > gpurun_out/ncu_raw_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page source --csv --print-source sass -k rx_prefilter 2>&1 | gzip -c > gpurun_out/ncu_sass_prefilter_$T.csv.gz
ls -la gpurun_out | tail
