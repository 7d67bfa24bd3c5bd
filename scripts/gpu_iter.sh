# iteration: GPU tests, bench, ncu full capture (CSV back)
set -x
T=${TAG:-x}
timeout 1200 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu_$T.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu_$T.log
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$T.log 2>&1; echo bench=$?
tail -1 gpurun_out/bench_$T.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 12 --csv --log-file gpurun_out/launches_$T.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
if [ -z "$NONCU" ]; then
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"rx_pass1|rx_prefilter" -c 2 \
  -o /tmp/prof_$T python bench.py --steps 1 --warmup 0 --no-cpu-baseline --length-mib 64 > gpurun_out/ncu_full_$T.log 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page details --csv > gpurun_out/ncu_details_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page raw --csv > gpurun_out/ncu_raw_$T.csv 2>&1
fi
