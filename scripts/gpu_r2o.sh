set -x
mkdir -p gpurun_out
T=r2o
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${T}.json 2>gpurun_out/bench_${T}.err; echo bench=$?
tail -1 gpurun_out/bench_${T}.json | cut -c1-2500; tail -3 gpurun_out/bench_${T}.err
timeout 600 python bench.py --config snort --batch 100000 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${T}_batch.json 2>gpurun_out/bench_${T}_batch.err; echo bench=$?
tail -1 gpurun_out/bench_${T}_batch.json | cut -c1-900; tail -3 gpurun_out/bench_${T}_batch.err
timeout 1200 python -m pytest -q -m gpu tests/test_gpu_batch.py tests/test_gpu_host.py tests/test_gpu_parity.py tests/test_prefilter.py > gpurun_out/pytest_${T}.log 2>&1; echo pytest=$?
tail -12 gpurun_out/pytest_${T}.log
export RX_LINEINFO=1
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:"rx_pass1" -s 1 -c 1 \
  -o /tmp/prof_$T python scripts/hot_group_profile.py 4 2 > gpurun_out/ncu_full_$T.log 2>&1; echo ncu=$?
ncu -i /tmp/prof_$T.ncu-rep --page raw --csv > gpurun_out/ncu_raw_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page source --csv --print-source sass -k rx_pass1 2>&1 | gzip -c > gpurun_out/ncu_sass_pass1_$T.csv.gz
