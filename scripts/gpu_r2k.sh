set -x
mkdir -p gpurun_out
T=r2k
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/int_peak scripts/int_peak.cu && /tmp/int_peak > gpurun_out/int_peak.json; echo intpeak=$?; cat gpurun_out/int_peak.json
timeout 600 python scripts/host_timing.py > gpurun_out/host_timing.log 2>&1; echo ht=$?; cat gpurun_out/host_timing.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${T}.json 2>gpurun_out/bench_${T}.err; echo bench=$?
tail -1 gpurun_out/bench_${T}.json | cut -c1-1500; tail -3 gpurun_out/bench_${T}.err
timeout 1500 python -m pytest -q -m gpu tests/test_prefilter.py tests/test_gpu_multiproc.py "tests/test_gpu_fullsize.py::test_full_size_every_regex_vs_golden[snort]" > gpurun_out/pytest_${T}.log 2>&1; echo pytest=$?
tail -15 gpurun_out/pytest_${T}.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches_$T.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch_$T.log 2>&1; echo ncu_launch=$?
timeout 1500 ncu --set full --clock-control none -k regex:"rx_pass1|rx_prefilter" -s 8 -c 2 \
  -o /tmp/prof_$T python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full_$T.log 2>&1; echo ncu=$?
ncu -i /tmp/prof_$T.ncu-rep --page details --csv > gpurun_out/ncu_details_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page raw --csv > gpurun_out/ncu_raw_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page source --csv --print-source sass -k rx_prefilter 2>&1 | gzip -c > gpurun_out/ncu_sass_prefilter_$T.csv.gz
