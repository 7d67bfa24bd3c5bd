set -x
mkdir -p gpurun_out
T=r2j
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${T}.json 2>gpurun_out/bench_${T}.err; echo bench=$?
tail -1 gpurun_out/bench_${T}.json | cut -c1-1200; tail -3 gpurun_out/bench_${T}.err
for R in 168 255; do
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --max-regs $R > gpurun_out/bench_${T}_r$R.json 2>gpurun_out/bench_${T}_r$R.err; echo bench=$?
tail -1 gpurun_out/bench_${T}_r$R.json | cut -c1-900; tail -3 gpurun_out/bench_${T}_r$R.err
done
timeout 600 python scripts/debug_chunks.py > gpurun_out/debug_chunks.log 2>&1; echo dbg=$?; tail -8 gpurun_out/debug_chunks.log
timeout 1500 python -m pytest -q -m gpu tests/test_prefilter.py tests/test_gpu_parity.py tests/test_gpu_batch.py "tests/test_gpu_fullsize.py::test_full_size_every_regex_vs_golden[snort]" > gpurun_out/pytest_${T}.log 2>&1; echo pytest=$?
tail -15 gpurun_out/pytest_${T}.log
timeout 1500 ncu --set full --clock-control none -k regex:"rx_pass1|rx_prefilter" -s 8 -c 2 \
  -o /tmp/prof_$T python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full_$T.log 2>&1; echo ncu=$?
ncu -i /tmp/prof_$T.ncu-rep --page details --csv > gpurun_out/ncu_details_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page raw --csv > gpurun_out/ncu_raw_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page source --csv --print-source sass -k rx_prefilter 2>&1 | gzip -c > gpurun_out/ncu_sass_prefilter_$T.csv.gz
LD_PRELOAD=$PWD/scripts/segv_trace.so timeout 900 python scripts/repro_multi.py > gpurun_out/repro_multi_$T.log 2>&1; echo repro=$?
tail -12 gpurun_out/repro_multi_$T.log
