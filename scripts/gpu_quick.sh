# quick perf check: Snort-like bench line, batch line, the batch/host/parity tests
set -x
T=${TAG:-q}
mkdir -p gpurun_out
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${T}.json 2>gpurun_out/bench_${T}.err; echo bench=$?
tail -1 gpurun_out/bench_${T}.json | cut -c1-300; tail -1 gpurun_out/bench_${T}.json | grep -o '"kernels_ms_per_step[^}]*}'; tail -1 gpurun_out/bench_${T}.json | grep -o '"e2e".*'
timeout 600 python bench.py --batch 100000 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${T}_batch.json 2>gpurun_out/bench_${T}_batch.err; echo bench=$?
tail -1 gpurun_out/bench_${T}_batch.json | cut -c1-200; tail -1 gpurun_out/bench_${T}_batch.json | grep -o '"kernels_ms_per_step[^}]*}'
timeout 1200 python -m pytest -q -m gpu tests/test_gpu_batch.py tests/test_gpu_host.py tests/test_gpu_parity.py tests/test_prefilter.py "tests/test_gpu_fullsize.py::test_full_size_every_regex_vs_golden[snort]" > gpurun_out/pytest_${T}.log 2>&1; echo pytest=$?
tail -5 gpurun_out/pytest_${T}.log
