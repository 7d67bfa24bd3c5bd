# quick check of a fix-up change: Snort-like and Dotstar-like bench lines and
# the tests that drive the fix-up hardest
set -x
mkdir -p gpurun_out
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_fx.json 2>gpurun_out/bench_fx.err; echo bench=$?
tail -1 gpurun_out/bench_fx.json | grep -o '"value": [0-9.]*' | head -1; tail -1 gpurun_out/bench_fx.json | grep -o '"kernels_ms_per_step[^}]*}'
timeout 900 python bench.py --config dotstar --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_fx_dotstar.json 2>&1; echo bench=$?
tail -1 gpurun_out/bench_fx_dotstar.json | grep -o '"value": [0-9.]*' | head -1; tail -1 gpurun_out/bench_fx_dotstar.json | grep -o '"kernels_ms_per_step[^}]*}'
timeout 1500 python -m pytest -q -m gpu tests/test_gpu_parity.py tests/test_gpu_multiproc.py tests/test_gpu_host.py "tests/test_gpu_fullsize.py::test_full_size_every_regex_vs_golden" > gpurun_out/pytest_fx.log 2>&1; echo pytest=$?
tail -5 gpurun_out/pytest_fx.log
