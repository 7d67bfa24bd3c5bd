set -x
T=${TAG:-ab}
mkdir -p gpurun_out
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${T}_lock.json 2>gpurun_out/bench_${T}_lock.err; echo bench=$?
tail -1 gpurun_out/bench_${T}_lock.json | cut -c1-900; tail -3 gpurun_out/bench_${T}_lock.err
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --ablate no_lockstep > gpurun_out/bench_${T}_nolock.json 2>gpurun_out/bench_${T}_nolock.err; echo bench=$?
tail -1 gpurun_out/bench_${T}_nolock.json | cut -c1-900
timeout 900 python -m pytest -q -m gpu tests/test_gpu_parity.py tests/test_prefilter.py "tests/test_gpu_fullsize.py::test_full_size_every_regex_vs_golden[snort]" > gpurun_out/pytest_$T.log 2>&1; echo pytest=$?
tail -5 gpurun_out/pytest_$T.log
