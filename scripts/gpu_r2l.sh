set -x
mkdir -p gpurun_out
T=r2l
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${T}.json 2>gpurun_out/bench_${T}.err; echo bench=$?
tail -1 gpurun_out/bench_${T}.json | cut -c1-1500; tail -3 gpurun_out/bench_${T}.err
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --max-regs 168 > gpurun_out/bench_${T}_r168.json 2>gpurun_out/bench_${T}_r168.err; echo bench=$?
tail -1 gpurun_out/bench_${T}_r168.json | cut -c1-1500
timeout 2700 python -m pytest -q -m gpu tests > gpurun_out/pytest_${T}.log 2>&1; echo pytest=$?
tail -15 gpurun_out/pytest_${T}.log
