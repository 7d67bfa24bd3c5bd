mkdir -p gpurun_out
timeout 900 python -m pytest -q -m gpu tests/test_gpu_parity.py -k register > gpurun_out/pytest_regs.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_regs.log
for R in 184 255; do
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --max-regs $R > gpurun_out/r$R.json 2> gpurun_out/r$R.err; echo "regs $R rc=$?"
tail -1 gpurun_out/r$R.json | grep -o '"value": [0-9.]*' | head -1; tail -1 gpurun_out/r$R.json | grep -o '"kernels_ms_per_step[^}]*}'; tail -2 gpurun_out/r$R.err
done
