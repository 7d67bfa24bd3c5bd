mkdir -p gpurun_out
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --max-regs 184 > gpurun_out/r184.json 2> gpurun_out/r184.err; echo rc=$?
tail -5 gpurun_out/r184.err; tail -1 gpurun_out/r184.json | cut -c1-200
