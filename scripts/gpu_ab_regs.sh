set -x
mkdir -p gpurun_out
for A in "" "--max-regs 168" "--max-regs 168 --ablate lockstep_round" "--ablate lockstep_round"; do
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline $A > /tmp/b.json 2>/tmp/b.err; echo "bench [$A] rc=$?"
tail -1 /tmp/b.json | grep -o '"value": [0-9.]*'; tail -1 /tmp/b.json | grep -o '"kernels_ms_per_step[^}]*}'
done
