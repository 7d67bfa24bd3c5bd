# Round-2 final: the measurement set (scripts/gpu_measure.sh), a register
# sweep, and a reduced ablation ladder on the Dotstar/Protomata-like set
set -x
mkdir -p gpurun_out
timeout 900 python -m pytest -q -m gpu tests/test_gpu_batch.py tests/test_gpu_host.py > gpurun_out/pytest_final_batch.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_final_batch.log
TAG=${TAG:-r2z} bash scripts/gpu_measure.sh
for R in 184 200; do
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --max-regs $R > /tmp/b.json 2>/tmp/b.err; echo "regs $R rc=$?"
tail -1 /tmp/b.json | grep -o '"value": [0-9.]*'; tail -1 /tmp/b.json | grep -o '"kernels_ms_per_step[^}]*}'
done > gpurun_out/regs_sweep.log 2>&1
cat gpurun_out/regs_sweep.log
CONFIGS=dotstar EXTRA="--length-mib 256" RUNGS="base zbs pf lock interval1 interval8 merge16" STEPS=3 \
  bash scripts/ablation.sh > gpurun_out/ablation_dotstar.log 2>&1; echo ablation=$?
tail -12 gpurun_out/ablation_dotstar.log
# functional check of bench.py's N > 1 paths on this one-GPU box (gloo, both
# ranks on cuda:0; not a performance number)
for S in chunk regex; do
RX_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
  --master-port 29531 bench.py --gpus 2 --steps 2 --warmup 1 --length-mib 64 --split $S --no-cpu-baseline \
  > gpurun_out/bench_n2_gloo_$S.json 2>gpurun_out/bench_n2_gloo_$S.err; echo n2_$S=$?
tail -1 gpurun_out/bench_n2_gloo_$S.json | cut -c1-600; tail -3 gpurun_out/bench_n2_gloo_$S.err
done
