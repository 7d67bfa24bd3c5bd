set -x
mkdir -p gpurun_out
T=r2p
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${T}.json 2>gpurun_out/bench_${T}.err; echo bench=$?
tail -1 gpurun_out/bench_${T}.json | cut -c1-600
for P in 64 128; do
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --piece-mib $P > gpurun_out/bench_${T}_p$P.json 2>&1; echo bench=$?
tail -1 gpurun_out/bench_${T}_p$P.json | grep -o '"e2e".*'
done
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --ablate lockstep_round > gpurun_out/bench_${T}_round.json 2>&1; echo bench=$?
tail -1 gpurun_out/bench_${T}_round.json | cut -c1-300; tail -1 gpurun_out/bench_${T}_round.json | grep -o '"kernels_ms_per_step[^}]*}'
timeout 600 python bench.py --config snort --batch 100000 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${T}_batch.json 2>gpurun_out/bench_${T}_batch.err; echo bench=$?
tail -1 gpurun_out/bench_${T}_batch.json | cut -c1-400; tail -1 gpurun_out/bench_${T}_batch.json | grep -o '"kernels_ms_per_step[^}]*}'
timeout 1200 python -m pytest -q -m gpu tests/test_gpu_batch.py > gpurun_out/pytest_${T}.log 2>&1; echo pytest=$?
tail -5 gpurun_out/pytest_${T}.log
