# Round-end style measurement on one B200: the bench line (with cpu_baseline),
# the reference arm, the other configs and the N3 batch line, the ncu launch
# list and one ncu --set full capture of rx_prefilter + rx_pass1.
# Usage: TAG=r2z bash scripts/gpu_measure.sh
set -x
T=${TAG:-r2}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 900 python bench.py > gpurun_out/bench_${T}.json 2>gpurun_out/bench_${T}.err; echo bench=$?
tail -1 gpurun_out/bench_${T}.json | cut -c1-3000; tail -3 gpurun_out/bench_${T}.err
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_${T}_ref.json 2>&1; echo ref=$?
tail -1 gpurun_out/bench_${T}_ref.json | cut -c1-800
for C in dotstar clamav; do
timeout 900 python bench.py --config $C --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${T}_$C.json 2>gpurun_out/bench_${T}_$C.err; echo bench=$?
tail -1 gpurun_out/bench_${T}_$C.json | cut -c1-400
done
timeout 600 python bench.py --outputs list --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${T}_list.json 2>gpurun_out/bench_${T}_list.err; echo bench=$?
tail -1 gpurun_out/bench_${T}_list.json | cut -c1-300
timeout 600 python bench.py --batch 100000 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${T}_batch.json 2>gpurun_out/bench_${T}_batch.err; echo bench=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches_$T.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch_$T.log 2>&1; echo ncu_launch=$?
timeout 1500 ncu --set full --clock-control none -k regex:"rx_pass1|rx_prefilter" -s 6 -c 2 \
  -o /tmp/prof_$T python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full_$T.log 2>&1; echo ncu=$?
ncu -i /tmp/prof_$T.ncu-rep --page details --csv > gpurun_out/ncu_details_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page raw --csv > gpurun_out/ncu_raw_$T.csv 2>&1
