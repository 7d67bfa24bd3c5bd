# K / register experiments on the Snort-like step with cluster lockstep, and
# an ncu --set full capture of rx_pass1 at the bench configuration
set -x
T=${TAG:-k}
mkdir -p gpurun_out
for K in 2 8; do
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --words-per-lane $K > gpurun_out/bench_${T}_k$K.json 2>gpurun_out/bench_${T}_k$K.err; echo bench=$?
tail -1 gpurun_out/bench_${T}_k$K.json | cut -c1-700; tail -2 gpurun_out/bench_${T}_k$K.err
done
timeout 1500 ncu --set full --clock-control none -k regex:"rx_pass1" -s 4 -c 1 \
  -o /tmp/prof_$T python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full_$T.log 2>&1; echo ncu=$?
tail -3 gpurun_out/ncu_full_$T.log
ncu -i /tmp/prof_$T.ncu-rep --page details --csv > gpurun_out/ncu_details_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page raw --csv > gpurun_out/ncu_raw_$T.csv 2>&1
