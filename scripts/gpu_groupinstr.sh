# experiment: group code-size cap (RX_GROUP_INSTR, rx_lower.cpp plan_groups) vs the
# instruction-fetch stall of rx_pass1 on the Snort-like step
nproc
for gi in 600 1000 3000; do
  RX_GROUP_INSTR=$gi timeout 500 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_gi$gi.json 2>&1
  echo gi=$gi rc=$?; tail -1 gpurun_out/bench_gi$gi.json | cut -c1-200
done
