# ncu --set full capture of the prefilter and the interleaved pass (64 MiB prefix of the Snort-like input)
set -x
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"rx_pass1|rx_prefilter" -c 2 \
  -o gpurun_out/prof_${TAG:-x} python bench.py --steps 1 --warmup 0 --no-cpu-baseline --length-mib 64 > gpurun_out/ncu_full_${TAG:-x}.log 2>&1
echo ncu=$?
