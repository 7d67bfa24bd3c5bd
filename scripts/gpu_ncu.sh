# ncu --set full capture of the prefilter and the interleaved pass (64 MiB prefix of the Snort-like input);
# the report stays on the box, its details/raw pages come back as CSV
set -x
T=${TAG:-x}
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"rx_pass1|rx_prefilter" -c 2 \
  -o /tmp/prof_$T python bench.py --steps 1 --warmup 0 --no-cpu-baseline --length-mib 64 > gpurun_out/ncu_full_$T.log 2>&1
echo ncu=$?
ncu -i /tmp/prof_$T.ncu-rep --page details --csv > gpurun_out/ncu_details_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page raw --csv > gpurun_out/ncu_raw_$T.csv 2>&1
ls -la /tmp/prof_$T.ncu-rep gpurun_out/
