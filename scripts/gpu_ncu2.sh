# ncu --set full of the three kernels on the Snort-like bench input (64 MiB prefix), with source lines
set -x
T=${TAG:-x}
export RX_LINEINFO=1
timeout 300 python bench.py --steps 1 --warmup 0 --no-cpu-baseline --length-mib 64 > /dev/null 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"rx_pass1|rx_fixup|rx_prefilter" -c 3 \
  -o /tmp/prof_$T python bench.py --steps 1 --warmup 0 --no-cpu-baseline --length-mib 64 > gpurun_out/ncu_full_$T.log 2>&1
echo ncu=$?
ncu -i /tmp/prof_$T.ncu-rep --page details --csv > gpurun_out/ncu_details_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page raw --csv > gpurun_out/ncu_raw_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page source --csv -k regex:rx_pass1 --print-source sass > gpurun_out/ncu_src_$T.csv 2>&1
ls -la gpurun_out/
