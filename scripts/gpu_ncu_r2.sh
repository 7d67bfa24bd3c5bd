# ncu --set full of one Snort-like step (prefilter + pass 1) with line info; SASS source page of rx_pass1
set -x
T=${TAG:-r2b}
nproc
export RX_LINEINFO=1
timeout 900 python scripts/stats_run.py snort 16 > /dev/null 2>&1   # compile (line info) outside ncu
timeout 1500 ncu --set full --import-source on --clock-control none -k regex:"rx_pass1|rx_prefilter" -c 2 \
  -o /tmp/prof_$T python bench.py --steps 1 --warmup 0 --no-cpu-baseline > gpurun_out/ncu_full_$T.log 2>&1; echo ncu=$?
tail -3 gpurun_out/ncu_full_$T.log
ncu -i /tmp/prof_$T.ncu-rep --page details --csv > gpurun_out/ncu_details_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page raw --csv > gpurun_out/ncu_raw_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page source --csv --print-source sass -k rx_pass1 > /tmp/src_$T.csv 2>&1
gzip -c /tmp/src_$T.csv > gpurun_out/ncu_sass_pass1_$T.csv.gz
ncu -i /tmp/prof_$T.ncu-rep --page source --csv --print-source sass -k rx_prefilter > /tmp/srcp_$T.csv 2>&1
gzip -c /tmp/srcp_$T.csv > gpurun_out/ncu_sass_prefilter_$T.csv.gz
ls -la gpurun_out | tail
