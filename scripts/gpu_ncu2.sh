# ncu --set full of the three kernels on the Snort-like bench input (64 MiB prefix), with source lines
set -x
T=${TAG:-x}
export RX_LINEINFO=1
timeout 300 python bench.py --steps 1 --warmup 0 --no-cpu-baseline --length-mib 64 > /dev/null 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"rx_pass1|rx_fixup|rx_prefilter" -c 4 \
  -o /tmp/prof_$T python bench.py --steps 1 --warmup 0 --no-cpu-baseline --length-mib 64 > gpurun_out/ncu_full_$T.log 2>&1
echo ncu=$?
ncu -i /tmp/prof_$T.ncu-rep --page details --csv > gpurun_out/ncu_details_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page raw --csv > /tmp/ncu_raw_$T.csv 2>&1
python -c "
import csv,sys
rows=list(csv.reader(open('/tmp/ncu_raw_$T.csv')))
keep=[i for i,c in enumerate(rows[0]) if any(k in c for k in ('Kernel Name','dram__bytes','gpu__time_duration.sum','smsp__pcsamp','sm__inst_executed_pipe','smsp__average_warp','launch__','sm__throughput','smsp__inst_executed.sum','l1tex__t_bytes','lts__t_bytes','smsp__thread_inst','sm__warps_active','smsp__issue_active'))]
w=csv.writer(open('gpurun_out/ncu_raw_$T.csv','w'))
for r in rows: w.writerow([r[i] for i in keep if i < len(r)])
"
ncu -i /tmp/prof_$T.ncu-rep --page source --csv -k regex:rx_pass1 --print-source sass > /tmp/ncu_src_$T.csv 2>&1
python scripts/ncu_trim.py /tmp/ncu_src_$T.csv gpurun_out/ncu_src_top_$T.csv 400
du -sh gpurun_out/
