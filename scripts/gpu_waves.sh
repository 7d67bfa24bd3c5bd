# waves x cluster-major sweep on the three configs, then ncu of the Dotstar-like pass 1
set -x
T=${TAG:-x}
for c in snort dotstar clamav; do
for kv in "RX_WAVES=2 RX_CMAJOR=1" "RX_WAVES=4 RX_CMAJOR=1" "RX_WAVES=8 RX_CMAJOR=1" "RX_WAVES=2 RX_CMAJOR=0" "RX_WAVES=4 RX_CMAJOR=0"; do
  env $kv timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline > /tmp/b.log 2>&1
  echo "$c $kv :: $(tail -1 /tmp/b.log | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"],2), d["roofline"]["kernels_ms_per_step"])')"
done
RX_STATS=1 timeout 300 python bench.py --config $c --steps 1 --warmup 0 --no-cpu-baseline 2>&1 | grep "rx stats" | head -1
done
export RX_LINEINFO=1
timeout 600 python bench.py --config dotstar --steps 1 --warmup 0 --no-cpu-baseline --length-mib 64 > /dev/null 2>&1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"rx_pass1" -c 1 \
  -o /tmp/prof_$T python bench.py --config dotstar --steps 1 --warmup 0 --no-cpu-baseline --length-mib 64 > gpurun_out/ncu_full_$T.log 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page details --csv > gpurun_out/ncu_details_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page raw --csv > /tmp/ncu_raw_$T.csv 2>&1
python -c "
import csv
rows=list(csv.reader(open('/tmp/ncu_raw_$T.csv')))
keep=[i for i,c in enumerate(rows[0]) if any(k in c for k in ('Kernel Name','dram__bytes','gpu__time_duration.sum','smsp__pcsamp','sm__inst_executed_pipe','launch__','smsp__inst_executed.sum','sm__warps_active','smsp__issue_active'))]
w=csv.writer(open('gpurun_out/ncu_raw_$T.csv','w'))
for r in rows: w.writerow([r[i] for i in keep if i < len(r)])
"
ncu -i /tmp/prof_$T.ncu-rep --page source --csv --print-source sass > /tmp/ncu_src_$T.csv 2>&1
python scripts/ncu_trim.py /tmp/ncu_src_$T.csv gpurun_out/ncu_src_top_$T.csv 300
du -sh gpurun_out
