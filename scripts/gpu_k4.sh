# Snort-like at K = 4 (bench.PROGRAM_OPTS): parity in the bench's launch configuration, bench line, launch list, ncu traffic
T=r1k4
timeout 900 python -m pytest tests/test_gpu_configs.py tests/test_gpu_fullsize.py -q -k "snort" > gpurun_out/pytest_$T.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_$T.log
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_snort_$T.json 2>gpurun_out/bench_snort_$T.err; echo bench=$?
tail -1 gpurun_out/bench_snort_$T.json | cut -c1-400
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 30 --csv --log-file gpurun_out/launches_snort_$T.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo launches=$?
timeout 900 ncu --set full --clock-control none -k regex:"rx_pass1|rx_fixup|rx_prefilter" -c 4 -o /tmp/prof_$T python bench.py --steps 1 --warmup 0 --no-cpu-baseline > gpurun_out/ncu_full_$T.log 2>&1; echo ncu=$?
ncu -i /tmp/prof_$T.ncu-rep --page details --csv > gpurun_out/ncu_details_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page raw --csv > /tmp/ncu_raw_$T.csv 2>&1
python scripts/ncu_traffic.py /tmp/ncu_raw_$T.csv "snort-like 1k regexes x 256 MiB payloads" 268435456 gpurun_out/ncu_traffic_$T.json
python -c "
import csv
rows=list(csv.reader(open('/tmp/ncu_raw_$T.csv')))
keep=[i for i,c in enumerate(rows[0]) if any(k in c for k in ('Kernel Name','dram__bytes','gpu__time_duration.sum','smsp__pcsamp','sm__inst_executed_pipe','launch__','smsp__inst_executed.sum','sm__warps_active','smsp__issue_active'))]
w=csv.writer(open('gpurun_out/ncu_raw_$T.csv','w'))
for r in rows: w.writerow([r[i] for i in keep if i < len(r)])
"
