# round measurement: smoke, bench (all arms), launch list, ncu --set full traffic of the Snort-like step, GPU tests
set -x
T=${TAG:-r1}
nproc; nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$T.log 2>&1; echo smoke=$?; tail -1 gpurun_out/smoke_$T.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_snort_$T.json 2>gpurun_out/bench_snort_$T.err; echo bench=$?
tail -1 gpurun_out/bench_snort_$T.json | cut -c1-3000
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/bench_ref_$T.json 2>&1; echo ref=$?
tail -1 gpurun_out/bench_ref_$T.json | cut -c1-600
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 30 --csv --log-file gpurun_out/launches_snort_$T.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo launches=$?
timeout 1800 ncu --set full --clock-control none -k regex:"rx_pass1|rx_fixup|rx_prefilter" -c 4 \
  -o /tmp/prof_$T python bench.py --steps 1 --warmup 0 --no-cpu-baseline > gpurun_out/ncu_full_$T.log 2>&1; echo ncu=$?
ncu -i /tmp/prof_$T.ncu-rep --page details --csv > gpurun_out/ncu_details_$T.csv 2>&1
ncu -i /tmp/prof_$T.ncu-rep --page raw --csv > /tmp/ncu_raw_$T.csv 2>&1
python scripts/ncu_traffic.py /tmp/ncu_raw_$T.csv "snort-like 1k regexes x 256 MiB payloads" 268435456 gpurun_out/ncu_traffic.json
python -c "
import csv
rows=list(csv.reader(open('/tmp/ncu_raw_$T.csv')))
keep=[i for i,c in enumerate(rows[0]) if any(k in c for k in ('Kernel Name','dram__bytes','gpu__time_duration.sum','smsp__pcsamp','sm__inst_executed_pipe','launch__','smsp__inst_executed.sum','sm__warps_active','smsp__issue_active'))]
w=csv.writer(open('gpurun_out/ncu_raw_$T.csv','w'))
for r in rows: w.writerow([r[i] for i in keep if i < len(r)])
"
for c in dotstar clamav; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${c}_$T.json 2>&1; echo bench_$c=$?
  tail -1 gpurun_out/bench_${c}_$T.json | cut -c1-400
done
timeout 3000 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu_$T.log 2>&1; echo pytest=$?
tail -5 gpurun_out/pytest_gpu_$T.log
du -sh gpurun_out
