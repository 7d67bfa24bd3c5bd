# where does pass-1 time go: counters + timing with parts disabled (results invalid under RX_DBG)
set -x
run() { echo "== $*"; env "$@" timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | grep -v "^\[rx stats" | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('RESULT', d['value'], d['ms_per_step'])"; }
RX_STATS=1 timeout 600 python bench.py --steps 1 --warmup 0 --no-cpu-baseline 2>&1 | grep "rx stats" | head -2
run RX_DBG=0
run RX_DBG=1
run RX_DBG=2
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 12 --csv --log-file gpurun_out/launches_dbg1.csv env RX_DBG=1 python bench.py --steps 1 --warmup 1 --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 12 --csv --log-file gpurun_out/launches_dbg2.csv env RX_DBG=2 python bench.py --steps 1 --warmup 1 --no-cpu-baseline > /dev/null 2>&1
