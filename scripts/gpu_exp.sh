# scheduling experiments on the Snort-like bench
set -x
run() { echo "== $*"; env "$@" timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('RESULT', d['value'], d['ms_per_step'], d['config']['groups'], d['config']['compile_s'])"; }
run RX_PF_LOCKSTEP=0
run RX_PF_LOCKSTEP=1
run RX_PF_LOCKSTEP=0 RX_GROUP_INSTR=400
run RX_PF_LOCKSTEP=1 RX_GROUP_INSTR=400
run RX_PF_LOCKSTEP=0 RX_GROUP_INSTR=150
