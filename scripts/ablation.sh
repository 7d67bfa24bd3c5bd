# the paper's ablation ladder (Sec. 8.3, Table 3 / Fig. 12,
# PAPER.md P:L441-470) and merge-size / interval sweeps (Table 6 / Fig. 13-14,
# P:L505-529) on the synthetic sets, as bench.py lines.  B200 rungs:
#   base      every group runs every window, no guards   (no_prefilter,no_guards)
#   +zbs      zero-block skipping guards (Sec. 6)         (no_prefilter)
#   +sr       + shift rebalancing (Sec. 5)                (no_prefilter,rebalance)
#   +pf       + cross-regex prefilter (first-factor gating) (no_lockstep)
#   +lock     + cluster lockstep = the default
#   +modeb    + output-gated clusters (opt-in)            (modeb)
# sweeps (default path): group size (merge size) 4/16/32, guard interval 1/2/4/8
# Usage: CONFIGS="snort dotstar" [EXTRA="--length-mib 256"] [RUNGS="base zbs ..."] bash scripts/ablation.sh
#   -> gpurun_out/ablation_<cfg>.jsonl
set -x
mkdir -p gpurun_out
for C in ${CONFIGS:-snort}; do
  OUT=gpurun_out/ablation_$C.jsonl
  : > $OUT
  run() {  # tag, extra bench args
    tag=$1; shift
    timeout ${RUNG_TIMEOUT:-900} python bench.py --config $C --steps ${STEPS:-3} --warmup 3 --no-cpu-baseline ${EXTRA:-} "$@" > /tmp/ab.json 2>/tmp/ab.err
    rc=$?
    echo "{\"rung\": \"$tag\", \"rc\": $rc, \"line\": $(tail -1 /tmp/ab.json | grep '^{' || echo null)}" >> $OUT
    tail -2 /tmp/ab.err
  }
  want() { [ -z "$RUNGS" ] || [[ " $RUNGS " == *" $1 "* ]]; }
  want base && run base --ablate no_prefilter,no_guards
  want zbs && run zbs --ablate no_prefilter
  want sr && run sr --ablate no_prefilter,rebalance
  want pf && run pf --ablate no_lockstep
  want lock && run lock
  want modeb && run modeb --ablate modeb
  for g in 4 16 32; do want merge$g && run merge$g --group-size $g; done
  for i in 1 2 4 8; do want interval$i && run interval$i --interval $i; done
  python - "$OUT" <<'PY'
import json, sys
for l in open(sys.argv[1]):
    d = json.loads(l)
    v = d["line"]
    print(d["rung"], d["rc"], None if v is None else round(v["value"], 2), None if v is None else round(v["ms_per_step"], 2))
PY
done
