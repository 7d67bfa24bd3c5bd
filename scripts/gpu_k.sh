# experiment: words per lane K (instructions amortised over 32*K positions) and group size
for a in "--words-per-lane 4" "--words-per-lane 1" "--group-size 16" "--words-per-lane 4 --config dotstar"; do
  timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline $a > gpurun_out/bench_k.json 2>&1
  echo "[$a] rc=$?"; tail -1 gpurun_out/bench_k.json | python -c "import json,sys;d=json.loads(sys.stdin.read());print(d['value'],d['config']['groups'],d['roofline']['kernels_ms_per_step'])" 2>&1 | tail -2
done
