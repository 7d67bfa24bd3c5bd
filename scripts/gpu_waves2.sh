# waves sweep (window-major sparse pass), GPU tests, window-major dotstar ncu
set -x
T=${TAG:-x}
for c in snort dotstar clamav; do
for kv in "RX_WAVES=4" "RX_WAVES=8" "RX_WAVES=16"; do
  env $kv timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline > /tmp/b.log 2>&1
  echo "$c $kv :: $(tail -1 /tmp/b.log | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"],2), d["roofline"]["kernels_ms_per_step"])')"
done
done
timeout 2400 python -m pytest tests -q -m gpu -x -k "not config5" > gpurun_out/pytest_gpu_$T.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu_$T.log
