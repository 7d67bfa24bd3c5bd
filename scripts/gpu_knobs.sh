# scheduling knob sweep on the Snort-like bench (then tests, then the other configs)
set -x
T=${TAG:-x}
for kv in "RX_CMAJOR=1 RX_CM_SYNC=1" "RX_CMAJOR=1 RX_CM_SYNC=0" "RX_CMAJOR=0" "RX_CMAJOR=1 RX_DYNAMIC=1" "RX_CMAJOR=0 RX_DYNAMIC=1"; do
  env $kv timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > /tmp/b.log 2>&1
  echo "$kv :: $(tail -1 /tmp/b.log | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"],2), d["roofline"]["kernels_ms_per_step"])')"
done
timeout 2400 python -m pytest tests -q -m gpu -x -k "not config5" > gpurun_out/pytest_gpu_$T.log 2>&1; echo pytest=$?
tail -5 gpurun_out/pytest_gpu_$T.log
for c in dotstar clamav; do
for kv in "RX_CMAJOR=1 RX_CM_SYNC=1" "RX_CMAJOR=1 RX_CM_SYNC=0" "RX_CMAJOR=0"; do
  env $kv timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline > /tmp/b.log 2>&1
  echo "$c $kv :: $(tail -1 /tmp/b.log | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"],2), d["roofline"]["kernels_ms_per_step"])')"
done
done
