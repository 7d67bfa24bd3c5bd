set -x
T=${TAG:-x}
for c in snort dotstar clamav; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${c}_$T.json 2>&1
  echo "$c :: $(tail -1 gpurun_out/bench_${c}_$T.json | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"],2), d["roofline"]["kernels_ms_per_step"])')"
done
timeout 2400 python -m pytest tests -q -m gpu -x -k "not config5" > gpurun_out/pytest_gpu_$T.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu_$T.log
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:rx_pass1 -c 1 --csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline 2>/dev/null | grep -E "dram__|gpu__time" | cut -c1-300
