set -x
mkdir -p gpurun_out
T=r2m
timeout 600 python scripts/stats_run.py snort > gpurun_out/stats_${T}.log 2>&1; echo stats=$?
grep -v "group " gpurun_out/stats_${T}.log | tail -4
for C in dotstar clamav; do
timeout 900 python bench.py --config $C --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_${T}_$C.json 2>gpurun_out/bench_${T}_$C.err; echo bench=$?
tail -1 gpurun_out/bench_${T}_$C.json | cut -c1-600
done
for TOOL in memcheck racecheck synccheck; do
timeout 900 compute-sanitizer --tool $TOOL --kernel-name regex:rx_ python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/sanitizer_${TOOL}.log 2>&1; echo $TOOL=$?
tail -4 gpurun_out/sanitizer_${TOOL}.log
done
