# copy the round-end style measurement (scripts/gpu_final_r2.sh) into profiles/
set -x
T=${TAG:-r2z}
W="snort-like 1k regexes x 256 MiB payloads"
python scripts/ncu_traffic.py gpurun_out/ncu_raw_$T.csv "$W" 268435456 profiles/ncu_traffic.json profiles/r2_final_ncu_snort.md > /dev/null
python scripts/ncu_summary.py gpurun_out/ncu_details_$T.csv gpurun_out/ncu_raw_$T.csv profiles/r2_final_ncu_snort.md \
  "Snort-like 1k x 256 MiB, round-2 final: ncu --set full of the timed step's rx_prefilter and rx_pass1"
cp gpurun_out/launches_$T.csv profiles/r2_final_launches_snort.csv
tail -1 gpurun_out/bench_$T.json > profiles/r2_final_bench_snort.json
tail -1 gpurun_out/bench_${T}_ref.json > profiles/r2_final_bench_reference.json
tail -1 gpurun_out/bench_${T}_dotstar.json > profiles/r2_final_bench_dotstar.json
tail -1 gpurun_out/bench_${T}_clamav.json > profiles/r2_final_bench_clamav.json
tail -1 gpurun_out/bench_${T}_list.json > profiles/r2_final_bench_list.json
tail -1 gpurun_out/bench_${T}_batch.json > profiles/r2_final_bench_batch.json
cp gpurun_out/regs_sweep.log profiles/r2_final_regs_sweep.log 2>/dev/null
cp gpurun_out/ablation_dotstar.jsonl profiles/r2_ablation_dotstar256.jsonl 2>/dev/null
for S in chunk regex; do tail -1 gpurun_out/bench_n2_gloo_$S.json > profiles/r2_n2_gloo_functional_$S.json 2>/dev/null; done
