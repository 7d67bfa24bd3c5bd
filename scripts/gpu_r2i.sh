set -x
mkdir -p gpurun_out
LD_PRELOAD=$PWD/scripts/segv_trace.so timeout 900 python scripts/repro_multi.py > gpurun_out/repro_multi.log 2>&1; echo repro=$?
tail -40 gpurun_out/repro_multi.log
timeout 1200 python -m pytest -q -m gpu tests/test_gpu_multiproc.py tests/test_rebalance.py > gpurun_out/pytest_r2i.log 2>&1; echo pytest=$?
tail -30 gpurun_out/pytest_r2i.log
CONFIGS=snort STEPS=3 bash scripts/ablation.sh > gpurun_out/ablation_snort.log 2>&1; echo ablation=$?
tail -20 gpurun_out/ablation_snort.log
