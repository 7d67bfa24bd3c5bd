mkdir -p gpurun_out
timeout 3000 python -m pytest tests -q -m gpu --durations=20 > gpurun_out/pytest_durations.log 2>&1; echo pytest=$?
tail -30 gpurun_out/pytest_durations.log
