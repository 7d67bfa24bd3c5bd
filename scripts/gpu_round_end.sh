# round-end style: smoke, the whole -m gpu suite, then the measurement set
set -x
TAG=${TAG:-r2end} PYTEST_TIMEOUT=3600 bash scripts/gpu_check.sh
TAG=${TAG:-r2end} bash scripts/gpu_measure.sh
