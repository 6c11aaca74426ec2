cd "$(dirname "$0")/.."
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -q -x 2>&1 | tail -3
WORKLOADS="1 2 3 5 4" STEPS=30 bash scripts/gpu_workloads.sh > /dev/null 2>&1
