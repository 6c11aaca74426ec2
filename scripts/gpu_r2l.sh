cd "$(dirname "$0")/.."
for W in 1 2 3 5; do MATH=fp32 WORKLOAD=$W python tools/plan_dump.py; done
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -q -x 2>&1 | tail -2
WORKLOADS="1 2 3 5 6" STEPS=30 bash scripts/gpu_workloads.sh > /dev/null 2>&1
