cd "$(dirname "$0")/.."
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -3
WORKLOADS="1 2 3 5" STEPS=30 bash scripts/gpu_workloads.sh > /dev/null 2>&1
timeout -s KILL 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launch_small_1.csv python bench.py --steps 1 --warmup 1 --workload 1 --math fp32 --no-cpu-baseline --no-e2e --no-graph --serial --no-extra-modes > /dev/null 2>&1
