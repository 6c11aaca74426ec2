set -x
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "fp32" 2>&1 | tail -30
timeout 300 python __graft_entry__.py smoke 2>&1 | tail -8
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e --math fp32 2>&1 | tail -3
