set -x
timeout 600 python bench.py --gpus 1 --steps 20 --warmup 5 2>&1 | tail -2
