cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "tree or leaf or staged or wgrad_cta" 2>&1 | grep -E "^E|passed|failed|Error" | head -20
for ex in nccl tree; do timeout 300 python bench.py --exchange $ex --steps 20 --warmup 5 --no-cpu-baseline --no-e2e --no-extra-modes 2>&1 | tail -1 > gpurun_out/ex_$ex.json; done
