cd "$(dirname "$0")/.."
MATH=fp32 WORKLOAD=5 python tools/plan_dump.py
WL=5 python tools/pass_time.py googlenet_conv_1:fwd fp32 '{}' '{"bn_model":0}' '{"cta_pairs":0}' '{"tile_units":4}'
WL=5 python tools/pass_time.py googlenet_conv_4:fwd fp32 '{}' '{"bn_model":0}' '{"cta_pairs":0}' '{"tile_units":4}'
WL=5 python tools/pass_time.py googlenet_conv_4:bwd_data fp32 '{}' '{"bn_model":0}' '{"cta_pairs":0}' '{"tile_units":4}'
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "group" 2>&1 | tail -2
WORKLOADS="5 6" STEPS=20 bash scripts/gpu_workloads.sh > /dev/null 2>&1
