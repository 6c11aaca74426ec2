#!/bin/bash
# quick loop: gpu tests, skip-mode probes of selected passes, default bench (no ncu)
cd "$(dirname "$0")"
mkdir -p gpurun_out
./scripts_gpu_check.sh
SKIPS="${SKIPS:-0 7}" timeout -s KILL 300 python tools/stage_probe.py ${PROBE:-caffenet_conv1:fwd caffenet_conv1:bwd_filter caffenet_conv2:fwd caffenet_conv2:bwd_data caffenet_conv2:bwd_filter} > gpurun_out/stage_probe.log 2>&1
echo "probe rc=$?"; cat gpurun_out/stage_probe.log | tail -20
STEPS=${STEPS:-30} ./scripts_gpu_bench.sh
