#!/bin/bash
# diagnostics: skip-mode stage timings + ncu full captures of selected igemm launches
cd "$(dirname "$0")"
mkdir -p gpurun_out
SKIPS="0 1 2 3 4 7" timeout -s KILL 300 python tools/stage_probe.py ${PROBE:-caffenet_conv1:fwd caffenet_conv1:bwd_filter} > gpurun_out/stage_probe.log 2>&1
echo "probe rc=$?"; cat gpurun_out/stage_probe.log | tail -20
TAG=${TAG:-p} SKIPS="${NCUSKIPS:-14 27}" ./scripts_gpu_ncu.sh
