#!/bin/bash
# targeted: selected gpu tests (-k expr), then quick probes + bench
cd "$(dirname "$0")"
mkdir -p gpurun_out
timeout -s KILL 600 python -m pytest tests -m gpu -q -x --timeout 240 -p no:cacheprovider -k "${TESTK:-halo}" > gpurun_out/pytest_k.log 2>&1; echo "pytest-k rc=$?" >> gpurun_out/pytest_k.log
tail -25 gpurun_out/pytest_k.log
if [ -z "$NOQUICK" ]; then ./scripts_gpu_quick.sh; fi
