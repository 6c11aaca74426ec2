#!/bin/bash
# GPU box: the whole -m gpu suite and smoke (bounded by timeouts so a hang cannot wedge the box)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout -s KILL 2400 python -m pytest tests -m gpu -q -x ${PYTEST_ARGS} > gpurun_out/gpu_tests.log 2>&1
echo "pytest rc=$?"; tail -25 gpurun_out/gpu_tests.log
timeout -s KILL 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
echo "smoke rc=$?"; tail -5 gpurun_out/smoke.log
