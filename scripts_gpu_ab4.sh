#!/bin/bash
# gpu tests, then A/B of builds on one box (AB as in scripts_gpu_ab3.sh)
cd "$(dirname "$0")"
mkdir -p gpurun_out
[ -z "$NOCHECK" ] && ./scripts_gpu_check.sh
[ -n "$PROBE" ] && SKIPS="${SKIPS:-0 8}" timeout -s KILL 300 python tools/stage_probe.py $PROBE 2>&1 | tail -8
AB=${AB:-"head|GLP_LIB=ab_libs/head.so;new|X=1"} ./scripts_gpu_ab3.sh
