#!/bin/bash
# tests + bench (+ optional ncu) in one call
cd "$(dirname "$0")"
./scripts_gpu_check.sh
./scripts_gpu_bench.sh
