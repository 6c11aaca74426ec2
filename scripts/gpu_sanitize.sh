#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over a bounded subset of the GPU parity tests
# (bf16, tf32 and 3xTF32 plans: im2col and halo kernels, CTA pairs, the SIMT anchor)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/sanitize
SEL=${SEL:-"(test_exact_integer_bitexact and (lenet_conv2 or caffenet_conv1_s4 or gnet_conv_1)) or (tree_exchange and small_filter and fp32)"}
for tool in memcheck racecheck synccheck; do
  timeout -s KILL ${TLIM:-900} compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 9 \
    python -m pytest tests/test_gpu_parity.py -q -x -k "$SEL" > gpurun_out/sanitize/$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|passed|failed" gpurun_out/sanitize/$tool.log | tail -3
done
