#!/bin/bash
# tests, epilogue-store floor probes (GLP_DEBUG_SKIP 8 = no output stores), default bench
cd "$(dirname "$0")"
mkdir -p gpurun_out
[ -z "$NOCHECK" ] && ./scripts_gpu_check.sh
SKIPS="${SKIPS:-0 8}" timeout -s KILL 300 python tools/stage_probe.py ${PROBE:-caffenet_conv1:fwd caffenet_conv2:fwd caffenet_conv2:bwd_data caffenet_conv4:fwd caffenet_conv4:bwd_data} > gpurun_out/stage_probe.log 2>&1
echo "probe rc=$?"; tail -20 gpurun_out/stage_probe.log
for i in 1 2; do
timeout -s KILL 600 python bench.py --no-cpu-baseline ${BENCHARGS} > gpurun_out/bench_p$i.json 2> gpurun_out/bench_p$i.err
echo "bench rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/bench_p$i.json')); print(d['value'], d['ms_per_step'], d['clocks'], d['roofline']['frac'], d['roofline']['kernel']); print([(k['layer'][-5:],k['pass'],k['avg_us']) for k in d['kernels']])"
done
