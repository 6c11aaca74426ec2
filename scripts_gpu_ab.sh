#!/bin/bash
# A/B: the same bench with an environment knob at two values, interleaved twice.
#   AB_VAR=GLP_CTA_GROUP AB_VALS="2 1"  (default: CTA pairs on / off)
#   AB_VAR=GLP_KSUB      AB_VALS="2 1"  (two / one k-blocks per pipeline stage)
cd "$(dirname "$0")"
mkdir -p gpurun_out
VAR=${AB_VAR:-GLP_CTA_GROUP}
for rep in 1 2; do
  for v in ${AB_VALS:-2 1}; do
    out=gpurun_out/ab_${VAR}_${v//\//_}_r${rep}.json
    env "$VAR=$v" timeout -s KILL 600 python bench.py --steps ${STEPS:-50} --warmup 5 --no-cpu-baseline --no-e2e ${BENCH_ARGS} > "$out" 2>/dev/null
    python3 - "$out" "$VAR=$v rep $rep" <<'PY'
import json,sys
d=json.load(open(sys.argv[1]))
print(sys.argv[2], d["value"], d["ms_per_step"], d["clocks"], " ".join(f"{k['layer'][-5:]}/{k['pass'][:5]}={k['avg_us']:.0f}" for k in d["kernels"]))
PY
  done
done
