#!/bin/bash
# A/B: the same bench with CTA pairs on (default) and off (GLP_CTA_GROUP=1), interleaved twice.
cd "$(dirname "$0")"
mkdir -p gpurun_out
for rep in 1 2; do
  for cg in 2 1; do
    GLP_CTA_GROUP=$cg timeout -s KILL 600 python bench.py --steps ${STEPS:-50} --warmup 5 --no-cpu-baseline --no-e2e ${BENCH_ARGS} > gpurun_out/ab_cg${cg}_r${rep}.json 2>/dev/null
    python3 - "$cg" "$rep" <<'PY'
import json,sys
d=json.load(open(f"gpurun_out/ab_cg{sys.argv[1]}_r{sys.argv[2]}.json"))
print("cg", sys.argv[1], "rep", sys.argv[2], d["value"], d["ms_per_step"], d["clocks"], " ".join(f"{k['layer'][-5:]}/{k['pass'][:5]}={k['avg_us']:.0f}" for k in d["kernels"]))
PY
  done
done
