#!/bin/bash
# A/B/C on one box: AB="label|ENV=val;label2|ENV=val" (default: previous build vs current vs
# current with the block s2d pack), interleaved 3 times, 100 steps each
cd "$(dirname "$0")"
AB=${AB:-"old|GLP_LIB=ab_libs/old.so;new|X=1;s2dblock|GLP_S2D_BLOCK=1"}
IFS=';' read -ra CASES <<< "$AB"
for rep in 1 2 3; do
for c in "${CASES[@]}"; do
  label="${c%%|*}"; envs="${c#*|}"
  env $envs timeout -s KILL 300 python bench.py --steps ${STEPS:-200} --warmup 10 --workload ${WORKLOAD:-4} --no-cpu-baseline --no-e2e > /tmp/ab.json 2>/dev/null
  python3 - "$label $rep" <<'PY'
import json,sys
d=json.loads(open('/tmp/ab.json').read().splitlines()[-1])
print(sys.argv[1], d["value"], d["ms_per_step"], d["clocks"]["sm_mhz"], " ".join(f"{k['layer'][-5:]}/{k['pass'][:5]}={k['avg_us']:.0f}" for k in d["kernels"]))
PY
done
done
