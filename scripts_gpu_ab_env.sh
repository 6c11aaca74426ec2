#!/bin/bash
# A/B of environment settings on one box: each line of $AB is "label|ENV=val ENV2=val"
cd "$(dirname "$0")"
mkdir -p gpurun_out
W=${WORKLOAD:-4}
IFS=';' read -ra CASES <<< "$AB"
for rep in 1 2; do
for c in "${CASES[@]}"; do
  label="${c%%|*}"; envs="${c#*|}"
  env $envs timeout -s KILL 300 python bench.py --steps ${STEPS:-40} --warmup 5 --workload $W --no-cpu-baseline --no-e2e > gpurun_out/ab_${label}.json 2>/dev/null
  echo "$rep $label: $(python -c "import json; d=json.loads(open('gpurun_out/ab_${label}.json').read().splitlines()[-1]); print(d['value'], d['ms_per_step'], d['clocks']['sm_mhz'] if d['clocks'] else None)" 2>&1 | tail -1)"
done
done
