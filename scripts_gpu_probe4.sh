#!/bin/bash
# per-pass timing of selected layer-passes under environment variants: VARIANTS="label|ENV=v;..."
cd "$(dirname "$0")"
IFS=';' read -ra CASES <<< "${VARIANTS:-base|X=1}"
for c in "${CASES[@]}"; do
  label="${c%%|*}"; envs="${c#*|}"
  echo "== $label ($envs)"
  env $envs SKIPS=0 timeout -s KILL 300 python tools/stage_probe.py ${PROBE} 2>&1 | tail -6
done
