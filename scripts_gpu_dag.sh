#!/bin/bash
# A/B: leveled step DAG vs chain for the branchy workloads
cd "$(dirname "$0")"
mkdir -p gpurun_out
for W in ${WLS:-5 6 4}; do
for V in dag chain; do
  X=""; [ $V = chain ] && X="--chain"
  timeout -s KILL 300 python bench.py --steps 30 --warmup 5 --workload $W --no-cpu-baseline --no-e2e $X > gpurun_out/dag_${W}_${V}.json 2> gpurun_out/dag_${W}_${V}.err
  echo "wl $W $V rc=$? $(python -c "import json; d=json.loads(open('gpurun_out/dag_${W}_${V}.json').read().splitlines()[-1]); print(d['value'], d['ms_per_step'], d['launch'])" 2>&1 | tail -1)"
done
done
