#!/bin/bash
# small workloads: ncu launch lists (per-kernel device time) of one serial step
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/small
for w in ${WORKLOADS:-1 3 5}; do
  timeout -s KILL 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/small/launch_w$w.csv python bench.py --workload $w --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-graph --serial --no-extra-modes ${BENCHARGS} > /dev/null 2>&1
  echo "w$w rc=$?"
done
