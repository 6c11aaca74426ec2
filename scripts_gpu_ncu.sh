#!/bin/bash
# ncu --set full captures of selected igemm launches (bench step order: fwd c1..c5, then
# dgrad/wgrad c5, c4, c3, c2, wgrad c1; 14 igemm launches per step, warmup 1 step).
cd "$(dirname "$0")"
mkdir -p gpurun_out
W=${WORKLOAD:-4}; MATH=${MATH:-bf16}
for S in ${SKIPS:-15 25}; do
  timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:igemm -s $S -c 1 \
    -o gpurun_out/prof_${TAG:-x}_s$S -f python bench.py --steps 2 --warmup 1 --workload $W --math $MATH --no-cpu-baseline --no-e2e --no-graph --serial > gpurun_out/ncu_s$S.log 2>&1
  echo "ncu s$S rc=$?"
done
