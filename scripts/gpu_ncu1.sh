#!/bin/bash
# ncu --set full capture of one kernel (regex K, skip S) of the serial eager bench step
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k "regex:${K:-hwgrad}" -s ${S:-1} -c 1 \
  -o gpurun_out/prof_${TAG:-one} -f python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-graph --serial ${BENCHARGS} > gpurun_out/ncu_${TAG:-one}.log 2>&1
echo "ncu rc=$?"; tail -2 gpurun_out/ncu_${TAG:-one}.log
