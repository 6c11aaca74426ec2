#!/bin/bash
# ncu launch list (time + dram bytes) of 2 serial eager bench steps, and optional full captures
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
W=${WORKLOAD:-4}; MATH=${MATH:-bf16}; TAGN=${TAG:-step}
timeout -s KILL 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launch_${TAGN}.csv python bench.py --steps 1 --warmup 1 --workload $W --math $MATH --no-cpu-baseline --no-e2e --no-graph --serial > gpurun_out/ncu_${TAGN}.log 2>&1
echo "launch rc=$?"
python tools/launch_table.py gpurun_out/launch_${TAGN}.csv 2>&1 | tail -25
for K in ${FULLK}; do
  timeout -s KILL 600 ncu --set full --clock-control none --import-source on -k regex:${K%%:*} -s ${K##*:} -c 1 -o gpurun_out/prof_${TAGN}_${K%%:*} -f python bench.py --steps 1 --warmup 1 --workload $W --math $MATH --no-cpu-baseline --no-e2e --no-graph --serial > /dev/null 2>&1
  echo "full $K rc=$?"
done
