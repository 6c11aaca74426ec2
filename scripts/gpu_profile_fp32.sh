#!/bin/bash
# fp32 (3xTF32) step: ncu launch list (time + dram bytes) of one serial eager step, and full
# captures of selected igemm launches (step order: fwd c1..c5, dgrad/wgrad c5..c2, wgrad c1)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
B="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-graph --serial --no-extra-modes ${BENCHARGS}"
timeout -s KILL 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launch_${TAG:-fp32}.csv $B > gpurun_out/ncu_launch_${TAG:-fp32}.log 2>&1
echo "launch rc=$?"
python tools/launch_table.py gpurun_out/launch_${TAG:-fp32}.csv ${PERSTEP:-43} 2>&1 | tail -30
for s in ${SKIPS:-1 13}; do
  timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k "regex:${K:-igemm}" -s $s -c 1 \
    -o gpurun_out/prof_${TAG:-fp32}_s$s -f $B > gpurun_out/ncu_full_${TAG:-fp32}_s$s.log 2>&1
  echo "full s=$s rc=$?"
done
