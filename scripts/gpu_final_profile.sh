#!/bin/bash
# Final round-2 profile evidence for the fp32 headline (CaffeNet conv1-5 b256): the ncu launch list
# of serial eager steps (time + DRAM bytes per launch) and --set full captures of the 14 GEMM
# launches of one step.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launch_fp32_final.csv python bench.py --steps 1 --warmup 1 --math fp32 --no-cpu-baseline --no-e2e --no-graph --serial --no-extra-modes > gpurun_out/ncu_fp32_final.log 2>&1
echo "launch rc=$?"
timeout -s KILL 1800 ncu --set full --clock-control none --import-source on -k "regex:igemm" -s 14 -c 14 \
  -o gpurun_out/prof_fp32_final -f python bench.py --steps 1 --warmup 1 --math fp32 --no-cpu-baseline --no-e2e --no-graph --serial --no-extra-modes > gpurun_out/ncu_full_fp32_final.log 2>&1
echo "full rc=$?"; tail -2 gpurun_out/ncu_full_fp32_final.log
