#!/bin/bash
# End-of-round evidence in one gpurun call (text summaries only, so gpurun_out stays < 64 MiB):
# smoke + the GPU suite, the default bench line, the bf16 / tf32 lines with per-kernel times, the
# reference (oracle) arm, the ncu launch list of one serial fp32 step and ncu --set full summaries
# of its 14 GEMM launches.  TAG names the output files.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
T=${TAG:-final}
./scripts/gpu_check.sh
timeout -s KILL 600 python bench.py > gpurun_out/bench_default_$T.json 2> gpurun_out/bench_default_$T.err
echo "bench rc=$?"; cut -c1-400 gpurun_out/bench_default_$T.json
for M in bf16 tf32; do
  timeout -s KILL 300 python bench.py --math $M --steps 50 --warmup 5 --no-cpu-baseline --no-e2e --no-extra-modes > gpurun_out/bench_${M}_$T.json 2>/dev/null
  echo "bench $M rc=$?"
done
timeout -s KILL 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_$T.json 2>/dev/null
echo "ref rc=$?"
A="--steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-graph --serial --no-extra-modes"
timeout -s KILL 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launch_fp32_$T.csv python bench.py $A > /dev/null 2>&1
echo "launch rc=$?"
python tools/launch_list.py gpurun_out/launch_fp32_$T.csv 38 > gpurun_out/launches_fp32_step_$T.txt 2>&1
tail -3 gpurun_out/launches_fp32_step_$T.txt
timeout -s KILL 1500 ncu --set full --clock-control none --import-source on -k "regex:igemm|hdgrad|hwgrad|hfwd" -s 14 -c 14 \
  -o gpurun_out/prof_fp32_$T -f python bench.py $A > /dev/null 2>&1
echo "full rc=$?"
python tools/profile_round.py ../gpurun_out/r02_$T gpurun_out/prof_fp32_$T.ncu-rep gpurun_out/launch_fp32_$T.csv fp32 > /dev/null 2>&1
echo "summary rc=$?"
cp profiles/traffic.json gpurun_out/r02_$T/traffic.json
rm -f gpurun_out/prof_fp32_$T.ncu-rep
cat gpurun_out/r02_$T/ncu_step_gemms.txt
