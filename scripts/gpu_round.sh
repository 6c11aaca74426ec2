#!/bin/bash
# Round evidence in one gpurun call: smoke + gpu tests, the default bench line, the reference
# (oracle) arm, the ncu launch list of one step (time + dram bytes) and ncu --set full captures
# of every GEMM launch of one step.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
TAGN=${TAG:-round}
[ -z "$NOCHECK" ] && ./scripts/gpu_check.sh
timeout -s KILL 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
echo "bench rc=$?"; cat gpurun_out/bench_default.json; tail -3 gpurun_out/bench_default.err
if [ -z "$NOREF" ]; then
  timeout -s KILL 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
  echo "ref rc=$?"; cat gpurun_out/bench_ref.json
fi
timeout -s KILL 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launch_${TAGN}.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-graph --serial > gpurun_out/ncu_${TAGN}.log 2>&1
echo "launch rc=$?"
python tools/launch_table.py gpurun_out/launch_${TAGN}.csv 2>&1 | tail -50
if [ -z "$NOFULL" ]; then
  timeout -s KILL 1200 ncu --set full --clock-control none --import-source on -k "regex:igemm|hwgrad|hfwd|hdgrad" -s ${SKIP:-0} -c ${CNT:-30} \
    -o gpurun_out/prof_${TAGN} -f python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-graph --serial > gpurun_out/ncu_full_${TAGN}.log 2>&1
  echo "full rc=$?"; tail -3 gpurun_out/ncu_full_${TAGN}.log
fi
