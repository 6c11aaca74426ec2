#!/bin/bash
# GPU-box bench: timed run, ncu launch list, one ncu --set full capture of a top kernel.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
W=${WORKLOAD:-4}
MATH=${MATH:-bf16}
timeout -s KILL 600 python bench.py --steps ${STEPS:-50} --warmup 5 --workload $W --math $MATH > gpurun_out/bench_w${W}_${MATH}.json 2> gpurun_out/bench_w${W}_${MATH}.err
echo "bench rc=$?"; cat gpurun_out/bench_w${W}_${MATH}.json; tail -3 gpurun_out/bench_w${W}_${MATH}.err
if [ -n "$NCU" ]; then
  timeout -s KILL 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/launches_w${W}_${MATH}.csv python bench.py --steps 2 --warmup 1 --workload $W --math $MATH --no-cpu-baseline --no-e2e --no-graph --serial > /dev/null 2>&1
  echo "ncu launches rc=$?"
  timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:igemm -s ${SKIP:-15} -c ${CNT:-1} \
    -o gpurun_out/prof_w${W}_${MATH} -f python bench.py --steps 2 --warmup 1 --workload $W --math $MATH --no-cpu-baseline --no-e2e > gpurun_out/ncu_full.log 2>&1
  echo "ncu full rc=$?"; tail -3 gpurun_out/ncu_full.log
fi
