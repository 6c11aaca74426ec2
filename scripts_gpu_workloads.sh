#!/bin/bash
# every BASELINE.json workload (bf16 + tf32), plus GoogLeNet without sibling fusion
cd "$(dirname "$0")"
mkdir -p gpurun_out
for W in ${WLS:-1 2 3 4 5 6 7}; do
  for M in ${MATHS:-bf16 tf32}; do
    timeout -s KILL 300 python bench.py --steps ${STEPS:-30} --warmup 5 --workload $W --math $M --no-cpu-baseline --no-e2e > gpurun_out/wl_${W}_${M}.json 2> gpurun_out/wl_${W}_${M}.err
    echo "wl $W $M rc=$? $(python -c "import json,sys; d=json.loads(open('gpurun_out/wl_${W}_${M}.json').read().splitlines()[-1]); print(d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['achieved'])" 2>&1 | tail -1)"
  done
done
if [ -z "$NONOFUSE" ]; then
timeout -s KILL 300 python bench.py --steps ${STEPS:-30} --warmup 5 --workload 5 --math bf16 --no-cpu-baseline --no-e2e --no-fuse > gpurun_out/wl_5_bf16_nofuse.json 2> gpurun_out/wl_5_nofuse.err
echo "wl 5 bf16 no-fuse rc=$? $(python -c "import json; d=json.loads(open('gpurun_out/wl_5_bf16_nofuse.json').read().splitlines()[-1]); print(d['value'], d['ms_per_step'])" 2>&1 | tail -1)"
fi
if [ -n "$POOL" ]; then
for W in ${POOLWLS:-1 2 3 4 5 6}; do
  timeout -s KILL 300 python bench.py --scheme pool --steps ${PSTEPS:-5} --warmup 2 --workload $W --math bf16 > gpurun_out/pool_${W}.json 2> gpurun_out/pool_${W}.err
  echo "pool wl $W rc=$? $(cat gpurun_out/pool_${W}.json | python -c "import json,sys; d=json.loads(sys.stdin.read().splitlines()[-1]); print(d['value'], d['ms_per_step_eager'], d['ms_per_step_graph'], d['config']['pool_streams'])" 2>&1 | tail -1)"
done
fi
