#!/bin/bash
# every BASELINE.json workload (and the NEXT-3 variants) through bench.py: the fp32 (3xTF32)
# headline line (mixed split / 3xTF32) with the bf16 / tf32 lines beside it
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/workloads
for w in ${WORKLOADS:-1 2 3 4 5 6 7 8 9}; do
  timeout -s KILL 600 python bench.py --workload $w --steps ${STEPS:-20} --warmup 5 --no-cpu-baseline --no-e2e ${BENCHARGS} \
    > gpurun_out/workloads/wl_$w.json 2> gpurun_out/workloads/wl_$w.err
  echo "workload $w rc=$?"; tail -c 400 gpurun_out/workloads/wl_$w.err
done
