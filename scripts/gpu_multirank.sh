#!/bin/bash
# the N-rank bench path on ONE GPU (gloo, every rank on cuda:0): exercises self-launch, sharding,
# bucketed all-reduce, weak-scaling line, the tree exchange's fallback transport, max over ranks
cd "$(dirname "$0")/.."
for ex in nccl tree; do
  timeout -s KILL 600 python bench.py --gpus 2 --dist-backend gloo --same-device --exchange $ex \
    --steps 3 --warmup 2 --no-cpu-baseline ${BENCHARGS} > gpurun_out/mr_$ex.json 2> gpurun_out/mr_$ex.err
  echo "exchange $ex rc=$?"; tail -c 600 gpurun_out/mr_$ex.err | grep -v NCCL | tail -5
  tail -c 700 gpurun_out/mr_$ex.json
done
