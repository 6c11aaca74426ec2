#!/bin/bash
# Bench every BASELINE.json workload (1..5) in bf16 and tf32 (short runs, no CPU baseline / e2e).
cd "$(dirname "$0")"
mkdir -p gpurun_out
for m in bf16 tf32; do
  for w in 1 2 3 4 5; do
    timeout -s KILL 300 python bench.py --workload $w --math $m --steps ${STEPS:-30} --warmup 5 \
      --no-cpu-baseline --no-e2e > gpurun_out/wl_${w}_${m}.json 2> gpurun_out/wl_${w}_${m}.err
    python3 - "$w" "$m" <<'PY'
import json, sys
w, m = sys.argv[1], sys.argv[2]
try:
    d = json.load(open(f"gpurun_out/wl_{w}_{m}.json"))
    best = max(d["kernels"], key=lambda k: k["tflops"])
    print(f"w{w} {m:4s} {d['config']['workload']:28s} {d['value']:10.1f} {d['unit']} {d['ms_per_step']:8.3f} ms "
          f"step {d['tflops_step']:7.1f} TF/s  best {best['layer']}/{best['pass']} {best['tflops']} TF/s "
          f"dom {d['roofline']['kernel']} frac {d['roofline']['frac']}")
except Exception as e:
    print(f"w{w} {m} FAILED {e}"); print(open(f"gpurun_out/wl_{w}_{m}.err").read()[-800:])
PY
  done
done
