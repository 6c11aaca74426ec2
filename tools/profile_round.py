"""Summarise one round's GPU evidence into profiles/<round>/ (run here, on reports brought back in
gpurun_out/ by scripts_gpu_round.sh):

  python tools/profile_round.py r01 gpurun_out/prof_round.ncu-rep gpurun_out/launch_round.csv

* ncu_step_gemms.txt  — every GEMM launch of one CaffeNet step from the `ncu --set full` capture
  (layer/pass mapped from the serial bench order), with duration, achieved TFLOP/s (algorithmic
  flops / duration), DRAM bytes, L2/L1 throughput, tensor-pipe activity, registers, grid;
* launches_step.txt   — the ncu launch list of one serial eager step (time + DRAM bytes per launch,
  cold-cache and serialised: shares of the step, not absolute bench times);
* profiles/traffic.json — dram read+write bytes per launch of each GEMM, keyed
  "workload/layer/pass/math" (bench.py puts the dominant kernel's entry in roofline.traffic).
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

# serial bench order of the GEMM launches of one CaffeNet step (bench.py step(concurrent=False))
ORDER = [("caffenet_conv1", "fwd"), ("caffenet_conv2", "fwd"), ("caffenet_conv3", "fwd"),
         ("caffenet_conv4", "fwd"), ("caffenet_conv5", "fwd"),
         ("caffenet_conv5", "bwd_data"), ("caffenet_conv5", "bwd_filter"),
         ("caffenet_conv4", "bwd_data"), ("caffenet_conv4", "bwd_filter"),
         ("caffenet_conv3", "bwd_data"), ("caffenet_conv3", "bwd_filter"),
         ("caffenet_conv2", "bwd_data"), ("caffenet_conv2", "bwd_filter"),
         ("caffenet_conv1", "bwd_filter")]
METRICS = {
    "dur_us": "gpu__time_duration.sum",
    "dram_rd": "dram__bytes_read.sum",
    "dram_wr": "dram__bytes_write.sum",
    "lts_pct": "lts__throughput.avg.pct_of_peak_sustained_elapsed",
    "l1_pct": "l1tex__throughput.avg.pct_of_peak_sustained_elapsed",
    "tensor_pct": "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "tensor_rt_pct": "TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
    "sm_ghz": "sm__cycles_elapsed.avg.per_second",
    "regs": "launch__registers_per_thread",
    "grid": "launch__grid_size",
    "cluster": "launch__cluster_dim_x",
}


def raw_rows(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    h, units = r[0], r[1]
    return [dict(zip(h, zip(units, row))) for row in r[2:]]


def num(d, key):
    if key not in d:
        return None
    u, v = d[key]
    try:
        x = float(v.replace(",", ""))
    except ValueError:
        return None
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-3, "usecond": 1,
             "msecond": 1e3, "cycle/nsecond": 1, "cycle/usecond": 1e-3, "Ghz": 1,
             "cycle/second": 1e-9}.get(u, 1)
    return x * scale


def main(rnd, rep, launches=None, workload=4, math="bf16"):
    from glp_workloads import config
    flops = {l.name: l.flops_per_pass() for l in config(workload)}
    outdir = os.path.join(ROOT, "profiles", rnd)
    os.makedirs(outdir, exist_ok=True)
    rows = [d for d in raw_rows(rep) if any(k in d["Kernel Name"][1] for k in ("igemm", "hwgrad", "hfwd", "hdgrad"))]
    # the capture may hold more than one step: take the last one that starts with conv1's forward
    starts = [i for i, d in enumerate(rows) if "hfwd" in d["Kernel Name"][1]]
    if starts and len(rows) - starts[-1] < len(ORDER):
        starts = starts[:-1]
    if starts:
        rows = rows[starts[-1]:starts[-1] + len(ORDER)]
    lines = [f"ncu --set full --clock-control none (cold cache, one launch at a time) of the GEMM "
             f"launches of one CaffeNet b256 {math} step; report {os.path.basename(rep)}",
             f"{'layer':15s} {'pass':10s} {'kernel':28s} {'us':>7s} {'TF/s':>6s} {'DRAM MB':>8s} "
             f"{'L2 %':>5s} {'L1 %':>5s} {'tens%':>5s} {'GHz':>5s} {'regs':>4s} {'grid':>4s} {'clu':>3s}"]
    traffic = {}
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tpath):
        traffic = json.load(open(tpath))
    for (layer, pas), d in zip(ORDER, rows):
        v = {k: num(d, m) for k, m in METRICS.items()}
        dram = (v["dram_rd"] or 0) + (v["dram_wr"] or 0)
        tf = flops[layer] / (v["dur_us"] * 1e-6) / 1e12 if v["dur_us"] else 0.0
        name = d["Kernel Name"][1].replace("void ", "").replace("glp::", "").split("(")[0][:28]
        tens = v["tensor_pct"] if v["tensor_pct"] is not None else v["tensor_rt_pct"]
        lines.append(f"{layer:15s} {pas:10s} {name:28s} {v['dur_us']:7.1f} {tf:6.0f} {dram / 1e6:8.1f} "
                     f"{v['lts_pct'] or 0:5.1f} {v['l1_pct'] or 0:5.1f} {tens or 0:5.1f} "
                     f"{v['sm_ghz'] or 0:5.2f} {int(v['regs'] or 0):4d} {int(v['grid'] or 0):4d} "
                     f"{int(v['cluster'] or 0):3d}")
        traffic[f"{workload}/{layer}/{pas}/{math}"] = dram
    open(os.path.join(outdir, "ncu_step_gemms.txt"), "w").write("\n".join(lines) + "\n")
    json.dump(traffic, open(tpath, "w"), indent=1, sort_keys=True)
    print("\n".join(lines))
    if launches:
        rows = list(csv.reader(open(launches)))
        hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
        h = rows[hi]
        ki, vi, ii, mi = (h.index("Kernel Name"), h.index("Metric Value"), h.index("ID"),
                          h.index("Metric Name"))
        per = {}
        for r in rows[hi + 1:]:
            e = per.setdefault(int(r[ii]), {"name": r[ki].split("(")[0].replace("void ", "").replace("glp::", "")})
            e[r[mi]] = float(r[vi].replace(",", ""))
        ids = sorted(per)
        # the last step starts at the last launch of the first layer's activation pack
        # (CaffeNet: conv1's space-to-depth pack opens every step)
        starts = [i for i in ids if per[i]["name"].startswith("pack_s2d")] or ids[:1]
        step = [per[i] for i in ids if i >= starts[-1] and "spin_kernel" not in per[i]["name"]]
        tot = sum(e["gpu__time_duration.sum"] for e in step) / 1e3
        with open(os.path.join(outdir, "launches_step.txt"), "w") as f:
            f.write("ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum "
                    "--clock-control none: one serial eager CaffeNet b256 step (cold cache, serialised)\n")
            for e in step:
                t = e["gpu__time_duration.sum"] / 1e3
                b = e.get("dram__bytes_read.sum", 0) + e.get("dram__bytes_write.sum", 0)
                f.write(f"{t:9.1f} us {100 * t / tot:5.1f}%  {b / 1e6:8.1f} MB  {e['name']}\n")
            f.write(f"{tot:9.1f} us total, {len(step)} launches per step\n")
        print(open(os.path.join(outdir, "launches_step.txt")).read())


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], sys.argv[3] if len(sys.argv) > 3 else None,
         math=sys.argv[4] if len(sys.argv) > 4 else "bf16")
