"""Summarise ncu reports / launch lists from gpurun_out/ into profiles/<round>/ (run here)."""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))
from launch_table import load  # noqa: E402

KEYS = ["gpu__time_duration.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sectors_srcunit_tex_op_read.sum",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__inst_executed.sum",
        "launch__registers_per_thread", "launch__grid_size", "launch__cluster_dim_x",
        "sm__cycles_elapsed.avg", "dram__throughput.avg.pct_of_peak_sustained_elapsed"]
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    return {h: (u, v) for h, u, v in zip(r[0], r[1], r[2])}


def main(rnd, reports, launches, per_step):
    outdir = os.path.join(ROOT, "profiles", rnd)
    os.makedirs(outdir, exist_ok=True)
    traffic = {}
    for key, rep in reports.items():
        d = raw(rep)
        lines = [f"report: {os.path.basename(rep)}  kernel: {d.get('Kernel Name', ('', ''))[1]}"]
        for k in KEYS:
            if k in d:
                lines.append(f"  {k:70s} {d[k][1]:>20s} {d[k][0]}")
        b = 0.0
        for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            u, v = d[k]
            b += float(v.replace(",", "")) * UNIT.get(u, 1)
        traffic[key] = b
        lines.append(f"  dram read+write per launch = {b / 1e6:.1f} MB")
        open(os.path.join(outdir, f"ncu_{key.replace('/', '_')}.txt"), "w").write("\n".join(lines) + "\n")
    json.dump(traffic, open(os.path.join(ROOT, "profiles", "traffic.json"), "w"), indent=1)
    if launches:
        out = load(launches)[-per_step:]
        with open(os.path.join(outdir, "launches_step.txt"), "w") as f:
            f.write("ncu --metrics gpu__time_duration.sum --clock-control none (cold-cache, serialised)\n")
            tot = sum(t for _, _, t in out)
            for i, n, t in out:
                f.write(f"{t:10.1f} us {100 * t / tot:5.1f}%  {n}\n")
            f.write(f"{tot:10.1f} us total, {len(out)} launches per step\n")


if __name__ == "__main__":
    cfg = json.loads(sys.argv[2])
    main(sys.argv[1], cfg, sys.argv[3] if len(sys.argv) > 3 else None,
         int(sys.argv[4]) if len(sys.argv) > 4 else 43)
