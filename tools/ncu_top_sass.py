"""Top SASS instructions of an ncu report by warp-stall samples (diagnostic; run on a report
brought back from the GPU box): python tools/ncu_top_sass.py REP [N]"""
import csv, io, subprocess, sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"],
                     capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(out)))
h, rows = r[1], r[2:]
base = int(rows[0][0], 16)
si = h.index("Warp Stall Sampling (All Samples)") if "Warp Stall Sampling (All Samples)" in h else None
cols = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
src = h.index("Source")
tot = sum(float(x[si] or 0) for x in rows)
print(f"total samples {tot:.0f}")
for x in sorted(rows, key=lambda x: -float(x[si] or 0))[:n]:
    top = sorted(((float(x[h.index(c)] or 0), c[6:]) for c in cols), reverse=True)[:2]
    print(f"{int(x[0],16)-base:6x} {float(x[si] or 0):7.0f} {x[src][:70]:70s} " +
          " ".join(f"{k}={v:.0f}" for v, k in top))
