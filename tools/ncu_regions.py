"""Attribute ncu stall samples of an igemm kernel to its roles (by SASS address range from the
cubin's line table) — run here on a report brought back from the GPU box."""
import csv, io, re, subprocess, sys
from collections import defaultdict

rep, lo_hi = sys.argv[1], sys.argv[2:]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"],
                     capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(out)))
h, rows = r[1], r[2:]
base = int(rows[0][0], 16)
cols = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
ranges = []
for spec in lo_hi:            # name:start-end (hex offsets)
    name, rr = spec.split(":")
    a, b = rr.split("-")
    ranges.append((name, int(a, 16), int(b, 16)))
agg = defaultdict(lambda: defaultdict(float))
for x in rows:
    off = int(x[0], 16) - base
    reg = next((n for n, a, b in ranges if a <= off < b), "other")
    for c in cols:
        v = x[h.index(c)]
        agg[reg][c] += float(v or 0)
    agg[reg]["_inst"] += float(x[h.index("Instructions Executed")] or 0)
for reg, d in agg.items():
    tot = sum(v for k, v in d.items() if k.startswith("stall"))
    top = sorted(((v, k) for k, v in d.items() if k.startswith("stall")), reverse=True)[:5]
    print(f"{reg:10s} samples={tot:8.0f} inst={d['_inst']:.3g} " + " ".join(f"{k[6:]}={v:.0f}" for v, k in top))
