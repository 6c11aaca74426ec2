"""Per-step kernel table from an ncu launch list (gpu__time_duration.sum, --csv log)."""
import csv
import sys
from collections import OrderedDict


def load(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, vi, ii, mi = h.index("Kernel Name"), h.index("Metric Value"), h.index("ID"), h.index("Metric Name")
    out = []
    for r in rows[hi + 1:]:
        if r[mi] == "gpu__time_duration.sum":
            name = r[ki].split("(")[0].replace("void ", "").replace("glp::", "")
            out.append((int(r[ii]), name, float(r[vi].replace(",", "")) / 1e3))
    return out


if __name__ == "__main__":
    out = load(sys.argv[1])
    per_step = int(sys.argv[2]) if len(sys.argv) > 2 else None
    step = out[-per_step:] if per_step else out
    tot = sum(t for _, _, t in step)
    agg = OrderedDict()
    for _, n, t in step:
        agg.setdefault(n, [0, 0.0])
        agg[n][0] += 1
        agg[n][1] += t
    for n, (c, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print(f"{t:10.1f} us {100 * t / tot:5.1f}%  x{c:<3d} {n}")
    print(f"{tot:10.1f} us total ({len(step)} launches)")
