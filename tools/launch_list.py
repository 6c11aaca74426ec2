"""Per-launch table (time, DRAM bytes, achieved DRAM GB/s) from an ncu --csv launch log with
gpu__time_duration.sum and dram__bytes_{read,write}.sum.  usage: launch_list.py log.csv [last_n]"""
import csv
import sys
from collections import OrderedDict


def load(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, vi, ii, mi, ui = (h.index("Kernel Name"), h.index("Metric Value"), h.index("ID"),
                          h.index("Metric Name"), h.index("Metric Unit"))
    out = OrderedDict()
    scale = {"ns": 1e-9, "us": 1e-6, "ms": 1e-3, "byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
             "msecond": 1e-3}
    for r in rows[hi + 1:]:
        i = int(r[ii])
        e = out.setdefault(i, {"name": r[ki].split("(")[0].replace("void ", "").replace("glp::", "")})
        e[r[mi]] = float(r[vi].replace(",", "")) * scale.get(r[ui], 1)
    return list(out.values())


if __name__ == "__main__":
    L = load(sys.argv[1])
    if len(sys.argv) > 2:
        L = L[-int(sys.argv[2]):]
    tot = 0
    for e in L:
        t = e.get("gpu__time_duration.sum", 0)
        b = e.get("dram__bytes_read.sum", 0) + e.get("dram__bytes_write.sum", 0)
        tot += t
        print(f"{t * 1e6:9.1f} us  {b / 1e6:8.1f} MB  {b / t / 1e9 if t else 0:7.0f} GB/s  {e['name'][:60]}")
    print(f"{tot * 1e6:9.1f} us total, {len(L)} launches")
