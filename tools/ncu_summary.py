"""Summarise an ncu --set full report: headline metrics + top stall PCs (run here, no GPU)."""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
        "TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
        "lts__t_sectors_srcunit_tex_op_read.sum", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__inst_executed.sum", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "sm__cycles_elapsed.avg",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed"]


def run(cmd):
    return subprocess.run(cmd, capture_output=True, text=True).stdout


def main(rep, top=25):
    raw = list(csv.reader(io.StringIO(run(["ncu", "-i", rep, "--page", "raw", "--csv"]))))
    h, u, v = raw[0], raw[1], raw[2]
    d = dict(zip(h, zip(u, v)))
    print("kernel:", d.get("Kernel Name", ("", ""))[1][:100])
    for k in KEYS:
        if k in d:
            print(f"  {k:90s} {d[k][1]:>18s} {d[k][0]}")
    st = [(float(d[k][1]), k) for k in d if k.startswith("smsp__pcsamp_warps_issue_stalled")
          and not k.endswith("not_issued") and d[k][1] not in ("", "n/a")]
    for val, k in sorted(st, reverse=True)[:8]:
        print(f"  stall {k[len('smsp__pcsamp_warps_issue_stalled_'):]:40s} {val:10.0f}")
    sass = list(csv.reader(io.StringIO(run(["ncu", "-i", rep, "--page", "source", "--csv",
                                             "--print-source=sass"]))))
    hh = sass[1]
    rows = sass[2:]
    si, src, ex = hh.index("Warp Stall Sampling (All Samples)"), hh.index("Source"), hh.index("Instructions Executed")
    tot = sum(float(r[si] or 0) for r in rows)
    print(f"  total stall samples {tot:.0f}; top PCs:")
    for r in sorted(rows, key=lambda r: -float(r[si] or 0))[:top]:
        print(f"   {float(r[si]):7.0f} {r[0][-5:]} {r[src][:70]:70s} ex={r[ex]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 25)
