"""Summaries of ncu output for profiles/ (run here, on the CPU box).

  python tools/summarize_ncu.py launches <launches.csv>        -> per-kernel share table
  python tools/summarize_ncu.py full <report.ncu-rep> [...]    -> key counters per kernel
"""
import collections
import csv
import io
import json
import subprocess
import sys

FULL_METRICS = [
    "gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
    "sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
    "sm__issue_active.avg.pct_of_peak_sustained_elapsed",
    "sm__warps_active.avg.pct_of_peak_sustained_active",
    "smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_dispatch_stall_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
    "dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem", "smsp__inst_executed.sum",
]


def _to_us(v, unit):
    v = float(v)
    return {"ns": v / 1e3, "us": v, "usecond": v, "ms": v * 1e3, "msecond": v * 1e3, "s": v * 1e6}.get(unit, v)


def launches(path):
    lines = [ln for ln in open(path) if not ln.startswith("==")]
    agg = collections.OrderedDict()
    for r in csv.DictReader(io.StringIO("".join(lines))):
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        name = r["Kernel Name"].split("(")[0].replace("void ", "")
        us = _to_us(r["Metric Value"], r["Metric Unit"])
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += us
    tot = sum(v[1] for v in agg.values())
    out = {"total_us": tot, "kernels": [
        {"kernel": k, "launches": v[0], "total_us": v[1], "mean_us": v[1] / v[0], "share": v[1] / tot}
        for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1])]}
    return out


def full(path):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    res = []
    for v in rows[2:]:
        d = {"kernel": v[hdr.index("Kernel Name")].split("(")[0]}
        for m in FULL_METRICS:
            if m in hdr:
                i = hdr.index(m)
                d[m] = "%s %s" % (v[i], units[i])
        res.append(d)
    return res


if __name__ == "__main__":
    mode = sys.argv[1]
    if mode == "launches":
        print(json.dumps(launches(sys.argv[2]), indent=1))
    else:
        print(json.dumps([full(p) for p in sys.argv[2:]], indent=1))
