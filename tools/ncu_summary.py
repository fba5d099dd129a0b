"""Summarise ncu outputs for profiles/ (run here, on the CPU box).

  python tools/ncu_summary.py launches <launches.csv> [--last N]   # per-kernel time share
  python tools/ncu_summary.py report <file.ncu-rep>                 # key metrics per kernel
"""
import csv
import io
import json
import subprocess
import sys
from collections import defaultdict


def launches(path, last=None):
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[h]
    ix = {k: i for i, k in enumerate(hdr)}
    recs = []
    for r in rows[h + 1:]:
        if len(r) != len(hdr) or r[ix["Metric Name"]] != "gpu__time_duration.sum":
            continue
        v = float(r[ix["Metric Value"]])
        unit = r[ix["Metric Unit"]]
        ns = v * {"ns": 1, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6}.get(unit, 1)
        name = r[ix["Kernel Name"]].split("(")[0].replace("void ", "")
        recs.append((name, ns, r[ix["Grid Size"]], r[ix["Block Size"]]))
    if last:
        recs = recs[-last:]
    agg = defaultdict(lambda: [0, 0.0])
    for name, ns, g, b in recs:
        key = f"{name} grid{g}"
        agg[key][0] += 1
        agg[key][1] += ns
    tot = sum(v[1] for v in agg.values())
    out = {"launches": len(recs), "total_us": round(tot / 1e3, 2),
           "kernels": [{"kernel": k, "count": c, "total_us": round(t / 1e3, 2), "share": round(t / tot, 4),
                        "mean_us": round(t / c / 1e3, 2)}
                       for k, (c, t) in sorted(agg.items(), key=lambda kv: -kv[1][1])]}
    return out


WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_bytes.sum",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__shared_mem_per_block_dynamic", "launch__cluster_dim_z", "sm__cycles_elapsed.avg.per_second",
        "smsp__average_warp_latency_issue_stalled_long_scoreboard"]


def report(path):
    txt = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    out = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")].split("(")[0]}
        for w in WANT:
            if w in hdr:
                i = hdr.index(w)
                d[w] = f"{r[i]} {units[i]}".strip()
        out.append(d)
    return out


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        last = int(sys.argv[sys.argv.index("--last") + 1]) if "--last" in sys.argv else None
        print(json.dumps(launches(sys.argv[2], last), indent=1))
    else:
        print(json.dumps(report(sys.argv[2]), indent=1))
