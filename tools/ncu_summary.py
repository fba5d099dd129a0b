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
        "smsp__average_warp_latency_issue_stalled_long_scoreboard", "pcie__read_bytes.sum.per_second",
        "syslts__t_sectors_srcunit_tex_aperture_sysmem_op_read_lookup_miss.sum",
        "l1tex__m_xbar2l1tex_read_bytes.sum"]


def report(path):
    if path.endswith(".csv"):  # the raw page exported on the GPU box (the .ncu-rep may not travel back)
        txt = open(path).read()
    else:
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


# algorithmic bytes / flops of the kbench shapes captured by tools/evidence.sh
ALGO = {
    "gemm_q": {"shape": "M128 N768 K768", "bytes": 2 * (768 * 768 + 128 * 768 + 128 * 768), "flops": 2 * 128 * 768 * 768},
    "gemm_fc1": {"shape": "M128 N3072 K768", "bytes": 2 * (3072 * 768 + 128 * 768 + 128 * 3072),
                 "flops": 2 * 128 * 3072 * 768},
    "gemm_fc2": {"shape": "M128 N768 K3072", "bytes": 2 * (768 * 3072 + 128 * 3072 + 128 * 768),
                 "flops": 2 * 128 * 768 * 3072},
    "skinny_dha": {"shape": "M128 N768 K768, W in pinned host memory", "host_bytes": 2 * 768 * 768},
    "embed_dha": {"shape": "S128 H768, tables in pinned host memory", "host_bytes": (2 * 128 + 3) * 768 * 2},
    "attention": {"shape": "B1 S128 H768 12 heads", "flops": 4 * 128 * 128 * 768},
    "layernorm": {"shape": "128 x 768", "bytes": 2 * 2 * 128 * 768},
    "lmhead_hbm": {"shape": "GPT-2 tied LM head, 1 row, V50257 H768, wte in HBM (streaming GEMV)",
                   "bytes": 2 * 50257 * 768},
    "attention_k5b": {"shape": "B1 S384 H1024 16 heads, 4 key-tile groups (K5b)", "flops": 4 * 384 * 384 * 1024},
    "pt_forward": {"shape": "32 MiB pinned host -> HBM, SM forwarder (K7)", "host_bytes": 32 << 20},
    # round 2 (tools/evidence_r02.sh)
    "gemm_M384_N4096_K1024": {"shape": "M384 N4096 K1024 (BERT-Large fc1 at S384)",
                              "bytes": 2 * (4096 * 1024 + 384 * 1024 + 384 * 4096), "flops": 2 * 384 * 4096 * 1024},
    "gemm_M1024_N4096_K1024": {"shape": "M1024 N4096 K1024 (GPT-2 Medium c_fc at S1024)",
                               "bytes": 2 * (4096 * 1024 + 1024 * 1024 + 1024 * 4096), "flops": 2 * 1024 * 4096 * 1024},
    "attention_s128": {"shape": "B1 S128 H768 12 heads (K5)", "flops": 4 * 128 * 128 * 768},
    "attention_s384": {"shape": "B1 S384 H1024 16 heads (K5b)", "flops": 4 * 384 * 384 * 1024},
    "attention_s1024_causal": {"shape": "B1 S1024 H1024 16 heads causal (K5b; half the S^2 term)",
                               "flops": 2 * 1024 * 1024 * 1024},
    "layernorm_dha": {"shape": "128 x 768, gamma/beta in pinned host memory (one cluster, DSMEM broadcast)",
                      "host_bytes": 2 * 2 * 768},
    "fp32_linear_dha": {"shape": "fp32 M128 N768 K768, W in pinned host memory (read once)",
                        "host_bytes": 4 * 768 * 768},
}


def bundle(d, launches_csv, peaks):
    """profiles/ summary: per-kernel ncu --set full metrics + algorithmic rooflines, and the
    per-kernel time shares of one bench step from the launch list."""
    out = {"kernels": {}, "bench_step_launches": launches(launches_csv, 86) if launches_csv else None}
    for name, algo in ALGO.items():
        path = f"{d}/full_{name}.ncu-rep"
        import os
        if not os.path.exists(path):
            path = f"{d}/full_{name}.raw.csv"
        try:
            r = report(path)[0]
        except Exception as e:  # noqa: BLE001
            out["kernels"][name] = {"error": str(e)}
            continue
        us = float(r["gpu__time_duration.sum"].split()[0])
        e = {"ncu": r, "algorithmic": algo, "duration_us": us}
        if "bytes" in algo:
            e["hbm_roofline"] = {"achieved_gbs": round(algo["bytes"] / us / 1e3, 1), "peak_gbs": peaks["hbm"],
                                 "frac": round(algo["bytes"] / us / 1e3 / peaks["hbm"], 4)}
        if "flops" in algo:
            e["tensor_roofline"] = {"achieved_tflops": round(algo["flops"] / us / 1e6, 2), "peak_tflops": peaks["tc"],
                                    "frac": round(algo["flops"] / us / 1e6 / peaks["tc"], 4)}
        if "host_bytes" in algo:
            sect = float(r["syslts__t_sectors_srcunit_tex_aperture_sysmem_op_read_lookup_miss.sum"].split()[0])
            e["host_link"] = {"algorithmic_bytes": algo["host_bytes"], "sysmem_read_bytes": int(sect * 32),
                              "achieved_gbs": round(algo["host_bytes"] / us / 1e3, 2), "peak_gbs": peaks["h2d"],
                              "frac": round(algo["host_bytes"] / us / 1e3 / peaks["h2d"], 4)}
        out["kernels"][name] = e
    return out


if __name__ == "__main__":
    if sys.argv[1] == "bundle":
        pk = json.load(open("MEASURED_PEAKS.json"))  # driver-measured; fp16 dense peak = bf16's (same rate)
        peaks = {"hbm": pk["hbm_gbs"], "tc": pk["bf16_tflops"], "h2d": 55.6}  # h2d: profiles/r01_linkprobe.json
        print(json.dumps(bundle(sys.argv[2], sys.argv[3] if len(sys.argv) > 3 else None, peaks), indent=1))
    elif sys.argv[1] == "launches":
        last = int(sys.argv[sys.argv.index("--last") + 1]) if "--last" in sys.argv else None
        print(json.dumps(launches(sys.argv[2], last), indent=1))
    else:
        print(json.dumps(report(sys.argv[2]), indent=1))
