"""Piece-granular pipeline model of a PT cold start (what one GPU cannot measure).

The planner's simulator lets every unit arrive on its own; the engine moves
PIECES (adjacent units of one link coalesced up to a cap, R18) and a unit is usable only when
its whole piece has landed.  On the primary's own link that costs little (the link never waits
for compute, so only the last piece matters -- hence the 2 MiB tail).  On a PT slot it can cost
a lot: if slot 1 is one 20 MB piece, none of slot 1's units can start before all 20 MB landed,
and everything after them waits too.  This model replays the engine's real piece schedules
(dp_transfer_schedule, the C++ code the engine runs) against a measured cost table, per
transport:
  dma  copy engine into a staging ring, then an NCCL send to the primary (the paper's 2 hops);
  ce   one copy-engine DMA straight into the primary's slot;
  sm   the forwarder kernel (host reads at the measured SM rate);
and prints the predicted cold-start latency for each PT piece cap.  Link constants are the
measured ones (profiles/r01_linkprobe*.json, r01_kbench_pt_forward.json); the NVLink/NCCL
constants are assumptions, stated below.

python tools/pt_piece_model.py profiles/r01_cost_tables.json [--warm=profiles/r01_warm_vs_torch_cublas.jsonl]
       [model:seq ...]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import paper_conf_eurosys_jeongba23_b200 as dp
import synth

BW_CE = 55.5e9 / 1e9    # B/ns, pinned H2D by the copy engine (measured)
BW_SM = 51.4e9 / 1e9    # B/ns, SM zero-copy host reads (measured)
C_CE = 3900             # ns of copy-engine time per DMA (measured)
C_SM = 5000             # ns per forwarder launch + drain (kernel, assumed)
BW_NVL = 700e9 / 1e9    # B/ns, NCCL point-to-point over NVLink 5 (assumption; 900 nominal)
C_NCCL = 8000           # ns per NCCL send/recv (assumption)
C_FLAG = 2000           # ns for a done word to reach the primary's wait kernel (assumption)


def predict(shape, cost, plan, k, transport, pt_cap, cap0=32 << 20, tail=2 << 20):
    n = len(cost["bytes"])
    method = np.asarray(plan.method)
    avail = np.zeros(n, dtype=np.int64)
    t0 = sum(int(cost["dha_link_ns"][i]) for i in range(n) if method[i] == dp.DHA)  # DHA reads on link 0
    for s in range(k):
        _, nb, fu, lu = dp.transfer_schedule(shape, plan, s, cap0 if s == 0 else pt_cap, tail)
        t_link, t_fwd = (t0 if s == 0 else 0), 0
        for b, f, l in zip(nb, fu, lu):
            b = int(b)
            if s == 0 or transport in ("dma", "ce"):
                t_link += C_CE + b / BW_CE
            else:
                t_link += C_SM + b / BW_SM
            if s == 0:
                land = t_link
            elif transport == "dma":
                t_fwd = max(t_fwd, t_link) + C_NCCL + b / BW_NVL
                land = t_fwd
            else:
                land = t_link + C_FLAG
            avail[f:l + 1] = int(land)
    t = 0
    for i in range(n):
        t = max(t, int(avail[i])) + int(cost["exe_dha_ns"][i] if method[i] == dp.DHA else cost["exe_mem_ns"][i])
    return t


def calibrate(cost, warm_ms):
    """Per-unit exe costs are profiled in isolation (L2 flushed, no PDL overlap with the
    neighbours), so their sum overstates the chained warm forward (BERT-Base: 1.22 ms summed
    vs 0.47 ms measured).  Scale every unit's in-HBM time by measured / summed; a DHA unit keeps
    its absolute extra link time (exe_dha - exe_mem)."""
    f = warm_ms * 1e6 / float(sum(cost["exe_mem_ns"]))
    c = dict(cost)
    mem = np.round(cost["exe_mem_ns"] * f).astype(np.int64)
    extra = cost["exe_dha_ns"] - cost["exe_mem_ns"]
    c["exe_mem_ns"] = mem
    c["exe_dha_ns"] = np.where(cost["exe_dha_ns"] >= (1 << 49), cost["exe_dha_ns"], np.maximum(mem + extra, 0))
    return c, f


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--warm=")]
    warm_file = next((a.split("=", 1)[1] for a in sys.argv[1:] if a.startswith("--warm=")), None)
    warm = {}
    if warm_file:  # measured warm forward per model:seq (tools/torch_warm_baseline.py output)
        for ln in open(warm_file):
            r = json.loads(ln)
            warm[f"{r['model']}:{r['seq']}"] = r["ours_warm_ms"]
    tables = json.load(open(args[0]))
    specs = args[1:] or [k for k in tables if ":" in k]
    caps = [1 << 20, 2 << 20, 4 << 20, 8 << 20, 16 << 20, 32 << 20]
    out = {"constants": {"BW_CE_GBs": BW_CE, "BW_SM_GBs": BW_SM, "C_CE_ns": C_CE, "C_SM_ns": C_SM,
                         "BW_NVL_GBs": BW_NVL, "C_NCCL_ns": C_NCCL, "C_FLAG_ns": C_FLAG}, "models": {}}
    for spec in specs:
        name = spec.split(":")[0]
        shape = synth.SHAPES[name]
        cost = {kk: np.asarray(v, dtype=np.int64) for kk, v in tables[spec].items()}
        res = {"T_warm_sum_exe_mem_ms": int(sum(cost["exe_mem_ns"])) / 1e6}
        if spec in warm:
            cost, f = calibrate(cost, warm[spec])
            res["calibrated_to_measured_warm_ms"] = warm[spec]
            res["exe_scale"] = round(f, 4)
        for mode in ("PT_DHA_LINK_STRIPE", "PT_DHA_STRIPE", "PT_DHA_LINK_BAL", "PT_DHA"):
            for k in (2, 4, 8):
                plan = dp.plan_generate(cost, mode, k)
                ideal = dp.plan_simulate(cost, plan)[0]
                row = {"planner_model_ms": ideal / 1e6}
                for tr in ("dma", "ce", "sm"):  # PT slots at cap c, the primary's link at 32 MiB (R18)
                    row[tr] = {f"{c >> 20}MiB": round(predict(shape, cost, plan, k, tr, c) / 1e6, 4) for c in caps}
                for tr in ("dma", "ce", "sm"):  # every link, the primary's included, at cap c
                    row[tr + "_all_links"] = {f"{c >> 20}MiB": round(predict(shape, cost, plan, k, tr, c, cap0=c) / 1e6, 4)
                                              for c in caps}
                res[f"{mode}/k{k}"] = row
        out["models"][spec] = res
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
