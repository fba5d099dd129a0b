"""Per-op timeline of the K6 persistent kernel (build with DP_NVCC_EXTRA=-DDP_PERSIST_TRACE).
python tools/persist_trace.py [model] [seq]  -> JSON lines: per op start/work/barrier (us)."""
import ctypes as C
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_jeongba23_b200 as dp
import synth

name = sys.argv[1] if len(sys.argv) > 1 else "bert_base"
S = int(sys.argv[2]) if len(sys.argv) > 2 else 128
m = synth.SHAPES[name]
w = synth.make_weights(m, seed=0)
ctx = dp.Context([0])
model = dp.Model(ctx, m, w)
n = model.n
ids = torch.from_numpy(synth.make_ids(m, 1, S)).cuda()
out = torch.empty(S, m.hidden, dtype=torch.float16, device="cuda")
pool = torch.empty(1, m.hidden, dtype=torch.float16, device="cuda") if m.family != "gpt2" else None
plan = dp._lib.PlanArrays(n, np.zeros(n, np.int8), np.zeros(n, np.int8), 1, 1)
model.infer_cold(plan, 0, ids, out, pool)
ctx.set_opts(use_graph=False, persistent=True)
for _ in range(5):
    model.infer_warm(0, ids, out, pool)
torch.cuda.synchronize()
G = torch.cuda.get_device_properties(0).multi_processor_count  # upper bound; CTAs never traced are dropped
L = m.layers
kinds = (["LN"] if m.family == "gpt2" else []) + ["GEMM_qkv", "ATTN", "GEMM_o", "LN_1", "GEMM_fc1", "GEMM_fc2",
                                                  "LN_2"] * L
nops = len(kinds)
buf = (C.c_uint64 * (G * nops * 8))()
rc = dp._lib.lib.dp_debug_persist_trace(buf, G, nops)
assert rc == 0, rc
t = np.frombuffer(buf, dtype=np.uint64).reshape(G, nops, 8).astype(np.int64)
t = t[t[:, 0, 0] > 0]  # the grid may be smaller than the SM count (whole clusters)
G = t.shape[0]
t0 = t[:, 0, 0].min()
rows = []
for o in range(nops):
    st = t[:, o, 0] - t0
    en = t[:, o, 1] - t0
    row = {"op": o, "kind": kinds[o], "start_min_us": st.min() / 1e3, "start_max_us": st.max() / 1e3}
    if o + 1 < nops:
        work = (en - st) / 1e3
        nxt = t[:, o + 1, 0] - t0
        if kinds[o].startswith("GEMM"):
            has = t[:, o, 2] > t[:, o, 0]
            row["acc_ready_med_us"] = float(np.median((t[has, o, 2] - t[has, o, 0]) / 1e3)) if has.any() else None
        for slot, nm in ((2, "acc"), (6, "staged"), (4, "p4"), (5, "p5")):
            has = t[:, o, slot] > t[:, o, 0]
            if has.any():
                d = (t[has, o, slot] - t[has, o, 0]) / 1e3
                row[nm] = [round(float(np.median(d)), 2), round(float(np.percentile(d, 90)), 2), round(float(d.max()), 2)]
        row["issued_med_us"] = float(np.median((t[:, o, 3] - t[:, o, 0]) / 1e3))
        row.update({"work_med_us": float(np.median(work)), "work_max_us": float(work.max()),
                    "end_max_us": en.max() / 1e3, "barrier_us": (nxt.min() - en.max()) / 1e3})
    rows.append(row)
for r in rows:
    print(json.dumps({k: (round(v, 2) if isinstance(v, float) else v) for k, v in r.items()}))
by = {}
for r in rows[:-1]:
    k = r["kind"].split("_")[0] + ("_" + r["kind"].split("_")[1] if "_" in r["kind"] else "")
    by.setdefault(k, []).append((r["work_max_us"], r["barrier_us"]))
print(json.dumps({"summary": {k: {"work_max_us_mean": round(float(np.mean([a for a, _ in v])), 2),
                                   "barrier_us_mean": round(float(np.mean([b for _, b in v])), 2), "n": len(v)}
                              for k, v in by.items()},
                  "total_us": round((t[:, -1, 0].max() - t0) / 1e3, 1)}))
