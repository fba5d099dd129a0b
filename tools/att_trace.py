"""Per-CTA phase timeline of the tcgen05 attention K5t (instrumented build:
DP_NVCC_EXTRA=-DDP_ATT_TRACE python paper_conf_eurosys_jeongba23_b200/build.py).
Stamps (us from the earliest CTA entry): entry, setup (after the PDL wait), each group's first
scores read, last P published, accumulator read; stored; the MMA / TMA warps done issuing.
python tools/att_trace.py S H heads causal [reps]"""
import ctypes
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_jeongba23_b200 as dp
from paper_conf_eurosys_jeongba23_b200 import _lib

S, H, heads, causal = (int(v) for v in sys.argv[1:5])
reps = int(sys.argv[5]) if len(sys.argv) > 5 else 10
qkv = torch.randn(S, 3 * H, device="cuda").half()
o = torch.empty(S, H, device="cuda").half()
for _ in range(reps):
    dp.attention_tc(qkv, 3 * H, o, 1, S, H, heads, causal)
torch.cuda.synchronize()
buf = np.zeros((2048, 64), dtype=np.uint64)
fn = _lib.lib.dp_debug_att_trace
assert fn(buf.ctypes.data_as(ctypes.c_void_p), 2048) == 0
rows = buf[(buf[:, 0] > 0) & (buf[:, 8] > 0)]
t0 = rows[:, 0].min()
rel = (rows[:, :11].astype(np.int64) - int(t0)) / 1e3
names = ["entry", "setup", "g0_first_s", "g1_first_s", "g0_last_p", "g1_last_p", "g0_o_read", "g1_o_read", "stored",
         "mma_issued", "tma_issued"]
out = {"S": S, "H": H, "causal": causal, "ctas": int(len(rows))}
nk = rows[:, 15].astype(np.int64)
for k in sorted(set(nk.tolist())):
    sel = rel[nk == k]
    out[f"nkt{k}"] = {n: round(float(np.median(sel[:, i])), 3) for i, n in enumerate(names)}
out["end_max"] = round(float(rel[:, 8].max()), 3)
# the longest CTA: per key tile j, S issued / P V issued (MMA warp) and S read (softmax group)
k = int(np.argmax(nk))
row = buf[(buf[:, 0] > 0) & (buf[:, 8] > 0)][k].astype(np.int64) - int(t0)
n = min(int(nk[k]), 16)
out["longest_g0_warp0"] = [[round(row[16 + 4 * i + k] / 1e3, 3) for k in range(4)] for i in range(min(n // 2, 8))]
out["longest_s_read"] = [round(row[48 + j] / 1e3, 3) for j in range(min(n, 8))]
out["longest_s_issue_start"] = [round(row[56 + j] / 1e3, 3) for j in range(min(n, 8))]
print(json.dumps(out))
