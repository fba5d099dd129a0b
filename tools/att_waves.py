"""Per-CTA entry / stored / cluster-merged / end stamps of K5t (instrumented build, DP_ATT_TRACE):
how many waves the grid ran in and where a CTA's time went.  python tools/att_waves.py S H heads causal"""
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
qkv = torch.randn(S, 3 * H, device="cuda").half()
o = torch.empty(S, H, device="cuda").half()
for _ in range(10):
    dp.attention_tc(qkv, 3 * H, o, 1, S, H, heads, causal)
torch.cuda.synchronize()
buf = np.zeros((2048, 64), dtype=np.uint64)
assert _lib.lib.dp_debug_att_trace(buf.ctypes.data_as(ctypes.c_void_p), 2048) == 0
rows = buf[(buf[:, 0] > 0) & (buf[:, 12] > 0)]
t0 = int(rows[:, 0].min())
rel = lambda c: (rows[:, c].astype(np.int64) - t0) / 1e3
entry, setup, stored, merged, end = rel(0), rel(1), rel(8), rel(11), rel(12)
out = {"S": S, "H": H, "heads": heads, "causal": causal, "ctas": int(len(rows)),
       "sms_used": int(len(set(rows[:, 14].tolist()))),
       "entry_quantiles": [round(float(np.quantile(entry, q)), 3) for q in (0, 0.25, 0.5, 0.75, 0.9, 1)],
       "stored_quantiles": [round(float(np.quantile(stored, q)), 3) for q in (0, 0.5, 0.9, 1)],
       "end_quantiles": [round(float(np.quantile(end, q)), 3) for q in (0, 0.5, 0.9, 1)],
       "setup_minus_entry_med": round(float(np.median(setup - entry)), 3),
       "merge_wait_med": round(float(np.median(np.where(merged > 0, merged - stored, 0))), 3),
       "merge_to_end_med": round(float(np.median(np.where(merged > 0, end - merged, end - stored))), 3),
       "nkt_hist": {int(k): int(v) for k, v in zip(*np.unique(rows[:, 15].astype(np.int64), return_counts=True))}}
print(json.dumps(out))
