"""Per-CTA phase timeline of the tcgen05 GEMM (needs the instrumented build:
DP_NVCC_EXTRA=-DDP_GEMM_TRACE python paper_conf_eurosys_jeongba23_b200/build.py).

Phases (globaltimer ns, relative to the earliest CTA entry): 0 entry, 1 W prefetch issued,
2 setup done (barriers, TMEM, CTA barrier), 3 after griddepcontrol.wait, 4 first stage landed,
5 all MMAs done, 6 fp32 tile in shared memory, 7 tile reduced (split-K cluster), 8 end.
The tile configuration is forced through dp_gemm_tc (bn 0 = the cost model's; < 0 a CTA pair).
python tools/gemm_trace.py M N K [reps] [bn] [split]"""
import ctypes
import json
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_jeongba23_b200 as dp
from paper_conf_eurosys_jeongba23_b200 import _lib

M, N, K = (int(v) for v in sys.argv[1:4])
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 20
bn = int(sys.argv[5]) if len(sys.argv) > 5 else 0
split = int(sys.argv[6]) if len(sys.argv) > 6 else 0
x = torch.randn(M, K, device="cuda").half()
w = (torch.randn(N, K, device="cuda") / math.sqrt(K)).half()
y = torch.empty(M, N, device="cuda").half()
for _ in range(reps):
    dp.gemm_tc(x, K, w, None, None, 0, y, N, M, N, K, bn=bn, split=split)
torch.cuda.synchronize()
buf = np.zeros((4096, 16), dtype=np.uint64)
assert _lib.lib.dp_debug_gemm_trace(buf.ctypes.data_as(ctypes.c_void_p), 4096) == 0
rows = buf[(buf[:, 0] > 0) & (buf[:, 8] > 0)]
t0 = rows[:, 0].min()
rel = (rows[:, :15].astype(np.int64) - int(t0)) / 1e3  # us (a phase a CTA did not record is negative)
names = ["entry", "w_issued", "setup", "pdl_wait", "first_stage", "mma_done", "tile_smem", "tile_reduced", "end",
         "epi_ld0", "epi_ld0_done", "epi_loop_done", "epi_fence_done", "after_done", "epi_entry"]
out = {"shape": [M, N, K], "ctas": int(len(rows)), "bn": bn, "split": split}
for i, n in enumerate(names):
    col = rel[:, i]
    out[n] = {"min": round(float(col.min()), 3), "med": round(float(np.median(col)), 3), "max": round(float(col.max()), 3)}
out["per_cta_active_us_med"] = round(float(np.median(rel[:, 8] - rel[:, 0])), 3)
print(json.dumps(out))
