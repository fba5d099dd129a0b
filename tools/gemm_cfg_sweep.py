"""Every tcgen05 GEMM tile configuration at the hot-path shapes, through dp_gemm_tc (release
build, no environment knobs): single-CTA K2 at BN 32..256 (split 1 and the cluster splits) and
the CTA-pair K2p at 256 x 64..256, beside the cost model's own choice (bn 0).  Device time
per launch, back-to-back launches held behind a sleep kernel (tools/kbench.py's timer), and
each configuration's output compared with the model's (max |diff|).

python tools/gemm_cfg_sweep.py [--reps 40] [--shapes M,N,K ...] [--out FILE]
"""
import argparse
import json
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_eurosys_jeongba23_b200 as dp

HOT = [(128, 2304, 768), (128, 768, 768), (128, 3072, 768), (128, 768, 3072),
       (384, 3072, 1024), (384, 1024, 1024), (384, 4096, 1024), (384, 1024, 4096),
       (1024, 3072, 1024), (1024, 1024, 1024), (1024, 4096, 1024), (1024, 1024, 4096),
       (256, 2304, 768), (256, 768, 3072), (256, 3072, 768)]


def timeit(fn, n):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda._sleep(int(2e6 + n * 40000))
    e0.record()
    for _ in range(n):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3 / n


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=40)
    ap.add_argument("--shapes", nargs="*", default=None)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    shapes = [tuple(int(v) for v in s.split(",")) for s in a.shapes] if a.shapes else HOT
    rows = []
    torch.manual_seed(0)
    for (M, N, K) in shapes:
        x = torch.randn(M, K, device="cuda").half()
        w = (torch.randn(N, K, device="cuda") / math.sqrt(K)).half()
        b = torch.randn(N, device="cuda").half()
        y0 = torch.empty(M, N, device="cuda").half()
        y = torch.empty_like(y0)
        dp.gemm_tc(x, K, w, b, None, 0, y0, N, M, N, K, bn=0)
        cfgs = [(0, 0)]
        for bn in (32, 64, 128, 256):
            if bn > 32 and M < bn // 2:
                continue
            for sp in (1, 2, 4):
                if sp > 1 and (bn > 128 or K // 64 < 2 * sp):
                    continue
                cfgs.append((bn, sp))
        if N % 256 == 0:
            cfgs += [(-bn, 0) for bn in (64, 128, 192, 256) if M > bn // 4]
        out = {"shape": [M, N, K], "us": {}}
        for bn, sp in cfgs:
            us = timeit(lambda: dp.gemm_tc(x, K, w, b, None, 0, y, N, M, N, K, bn=bn, split=sp), a.reps)
            torch.cuda.synchronize()
            diff = float((y.float() - y0.float()).abs().max())
            key = "model" if bn == 0 else (f"pair{-bn}" if bn < 0 else f"bn{bn}_s{sp}")
            out["us"][key] = round(us, 2)
            out.setdefault("maxdiff_vs_model", {})[key] = diff
        best = min((v, k) for k, v in out["us"].items())
        out["best"] = best[1]
        out["model_over_best"] = round(out["us"]["model"] / best[0], 3)
        out["tflops_best"] = round(2 * M * N * K / best[0] / 1e6, 1)
        rows.append(out)
        print(json.dumps(out), flush=True)
    if a.out:
        with open(a.out, "w") as f:
            for r in rows:
                f.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
