"""Kernel determinism under SM contention: every hot kernel is run many times while a noise
kernel (the PT forwarder streaming a pinned buffer, 2 CTAs per SM) occupies the SMs from
another stream; each output must equal the noise-free output bit for bit.  A kernel whose
correctness depends on timing (a missing barrier, an unguarded shared/DSMEM slot reuse) shows
up here.  python tools/stress_concurrency.py [reps]"""
import json
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_eurosys_jeongba23_b200 as dp

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 200
torch.manual_seed(0)
noise_src = torch.empty(256 << 20, dtype=torch.uint8).pin_memory()
noise_dst = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
side = torch.cuda.Stream()
main = torch.cuda.Stream()


def check(name, fn, out):
    with torch.cuda.stream(main):
        fn()
    torch.cuda.synchronize()
    ref = out.clone()
    bad, nan = 0, 0
    for i in range(reps):
        with torch.cuda.stream(side):
            dp.pt_forward(noise_src, noise_dst, (64 << 20) + (i % 7) * 4096, stream=side)
        with torch.cuda.stream(main):
            out.fill_(0) if i % 2 else None
            fn()
        if i % 16 == 15:
            torch.cuda.synchronize()
        torch.cuda.current_stream().wait_stream(main)
        if not torch.equal(out, ref):
            bad += 1
            nan += int(not bool(torch.isfinite(out).all()))
    torch.cuda.synchronize()
    r = {"kernel": name, "reps": reps, "mismatches": bad, "nonfinite": nan}
    print(json.dumps(r), flush=True)
    return r


res = []
for (M, N, K) in [(384, 1024, 1024), (384, 4096, 1024), (384, 1024, 4096), (128, 768, 3072), (128, 3072, 768),
                  (1024, 1024, 4096)]:
    x = torch.randn(M, K, device="cuda").half()
    w = (torch.randn(N, K, device="cuda") / math.sqrt(K)).half()
    b = torch.randn(N, device="cuda").half()
    r = torch.randn(M, N, device="cuda").half()
    y = torch.empty(M, N, device="cuda").half()
    res.append(check(f"gemm_tc M{M} N{N} K{K}", lambda: dp.linear(x, K, w, b, r, N, y, N, M, N, K, path=0, stream=main),
                     y))
    y2 = torch.empty(M, N, device="cuda").half()
    res.append(check(f"skinny M{M} N{N} K{K}",
                     lambda: dp.linear(x, K, w, b, None, 0, y2, N, M, N, K, path=1, stream=main), y2))
for B, S, H, heads, causal in [(1, 128, 768, 12, 0), (1, 384, 1024, 16, 0), (1, 1024, 1024, 16, 1)]:
    qkv = torch.randn(B * S, 3 * H, device="cuda").half()
    o = torch.empty(B * S, H, device="cuda").half()
    res.append(check(f"attention S{S} H{H}", lambda: dp.attention(qkv, 3 * H, o, B, S, H, heads, causal, stream=main),
                     o))
for rows, n in [(384, 1024), (128, 768)]:
    x = torch.randn(rows, n, device="cuda").half()
    rr = torch.randn(rows, n, device="cuda").half()
    g = torch.randn(n, device="cuda").half()
    bb = torch.randn(n, device="cuda").half()
    yy = torch.empty_like(x)
    res.append(check(f"layernorm {rows}x{n}", lambda: dp.layernorm(x, rr, g, bb, yy, rows, n, 1e-5, stream=main), yy))
print(json.dumps({"summary": sum(r["mismatches"] for r in res)}))
