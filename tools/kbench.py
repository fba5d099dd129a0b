"""Per-kernel device timings through the C-ABI hooks (CUDA events around back-to-back
launches on one stream, after warm-up).  Used with ncu too:
  ncu --set full -k regex:gemm_tc -c 3 python tools/kbench.py gemm
python tools/kbench.py [all|gemm|ln|attn|skinny|embed|lmhead|ptfwd] [reps]"""
import json
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_jeongba23_b200 as dp

which = sys.argv[1] if len(sys.argv) > 1 else "all"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 50
torch.manual_seed(0)
res = {}


def timeit(fn, n=reps):
    """Device time per launch: a sleep kernel holds the stream while the host enqueues the
    n launches, so the interval between the events contains no host launch latency."""
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
    return e0.elapsed_time(e1) * 1e3 / n  # us per launch


if which in ("all", "gemm"):
    for (M, N, K) in [(128, 768, 768), (128, 3072, 768), (128, 768, 3072), (384, 1024, 1024), (384, 4096, 1024),
                      (384, 1024, 4096), (1024, 3072, 1024), (1024, 4096, 1024), (1024, 1024, 4096)]:
        x = torch.randn(M, K, device="cuda").half()
        w = (torch.randn(N, K, device="cuda") / math.sqrt(K)).half()
        b = torch.randn(N, device="cuda").half()
        y = torch.empty(M, N, device="cuda").half()
        for bn in (0,):
            us = timeit(lambda: dp.linear(x, K, w, b, None, 0, y, N, M, N, K, path=0))
            flops = 2 * M * N * K
            byts = 2 * (N * K + M * K + M * N)
            res[f"gemm_tc M{M} N{N} K{K}"] = {"us": round(us, 2), "tflops": round(flops / us / 1e6, 1),
                                             "gbs": round(byts / us / 1e3, 1)}
        ref_us = timeit(lambda: torch.nn.functional.linear(x, w, b))
        res[f"torch(cuBLAS) M{M} N{N} K{K}"] = {"us": round(ref_us, 2)}
if which in ("all", "ln"):
    for rows, n in [(128, 768), (384, 1024), (1024, 1024)]:
        x = torch.randn(rows, n, device="cuda").half()
        g = torch.ones(n, device="cuda").half()
        bb = torch.zeros(n, device="cuda").half()
        y = torch.empty_like(x)
        us = timeit(lambda: dp.layernorm(x, None, g, bb, y, rows, n, 1e-5))
        res[f"layernorm {rows}x{n}"] = {"us": round(us, 2), "gbs": round(4 * rows * n / us / 1e3, 1)}
if which in ("all", "attn"):
    for B, S, H, heads, causal in [(1, 128, 768, 12, 0), (1, 384, 1024, 16, 0), (1, 1024, 1024, 16, 1)]:
        qkv = torch.randn(B * S, 3 * H, device="cuda").half()
        o = torch.empty(B * S, H, device="cuda").half()
        us = timeit(lambda: dp.attention(qkv, 3 * H, o, B, S, H, heads, causal))
        fl = 4 * S * S * H * B * (0.5 if causal else 1)
        res[f"attention S{S} H{H} causal{causal}"] = {"us": round(us, 2), "tflops": round(fl / us / 1e6, 2)}
if which in ("all", "attn", "attn_tc"):  # K5t (tcgen05; opts.attention_tc) at the same shapes
    for B, S, H, heads, causal in [(1, 128, 768, 12, 0), (1, 384, 1024, 16, 0), (1, 1024, 1024, 16, 1)]:
        qkv = torch.randn(B * S, 3 * H, device="cuda").half()
        o = torch.empty(B * S, H, device="cuda").half()
        us = timeit(lambda: dp.attention_tc(qkv, 3 * H, o, B, S, H, heads, causal))
        fl = 4 * S * S * H * B * (0.5 if causal else 1)
        res[f"attention_tc S{S} H{H} causal{causal}"] = {"us": round(us, 2), "tflops": round(fl / us / 1e6, 2)}
if which in ("all", "skinny"):
    for (M, N, K) in [(128, 768, 768), (128, 3072, 768), (128, 768, 3072), (1, 768, 768)]:
        x = torch.randn(M, K, device="cuda").half()
        wh = dp.host_alloc(N * K * 2)
        wd = torch.randn(N, K, device="cuda").half()
        y = torch.empty(M, N, device="cuda").half()
        us_h = timeit(lambda: dp.linear(x, K, wh, None, None, 0, y, N, M, N, K, path=1), n=20)
        us_d = timeit(lambda: dp.linear(x, K, wd, None, None, 0, y, N, M, N, K, path=1), n=20)
        res[f"skinny M{M} N{N} K{K}"] = {"us_host": round(us_h, 2), "pcie_gbs": round(N * K * 2 / us_h / 1e3, 1),
                                        "us_hbm": round(us_d, 2)}
        dp.host_free(wh)
if which in ("all", "lmhead"):
    # GPT-2 tied LM head (dp_lm_head's kernel): wte [V, H] read once, from HBM or from host
    for (V, H, M) in [(50257, 768, 1), (50257, 1024, 1), (50257, 1024, 8)]:
        x = torch.randn(M, H, device="cuda").half()
        wh = dp.host_alloc(V * H * 2)
        wd = (torch.randn(V, H, device="cuda") * 0.02).half()
        y = torch.empty(M, V, device="cuda", dtype=torch.float32)
        us_h = timeit(lambda: dp.linear(x, H, wh, None, None, 0, y, V, M, V, H, path=1, io=2), n=10)
        us_d = timeit(lambda: dp.linear(x, H, wd, None, None, 0, y, V, M, V, H, path=1, io=2), n=20)
        res[f"lm_head V{V} H{H} rows{M}"] = {"us_host": round(us_h, 1), "pcie_gbs": round(V * H * 2 / us_h / 1e3, 1),
                                            "us_hbm": round(us_d, 2), "hbm_gbs": round(V * H * 2 / us_d / 1e3, 1)}
        dp.host_free(wh)
if which in ("all", "embed"):
    V, P, H, S = 30522, 512, 768, 128
    word = dp.host_alloc(V * H * 2)
    pos = dp.host_alloc(P * H * 2)
    typ = dp.host_alloc(2 * H * 2)
    g = dp.host_alloc(H * 2)
    bb = dp.host_alloc(H * 2)
    ids = torch.randint(0, V, (S,), device="cuda", dtype=torch.int32)
    out = torch.empty(S, H, device="cuda").half()
    us = timeit(lambda: dp.embed(ids, S, word, pos, typ, g, bb, H, 1e-12, out), n=20)
    res["embed DHA S128 H768"] = {"us": round(us, 2), "pcie_gbs": round((2 * S + 3) * H * 2 / us / 1e3, 1)}

if which in ("all", "lnhost"):
    # DHA LayerNorm: gamma / beta host-mapped, read once per launch (one cluster, DSMEM broadcast)
    for rows, n in [(128, 768), (384, 1024)]:
        x = torch.randn(rows, n, device="cuda").half()
        g = dp.host_alloc(n * 2)
        bb = dp.host_alloc(n * 2)
        y = torch.empty_like(x)
        us = timeit(lambda: dp.layernorm(x, None, g, bb, y, rows, n, 1e-5), n=20)
        res[f"layernorm DHA {rows}x{n}"] = {"us": round(us, 2), "host_bytes": 4 * n}
        dp.host_free(g)
        dp.host_free(bb)
if which in ("all", "fp32"):
    # fp32 storage (DP_FP32): the CUDA-core linear with weights from host (DHA) and HBM, attention
    for (M, N, K) in [(128, 768, 768), (128, 3072, 768)]:
        x = torch.randn(M, K, device="cuda")
        wh = dp.host_alloc(N * K * 4)
        wd = torch.randn(N, K, device="cuda")
        y = torch.empty(M, N, device="cuda")
        us_h = timeit(lambda: dp.linear(x, K, wh, None, None, 0, y, N, M, N, K, path=1, dtype="fp32"), n=10)
        us_d = timeit(lambda: dp.linear(x, K, wd, None, None, 0, y, N, M, N, K, path=1, dtype="fp32"), n=20)
        res[f"fp32 linear M{M} N{N} K{K}"] = {"us_host": round(us_h, 2), "pcie_gbs": round(N * K * 4 / us_h / 1e3, 1),
                                             "us_hbm": round(us_d, 2), "tflops_hbm": round(2 * M * N * K / us_d / 1e6, 2)}
        dp.host_free(wh)
    for S, causal in ((128, 0), (1024, 1)):
        H, heads = 768, 12
        qkv = torch.randn(S, 3 * H, device="cuda")
        o = torch.empty(S, H, device="cuda")
        us = timeit(lambda: dp.attention(qkv, 3 * H, o, 1, S, H, heads, causal, dtype="fp32"), n=10)
        res[f"fp32 attention S{S} causal{causal}"] = {"us": round(us, 2)}
if which in ("all", "ptfwd"):
    # SM-driven PT forwarder vs the copy engine, host -> this GPU's HBM (on one GPU
    # the NVLink hop of the multi-GPU case is a local store): the per-link read side of PT.
    for mb in (1, 4, 32, 128):
        nb = mb << 20
        src = torch.empty(nb, dtype=torch.uint8).pin_memory()
        src.random_(0, 255)
        dst = torch.empty(nb, dtype=torch.uint8, device="cuda")
        us_f = timeit(lambda: dp.pt_forward(src, dst, nb), n=max(3, min(reps, 2048 // mb)))
        us_d = timeit(lambda: dst.copy_(src, non_blocking=True), n=max(3, min(reps, 2048 // mb)))
        assert torch.equal(dst.cpu(), src)
        res[f"pt_forward {mb} MiB"] = {"us": round(us_f, 2), "gbs": round(nb / us_f / 1e3, 2),
                                       "dma_us": round(us_d, 2), "dma_gbs": round(nb / us_d / 1e3, 2)}

print(json.dumps(res, indent=1))
