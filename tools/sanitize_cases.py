"""Small invocations of every hand-written kernel for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck): the tcgen05 GEMM with cluster split-K (DSMEM pushes), the DHA skinny
linear with cluster split-K, the cluster-broadcast LayerNorm and embedding (host-mapped
gamma / beta), attention (K5 / K5b / fp32), the fp32 linear, the SM PT forwarder (with its flag
protocol in loopback), and one tiny cold start per plan family.  Run under the sanitizer by
tools/sanitize.sh; exits non-zero on a Python-level error."""
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_eurosys_jeongba23_b200 as dp
import synth


def main():
    torch.manual_seed(0)
    dev = "cuda"
    # tcgen05 GEMM: plain, split-K over a cluster (K=3072 at M=128 picks splits), grouped q/k/v
    for M, N, K in ((128, 768, 3072), (96, 256, 512), (200, 384, 1024)):
        x = torch.randn(M, K, device=dev).half()
        w = (torch.randn(N, K, device=dev) / math.sqrt(K)).half()
        b = torch.randn(N, device=dev).half()
        r = torch.randn(M, N, device=dev).half()
        y = torch.zeros(M, N, device=dev).half()
        dp.linear(x, K, w, b, r, N, y, N, M, N, K, act="gelu_erf", path=0)
        # skinny (cluster split-K for K > 768), device and host-mapped weights
        dp.linear(x, K, w, b, r, N, y, N, M, N, K, path=1)
        hw = dp.host_alloc(N * K * 2)
        dp.linear(x, K, hw, None, None, 0, y, N, M, N, K, path=1)
        torch.cuda.synchronize()
        dp.host_free(hw)
    # round 2: forced tile widths incl. 96 / 192 and K ranges ending in a partial 3D-box stage
    for M, N, K, bn, sp in ((384, 512, 1024, 96, 1), (300, 512, 320, 192, 1), (128, 768, 768, 32, 4),
                            (100, 256, 192, 64, 2)):
        x = torch.randn(M, K, device=dev).half()
        w = (torch.randn(N, K, device=dev) / math.sqrt(K)).half()
        b = torch.randn(N, device=dev).half()
        r = torch.randn(M, N, device=dev).half()
        y = torch.zeros(M, N, device=dev).half()
        dp.gemm_tc(x, K, w, b, r, N, y, N, M, N, K, act="gelu_tanh", bn=bn, split=sp)
        torch.cuda.synchronize()
    # K5t: no split, key split over clusters of 2 and 4 (bulk DSMEM push + merge), causal and not
    for S, H, heads in ((384, 1024, 16), (512, 256, 4), (1024, 256, 4)):
        qkv = torch.randn(S, 3 * H, device=dev).half()
        o = torch.zeros(S, H, device=dev).half()
        for causal in (False, True):
            dp.attention_tc(qkv, 3 * H, o, 1, S, H, heads, causal)
        torch.cuda.synchronize()
    # LayerNorm / embedding with host-mapped gamma / beta (cluster DSMEM broadcast) and device ones
    for rows in (77, 384):
        n = 768
        x = torch.randn(rows, n, device=dev).half()
        y = torch.zeros_like(x)
        g = dp.host_alloc(n * 2)
        bb = dp.host_alloc(n * 2)
        dp.layernorm(x, None, g, bb, y, rows, n, 1e-12)
        dp.layernorm(x, x, torch.ones(n, device=dev).half(), torch.zeros(n, device=dev).half(), y, rows, n, 1e-12)
        torch.cuda.synchronize()
        dp.host_free(g)
        dp.host_free(bb)
    m = synth.SHAPES["tiny_bert"]
    w = synth.make_weights(m, seed=0)
    ctx = dp.Context([0])
    model = dp.Model(ctx, m, w)
    ids = torch.from_numpy(synth.make_ids(m, 2, 40)).cuda()
    out = torch.zeros(80, m.hidden, dtype=torch.float16, device=dev)
    pool = torch.zeros(2, m.hidden, dtype=torch.float16, device=dev)
    n = model.n
    kinds = [u["kind"] for u in model.units()]
    for meth in (np.zeros(n, np.int8), np.array([1 if k != "linear" else 0 for k in kinds], np.int8), np.ones(n, np.int8)):
        plan = dp._lib.PlanArrays(n, meth, None, 3, 1)
        model.infer_cold(plan, 0, ids, out, pool)
        torch.cuda.synchronize()
        model.infer_warm(0, ids, out, pool)
        torch.cuda.synchronize()
        model.evict(0)
    # PT in loopback through every transport (SM forwarder flags, staging ring, direct DMA)
    slot = np.array([i % 2 for i in range(n)], np.int8)
    for t in ("sm", "ce", "dma"):
        ctx.set_opts(pt_transport=t)
        plan = dp._lib.PlanArrays(n, np.zeros(n, np.int8), slot, 10, 2)
        model.infer_cold(plan, 0, ids, out, pool, secondaries=[0])
        torch.cuda.synchronize()
        model.evict(0)
    # attention: K5 (2 key tiles), K5b (groups), causal; fp32 path
    for S, causal in ((128, False), (384, False), (300, True)):
        H, heads = 256, 4
        qkv = torch.randn(S, 3 * H, device=dev).half()
        o = torch.zeros(S, H, device=dev).half()
        dp.attention(qkv, 3 * H, o, 1, S, H, heads, causal)
        o32 = torch.zeros(S, H, device=dev)
        dp.attention(qkv.float(), 3 * H, o32, 1, S, H, heads, causal, dtype="fp32")
    w32 = synth.make_weights(m, seed=0, dtype="fp32")
    model32 = dp.Model(ctx, m, w32, "fp32")
    out32 = torch.zeros(80, m.hidden, device=dev)
    pool32 = torch.zeros(2, m.hidden, device=dev)
    model32.infer_cold(dp._lib.PlanArrays(n, np.zeros(n, np.int8), None, 1, 1), 0, ids, out32, pool32)
    torch.cuda.synchronize()
    model32.evict(0)
    model32.close()
    model.close()
    ctx.close()
    print("sanitize cases done")


if __name__ == "__main__":
    main()
