"""GPU parity of each hot-path kernel against the fp64 oracle, through the C-ABI.

Tolerances: both sides see the same storage-rounded inputs; the kernel
accumulates in fp32 and rounds its output once to fp16/bf16, so an element may differ
from the fp64 value by half an output ulp plus the fp32 accumulation error:
  |y - ref| <= 2^-10 |ref| + K * 2^-22 * max|x w|  (fp16)   /  2^-7 |ref| + ...  (bf16).
Direct-host-access changes only WHERE the weights are read from, so the same kernel on a
host-mapped pointer and on a device pointer must give bit-identical results.
"""
import math

import numpy as np
import pytest

import synth
from oracle import forward as F

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

DT = {"fp16": torch.float16, "bf16": torch.bfloat16}
EPS_OUT = {"fp16": 2.0 ** -10, "bf16": 2.0 ** -7}


def dp():
    import paper_conf_eurosys_jeongba23_b200 as m
    return m


def to_t(a, dtype, dev="cuda"):
    if dtype == "bf16":
        t = torch.from_numpy(a.view(np.int16).copy()).view(torch.bfloat16)
    else:
        t = torch.from_numpy(np.ascontiguousarray(a))
    return t.to(dev)


def f64(t):
    return t.float().cpu().numpy().astype(np.float64)


class HostBuf:
    """Pinned + mapped host memory from the library (a DHA weight location)."""

    def __init__(self, arr: np.ndarray):
        self.nbytes = arr.nbytes
        self.ptr = dp().host_alloc(self.nbytes)
        np.ctypeslib.as_array((np.ctypeslib.ctypes.c_uint8 * self.nbytes).from_address(self.ptr))[:] = \
            np.frombuffer(np.ascontiguousarray(arr).tobytes(), dtype=np.uint8)

    def free(self):
        dp().host_free(self.ptr)


def close(y, ref, dtype, K=1, scale=1.0):
    tol = EPS_OUT[dtype] * np.abs(ref) + K * 2.0 ** -22 * scale + 1e-6
    err = np.abs(y - ref)
    assert np.all(err <= tol), f"max err {err.max():.3e}, worst tol {tol.flat[np.argmax(err - tol)]:.3e}"


# ---------------------------------------------------------------------------------------
# K1 embedding
# ---------------------------------------------------------------------------------------

@pytest.mark.parametrize("name,B,S", [("tiny_bert", 2, 33), ("bert_base", 1, 128), ("tiny_roberta", 1, 100),
                                      ("tiny_gpt2", 3, 17), ("bert_large", 1, 384)])
@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
def test_embed_parity_and_dha_bit_identity(name, B, S, dtype):
    m = synth.SHAPES[name]
    w = synth.make_weights(m, seed=1, dtype=dtype, recipe="scaled")
    ids = synth.make_ids(m, B, S, seed=2)
    ref = F.embed(m, w, ids, dtype).reshape(B * S, m.hidden)
    gpt = m.family == "gpt2"
    names = (["wte.weight", "wpe.weight"] if gpt else
             ["embeddings.word_embeddings.weight", "embeddings.position_embeddings.weight",
              "embeddings.token_type_embeddings.weight", "embeddings.LayerNorm.weight",
              "embeddings.LayerNorm.bias"])
    dev_t = {n: to_t(w[n], dtype) for n in names}
    host_b = {n: HostBuf(w[n]) for n in names}
    ids_t = torch.from_numpy(ids.reshape(-1)).cuda()
    pos_off = m.pad_idx + 1 if m.family == "roberta" else 0
    outs = []
    for where in ("device", "host"):
        P = (lambda n: dev_t[n].data_ptr()) if where == "device" else (lambda n: host_b[n].ptr)
        out = torch.empty(B * S, m.hidden, dtype=DT[dtype], device="cuda")
        if gpt:
            dp().embed(ids_t, S, P(names[0]), P(names[1]), None, None, None, m.hidden, 0.0, out, dtype)
        else:
            dp().embed(ids_t, S, P(names[0]), P(names[1]), P(names[2]), P(names[3]), P(names[4]), m.hidden,
                       m.ln_eps, out, dtype, pos_offset=pos_off)
        torch.cuda.synchronize()
        outs.append(out)
    assert torch.equal(outs[0].view(torch.int16), outs[1].view(torch.int16))
    y = f64(outs[0])
    # LN output: fp32 statistics + one output rounding
    tol = EPS_OUT[dtype] * np.abs(ref) + 2e-4 * (1 if gpt else np.abs(ref).max())
    assert np.all(np.abs(y - ref) <= tol), np.abs(y - ref).max()
    for b in host_b.values():
        b.free()


# ---------------------------------------------------------------------------------------
# K2 / K3 linear
# ---------------------------------------------------------------------------------------

SHAPES_LIN = [(1, 128, 64), (7, 256, 128), (32, 768, 768), (100, 384, 128), (128, 768, 768), (128, 3072, 768),
              (128, 768, 3072), (200, 1024, 1024), (384, 4096, 1024), (1024, 1024, 4096), (333, 2304, 768),
              # K ranges that are not a multiple of a ring stage's 3 / 2 chunks of 64 (the last 3D TMA
              # box zero-fills past K), a single chunk, and the 96 / 192-token tiles of the measured table
              (64, 256, 64), (48, 384, 192), (300, 512, 320), (200, 256, 64), (384, 4096, 1024),
              (1024, 3072, 1024)]


@pytest.mark.parametrize("M,N,K", SHAPES_LIN)
@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
def test_linear_tcgen05_parity(M, N, K, dtype):
    rng = np.random.default_rng(M * 7 + N + K)
    x = synth.round_to(rng.standard_normal((M, K)).astype(np.float32), dtype)
    wt = synth.round_to((rng.standard_normal((N, K)) / math.sqrt(K)).astype(np.float32), dtype)
    b = synth.round_to((0.1 * rng.standard_normal(N)).astype(np.float32), dtype)
    r = synth.round_to(rng.standard_normal((M, N)).astype(np.float32), dtype)
    X, W, Bt, R = (to_t(a, dtype) for a in (x, wt, b, r))
    x64, w64, b64, r64 = (synth.storage_to_f64(a, dtype) for a in (x, wt, b, r))
    for act, res in (("none", False), ("gelu_erf", False), ("none", True), ("gelu_tanh", True)):
        Y = torch.empty(M, N, dtype=DT[dtype], device="cuda")
        dp().linear(X, K, W, Bt, R if res else None, N, Y, N, M, N, K, act=act, path=0, dtype=dtype)
        torch.cuda.synchronize()
        ref = F.linear(x64, w64, b64, act, r64 if res else None)
        close(f64(Y), ref, dtype, K=K, scale=np.abs(x64).max() * np.abs(w64).max() * 4)


@pytest.mark.parametrize("M,N,K", [(1, 768, 768), (5, 128, 64), (128, 768, 768), (128, 3072, 768),
                                   (128, 768, 3072), (384, 1024, 4096), (17, 2304, 768),
                                   # M <= 8, K in 256..1024: the streaming GEMV (pooler, LM head), ragged N
                                   (2, 1001, 256), (3, 50257, 1024), (4, 129, 512), (6, 3072, 1024), (8, 777, 768)])
@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
def test_linear_skinny_dha_parity_and_bit_identity(M, N, K, dtype):
    rng = np.random.default_rng(M + 3 * N + K)
    x = synth.round_to(rng.standard_normal((M, K)).astype(np.float32), dtype)
    wt = synth.round_to((rng.standard_normal((N, K)) / math.sqrt(K)).astype(np.float32), dtype)
    b = synth.round_to((0.1 * rng.standard_normal(N)).astype(np.float32), dtype)
    X, W, Bt = (to_t(a, dtype) for a in (x, wt, b))
    hw, hb = HostBuf(wt), HostBuf(b)
    Y0 = torch.empty(M, N, dtype=DT[dtype], device="cuda")
    Y1 = torch.empty_like(Y0)
    dp().linear(X, K, W, Bt, None, 0, Y0, N, M, N, K, act="tanh", path=1, dtype=dtype)
    dp().linear(X, K, hw.ptr, hb.ptr, None, 0, Y1, N, M, N, K, act="tanh", path=1, dtype=dtype)
    torch.cuda.synchronize()
    assert torch.equal(Y0.view(torch.int16), Y1.view(torch.int16))
    ref = F.linear(*(synth.storage_to_f64(a, dtype) for a in (x, wt, b)), act="tanh")
    close(f64(Y0), ref, dtype, K=K, scale=4 * np.abs(synth.storage_to_f64(x, dtype)).max())
    hw.free()
    hb.free()


@pytest.mark.parametrize("M,N,K", [(300, 256, 1536), (129, 64, 2304), (257, 128, 6144), (45, 32, 48)])
def test_linear_skinny_split_k_cluster_residual(M, N, K):
    """K split over a thread-block cluster (cs = 2, 3, 8) and one CTA (K = 48, a ragged last
    chunk), ragged token blocks, fp32 residual read and written in place (the GPT-2 stream)."""
    dtype = "fp16"
    rng = np.random.default_rng(M + N + K)
    x = synth.round_to(rng.standard_normal((M, K)).astype(np.float32), dtype)
    wt = synth.round_to((rng.standard_normal((N, K)) / math.sqrt(K)).astype(np.float32), dtype)
    b = synth.round_to((0.1 * rng.standard_normal(N)).astype(np.float32), dtype)
    r = rng.standard_normal((M, N))
    X, W, Bt = (to_t(a, dtype) for a in (x, wt, b))
    hw = HostBuf(wt)
    outs = []
    for wptr in (W, hw.ptr):
        Rf = torch.from_numpy(r.astype(np.float32)).cuda()
        dp().linear(X, K, wptr, Bt, Rf, N, Rf, N, M, N, K, act="gelu_erf", path=1, dtype=dtype, io=3)
        torch.cuda.synchronize()
        outs.append(Rf)
    assert torch.equal(outs[0], outs[1])
    x64, w64, b64 = (synth.storage_to_f64(a, dtype) for a in (x, wt, b))
    ref = F.linear(x64, w64, b64, "gelu_erf", r.astype(np.float32).astype(np.float64))
    err = np.abs(outs[0].double().cpu().numpy() - ref).max()
    assert err <= 1e-4 * math.sqrt(K) * (1 + np.abs(ref).max()), err
    hw.free()


def test_linear_strided_output_and_input():
    """q/k/v write into column blocks of the [T, 3H] buffer; the pooler reads every S-th row."""
    dtype = "fp16"
    rng = np.random.default_rng(5)
    T, H = 96, 256
    x = synth.round_to(rng.standard_normal((T, H)).astype(np.float32), dtype)
    wt = synth.round_to((rng.standard_normal((H, H)) / 16).astype(np.float32), dtype)
    X, W = to_t(x, dtype), to_t(wt, dtype)
    qkv = torch.zeros(T, 3 * H, dtype=torch.float16, device="cuda")
    dp().linear(X, H, W, None, None, 0, qkv[:, H:].data_ptr(), 3 * H, T, H, H, path=0, dtype=dtype)
    torch.cuda.synchronize()
    ref = F.linear(x.astype(np.float64), wt.astype(np.float64))
    close(f64(qkv[:, H:2 * H]), ref, dtype, K=H, scale=16)
    assert torch.count_nonzero(qkv[:, :H]) == 0 and torch.count_nonzero(qkv[:, 2 * H:]) == 0
    # strided input (every 32nd row) through the skinny kernel
    Y = torch.empty(3, H, dtype=torch.float16, device="cuda")
    dp().linear(X, 32 * H, W, None, None, 0, Y, H, 3, H, H, path=1, dtype=dtype)
    torch.cuda.synchronize()
    close(f64(Y), ref[::32], dtype, K=H, scale=16)


# ---------------------------------------------------------------------------------------
# K4 LayerNorm, K5 attention
# ---------------------------------------------------------------------------------------

@pytest.mark.parametrize("rows,n", [(1, 128), (37, 768), (128, 1024), (1000, 768)])
def test_layernorm_parity_and_dha(rows, n):
    dtype = "fp16"
    rng = np.random.default_rng(rows + n)
    x = synth.round_to((3 * rng.standard_normal((rows, n)) + 1).astype(np.float32), dtype)
    r = synth.round_to(rng.standard_normal((rows, n)).astype(np.float32), dtype)
    g = synth.round_to((1 + 0.1 * rng.standard_normal(n)).astype(np.float32), dtype)
    b = synth.round_to((0.1 * rng.standard_normal(n)).astype(np.float32), dtype)
    X, R, G, Bt = (to_t(a, dtype) for a in (x, r, g, b))
    hg, hb = HostBuf(g), HostBuf(b)
    Y0 = torch.empty(rows, n, dtype=torch.float16, device="cuda")
    Y1 = torch.empty_like(Y0)
    dp().layernorm(X, R, G, Bt, Y0, rows, n, 1e-5)
    dp().layernorm(X, R, hg.ptr, hb.ptr, Y1, rows, n, 1e-5)
    torch.cuda.synchronize()
    assert torch.equal(Y0, Y1)
    ref = F.layer_norm(x.astype(np.float64) + r.astype(np.float64), g.astype(np.float64), b.astype(np.float64),
                       1e-5)
    close(f64(Y0), ref, dtype, K=n, scale=8)
    hg.free()
    hb.free()


@pytest.mark.parametrize("B,S,H,heads", [(1, 1, 128, 2), (2, 5, 128, 2), (1, 64, 768, 12), (2, 100, 256, 4),
                                         (1, 128, 768, 12), (1, 384, 1024, 16), (1, 1024, 1024, 16),
                                         (3, 200, 256, 4)])
@pytest.mark.parametrize("causal", [False, True])
@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
def test_attention_parity(B, S, H, heads, causal, dtype):
    rng = np.random.default_rng(B * 1000 + S + H)
    qkv = synth.round_to((1.5 * rng.standard_normal((B * S, 3 * H))).astype(np.float32), dtype)
    Q = to_t(qkv, dtype)
    O = torch.empty(B * S, H, dtype=DT[dtype], device="cuda")
    dp().attention(Q, 3 * H, O, B, S, H, heads, causal, dtype)
    torch.cuda.synchronize()
    q64 = synth.storage_to_f64(qkv, dtype).reshape(B, S, 3 * H)
    ref = F.attention(q64[..., :H], q64[..., H:2 * H], q64[..., 2 * H:], heads, causal).reshape(B * S, H)
    # P is rounded to fp16/bf16 before the P.V product (flash attention), hence the looser bound
    tol = (4 if dtype == "fp16" else 8) * EPS_OUT[dtype] * (np.abs(ref) + np.abs(q64).max())
    err = np.abs(f64(O) - ref)
    assert np.all(err <= tol), err.max()


@pytest.mark.parametrize("B,S,H,heads", [(1, 1, 128, 2), (2, 5, 128, 2), (1, 32, 128, 2), (1, 64, 768, 12),
                                         (1, 65, 128, 2), (2, 77, 256, 4), (1, 128, 768, 12), (1, 192, 256, 4),
                                         (1, 384, 1024, 16), (1, 1024, 1024, 16), (3, 200, 256, 4),
                                         (1, 512, 256, 4), (1, 700, 512, 8), (1, 1024, 256, 4)])
@pytest.mark.parametrize("causal", [False, True])
@pytest.mark.parametrize("dtype", ["fp16", "bf16"])
def test_attention_tc_parity(B, S, H, heads, causal, dtype):
    """K5t (tcgen05: S and P.V in TMEM, one softmax row per thread) against the oracle, same bound as
    K5 (P is rounded to the storage type before P.V).  The shapes cover every key-range split the
    launcher picks (1 CTA per query tile; a cluster of 2 / 4 CTAs merging over DSMEM: S512 x 4
    heads and S700 x 8 heads (ragged) -> 2, S1024 x 4 heads -> 4, where causal query tile 0 leaves
    CTAs with no key tile at all and rows fully masked in a CTA's range)."""
    rng = np.random.default_rng(B * 1000 + S + H + 7)
    qkv = synth.round_to((1.5 * rng.standard_normal((B * S, 3 * H))).astype(np.float32), dtype)
    Q = to_t(qkv, dtype)
    O = torch.empty(B * S, H, dtype=DT[dtype], device="cuda")
    dp().attention_tc(Q, 3 * H, O, B, S, H, heads, causal, dtype)
    torch.cuda.synchronize()
    q64 = synth.storage_to_f64(qkv, dtype).reshape(B, S, 3 * H)
    ref = F.attention(q64[..., :H], q64[..., H:2 * H], q64[..., 2 * H:], heads, causal).reshape(B * S, H)
    tol = (4 if dtype == "fp16" else 8) * EPS_OUT[dtype] * (np.abs(ref) + np.abs(q64).max())
    err = np.abs(f64(O) - ref)
    assert np.all(err <= tol), err.max()


def test_fp32_residual_stream_io():
    """GPT-2's pre-LN residual stream stays fp32: linear with fp32 residual+output (io=3),
    LayerNorm reading fp32, embedding writing fp32."""
    rng = np.random.default_rng(77)
    M, N, K = 130, 256, 512
    x = synth.round_to(rng.standard_normal((M, K)).astype(np.float32), "fp16")
    wt = synth.round_to((rng.standard_normal((N, K)) / 22).astype(np.float32), "fp16")
    r = (rng.standard_normal((M, N)) * 3).astype(np.float32)
    X, W = to_t(x, "fp16"), to_t(wt, "fp16")
    for path in (0, 1):
        R = torch.from_numpy(r.copy()).cuda()
        dp().linear(X, K, W, None, R, N, R, N, M, N, K, path=path, io=3)  # in place, fp32
        torch.cuda.synchronize()
        ref = F.linear(x.astype(np.float64), wt.astype(np.float64), None, "none", r.astype(np.float64))
        err = np.abs(R.cpu().numpy().astype(np.float64) - ref)
        assert err.max() <= 1e-4 * (1 + np.abs(ref).max()), err.max()
    g = synth.round_to((1 + 0.1 * rng.standard_normal(N)).astype(np.float32), "fp16")
    b = synth.round_to((0.1 * rng.standard_normal(N)).astype(np.float32), "fp16")
    Rt = torch.from_numpy(r).cuda()
    Y = torch.empty(M, N, dtype=torch.float16, device="cuda")
    dp().layernorm(Rt, None, to_t(g, "fp16"), to_t(b, "fp16"), Y, M, N, 1e-5, x_f32=True)
    torch.cuda.synchronize()
    ref = F.layer_norm(r.astype(np.float64), g.astype(np.float64), b.astype(np.float64), 1e-5)
    close(f64(Y), ref, "fp16", K=N, scale=8)


def _gemm_forced_case(bn, split, M, N, K, act, res, dtype, seed):
    """One forced tile configuration through dp_gemm_tc: parity with the oracle (the module's
    fp32-accumulation bound) and run-to-run bit equality (every reduction order is fixed)."""
    rng = np.random.default_rng(seed)
    x = synth.round_to(rng.standard_normal((M, K)).astype(np.float32), dtype)
    w = synth.round_to((rng.standard_normal((N, K)) / math.sqrt(K)).astype(np.float32), dtype)
    b = synth.round_to((0.1 * rng.standard_normal(N)).astype(np.float32), dtype)
    r = synth.round_to(rng.standard_normal((M, N)).astype(np.float32), dtype)
    X, W, B, R = (to_t(a, dtype) for a in (x, w, b, r))
    Y = torch.empty(M, N, dtype=DT[dtype], device="cuda")
    Y2 = torch.empty_like(Y)
    for out in (Y, Y2):
        dp().gemm_tc(X, K, W, B, R if res else None, N, out, N, M, N, K, act=act, bn=bn, split=split, dtype=dtype)
    torch.cuda.synchronize()
    assert torch.equal(Y, Y2), "forced GEMM configuration not deterministic"
    x64, w64, b64, r64 = (synth.storage_to_f64(a, dtype) for a in (x, w, b, r))
    ref = F.linear(x64, w64, b64, act, r64 if res else None)
    close(f64(Y), ref, dtype, K=K, scale=np.abs(x64).max() * np.abs(w64).max() * 4)


@pytest.mark.parametrize("bn,split,M,N,K", [(32, 2, 128, 768, 768), (32, 4, 128, 768, 3072), (32, 8, 100, 256, 1024),
                                             (64, 4, 200, 512, 2048), (128, 2, 384, 1024, 1024),
                                             (128, 4, 333, 768, 4096), (64, 8, 64, 128, 4096)])
def test_gemm_split_k_cluster_configs(bn, split, M, N, K):
    """Every (BN, split) the cluster split-K path can take, forced through dp_gemm_tc."""
    _gemm_forced_case(bn, split, M, N, K, "gelu_erf", True, "fp16", M + N + K)


@pytest.mark.parametrize("bn", [32, 64, 96, 128, 192, 256])
@pytest.mark.parametrize("M,N,K", [(100, 256, 512), (384, 1024, 1024), (1024, 512, 128)])
def test_gemm_single_cta_tile_widths(bn, M, N, K):
    """Every single-CTA tile width (K2) forced, ragged token tails included."""
    _gemm_forced_case(bn, 1, M, N, K, "gelu_tanh", True, "bf16", bn + M + N + K)


@pytest.mark.parametrize("bn", [-64, -128, -192, -256])
@pytest.mark.parametrize("M,N,K,dtype", [(1024, 4096, 1024, "fp16"), (384, 1024, 4096, "bf16"), (333, 2304, 768, "fp16"),
                                         (1, 256, 64, "fp16"), (100, 512, 64, "bf16"), (1000, 768, 3072, "fp16")])
def test_gemm_cta_pair_parity(bn, M, N, K, dtype):
    """K2p (tcgen05 cta_group::2, one 256 x |bn| tile per CTA pair): parity at the large models'
    shapes and ragged cases -- a token tile where only the leader's half holds rows (M = 1,
    M = 100 < |bn| / 2 for some widths), K = 64 (one k-block), a tail past M."""
    for act, res in (("none", False), ("gelu_erf", True)):
        _gemm_forced_case(bn, 0, M, N, K, act, res, dtype, -bn + M + N + K)


def test_gemm_cta_pair_rejects_odd_tile_count():
    X = torch.zeros(128, 64, dtype=torch.float16, device="cuda")
    W = torch.zeros(384, 64, dtype=torch.float16, device="cuda")
    Y = torch.empty(128, 384, dtype=torch.float16, device="cuda")
    with pytest.raises(dp().DeepPlanError, match="N % 256"):
        dp().gemm_tc(X, 64, W, None, None, 0, Y, 384, 128, 384, 64, bn=-128)
    with pytest.raises(dp().DeepPlanError, match="bn must be"):
        dp().gemm_tc(X, 64, W, None, None, 0, Y, 384, 128, 384, 64, bn=48)
