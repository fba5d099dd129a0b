"""Pins of the single-linear oracle `oracle.forward.linear` (the reference of every K2 / K3
kernel test) against things other than itself:

* brute force: explicit triple loops over (m, n, k) in pure Python floats, with the bias added,
  then the activation, then the residual -- the order the paper's models use it in
  (BERT: LN(x + dense(c)) takes the residual after a plain linear; BERT/GPT-2 MLPs apply GELU
  to x W^T + b before anything else, P:241 / HF [35]);
* torch's float64 `torch.nn.functional.linear` + `torch.nn.functional.gelu` (erf and tanh
  approximations) + `torch.tanh`: the special case that reduces to a library routine;
* the GPT-2 Conv1D layout ([in, out], y = x W + b) equals `linear` on the transpose -- the
  arena stores Conv1D weights transposed ([out, in]) and the kernels read them that way;
* a plausible mistake would fail: transposed weight, dropped bias, activation after the
  residual, wrong GELU variant.
"""
import math

import numpy as np
import pytest

from oracle import forward as F

torch = pytest.importorskip("torch")


def brute(x, w, b, act, res):
    M, K = x.shape
    N = w.shape[0]
    y = np.zeros((M, N))
    for m in range(M):
        for n in range(N):
            s = 0.0
            for k in range(K):
                s += float(x[m, k]) * float(w[n, k])
            if b is not None:
                s += float(b[n])
            if act == "gelu_erf":
                s = 0.5 * s * (1.0 + math.erf(s / math.sqrt(2.0)))
            elif act == "gelu_tanh":
                s = 0.5 * s * (1.0 + math.tanh(math.sqrt(2.0 / math.pi) * (s + 0.044715 * s ** 3)))
            elif act == "tanh":
                s = math.tanh(s)
            if res is not None:
                s += float(res[m, n])
            y[m, n] = s
    return y


def rand(rng, *shape):
    return rng.standard_normal(shape)


@pytest.mark.parametrize("act", ["none", "gelu_erf", "gelu_tanh", "tanh"])
@pytest.mark.parametrize("with_bias", [True, False])
@pytest.mark.parametrize("with_res", [True, False])
@pytest.mark.parametrize("M,N,K", [(1, 1, 1), (3, 5, 7), (4, 2, 9)])
def test_linear_vs_brute_force(act, with_bias, with_res, M, N, K):
    rng = np.random.default_rng(M * 100 + N * 10 + K)
    x, w = rand(rng, M, K), rand(rng, N, K)
    b = rand(rng, N) if with_bias else None
    r = rand(rng, M, N) if with_res else None
    y = F.linear(x, w, b, act=act, residual=r)
    assert y.shape == (M, N)
    np.testing.assert_allclose(y, brute(x, w, b, act, r), rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("act", ["none", "gelu_erf", "gelu_tanh", "tanh"])
def test_linear_vs_torch_f64(act):
    rng = np.random.default_rng(5)
    M, N, K = 37, 29, 64
    x, w, b, r = rand(rng, M, K), rand(rng, N, K), rand(rng, N), rand(rng, M, N)
    t = torch.nn.functional.linear(torch.from_numpy(x), torch.from_numpy(w), torch.from_numpy(b))
    if act == "gelu_erf":
        t = torch.nn.functional.gelu(t)
    elif act == "gelu_tanh":
        t = torch.nn.functional.gelu(t, approximate="tanh")
    elif act == "tanh":
        t = torch.tanh(t)
    t = t + torch.from_numpy(r)
    np.testing.assert_allclose(F.linear(x, w, b, act=act, residual=r), t.numpy(), rtol=1e-13, atol=1e-13)


def test_gpt2_conv1d_layout_is_linear_on_the_transpose():
    """HF GPT-2 Conv1D: y = x W + b with W [in, out]; the library stores W^T ([out, in])."""
    rng = np.random.default_rng(6)
    x, wc, b = rand(rng, 11, 16), rand(rng, 16, 48), rand(rng, 48)
    conv = x @ wc + b  # Conv1D definition
    np.testing.assert_allclose(F.linear(x, wc.T, b), conv, rtol=1e-13, atol=1e-13)
    # the transposed operand is not interchangeable (a square case makes the mistake type-check)
    ws = rand(rng, 16, 16)
    assert np.abs(F.linear(x, ws, None) - x @ ws).max() > 1e-3


def test_linear_plausible_mistakes_are_caught():
    rng = np.random.default_rng(7)
    x, w, b, r = rand(rng, 5, 8), rand(rng, 6, 8), rand(rng, 6), rand(rng, 5, 6)
    ref = brute(x, w, b, "gelu_erf", r)
    y = F.linear(x, w, b, act="gelu_erf", residual=r)
    np.testing.assert_allclose(y, ref, rtol=1e-12, atol=1e-12)
    dropped_bias = brute(x, w, None, "gelu_erf", r)
    act_after_res = F.gelu_erf(x @ w.T + b + r)
    wrong_gelu = brute(x, w, b, "gelu_tanh", r)
    for bad in (dropped_bias, act_after_res, wrong_gelu):
        assert np.abs(bad - ref).max() > 1e-4
