"""Pins for oracle/ops.py against independent definitions (not the oracle itself).

- GEMM: brute-force triple loops with math.fsum in every transpose mode + ACC.
- softmax-CE: torch.nn.functional.cross_entropy (fp64) and its autograd gradient;
  closed form ln C for zero logits (SURVEY.md 8(c) pins: ln 10 = 2.302585...);
  dlogits rows sum to 0.
- whole-network gradient: central finite differences (h = 1e-6) of the fp64 oracle
  loss on 2-3-2 and 5-7-3 MLPs (catches transposed operands, sign and index errors
  in GEMM / bias / ReLU backward / softmax-CE backward).
- SGD-momentum closed form for a constant gradient:
      a_t = g (1 - mu^t) / (1 - mu),  w_t = w_0 - lr g sum_{s=1..t} (1 - mu^s) / (1 - mu).
- Adam closed form for a constant gradient (TF form, reading Q8):
      w_t = w_0 - sum_{s=1..t} lr g sqrt(1-b2^s) / (|g| sqrt(1-b2^s) + eps);
  g = 0 leaves w bitwise unchanged.
- ReLU backward at h = 0 passes no gradient (reading Q10, TF ReluGrad).
- GELU (exact erf form): torch.nn.functional.gelu(approximate="none") in fp64 and its
  autograd derivative; identities gelu(0) = 0, gelu(u) - gelu(-u) = u (Phi(u) + Phi(-u)
  = 1), gelu'(0) = 1/2; the whole-MLP finite differences run with GELU layers too.
"""
import math

import numpy as np
import pytest
import torch

from oracle import ops as O
from oracle import graph as OG
from sf_inputs import graphs as G, data as D
from sf_inputs.ir import ACC, TA, TB, SGD_MOM, ADAM, STEP_INC, PARAM


def brute_gemm(A, B, C, flags):
    a = A.T if flags & TA else A
    b = B.T if flags & TB else B
    M, K = a.shape
    N = b.shape[1]
    out = np.zeros((M, N))
    for i in range(M):
        for j in range(N):
            terms = [float(a[i, k]) * float(b[k, j]) for k in range(K)]
            if flags & ACC:
                terms.append(float(C[i, j]))
            out[i, j] = math.fsum(terms)
    return out


@pytest.mark.parametrize("flags", [0, TA, TB, TA | TB, ACC, TA | ACC, TB | ACC, TA | TB | ACC])
def test_gemm_brute_force(flags):
    rng = np.random.default_rng(11 + flags)
    M, N, K = 5, 3, 7
    A = rng.standard_normal((K, M) if flags & TA else (M, K)).astype(np.float32)
    B = rng.standard_normal((N, K) if flags & TB else (K, N)).astype(np.float32)
    C = rng.standard_normal((M, N)).astype(np.float32)
    got = O.gemm(A, B, C, flags)
    assert got.dtype == np.float32 and got.shape == (M, N)
    ref = brute_gemm(A, B, C, flags)
    np.testing.assert_allclose(got, ref, rtol=1e-6, atol=1e-6)
    # exactly one rounding: the fp32 result is the nearest float to the fp64 value
    assert np.array_equal(got, ref.astype(np.float32))


def test_softmax_ce_vs_torch():
    rng = np.random.default_rng(5)
    B, C = 9, 13
    l = (rng.standard_normal((B, C)) * 4).astype(np.float32)
    y = rng.integers(0, C, size=(B, 1)).astype(np.int32)
    loss, d = O.softmax_ce(l, y)
    lt = torch.tensor(l, dtype=torch.float64, requires_grad=True)
    ref = torch.nn.functional.cross_entropy(lt, torch.tensor(y[:, 0], dtype=torch.long))
    ref.backward()
    assert abs(float(loss[0, 0]) - ref.item()) <= 1e-6 * abs(ref.item())
    np.testing.assert_allclose(d, lt.grad.numpy(), rtol=1e-6, atol=1e-8)
    np.testing.assert_allclose(d.astype(np.float64).sum(axis=1), 0.0, atol=1e-7)


def test_softmax_ce_zero_logits_is_ln_c():
    for C in (10, 1000, 30522):
        loss, d = O.softmax_ce(np.zeros((4, C), np.float32), np.zeros((4, 1), np.int32))
        assert float(loss[0, 0]) == np.float32(math.log(C))
        assert np.isclose(float(d[0, 1]), 1.0 / C / 4, rtol=1e-6)


def test_softmax_large_logits_stable():
    l = np.array([[1000.0, 0.0, -1000.0]], np.float32)
    p = O.softmax(l)
    assert np.all(np.isfinite(p)) and p[0, 0] == 1.0
    loss, d = O.softmax_ce(l, np.array([[2]], np.int32))
    assert np.isfinite(loss).all() and abs(float(loss[0, 0]) - 2000.0) < 1e-3


def test_relu_backward_at_zero_passes_nothing():
    dz, db = O.bias_act_bwd(np.ones((2, 3), np.float32),
                            np.array([[0.0, 1.0, -0.0], [2.0, 0.0, 3.0]], np.float32))
    assert dz.tolist() == [[0.0, 1.0, 0.0], [1.0, 0.0, 1.0]]
    assert db.tolist() == [[1.0, 1.0, 1.0]]


def test_identity_weights_pass_input_through():
    x = np.random.default_rng(2).random((4, 6)).astype(np.float32)
    z = O.gemm(x, np.eye(6, dtype=np.float32), None, 0)
    assert np.array_equal(z, x)


def _fwd_bwd(g, T, parts, exact=True, with_bwd=True):
    shapes = {i: (t.rows, t.cols) for i, t in enumerate(g.tensors)}
    for (a, b) in parts:
        for j in range(a, b):
            op = g.ops[j]
            if op.type in (SGD_MOM, ADAM, STEP_INC):
                continue
            O.apply_op(op, T, shapes, exact)


@pytest.mark.parametrize("act", ["relu", "gelu"])
@pytest.mark.parametrize("widths,batch", [((2, 3, 2), 4), ((5, 7, 3), 6), ((4, 6, 5, 3), 5)])
def test_finite_difference_whole_mlp(widths, batch, act):
    g = G.mlp_train(widths, batch=batch, pool=1, act=act)
    OG.validate(g)
    parts = OG.partition(g)
    st = D.init_state(g, seed=21)
    ds = D.datasets(g, seed=22)
    rng = np.random.default_rng(3)
    # non-zero biases so every term of the bias gradient is exercised
    for i, t in enumerate(g.tensors):
        if t.kind == PARAM and t.rows == 1:
            st[i] = rng.standard_normal((1, t.cols)).astype(np.float32) * 0.1

    def tensors():
        T = {i: a.astype(np.float64) if a.dtype == np.float32 else a.copy() for i, a in st.items()}
        T.update({i: a.astype(np.float64) if a.dtype == np.float32 else a for i, a in ds.items()})
        return T

    T = tensors()
    _fwd_bwd(g, T, parts)
    loss_id = g.tid("loss")
    L = len(widths) - 1
    h = 1e-6
    for li in range(1, L + 1):
        for pname, gname in ((f"W{li}", f"dW{li}"), (f"b{li}", f"db{li}")):
            p, gr = g.tid(pname), g.tid(gname)
            grad = T[gr]
            fd = np.zeros_like(grad)
            for idx in np.ndindex(*grad.shape):
                vals = []
                for sgn in (+1, -1):
                    T2 = tensors()
                    T2[p] = T2[p].copy()
                    T2[p][idx] += sgn * h
                    _fwd_bwd(g, T2, parts)
                    vals.append(T2[loss_id][0, 0])
                fd[idx] = (vals[0] - vals[1]) / (2 * h)
            scale = max(np.abs(fd).max(), 1e-12)
            assert np.abs(fd - grad).max() / scale < 1e-6, (pname, fd, grad)


def test_sgd_momentum_closed_form():
    lr, mu = 0.01, 0.9
    w0 = np.array([[1.5, -2.0, 0.25]], np.float32)
    g = np.array([[0.3, -0.7, 1e-3]], np.float32)
    w, a = w0.copy(), np.zeros_like(w0)
    for t in range(1, 31):
        w, a = O.sgd_momentum(w, a, g, lr, mu, exact=True)
        a_cf = g.astype(np.float64) * (1 - mu ** t) / (1 - mu)
        w_cf = w0.astype(np.float64) - lr * g.astype(np.float64) * sum(
            (1 - mu ** s) / (1 - mu) for s in range(1, t + 1))
        np.testing.assert_allclose(a, a_cf, rtol=1e-12)
        np.testing.assert_allclose(w, w_cf, rtol=1e-12)


def test_adam_closed_form_and_zero_grad():
    lr, b1, b2, eps = 1e-3, 0.9, 0.999, 1e-8
    w0 = np.array([[0.5, -1.0, 2.0, 0.0]], np.float32)
    g = np.array([[0.2, -3.0, 1e-4, 5.0]], np.float32)
    w, m, v = w0.copy(), np.zeros_like(w0), np.zeros_like(w0)
    for t in range(1, 21):
        step = np.array([[t - 1]], np.int32)
        w, m, v = O.adam(w, m, v, g, step, lr, b1, b2, eps, exact=True)
        gg = g.astype(np.float64)
        cf = w0.astype(np.float64) - sum(
            lr * gg * math.sqrt(1 - b2 ** s) / (np.abs(gg) * math.sqrt(1 - b2 ** s) + eps)
            for s in range(1, t + 1))
        np.testing.assert_allclose(w, cf, rtol=1e-10, atol=1e-12)
    # t = 1: update ~= lr * sign(g)
    w1, _, _ = O.adam(w0, np.zeros_like(w0), np.zeros_like(w0), g, np.array([[0]], np.int32),
                      lr, b1, b2, eps, exact=True)
    big = np.abs(g) >= 0.1  # lr*sign(g) holds where |g| sqrt(1-b2) >> eps
    np.testing.assert_allclose((w0 - w1)[big], (lr * np.sign(g))[big], rtol=1e-5)
    # g = 0 from the start: bitwise unchanged (fp32 path)
    z = np.zeros_like(w0)
    w2, m2, v2 = O.adam(w0, z, z, z, np.array([[7]], np.int32), lr, b1, b2, eps)
    assert w2.tobytes() == w0.tobytes() and not m2.any() and not v2.any()


def test_feed_cycles_through_pool():
    pool = np.arange(12, dtype=np.float32).reshape(6, 2)
    assert O.feed(pool, np.array([[0]]), 2).tolist() == [[0, 1], [2, 3]]
    assert O.feed(pool, np.array([[4]]), 2).tolist() == [[4.0, 5.0], [6.0, 7.0]]
    assert O.feed(pool, np.array([[5]]), 2).tolist() == [[8.0, 9.0], [10.0, 11.0]]


def test_gelu_vs_torch_and_identities():
    rng = np.random.default_rng(8)
    u = (rng.standard_normal((7, 11)) * 3).astype(np.float32)
    ut = torch.tensor(u, dtype=torch.float64, requires_grad=True)
    ref = torch.nn.functional.gelu(ut, approximate="none")
    h = O.gelu(u)
    np.testing.assert_allclose(h, ref.detach().numpy(), rtol=1e-6, atol=1e-7)
    assert np.array_equal(h, ref.detach().numpy().astype(np.float32))  # one rounding
    dh = rng.standard_normal((7, 11)).astype(np.float32)
    ref.backward(torch.tensor(dh, dtype=torch.float64))
    dz, db = O.gelu_bwd(dh, u)
    np.testing.assert_allclose(dz, ut.grad.numpy(), rtol=1e-6, atol=1e-7)
    np.testing.assert_allclose(db[0], ut.grad.numpy().sum(axis=0), rtol=1e-6, atol=1e-6)
    x = np.linspace(-6, 6, 101)
    e = O.gelu(x, exact=True) - O.gelu(-x, exact=True)
    np.testing.assert_allclose(e, x, atol=1e-14)
    assert O.gelu(np.zeros((1, 1)), exact=True)[0, 0] == 0.0
    d0, _ = O.gelu_bwd(np.ones((1, 1)), np.zeros((1, 1)), exact=True)
    assert d0[0, 0] == 0.5
    h, uu = O.bias_gelu(np.zeros((2, 3), np.float32), [np.full((1, 3), 10.0, np.float32)])
    assert np.all(uu == 10.0) and np.all(h == 10.0)
