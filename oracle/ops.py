"""Oracle op semantics (test infrastructure only; see oracle/__init__.py).

Each op reads fp32/int32 arrays, computes in fp64 and rounds its outputs once to
fp32 (SURVEY.md reading Q12).  With ``exact=True`` the arrays stay fp64 (used by
the finite-difference pins).  The paper runs these as TF ops backed by cuBLAS /
cuDNN (section 2.1); it fixes no formula, so the formulas are the
textbook / TF definitions named per function (readings Q8-Q10 in DESIGN.md).

Pins (tests/test_oracle_ops.py): GEMM vs brute-force loops in every transpose mode;
softmax-CE vs torch.nn.functional.cross_entropy in fp64 and the zero-weight closed
form ln C; whole-MLP central finite differences; SGD-momentum and Adam closed forms
for constant gradients; Adam bitwise no-op for g = 0.
"""
from __future__ import annotations

import numpy as np

from scipy.special import erf

from sf_inputs.ir import (ACC, ADAM, BIAS_ACT, BIAS_ACT_BWD, COLSUM, FEED, GELU, GEMM, RELU,
                          SGD_MOM, SOFTMAX, SOFTMAX_CE, STEP_INC, TA, TB)


def _f(x, exact):
    """Widen to fp64 (both modes accumulate in fp64)."""
    return np.asarray(x, dtype=np.float64)


def _out(x, exact):
    """Round once to fp32 (or keep fp64 in exact mode)."""
    return np.asarray(x, dtype=np.float64) if exact else np.asarray(x, dtype=np.float32)


def gemm(A, B, C_old, flags, exact=False):
    """C = op(A) @ op(B) [+ C_old]; op = transpose when TA / TB is set.

    Textbook matrix product (the paper's dense layers run as cuBLAS GEMMs,
    PAPER.md:321-323).  op(A) is [M, K], op(B) is [K, N].
    """
    a = _f(A, exact)
    b = _f(B, exact)
    if flags & TA:
        a = a.T
    if flags & TB:
        b = b.T
    c = a @ b
    if flags & ACC:
        c = c + _f(C_old, exact)
    return _out(c, exact)


def bias_act(z, biases, relu, exact=False):
    """h = act(z + b1 [+ b2 + b3]), biases broadcast over rows; act = ReLU or identity.

    TF BiasAdd + Relu.  Extra biases are BN/LN gamma/beta used additively (Q16).
    """
    s = _f(z, exact).copy()
    for b in biases:
        s = s + _f(b, exact)
    if relu:
        s = np.maximum(s, 0.0)
    return _out(s, exact)


def gelu(u, exact=False):
    """GELU, exact erf form (Hendrycks & Gimpel; BERT's activation; TF gelu with
    approximate=False): gelu(u) = u Phi(u) = 0.5 u (1 + erf(u / sqrt 2))."""
    x = _f(u, exact)
    return _out(0.5 * x * (1.0 + erf(x / np.sqrt(2.0))), exact)


def bias_gelu(z, biases, exact=False):
    """u = z + b1 [+ b2 + b3]; h = gelu(u).  Returns (h, u): u is kept for the backward."""
    s = _f(z, exact).copy()
    for b in biases:
        s = s + _f(b, exact)
    u = _out(s, exact)
    return gelu(u, exact), u


def gelu_bwd(dh, u, exact=False):
    """dz = dh * gelu'(u), gelu'(u) = Phi(u) + u phi(u) (product rule on u Phi(u));
    db = column sum of dz."""
    x = _f(u, exact)
    d = 0.5 * (1.0 + erf(x / np.sqrt(2.0))) + x * np.exp(-0.5 * x * x) / np.sqrt(2.0 * np.pi)
    dz = _f(dh, exact) * d
    return _out(dz, exact), _out(dz.sum(axis=0, keepdims=True), exact)


def bias_act_bwd(dh, h, exact=False):
    """dz = dh * [h > 0] (TF ReluGrad: gradient only where the output is > 0, Q10);
    db = column sum of dz."""
    dz = _f(dh, exact) * (_f(h, exact) > 0.0)
    db = dz.sum(axis=0, keepdims=True)
    return _out(dz, exact), _out(db, exact)


def colsum(x, exact=False):
    """s = column sum of x (bias gradient of an identity-activation layer)."""
    return _out(_f(x, exact).sum(axis=0, keepdims=True), exact)


def softmax_ce(logits, labels, exact=False):
    """Sparse softmax cross-entropy, mean over the batch (reading Q9).

    loss = (1/B) sum_i [ logsumexp(l_i) - l_i[y_i] ] with the row max subtracted;
    dlogits = (softmax(l) - onehot(y)) / B.
    """
    l = _f(logits, exact)
    y = np.asarray(labels).reshape(-1).astype(np.int64)
    B = l.shape[0]
    m = l.max(axis=1, keepdims=True)
    e = np.exp(l - m)
    s = e.sum(axis=1, keepdims=True)
    lse = m + np.log(s)
    loss = (lse[:, 0] - l[np.arange(B), y]).sum() / B
    p = e / s
    p[np.arange(B), y] -= 1.0
    d = p / B
    return _out(np.array([[loss]]), exact), _out(d, exact)


def softmax(logits, exact=False):
    """Row-wise softmax with the row max subtracted (inference output)."""
    l = _f(logits, exact)
    e = np.exp(l - l.max(axis=1, keepdims=True))
    return _out(e / e.sum(axis=1, keepdims=True), exact)


def sgd_momentum(w, a, g, lr, mu, exact=False):
    """TF MomentumOptimizer, non-Nesterov (reading Q8): a <- mu a + g; w <- w - lr a.

    Each output is rounded once; w uses the rounded a (what the framework stores).
    """
    a_new = _out(mu * _f(a, exact) + _f(g, exact), exact)
    w_new = _out(_f(w, exact) - lr * _f(a_new, exact), exact)
    return w_new, a_new


def adam(w, m, v, g, step, lr, b1, b2, eps, exact=False):
    """TF AdamOptimizer (reading Q8), t = step + 1:

    m <- b1 m + (1-b1) g;  v <- b2 v + (1-b2) g^2;
    lr_t = lr sqrt(1 - b2^t) / (1 - b1^t);  w <- w - lr_t m / (sqrt(v) + eps).
    """
    t = float(int(np.asarray(step).reshape(-1)[0]) + 1)
    g64 = _f(g, exact)
    m_new = _out(b1 * _f(m, exact) + (1.0 - b1) * g64, exact)
    v_new = _out(b2 * _f(v, exact) + (1.0 - b2) * g64 * g64, exact)
    lr_t = lr * np.sqrt(1.0 - b2 ** t) / (1.0 - b1 ** t)
    w_new = _out(_f(w, exact) - lr_t * _f(m_new, exact) / (np.sqrt(_f(v_new, exact)) + eps),
                 exact)
    return w_new, m_new, v_new


def feed(pool, step, rows):
    """x = pool[(step mod P) * rows : +rows], P = pool.rows / rows (data cursor, Q3/Q11)."""
    P = pool.shape[0] // rows
    s = int(np.asarray(step).reshape(-1)[0]) % P
    return np.array(pool[s * rows:(s + 1) * rows], copy=True)


def step_inc(step):
    return (np.asarray(step, dtype=np.int64) + 1).astype(np.int32)


def apply_op(op, T, shapes, exact=False):
    """Execute one graph op in place on the tensor dict ``T`` (id -> ndarray)."""
    t, ins, outs = op.type, op.ins, op.outs
    if t == GEMM:
        T[outs[0]] = gemm(T[ins[0]], T[ins[1]], T.get(outs[0]), op.flags, exact)
    elif t == BIAS_ACT and op.flags & GELU:
        h, u = bias_gelu(T[ins[0]], [T[i] for i in ins[1:]], exact)
        T[outs[0]] = h
        if len(outs) > 1:
            T[outs[1]] = u
    elif t == BIAS_ACT:
        T[outs[0]] = bias_act(T[ins[0]], [T[i] for i in ins[1:]], bool(op.flags & RELU), exact)
    elif t == BIAS_ACT_BWD and op.flags & GELU:
        T[outs[0]], T[outs[1]] = gelu_bwd(T[ins[0]], T[ins[1]], exact)
    elif t == BIAS_ACT_BWD:
        T[outs[0]], T[outs[1]] = bias_act_bwd(T[ins[0]], T[ins[1]], exact)
    elif t == COLSUM:
        T[outs[0]] = colsum(T[ins[0]], exact)
    elif t == SOFTMAX_CE:
        T[outs[0]], T[outs[1]] = softmax_ce(T[ins[0]], T[ins[1]], exact)
    elif t == SOFTMAX:
        T[outs[0]] = softmax(T[ins[0]], exact)
    elif t == SGD_MOM:
        T[outs[0]], T[outs[1]] = sgd_momentum(T[outs[0]], T[outs[1]], T[ins[0]],
                                              op.f[0], op.f[1], exact)
    elif t == ADAM:
        T[outs[0]], T[outs[1]], T[outs[2]] = adam(T[outs[0]], T[outs[1]], T[outs[2]],
                                                  T[ins[0]], T[ins[1]], *op.f[:4], exact=exact)
    elif t == FEED:
        T[outs[0]] = feed(T[ins[0]], T[ins[1]], shapes[outs[0]][0])
    elif t == STEP_INC:
        T[outs[0]] = step_inc(T[outs[0]])
    else:
        raise ValueError(f"unsupported op type {t}")
