"""GPU parity of every hot-path kernel against the oracle, through the C ABI (sf_op_*).

Bars (BASELINE.json north_star):
  - byte work (pack / unpack / peer-store walk, fill): bit-exact;
  - fp32 ops: per-tensor max|gpu - ref| / max(max|ref|, 1e-30) <= 1e-4 (reading Q12);
  - determinism: two launches give identical bits.
Shapes span several tiles with ragged tails (M, N, K not multiples of 128 / 64 / 32),
degenerate sizes (K < 8, N = 1 .. 10, M = 1) and the C1 / C2 / C3 layer shapes.
"""
import numpy as np
import pytest
import torch

from oracle import ops as O
from sf_inputs.ir import ACC, TA, TB

pytestmark = pytest.mark.gpu

TOL = 1e-4


def rel(a, b):
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    return float(np.abs(a - b).max() / max(np.abs(b).max(), 1e-30))


@pytest.fixture(scope="module")
def ops():
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_middleware_wur0hdh21_b200 import ops as K
    return K


def cu(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


# ---- multi-tensor copy (pack / unpack / peer store) -------------------------------------
def test_mtcopy_adversarial_sizes_bit_exact(ops):
    rng = np.random.default_rng(7)
    sizes = [4, 8, 12, 16, 20, 40, 256, 4096, 4100, 65536 + 12, 9 * 2 ** 20, 3 * 2 ** 20 + 4]
    sizes += [int(4 * rng.integers(1, 5000)) for _ in range(200)]
    src_host = rng.integers(0, 256, size=sum(-(-s // 256) * 256 for s in sizes), dtype=np.uint8)
    src = cu(src_host)
    dst = torch.full((len(src_host) + 4096,), 0xAB, dtype=torch.uint8, device="cuda")
    descs, expect = [], np.full(len(src_host) + 4096, 0xAB, np.uint8)
    so = do = 0
    for s in sizes:
        span = -(-s // 256) * 256
        descs.append((src.data_ptr() + so, dst.data_ptr() + do, s, span))
        expect[do:do + s] = src_host[so:so + s]
        expect[do + s:do + span] = 0
        so += -(-s // 256) * 256
        do += span
    ops.mtcopy(descs)
    torch.cuda.synchronize()
    assert np.array_equal(dst.cpu().numpy(), expect)


def test_mtcopy_windowed_walk_above_3gb_bit_exact(ops):
    """Live sets above 3 GB are walked in 2 GB windows (one launch each):
    3 descriptors straddling the window boundaries, ragged tails and zero padding, bit-exact."""
    sizes = [1_300_000_004, 1_400_000_000, 1_000_012]
    spans = [-(-s // 256) * 256 for s in sizes]
    total = sum(spans)
    g = torch.Generator(device="cuda").manual_seed(3)
    src = torch.randint(0, 256, (total,), dtype=torch.uint8, device="cuda", generator=g)
    dst = torch.full((total,), 0xAB, dtype=torch.uint8, device="cuda")
    descs, o = [], 0
    for s_, sp in zip(sizes, spans):
        descs.append((src.data_ptr() + o, dst.data_ptr() + o, s_, sp))
        o += sp
    ops.mtcopy(descs)
    torch.cuda.synchronize()
    o = 0
    for s_, sp in zip(sizes, spans):
        assert torch.equal(dst[o:o + s_], src[o:o + s_])
        assert not bool(dst[o + s_:o + sp].any())  # zero padding
        o += sp
    del src, dst
    torch.cuda.empty_cache()


def test_mtcopy_patch_iter(ops):
    src = cu(np.arange(64, dtype=np.uint8))
    dst = torch.zeros(64, dtype=torch.uint8, device="cuda")
    ops.mtcopy([(src.data_ptr(), dst.data_ptr(), 64, 64)], patch_iter=0x0102030405060708)
    out = dst.cpu().numpy()
    assert out[16:24].tobytes() == (0x0102030405060708).to_bytes(8, "little")
    assert np.array_equal(out[:16], np.arange(16)) and np.array_equal(out[24:], np.arange(24, 64))


def test_fill(ops):
    t = torch.zeros(1000 * 16 + 7, dtype=torch.uint8, device="cuda")
    ops.fill(t, 0xFF)
    assert bool((t == 0xFF).all())


# ---- GEMM (tcgen05 3xTF32) ---------------------------------------------------------------
GEMM_SHAPES = [
    (64, 256, 784, 0), (64, 10, 256, 0), (256, 10, 64, TA), (64, 256, 10, TB), (784, 256, 64, TA),
    (1, 4096, 2048, 0), (3, 17, 5, 0), (129, 65, 33, 0), (300, 200, 100, TA | TB),
    (128, 128, 32, ACC), (1000, 64, 576, 0), (576, 64, 3000, TA), (512, 1024, 1024, 0),
    (512, 300, 1024, TB), (7, 1000, 2048, 0), (1, 10, 256, ACC), (130, 8, 4, TA),
    # GEMV paths (M <= 8): cluster kernel incl. empty K ranks, K tails, ACC; K/8 > 512 falls back
    (8, 4096, 4096, 0), (4, 12, 13, 0), (1, 4, 1, 0), (5, 1024, 999, ACC), (2, 1000, 4100, 0),
    (3, 516, 64, 0), (1, 2048, 20000, 0),
    # row-contiguous GEMV (M <= 8, TB): ragged rows per CTA, N < #SMs, K*4 = 32 KB, K % 4 != 0 and
    # M*K*4 > 64 KB fall back to the tiled path
    (1, 4096, 2048, TB), (8, 1000, 2048, TB), (3, 17, 8, TB), (1, 1, 4096, TB), (2, 300, 8192, TB),
    (4, 100, 13, TB), (5, 30, 8192, TB), (1, 1000, 4096, TB | ACC),
]


@pytest.mark.parametrize("M,N,K,flags", GEMM_SHAPES)
def test_gemm_vs_oracle(ops, M, N, K, flags):
    rng = np.random.default_rng(M * 7 + N * 3 + K + flags)
    A = rng.standard_normal((K, M) if flags & TA else (M, K)).astype(np.float32)
    B = rng.standard_normal((N, K) if flags & TB else (K, N)).astype(np.float32)
    C0 = rng.standard_normal((M, N)).astype(np.float32)
    ref = O.gemm(A, B, C0, flags)
    Ct = cu(C0)
    ops.gemm(cu(A), cu(B), Ct, flags)
    got = Ct.cpu().numpy()
    assert rel(got, ref) <= TOL, rel(got, ref)
    # deterministic
    Ct2 = cu(C0)
    ops.gemm(cu(A), cu(B), Ct2, flags)
    assert torch.equal(Ct, Ct2)


# Shapes that take the default 128x256-tile path (use_bn256: N >= 256, no split-K at BN=256,
# >= 100 tiles) in all four operand majorness instantiations gemm_tma_kernel<256, A_MN, B_MN>:
# the C3 FFN / head weight gradients (TA: both operands MN-major), forward NN, the NT head,
# TA|TB; ragged M / N / K tails; accumulate.  Each case asserts the path it took.
GEMM_BN256 = [
    (1024, 4096, 512, TA, True, True),        # C3 FFN dW (intermediate)
    (4096, 1024, 512, TA, True, True),        # C3 FFN dW (output)
    (30520, 1024, 512, TA, True, True),       # C3 head dW (word embedding, pitch-padded vocab)
    (512, 30520, 1024, TB, False, False),     # C3 NT head: logits = h . word^T
    (4096, 1024, 1024, 0, False, True),       # forward NN
    (1024, 4096, 256, TA | TB, True, False),
    (1100, 3000, 300, TA, True, True),        # ragged M, N, K
    (1100, 3000, 300, 0, False, True),
    (1024, 4096, 512, TA | ACC, True, True),  # accumulate
    (1100, 3000, 300, TB | ACC, False, False),
]


@pytest.mark.parametrize("M,N,K,flags,a_mn,b_mn", GEMM_BN256)
def test_gemm_bn256_tile_path_vs_oracle(ops, M, N, K, flags, a_mn, b_mn):
    rng = np.random.default_rng(M + 5 * N + 11 * K + flags)
    A = rng.standard_normal((K, M) if flags & TA else (M, K)).astype(np.float32)
    B = rng.standard_normal((N, K) if flags & TB else (K, N)).astype(np.float32)
    C0 = rng.standard_normal((M, N)).astype(np.float32)
    ref = O.gemm(A, B, C0, flags)
    Ct = cu(C0)
    ops.gemm(cu(A), cu(B), Ct, flags)
    path = ops.last_gemm_path()
    assert path == {"kind": "tma", "bn": 256, "splits": 1, "a_mn": a_mn, "b_mn": b_mn}, path
    got = Ct.cpu().numpy()
    assert rel(got, ref) <= TOL, rel(got, ref)
    Ct2 = cu(C0)
    ops.gemm(cu(A), cu(B), Ct2, flags)
    assert torch.equal(Ct, Ct2)


def test_gemm_paths_of_existing_shapes(ops):
    """The tile widths / split-K factors the planner picks for the C1 / C2 / C3 shapes of
    GEMM_SHAPES (documents which instantiation each oracle case exercises)."""
    seen = set()
    for (M, N, K, flags) in GEMM_SHAPES:
        A = torch.zeros((K, M) if flags & TA else (M, K), device="cuda")
        B = torch.zeros((N, K) if flags & TB else (K, N), device="cuda")
        C = torch.zeros((M, N), device="cuda")
        ops.gemm(A, B, C, flags)
        p = ops.last_gemm_path()
        seen.add((p["kind"], p["bn"], p["a_mn"], p["b_mn"], p["splits"] > 1))
    kinds = {s[0] for s in seen}
    assert {"tma", "gemv_tma", "gemv_rows"} <= kinds, seen
    # 128- and 64-wide tiles, with and without split-K
    assert any(s[0] == "tma" and s[1] == 128 for s in seen) and any(s[0] == "tma" and s[1] == 64 for s in seen)
    assert any(s[0] == "tma" and s[4] for s in seen) and any(s[0] == "tma" and not s[4] for s in seen)


GEMM_EPI_SHAPES = [(1, 4096, 2048, 1, True), (1, 1000, 4096, 1, False), (8, 256, 784, 2, True),
                   (5, 516, 333, 3, True), (64, 256, 784, 1, True), (130, 96, 40, 2, False)]


@pytest.mark.parametrize("M,N,K,nb,relu", GEMM_EPI_SHAPES)
def test_gemm_bias_act_vs_oracle(ops, M, N, K, nb, relu):
    """Forward layer with its epilogue: fused into the GEMV reduction for M <= 8, a second
    elementwise kernel otherwise; both equal the oracle's gemm -> bias_act."""
    rng = np.random.default_rng(M + N + K + nb)
    A = rng.standard_normal((M, K)).astype(np.float32)
    B = rng.standard_normal((K, N)).astype(np.float32)
    bs = [rng.standard_normal((1, N)).astype(np.float32) for _ in range(nb)]
    z = O.gemm(A, B, None, 0)
    ref = O.bias_act(z, bs, relu)
    C = torch.full((M, N), 7.0, device="cuda")
    ops.gemm_bias_act(cu(A), cu(B), C, [cu(b) for b in bs], relu)
    assert rel(C.cpu().numpy(), ref) <= TOL
    C2 = torch.full((M, N), 7.0, device="cuda")
    ops.gemm_bias_act(cu(A), cu(B), C2, [cu(b) for b in bs], relu)
    assert torch.equal(C, C2)


GEMV_ROWS_EPI = [(1, 4096, 2048, 1, True), (1, 1000, 4096, 1, False), (8, 260, 784, 3, True),
                 (2, 7, 1024, 2, True)]


@pytest.mark.parametrize("M,N,K,nb,relu", GEMV_ROWS_EPI)
def test_gemv_rows_bias_act_vs_oracle(ops, M, N, K, nb, relu):
    """Row-contiguous GEMV (weights [N][K], TB) with the fused bias / ReLU epilogue."""
    rng = np.random.default_rng(M + 3 * N + K + nb)
    A = rng.standard_normal((M, K)).astype(np.float32)
    Bt = rng.standard_normal((N, K)).astype(np.float32)
    bs = [rng.standard_normal((1, N)).astype(np.float32) for _ in range(nb)]
    ref = O.bias_act(O.gemm(A, Bt, None, TB), bs, relu)
    C = torch.full((M, N), 7.0, device="cuda")
    ops.gemm_bias_act(cu(A), cu(Bt), C, [cu(b) for b in bs], relu, TB)
    assert rel(C.cpu().numpy(), ref) <= TOL
    C2 = torch.full((M, N), 7.0, device="cuda")
    ops.gemm_bias_act(cu(A), cu(Bt), C2, [cu(b) for b in bs], relu, TB)
    assert torch.equal(C, C2)


_GEMV_CHILD = r"""
import sys, numpy as np, torch
sys.path.insert(0, '.')
from paper_conf_middleware_wur0hdh21_b200 import ops as K
out = {}
for (M, N, Kd, acc) in [(1, 4096, 2048, 0), (8, 1000, 4096, 1), (3, 12, 13, 0), (2, 516, 999, 1)]:
    rng = np.random.default_rng(M * 100 + N + Kd)
    A = rng.standard_normal((M, Kd)).astype(np.float32)
    B = rng.standard_normal((Kd, N)).astype(np.float32)
    C0 = rng.standard_normal((M, N)).astype(np.float32)
    b = rng.standard_normal((1, N)).astype(np.float32)
    C = torch.from_numpy(C0).cuda()
    K.gemm_bias_act(torch.from_numpy(A).cuda(), torch.from_numpy(B).cuda(), C,
                    [torch.from_numpy(b).cuda()], True, 4 if acc else 0)
    out[f"{M}_{N}_{Kd}"] = C.cpu().numpy()
np.savez(sys.argv[1], **out)
"""


@pytest.mark.parametrize("path", ["tma", "cluster", "split"])
def test_gemv_paths_agree_with_oracle(path, tmp_path):
    """Every M <= 8 path (SF_GEMV=tma|cluster|split, read once per process) meets the bar."""
    import os, subprocess, sys
    f = tmp_path / "out.npz"
    env = dict(os.environ, SF_GEMV=path)
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    subprocess.run([sys.executable, "-c", _GEMV_CHILD, str(f)], cwd=root, env=env, check=True,
                   timeout=120)
    got = np.load(f)
    for key in got.files:
        M, N, Kd = map(int, key.split("_"))
        rng = np.random.default_rng(M * 100 + N + Kd)
        A = rng.standard_normal((M, Kd)).astype(np.float32)
        B = rng.standard_normal((Kd, N)).astype(np.float32)
        C0 = rng.standard_normal((M, N)).astype(np.float32)
        b = rng.standard_normal((1, N)).astype(np.float32)
        acc = key in ("8_1000_4096", "2_516_999")
        ref = O.bias_act(O.gemm(A, B, C0 if acc else None, ACC if acc else 0), [b], True)
        assert rel(got[key], ref) <= TOL, (path, key)


CHAIN_CASES = [
    ((2048, 4096, 4096, 1000), 1, True, True),   # C4 preempter model
    ((784, 256, 12), 1, True, True),              # C1-like head (N % 4 == 0 for TMA)
    ((100, 36, 516, 12), 2, True, False),         # ragged K / N, no softmax
    ((256, 1024, 64, 1000), 8, False, True),      # M = 8, no biases
    ((129, 260, 132, 8), 3, True, True),          # K tails inside a 128-row unit
    ((2048, 4096, 1000), 8, True, True),          # M = 8 at full width
    ((64, 64, 64, 64, 64, 64, 16), 5, True, True),  # 6 layers
]


@pytest.mark.parametrize("widths,M,biases,softmax", CHAIN_CASES)
def test_mlp_chain_vs_oracle(ops, widths, M, biases, softmax):
    """The fused chain equals the oracle's layer-by-layer gemm -> bias_act -> ... -> softmax;
    every intermediate h is materialised and checked; two launches are bit-identical."""
    rng = np.random.default_rng(sum(widths) + M)
    n = len(widths) - 1
    x = rng.standard_normal((M, widths[0])).astype(np.float32)
    Ws = [(rng.standard_normal((widths[i], widths[i + 1])) / np.sqrt(widths[i])).astype(np.float32)
          for i in range(n)]
    bs = [rng.standard_normal((1, widths[i + 1])).astype(np.float32) if biases else None for i in range(n)]
    relu = [i < n - 1 for i in range(n)]
    refs, h = [], x
    for i in range(n):
        z = O.gemm(h, Ws[i], None, 0)
        h = O.bias_act(z, [bs[i]] if biases else [], relu[i]) if (biases or relu[i]) else z
        refs.append(h)
    outs = []
    for _ in range(2):
        hs = [torch.full((M, widths[i + 1]), float("nan"), device="cuda") for i in range(n)]
        probs = torch.full((M, widths[-1]), float("nan"), device="cuda") if softmax else None
        ops.mlp_chain(cu(x), [cu(W) for W in Ws], [cu(b) if b is not None else None for b in bs],
                      relu, hs, probs)
        torch.cuda.synchronize()
        outs.append((hs, probs))
    hs, probs = outs[0]
    for i in range(n):
        assert rel(hs[i].cpu().numpy(), refs[i]) <= TOL, (i, rel(hs[i].cpu().numpy(), refs[i]))
        assert torch.equal(hs[i], outs[1][0][i])
    if softmax:
        assert rel(probs.cpu().numpy(), O.softmax(refs[-1])) <= TOL
        assert torch.equal(probs, outs[1][1])


def test_mlp_chain_rejects_unsupported_shapes(ops):
    """N % 4 != 0 on a row-split layer (layers >= 1 stream whole float4 rows) and more than 6
    layers are refused, not silently wrong."""
    from paper_conf_middleware_wur0hdh21_b200._abi import SFError
    x = torch.zeros(1, 64, device="cuda")
    with pytest.raises(SFError):
        ops.mlp_chain(x, [torch.zeros(64, 8, device="cuda"), torch.zeros(8, 10, device="cuda")],
                      [None, None], [True, False],
                      [torch.zeros(1, 8, device="cuda"), torch.zeros(1, 10, device="cuda")])
    Ws = [torch.zeros(64, 64, device="cuda") for _ in range(7)]
    with pytest.raises(SFError):
        ops.mlp_chain(x, Ws, [None] * 7, [True] * 7, [torch.zeros(1, 64, device="cuda") for _ in range(7)])


def test_gemm_plain_tf32_would_fail_the_bar(ops):
    """Control: single-pass TF32 (torch allow_tf32) misses 1e-4 where 3xTF32 passes."""
    rng = np.random.default_rng(1)
    A = rng.standard_normal((256, 1024)).astype(np.float32)
    B = rng.standard_normal((1024, 256)).astype(np.float32)
    ref = O.gemm(A, B, None, 0)
    C = torch.zeros(256, 256, device="cuda")
    ops.gemm(cu(A), cu(B), C, 0)
    ours = rel(C.cpu().numpy(), ref)
    tf32 = torch.backends.cuda.matmul.allow_tf32
    torch.backends.cuda.matmul.allow_tf32 = True
    try:
        plain = rel((cu(A) @ cu(B)).cpu().numpy(), ref)
    finally:
        torch.backends.cuda.matmul.allow_tf32 = tf32
    assert ours <= TOL
    assert ours < plain / 10  # plain tf32 is ~1e-3


# ---- elementwise / reductions -------------------------------------------------------------
@pytest.mark.parametrize("rows,cols,nb", [(64, 256, 1), (512, 4096, 2), (5, 7, 3), (1001, 64, 1)])
def test_bias_gelu_and_backward(ops, rows, cols, nb):
    """GELU: erff/expf kernels vs the fp64 oracle at 1e-4."""
    rng = np.random.default_rng(rows + 3 * cols)
    z = (rng.standard_normal((rows, cols)) * 2).astype(np.float32)
    bs = [rng.standard_normal((1, cols)).astype(np.float32) for _ in range(nb)]
    h = torch.empty(rows, cols, device="cuda")
    ops.bias_act(cu(z), [cu(b) for b in bs], h, 2)
    rh, ru = O.bias_gelu(z, bs)
    assert rel(h.cpu().numpy(), rh) <= TOL
    dh = rng.standard_normal((rows, cols)).astype(np.float32)
    dz = torch.empty(rows, cols, device="cuda")
    db = torch.empty(1, cols, device="cuda")
    ops.gelu_bwd(cu(dh), cu(ru), dz, db)
    rdz, rdb = O.gelu_bwd(dh, ru)
    assert rel(dz.cpu().numpy(), rdz) <= TOL
    assert rel(db.cpu().numpy(), rdb) <= TOL


@pytest.mark.parametrize("rows,cols,nb,relu", [(64, 256, 1, True), (64, 10, 1, False),
                                                (1001, 64, 3, False), (5, 7, 2, True)])
def test_bias_act(ops, rows, cols, nb, relu):
    rng = np.random.default_rng(rows + cols)
    z = rng.standard_normal((rows, cols)).astype(np.float32)
    bs = [rng.standard_normal((1, cols)).astype(np.float32) for _ in range(nb)]
    h = torch.empty(rows, cols, device="cuda")
    ops.bias_act(cu(z), [cu(b) for b in bs], h, relu)
    assert rel(h.cpu().numpy(), O.bias_act(z, bs, relu)) <= TOL


@pytest.mark.parametrize("rows,cols", [(64, 256), (25088, 64), (3, 1000), (513, 33), (1, 5),
                                       (100352, 64), (17, 4), (4097, 2048), (7, 12)])
def test_bias_act_bwd_and_colsum(ops, rows, cols):
    rng = np.random.default_rng(rows * cols)
    dh = rng.standard_normal((rows, cols)).astype(np.float32)
    h = np.maximum(rng.standard_normal((rows, cols)), 0).astype(np.float32)
    dz = torch.empty(rows, cols, device="cuda")
    db = torch.empty(1, cols, device="cuda")
    ops.bias_act_bwd(cu(dh), cu(h), dz, db)
    rdz, rdb = O.bias_act_bwd(dh, h)
    assert np.array_equal(dz.cpu().numpy(), rdz)  # masking is exact
    assert rel(db.cpu().numpy(), rdb) <= TOL
    s = torch.empty(1, cols, device="cuda")
    ops.colsum(cu(dh), s)
    assert rel(s.cpu().numpy(), O.colsum(dh)) <= TOL
    s2 = torch.empty(1, cols, device="cuda")
    ops.colsum(cu(dh), s2)
    assert torch.equal(s, s2)


@pytest.mark.parametrize("rows,cols", [(64, 10), (1, 1000), (3136, 256), (512, 30522), (7, 3),
                                       (20000, 64), (33, 16), (5, 128), (9, 4), (100, 8)])
def test_softmax_ce_and_softmax(ops, rows, cols):
    rng = np.random.default_rng(rows + cols)
    l = (rng.standard_normal((rows, cols)) * 3).astype(np.float32)
    y = rng.integers(0, cols, size=(rows, 1)).astype(np.int32)
    loss = torch.empty(1, 1, device="cuda")
    d = torch.empty(rows, cols, device="cuda")
    ops.softmax_ce(cu(l), cu(y), loss, d)
    rloss, rd = O.softmax_ce(l, y)
    assert rel(loss.cpu().numpy(), rloss) <= TOL
    assert rel(d.cpu().numpy(), rd) <= TOL
    p = torch.empty(rows, cols, device="cuda")
    ops.softmax(cu(l), p)
    assert rel(p.cpu().numpy(), O.softmax(l)) <= TOL


def test_softmax_ce_zero_logits_ln_c(ops):
    loss = torch.empty(1, 1, device="cuda")
    d = torch.empty(64, 10, device="cuda")
    ops.softmax_ce(torch.zeros(64, 10, device="cuda"), torch.zeros(64, 1, dtype=torch.int32, device="cuda"),
                   loss, d)
    assert abs(loss.item() - np.log(10.0)) <= 1e-6


@pytest.mark.parametrize("n", [1, 3, 4, 1000, 200704 + 3])
def test_sgd_momentum(ops, n):
    rng = np.random.default_rng(n)
    w, a, g = (rng.standard_normal((1, n)).astype(np.float32) for _ in range(3))
    rw, ra = O.sgd_momentum(w, a, g, 0.01, 0.9)
    tw, ta = cu(w), cu(a)
    ops.sgd_mom(tw, ta, cu(g), 0.01, 0.9)
    assert rel(ta.cpu().numpy(), ra) <= TOL and rel(tw.cpu().numpy(), rw) <= TOL


@pytest.mark.parametrize("n,step", [(5, 0), (1024, 9), (4096 * 3 + 1, 1000)])
def test_adam(ops, n, step):
    rng = np.random.default_rng(n)
    w, g = (rng.standard_normal((1, n)).astype(np.float32) for _ in range(2))
    m = (rng.standard_normal((1, n)) * 0.1).astype(np.float32)
    v = (rng.random((1, n)) * 0.1).astype(np.float32)
    st = np.array([[step]], np.int32)
    rw, rm, rv = O.adam(w, m, v, g, st, 1e-3, 0.9, 0.999, 1e-8)
    tw, tm, tv = cu(w), cu(m), cu(v)
    ops.adam(tw, tm, tv, cu(g), cu(st), 1e-3, 0.9, 0.999, 1e-8)
    assert rel(tm.cpu().numpy(), rm) <= TOL and rel(tv.cpu().numpy(), rv) <= TOL
    assert rel(tw.cpu().numpy(), rw) <= TOL  # per-tensor bar (reading Q12)
    # the update itself, up to fp32 rounding of w (|dw| ~ lr, ulp(w) ~ 1e-7)
    assert rel(tw.cpu().numpy() - w, rw - w) <= 1e-3


def test_adam_zero_grad_bitwise_noop(ops):
    w = cu(np.random.default_rng(0).standard_normal((1, 999)).astype(np.float32))
    w0 = w.clone()
    z = torch.zeros_like(w)
    ops.adam(w, z.clone(), z.clone(), z, torch.tensor([[5]], dtype=torch.int32, device="cuda"),
             1e-4, 0.9, 0.999, 1e-8)
    assert torch.equal(w, w0)
