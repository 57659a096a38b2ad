"""Direct kernel entry points (sf_op_*) on torch CUDA tensors — marshalling only."""
from __future__ import annotations

import ctypes as C
from typing import Optional, Sequence, Tuple

import torch

from . import _abi as A
from ._abi import check, lib

TA, TB, ACC = 1, 2, 4


def _p(t: Optional[torch.Tensor]):
    return C.c_void_p(t.data_ptr()) if t is not None else None


def _s(stream: Optional[torch.cuda.Stream]):
    s = stream if stream is not None else torch.cuda.current_stream()
    return C.c_void_p(s.cuda_stream)


def _need_cuda(*ts):
    for t in ts:
        if t is not None and (not t.is_cuda or not t.is_contiguous()):
            raise ValueError("sf ops take contiguous CUDA tensors")


def gemm(A_: torch.Tensor, B: torch.Tensor, C_: torch.Tensor, flags: int = 0, stream=None) -> None:
    """C = op(A) op(B) (+C if ACC), fp32 via tcgen05 3xTF32 (batch<=8: GEMV)."""
    _need_cuda(A_, B, C_)
    M, N = C_.shape
    K = A_.shape[0] if flags & TA else A_.shape[1]
    check(lib().sf_op_gemm(_p(A_), _p(B), _p(C_), M, N, K, A_.shape[1], B.shape[1], C_.shape[1],
                           flags, _s(stream)), "sf_op_gemm")


GEMM_PATH_KINDS = {1: "tma", 2: "ldg", 3: "gemv_tma", 4: "gemv_rows", 5: "gemv_cluster",
                   6: "gemv_split", 7: "gemv", 8: "gemv_blocked"}


def last_gemm_path() -> dict:
    """Kernel path of the last GEMM this thread launched (sf_last_gemm_path, diagnostics)."""
    p = A.sf_gemm_path()
    check(lib().sf_last_gemm_path(C.byref(p)), "sf_last_gemm_path")
    return {"kind": GEMM_PATH_KINDS.get(p.kind, "none"), "bn": p.bn, "splits": p.splits,
            "a_mn": bool(p.a_mn), "b_mn": bool(p.b_mn)}


def gemm_bias_act(A_: torch.Tensor, B: torch.Tensor, C_: torch.Tensor, biases: Sequence[torch.Tensor],
                  relu: bool, flags: int = 0, stream=None) -> None:
    """C = act(op(A) op(B) (+C if ACC) + sum(biases)) — forward layer with fused epilogue."""
    bs = list(biases) + [None] * (3 - len(biases))
    _need_cuda(A_, B, C_, *bs)
    M, N = C_.shape
    K = A_.shape[0] if flags & TA else A_.shape[1]
    check(lib().sf_op_gemm_bias_act(_p(A_), _p(B), _p(C_), M, N, K, A_.shape[1], B.shape[1],
                                    C_.shape[1], flags, _p(bs[0]), _p(bs[1]), _p(bs[2]), int(relu),
                                    _s(stream)), "sf_op_gemm_bias_act")


def mlp_chain(x: torch.Tensor, Ws: Sequence[torch.Tensor], bs: Sequence[Optional[torch.Tensor]],
              relu: Sequence[bool], hs: Sequence[torch.Tensor], probs: Optional[torch.Tensor] = None,
              stream=None) -> None:
    """Fused batch-M MLP forward (+ softmax) in one persistent kernel (sf_op_mlp_chain)."""
    n = len(Ws)
    _need_cuda(x, *Ws, *[b for b in bs if b is not None], *hs, probs)
    widths = (C.c_int32 * (n + 1))(*([x.shape[1]] + [W.shape[1] for W in Ws]))
    Wp = (C.c_void_p * n)(*[W.data_ptr() for W in Ws])
    bp = (C.c_void_p * n)(*[(b.data_ptr() if b is not None else None) for b in bs])
    rl = (C.c_int32 * n)(*[int(r) for r in relu])
    hp = (C.c_void_p * n)(*[h.data_ptr() for h in hs])
    check(lib().sf_op_mlp_chain(_p(x), x.shape[0], n, widths, Wp, bp, rl, hp, _p(probs), _s(stream)),
          "sf_op_mlp_chain")


def bias_act(z, biases: Sequence[torch.Tensor], h, relu, stream=None) -> None:
    """relu: False / True, or the act code (0 identity, 1 ReLU, 2 GELU)."""
    bs = list(biases) + [None] * (3 - len(biases))
    _need_cuda(z, h, *bs)
    check(lib().sf_op_bias_act(_p(z), _p(bs[0]), _p(bs[1]), _p(bs[2]), _p(h), z.shape[0], z.shape[1],
                               int(relu), _s(stream)), "sf_op_bias_act")


def gelu_bwd(dh, u, dz, db, stream=None) -> None:
    _need_cuda(dh, u, dz, db)
    check(lib().sf_op_gelu_bwd(_p(dh), _p(u), _p(dz), _p(db), dh.shape[0], dh.shape[1],
                               _s(stream)), "sf_op_gelu_bwd")


def bias_act_bwd(dh, h, dz, db, stream=None) -> None:
    _need_cuda(dh, h, dz, db)
    check(lib().sf_op_bias_act_bwd(_p(dh), _p(h), _p(dz), _p(db), dh.shape[0], dh.shape[1],
                                   _s(stream)), "sf_op_bias_act_bwd")


def colsum(x, s, stream=None) -> None:
    _need_cuda(x, s)
    check(lib().sf_op_colsum(_p(x), _p(s), x.shape[0], x.shape[1], _s(stream)), "sf_op_colsum")


def softmax_ce(logits, labels, loss, dlogits, stream=None) -> None:
    _need_cuda(logits, labels, loss, dlogits)
    check(lib().sf_op_softmax_ce(_p(logits), _p(labels), _p(loss), _p(dlogits), logits.shape[0],
                                 logits.shape[1], _s(stream)), "sf_op_softmax_ce")


def softmax(logits, probs, stream=None) -> None:
    _need_cuda(logits, probs)
    check(lib().sf_op_softmax(_p(logits), _p(probs), logits.shape[0], logits.shape[1], _s(stream)),
          "sf_op_softmax")


def sgd_mom(w, a, g, lr: float, mu: float, stream=None) -> None:
    _need_cuda(w, a, g)
    check(lib().sf_op_sgd_mom(_p(w), _p(a), _p(g), w.numel(), lr, mu, _s(stream)), "sf_op_sgd_mom")


def adam(w, m, v, g, step, lr, b1, b2, eps, stream=None) -> None:
    _need_cuda(w, m, v, g, step)
    check(lib().sf_op_adam(_p(w), _p(m), _p(v), _p(g), _p(step), w.numel(), lr, b1, b2, eps,
                           _s(stream)), "sf_op_adam")


def mtcopy(descs: Sequence[Tuple[int, int, int, int]], patch_iter: int = -1, stream=None) -> None:
    """descs: (src_ptr, dst_ptr, nbytes, span) — the pack / unpack / peer-store walk."""
    arr = (A.sf_copy_desc * max(1, len(descs)))()
    for i, (s, d, nb, sp) in enumerate(descs):
        arr[i].src, arr[i].dst, arr[i].nbytes, arr[i].span = s, d, nb, sp
    check(lib().sf_op_mtcopy(arr, len(descs), patch_iter, _s(stream)), "sf_op_mtcopy")


def fill(t: torch.Tensor, value: int, stream=None) -> None:
    check(lib().sf_op_fill(_p(t), t.numel() * t.element_size(), value, _s(stream)), "sf_op_fill")
