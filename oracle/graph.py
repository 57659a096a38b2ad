"""Oracle graph analysis: validation, partition into subgraphs, live sets (test infra).

* Partition — PAPER.md:323-325 (section 2.1: "Session also optimizes graph execution
  by partitioning the full graph into subgraphs, which can be independently executed
  by executors") and PAPER.md:635-637 (section 3.2: one executor per device for every
  subgraph).  Granularity within a device is not specified by the paper; reading Q2:
  PER_LAYER_PHASE = maximal runs of ops with equal phase id; MAX_OPS = n splits each
  run into chunks of at most n ops, except that a run containing optimizer ops
  (SGD_MOM / ADAM / STEP_INC) is kept whole unless ``update_chunks`` > 1, which splits it
  into byte-balanced chunks (``_split_update``); resuming inside it continues with the
  remaining updates, so nothing is applied twice or lost.
* Live set — PAPER.md:734-744 (section 3.3 "Context saving": persistent variables are
  tracked and saved; intermediate data is discarded at iteration end) extended by
  north_star to in-flight activations crossing the cut (reading Q1/Q3):
      L_k = persistent (PARAM, SLOT, SCALAR_STATE)
          U { t : some op at or after S_k reads t before any op at or after S_k
                  overwrites it, and t was written before S_k in this iteration }
          U { OUTPUT tensors written before S_k (fetched at iteration end) }.
  Externally fed INPUT/LABEL tensors (no writer op) count as written at the start of
  S_0.  DATASET tensors are replicated read-only and never live.  Order: tensor id.

Pins (tests/test_oracle_graph.py): SURVEY.md 8(c) step 3's C1 live table (plus the
data cursor, reading Q3) as a golden fixture; brute-force restore-from-poison at
every cut of every iteration on tiny graphs; minimality (dropping any non-persistent
member of L_k changes the result); Table 1 identity stateful bytes = 2 x params x 4 B.
"""
from __future__ import annotations

from typing import List, Tuple

from sf_inputs.ir import (ACC, ADAM, BIAS_ACT, BIAS_ACT_BWD, COLSUM, DATASET, F32, FEED,
                          GELU, GEMM, I32, RELU, INPUT, LABEL, OUTPUT, PERSISTENT_KINDS, SGD_MOM,
                          SOFTMAX, SOFTMAX_CE, STEP_INC, TA, TB, Graph)

OPTIMIZER_OPS = (SGD_MOM, ADAM, STEP_INC)


class GraphError(ValueError):
    pass


def op_reads(op) -> List[int]:
    r = list(op.ins)
    if op.type == GEMM and op.flags & ACC:
        r.append(op.outs[0])
    if op.type in (SGD_MOM, ADAM, STEP_INC):
        r.extend(op.outs)
    return r


def op_writes(op) -> List[int]:
    return list(op.outs)


def validate(g: Graph) -> None:
    """Shape/dtype/kind checks and read-before-write within one iteration."""
    T = g.tensors
    n = len(T)

    def chk(c, msg):
        if not c:
            raise GraphError(msg)

    for j, op in enumerate(g.ops):
        for t in op.ins + op.outs:
            chk(0 <= t < n, f"op {j}: tensor id {t} out of range")
        for t in op.outs:
            chk(T[t].kind != DATASET, f"op {j}: writes DATASET {T[t].name}")
            if T[t].kind in PERSISTENT_KINDS:
                chk(op.type in OPTIMIZER_OPS, f"op {j}: only optimizer ops write state")
        if op.type == GEMM:
            chk(len(op.ins) == 2 and len(op.outs) == 1, f"op {j}: gemm arity")
            A, B, C = T[op.ins[0]], T[op.ins[1]], T[op.outs[0]]
            M, K = (A.cols, A.rows) if op.flags & TA else (A.rows, A.cols)
            K2, N = (B.cols, B.rows) if op.flags & TB else (B.rows, B.cols)
            chk(K == K2 and C.rows == M and C.cols == N, f"op {j}: gemm shape mismatch")
            chk(A.dtype == B.dtype == C.dtype == F32, f"op {j}: gemm dtype")
        elif op.type == BIAS_ACT:
            n_out = (1, 2) if op.flags & GELU else (1,)
            chk(2 <= len(op.ins) <= 4 and len(op.outs) in n_out, f"op {j}: bias_act arity")
            chk(not (op.flags & RELU and op.flags & GELU), f"op {j}: one activation")
            z = T[op.ins[0]]
            for o in op.outs:
                chk((z.rows, z.cols) == (T[o].rows, T[o].cols), f"op {j}: bias_act shape")
            for b in op.ins[1:]:
                chk((T[b].rows, T[b].cols) == (1, z.cols), f"op {j}: bias shape")
        elif op.type == BIAS_ACT_BWD:
            dh, h, dz, db = (T[op.ins[0]], T[op.ins[1]], T[op.outs[0]], T[op.outs[1]])
            chk((dh.rows, dh.cols) == (h.rows, h.cols) == (dz.rows, dz.cols),
                f"op {j}: bias_act_bwd shape")
            chk((db.rows, db.cols) == (1, dh.cols), f"op {j}: db shape")
        elif op.type == COLSUM:
            x, s = T[op.ins[0]], T[op.outs[0]]
            chk((s.rows, s.cols) == (1, x.cols), f"op {j}: colsum shape")
        elif op.type == SOFTMAX_CE:
            l, y, loss, d = (T[op.ins[0]], T[op.ins[1]], T[op.outs[0]], T[op.outs[1]])
            chk(y.dtype == I32 and (y.rows, y.cols) == (l.rows, 1), f"op {j}: labels")
            chk((loss.rows, loss.cols) == (1, 1), f"op {j}: loss shape")
            chk((d.rows, d.cols) == (l.rows, l.cols), f"op {j}: dlogits shape")
        elif op.type == SOFTMAX:
            chk((T[op.ins[0]].rows, T[op.ins[0]].cols) == (T[op.outs[0]].rows, T[op.outs[0]].cols),
                f"op {j}: softmax shape")
        elif op.type == SGD_MOM:
            g_, w, a = T[op.ins[0]], T[op.outs[0]], T[op.outs[1]]
            chk((g_.rows, g_.cols) == (w.rows, w.cols) == (a.rows, a.cols), f"op {j}: sgd shape")
            chk(len(op.f) >= 2, f"op {j}: sgd params")
        elif op.type == ADAM:
            g_, st = T[op.ins[0]], T[op.ins[1]]
            w, m, v = (T[t] for t in op.outs)
            chk((g_.rows, g_.cols) == (w.rows, w.cols) == (m.rows, m.cols) == (v.rows, v.cols),
                f"op {j}: adam shape")
            chk(st.dtype == I32 and st.numel == 1, f"op {j}: adam step")
            chk(len(op.f) >= 4, f"op {j}: adam params")
        elif op.type == FEED:
            pool, st, x = T[op.ins[0]], T[op.ins[1]], T[op.outs[0]]
            chk(pool.kind == DATASET and pool.cols == x.cols and pool.rows % x.rows == 0
                and pool.dtype == x.dtype, f"op {j}: feed shape")
            chk(st.dtype == I32 and st.numel == 1, f"op {j}: feed step")
        elif op.type == STEP_INC:
            chk(len(op.outs) == 1 and T[op.outs[0]].dtype == I32, f"op {j}: step_inc")
        else:
            raise GraphError(f"op {j}: unsupported type {op.type}")
    # read-before-write within an iteration
    written = set()
    for j, op in enumerate(g.ops):
        for t in op_reads(op):
            k = T[t].kind
            if k in PERSISTENT_KINDS or k == DATASET or t in written:
                continue
            if k in (INPUT, LABEL) and not any(t in o.outs for o in g.ops):
                continue  # externally fed
            raise GraphError(f"op {j}: reads {T[t].name} before it is written")
        written.update(op_writes(op))


def _split_update(g: Graph, a: int, b: int, chunks: int) -> List[Tuple[int, int]]:
    """Split an optimizer run into byte-balanced chunks (reading Q2, update_chunks > 1).

    Op j gets weight w_j = nbytes of its updated variable (0 for STEP_INC); with
    C_j = sum of weights of the run's ops before j and W the run total, op j belongs to
    chunk min(U - 1, floor(U * C_j / W)); maximal equal-chunk runs are the subgraphs.
    """
    w = [g.tensors[g.ops[j].outs[0]].nbytes if g.ops[j].type in (SGD_MOM, ADAM) else 0
         for j in range(a, b)]
    W = sum(w)
    if chunks <= 1 or W == 0:
        return [(a, b)]
    out, c, start, prev = [], 0, a, None
    for i, j in enumerate(range(a, b)):
        ch = min(chunks - 1, (chunks * c) // W)
        if prev is not None and ch != prev:
            out.append((start, j))
            start = j
        prev = ch
        c += w[i]
    out.append((start, b))
    return out


def partition(g: Graph, policy: str = "phase", max_ops: int = 0,
              update_chunks: int = 1) -> List[Tuple[int, int]]:
    """Contiguous op ranges [start, end) for S_0..S_{n-1} (reading Q2)."""
    runs = []
    s = 0
    for j in range(1, len(g.ops) + 1):
        if j == len(g.ops) or g.ops[j].phase != g.ops[s].phase:
            runs.append((s, j))
            s = j
    if update_chunks > 1:
        split = []
        for (a, b) in runs:
            if any(g.ops[j].type in OPTIMIZER_OPS for j in range(a, b)):
                split.extend(_split_update(g, a, b, update_chunks))
            else:
                split.append((a, b))
        runs = split
    if policy == "phase":
        return runs
    if policy != "max_ops" or max_ops <= 0:
        raise GraphError(f"unknown partition policy {policy!r}")
    out = []
    for (a, b) in runs:
        if any(g.ops[j].type in OPTIMIZER_OPS for j in range(a, b)):
            out.append((a, b))  # optimizer runs are split only by update_chunks
            continue
        for c in range(a, b, max_ops):
            out.append((c, min(b, c + max_ops)))
    return out


def live_set(g: Graph, parts: List[Tuple[int, int]], k: int) -> List[int]:
    """L_k: tensor ids live at cut k (before S_k), ascending (module docstring)."""
    start = parts[k][0]
    ops = g.ops
    fed_ext = {i for i, t in enumerate(g.tensors)
               if t.kind in (INPUT, LABEL) and not any(i in o.outs for o in ops)}
    live = []
    for i, t in enumerate(g.tensors):
        if t.kind in PERSISTENT_KINDS:
            live.append(i)
            continue
        if t.kind == DATASET:
            continue
        written_before = (i in fed_ext and start > 0) or any(i in ops[j].outs for j in range(start))
        if not written_before:
            continue
        if t.kind == OUTPUT:
            live.append(i)
            continue
        # needed: read at/after S_k before being overwritten at/after S_k
        needed = False
        for j in range(start, len(ops)):
            if i in op_reads(ops[j]):
                needed = True
                break
            if i in op_writes(ops[j]):
                break
        if needed:
            live.append(i)
    return live


def live_bytes(g: Graph, ids: List[int]) -> int:
    return sum(g.tensors[i].nbytes for i in ids)
