"""Graph IR shared by the oracle and the CUDA path as *input description only*.

This module is the workload spec: which tensors a static training/inference graph
has and which ops (from the fixed op set of BASELINE.json north_star) run in which
order.  It holds none of the method's arithmetic: no op semantics, no partitioning,
no live-set analysis, no staging layout.  The oracle (``oracle/``) and the C++
runtime (``paper_conf_middleware_wur0hdh21_b200/csrc``) each implement those
independently from PAPER.md.

Graph model: PAPER.md:279-291 (section 2, "computation graphs ... nodes describe
operations while edges specify dataflows").  Tensor kinds follow the paper's split
between persistent variables kept across session runs (section 3.3
"Context saving") and intermediate data discarded at iteration end.

The integer codes below are the C-ABI enum values declared in include/sf.h; a
not-gpu test parses the header and checks they agree.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import List, Optional

# ---- dtypes (include/sf.h: sf_dtype) ------------------------------------------
F32 = 0
I32 = 1
DTYPE_BYTES = {F32: 4, I32: 4}
DTYPE_NAMES = {F32: "f32", I32: "i32"}

# ---- tensor kinds (include/sf.h: sf_tensor_kind) ------------------------------
PARAM = 0         # persistent variable (weights, BN statistics)
SLOT = 1          # persistent optimizer slot (momentum, Adam m/v)
SCALAR_STATE = 2  # persistent scalar state (step / data cursor)
DATASET = 3       # read-only, replicated on every candidate device, never migrated
INPUT = 4         # fed each iteration (FEED op or request copy)
LABEL = 5         # fed each iteration
ACT = 6           # intermediate activation
GRAD = 7          # intermediate gradient
OUTPUT = 8        # fetched result (loss, probabilities): live until iteration end
KIND_NAMES = {PARAM: "param", SLOT: "slot", SCALAR_STATE: "scalar_state",
              DATASET: "dataset", INPUT: "input", LABEL: "label", ACT: "act",
              GRAD: "grad", OUTPUT: "output"}
PERSISTENT_KINDS = (PARAM, SLOT, SCALAR_STATE)

# ---- op types (include/sf.h: sf_op_type) --------------------------------------
GEMM = 1          # ins [A, B]; outs [C]; flags TA|TB|ACC
BIAS_ACT = 2      # ins [z, b1, (b2), (b3)]; outs [h] (GELU: [h, u]); flags RELU | GELU
BIAS_ACT_BWD = 3  # ins [dh, h] (GELU: [dh, u]); outs [dz, db]   (act backward + bias grad)
COLSUM = 4        # ins [x]; outs [s]
SOFTMAX_CE = 5    # ins [logits, labels]; outs [loss, dlogits]
SOFTMAX = 6       # ins [logits]; outs [probs]
SGD_MOM = 7       # ins [g]; outs [w, a]          f = [lr, mu]
ADAM = 8          # ins [g, step]; outs [w, m, v] f = [lr, beta1, beta2, eps]
FEED = 9          # ins [pool, step]; outs [x]
STEP_INC = 10     # ins []; outs [step]
OP_NAMES = {GEMM: "gemm", BIAS_ACT: "bias_act", BIAS_ACT_BWD: "bias_act_bwd",
            COLSUM: "colsum", SOFTMAX_CE: "softmax_ce", SOFTMAX: "softmax",
            SGD_MOM: "sgd_mom", ADAM: "adam", FEED: "feed", STEP_INC: "step_inc"}

# GEMM flags
TA = 1
TB = 2
ACC = 4
# BIAS_ACT flags
RELU = 1
GELU = 2          # BIAS_ACT / BIAS_ACT_BWD flag: exact-erf GELU


@dataclass
class Tensor:
    name: str
    rows: int
    cols: int
    dtype: int = F32
    kind: int = ACT

    @property
    def numel(self) -> int:
        return self.rows * self.cols

    @property
    def nbytes(self) -> int:
        return self.numel * DTYPE_BYTES[self.dtype]


@dataclass
class Op:
    type: int
    ins: List[int]
    outs: List[int]
    flags: int = 0
    f: List[float] = field(default_factory=list)
    phase: int = 0


@dataclass
class Graph:
    name: str
    tensors: List[Tensor] = field(default_factory=list)
    ops: List[Op] = field(default_factory=list)

    def add(self, name: str, rows: int, cols: int, dtype: int = F32, kind: int = ACT) -> int:
        self.tensors.append(Tensor(name, rows, cols, dtype, kind))
        return len(self.tensors) - 1

    def op(self, type_: int, ins, outs, flags: int = 0, f=(), phase: int = 0) -> None:
        self.ops.append(Op(type_, list(ins), list(outs), flags, list(f), phase))

    def tid(self, name: str) -> int:
        for i, t in enumerate(self.tensors):
            if t.name == name:
                return i
        raise KeyError(name)

    def ids_of_kind(self, *kinds) -> List[int]:
        return [i for i, t in enumerate(self.tensors) if t.kind in kinds]

    def param_count(self) -> int:
        return sum(t.numel for t in self.tensors if t.kind == PARAM)

    def phases(self) -> List[int]:
        return [o.phase for o in self.ops]


def find_op_tensor(g: Graph, name: str) -> Optional[int]:
    for i, t in enumerate(g.tensors):
        if t.name == name:
            return i
    return None
