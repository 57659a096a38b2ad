"""Oracle execution: partitioned training under a preemption schedule (test infra).

The method's defining property is that preemption moves *where* subgraphs run and
nothing else: "The new session is populated with the tasks of the aborted session run
so that no work is lost" (section 3.3); "subsequent sessions of
job2 will be run on a different device".  So the oracle is the
plain definition: run S_0..S_{n-1} of every iteration in order on the "current
device"; at each scheduled cut (iter, k, target):

  1. pack L_k from the current device into staging bytes
  2. poison the target device's tensors (0xFF bytes: NaN / -1)
  3. unpack the staging bytes into the target device
  4. target becomes the current device (peer tier) — or, for the host tier
     (target == HOST), the current device itself is poisoned and restored from the
     host copy after the preempter ran (reading Q4: park and swap back).

Every simulated device holds its own copy of the DATASET tensors (replicated,
read-only).  Persistent state starts on device ``home``.

Pins (tests/test_oracle_runner.py): preempted run == unpreempted run bitwise for every
cut k of several iterations (tiny MLPs, C1, a C2 prefix); GPU-free trajectory sanity
(loss decreases on C1); inference vs brute-force forward.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Callable, Dict, List, Optional, Sequence, Tuple

import numpy as np

from sf_inputs.ir import DATASET, F32, OUTPUT, PERSISTENT_KINDS, Graph
from . import graph as G
from . import ops as O
from . import staging as S

HOST = -1


def poison_like(a: np.ndarray) -> np.ndarray:
    """0xFF bytes of the same dtype/shape: NaN for fp32, -1 for int32."""
    return np.frombuffer(b"\xff" * a.nbytes, dtype=a.dtype).reshape(a.shape).copy()


@dataclass
class Trajectory:
    outputs: List[Dict[str, np.ndarray]] = field(default_factory=list)  # per iteration
    state: Dict[int, np.ndarray] = field(default_factory=dict)          # final persistent
    stagings: List[Tuple[int, int, int, bytes]] = field(default_factory=list)  # (it,k,tgt,buf)
    trace: List[Tuple[int, int, int]] = field(default_factory=list)     # (device, it, k)
    device: int = 0


def _empty(g: Graph, dev_data: Dict[int, np.ndarray]) -> Dict[int, np.ndarray]:
    T = {}
    for i, t in enumerate(g.tensors):
        if t.kind == DATASET:
            T[i] = dev_data[i]
        else:
            dt = np.float32 if t.dtype == F32 else np.int32
            T[i] = poison_like(np.zeros((t.rows, t.cols), dt))
    return T


def run(g: Graph, iters: int, state0: Dict[int, np.ndarray], data: Dict[int, np.ndarray],
        schedule: Sequence[Tuple[int, int, int]] = (), parts=None, n_devices: int = 2,
        home: int = 0, exact: bool = False, keep_stagings: bool = True,
        omit: Sequence[int] = (),
        inference: Optional[Tuple[Graph, Dict[int, np.ndarray], np.ndarray]] = None,
        feeds: Optional[Callable[[int], Dict[int, np.ndarray]]] = None
        ) -> Trajectory:
    """Run ``iters`` iterations; ``schedule`` = [(iter, k, target)] cuts (target or HOST).

    ``feeds(it)`` -> {tensor id: array}: externally fed INPUT / LABEL tensors written
    into the current device at the start of S_0 of iteration ``it`` (host input stage).

    ``omit`` drops tensor ids from every migrated live set (minimality pin only).
    """
    G.validate(g)
    parts = parts or G.partition(g)
    shapes = {i: (t.rows, t.cols) for i, t in enumerate(g.tensors)}
    devs = [_empty(g, data) for _ in range(n_devices)]
    for i, a in state0.items():
        devs[home][i] = np.array(a, dtype=np.float64 if exact and a.dtype == np.float32 else a.dtype,
                                 copy=True)
    if exact:
        for d in devs:
            for i in list(d):
                if d[i].dtype == np.float32:
                    d[i] = d[i].astype(np.float64)
    cur = home
    sched = {(it, k): tgt for (it, k, tgt) in schedule}
    tr = Trajectory()
    outputs_ids = [i for i, t in enumerate(g.tensors) if t.kind == OUTPUT]
    for it in range(iters):
        for k, (a, b) in enumerate(parts):
            if (it, k) in sched:
                tgt = sched[(it, k)]
                live = [i for i in G.live_set(g, parts, k) if i not in omit]
                buf = S.pack(g, live, {i: devs[cur][i].astype(np.float32)
                                       if exact and devs[cur][i].dtype == np.float64
                                       else devs[cur][i] for i in live}, k, it)
                if keep_stagings:
                    tr.stagings.append((it, k, tgt, buf))
                dst = cur if tgt == HOST else tgt
                for i, t in enumerate(g.tensors):
                    if t.kind != DATASET:
                        devs[dst][i] = poison_like(devs[dst][i])
                if inference is not None:
                    run_inference(*inference)  # the preempter runs at the cut
                got = {}
                S.unpack(g, buf, got)
                for i, arr in got.items():
                    devs[dst][i] = arr.astype(np.float64) if exact and arr.dtype == np.float32 else arr
                cur = dst
            if k == 0 and feeds is not None:
                for i, arr in feeds(it).items():
                    devs[cur][i] = np.array(arr, copy=True)
            for j in range(a, b):
                O.apply_op(g.ops[j], devs[cur], shapes, exact)
            tr.trace.append((cur, it, k))
        tr.outputs.append({g.tensors[i].name: np.array(devs[cur][i], copy=True)
                           for i in outputs_ids})
    tr.state = {i: np.array(devs[cur][i], copy=True)
                for i, t in enumerate(g.tensors) if t.kind in PERSISTENT_KINDS}
    tr.device = cur
    return tr


def run_inference(g: Graph, params: Dict[int, np.ndarray], x: np.ndarray) -> np.ndarray:
    """Batch-1 forward of an inference graph (one subgraph); returns its OUTPUT tensor."""
    G.validate(g)
    shapes = {i: (t.rows, t.cols) for i, t in enumerate(g.tensors)}
    T = dict(params)
    xin = [i for i, t in enumerate(g.tensors) if t.kind == 4]
    T[xin[0]] = np.asarray(x, dtype=np.float32).reshape(shapes[xin[0]])
    for op in g.ops:
        O.apply_op(op, T, shapes)
    outs = [i for i, t in enumerate(g.tensors) if t.kind == OUTPUT]
    return T[outs[0]]
