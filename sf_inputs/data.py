"""Seeded synthetic data and initial state for the workload graphs.

Input generation only (SURVEY.md reading Q11): glorot-uniform weights (Keras
default, limit sqrt(6/(fan_in+fan_out))), zero biases, BN gamma = 1 / beta = 0 /
moving mean = 0 / moving var = 1, zero optimizer slots, step = 0; features
x ~ U[0, 1), labels = floor(u * C).  Generated once on the host and fed identically
to the GPU path and the oracle.  No op of the method is computed here.
"""
from __future__ import annotations

from typing import Dict

import numpy as np

from .ir import DATASET, F32, I32, INPUT, PARAM, SCALAR_STATE, SLOT, Graph

SEED_DATA = 1
SEED_INIT = 3
SEED_INFER = 4


def _glorot(rng: np.random.Generator, rows: int, cols: int, name: str) -> np.ndarray:
    fan_in, fan_out = rows, cols
    limit = np.sqrt(6.0 / (fan_in + fan_out))
    return rng.uniform(-limit, limit, size=(rows, cols)).astype(np.float32)


def init_state(g: Graph, seed: int = SEED_INIT) -> Dict[int, np.ndarray]:
    """Initial persistent state (PARAM, SLOT, SCALAR_STATE) keyed by tensor id."""
    rng = np.random.Generator(np.random.PCG64(seed))
    out: Dict[int, np.ndarray] = {}
    for i, t in enumerate(g.tensors):
        if t.kind == PARAM:
            nm = t.name
            if t.rows == 1:  # vectors: biases, BN/LN gamma & beta, BN moving stats
                if "gamma" in nm or nm.endswith("moving_var"):
                    out[i] = np.ones((t.rows, t.cols), np.float32)
                else:
                    out[i] = np.zeros((t.rows, t.cols), np.float32)
            else:
                out[i] = _glorot(rng, t.rows, t.cols, nm)
        elif t.kind == SLOT:
            out[i] = np.zeros((t.rows, t.cols), np.float32)
        elif t.kind == SCALAR_STATE:
            out[i] = np.zeros((t.rows, t.cols), np.int32)
    return out


def _n_classes(g: Graph, label_tid: int) -> int:
    """Classes for a label tensor = width of the logits it is consumed with."""
    from .ir import FEED, SOFTMAX_CE
    for o in g.ops:
        if o.type == SOFTMAX_CE and o.ins[1] == label_tid:
            return g.tensors[o.ins[0]].cols
        if o.type == FEED and o.ins[0] == label_tid:
            return _n_classes(g, o.outs[0])
    raise ValueError(f"label {g.tensors[label_tid].name} not consumed by softmax_ce")


def datasets(g: Graph, seed: int = SEED_DATA) -> Dict[int, np.ndarray]:
    """Read-only DATASET tensors: features U[0,1), int32 labels U{0..C-1}."""
    rng = np.random.Generator(np.random.PCG64(seed))
    out: Dict[int, np.ndarray] = {}
    for i, t in enumerate(g.tensors):
        if t.kind != DATASET:
            continue
        if t.dtype == F32:
            out[i] = rng.random((t.rows, t.cols), dtype=np.float32)
        else:
            c = _n_classes(g, i)
            out[i] = np.floor(rng.random((t.rows, t.cols)) * c).astype(np.int32)
            np.clip(out[i], 0, c - 1, out=out[i])
    return out


def infer_inputs(g: Graph, n: int, seed: int = SEED_INFER) -> np.ndarray:
    """n request inputs for an inference graph's single INPUT tensor: [n, rows, cols]."""
    rng = np.random.Generator(np.random.PCG64(seed))
    xs = [t for t in g.tensors if t.kind == INPUT]
    assert len(xs) == 1
    t = xs[0]
    return rng.random((n, t.rows, t.cols), dtype=np.float32)


def random_bytes(n: int, seed: int) -> np.ndarray:
    """Arbitrary byte contents (pack/unpack parity inputs)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    return rng.integers(0, 256, size=n, dtype=np.uint8)


def preemption_schedule(n_iters: int, n_subgraphs: int, n_preempt: int, targets,
                        seed: int = 7):
    """Seeded random preemption points [(iter, k, target)], sorted, distinct."""
    rng = np.random.Generator(np.random.PCG64(seed))
    pts = set()
    while len(pts) < min(n_preempt, n_iters * n_subgraphs):
        it = int(rng.integers(0, n_iters))
        k = int(rng.integers(0, n_subgraphs))
        pts.add((it, k))
    pts = sorted(pts)
    return [(it, k, targets[j % len(targets)]) for j, (it, k) in enumerate(pts)]


def poisson_arrivals(n: int, rate_per_s: float, seed: int = 7) -> np.ndarray:
    """Open-loop Poisson arrival offsets in seconds."""
    rng = np.random.Generator(np.random.PCG64(seed))
    return np.cumsum(rng.exponential(1.0 / rate_per_s, size=n))


def u8_images(n: int, cols: int, classes: int, seed: int = SEED_DATA):
    """Synthetic u8 image pool for the host input stage (reading Q27): pixels U{0..255},
    labels U{0..classes-1}."""
    rng = np.random.Generator(np.random.PCG64(seed))
    return (rng.integers(0, 256, size=(n, cols), dtype=np.uint8),
            rng.integers(0, classes, size=(n, 1), dtype=np.int32))
