"""Oracle of the host input stage (test infrastructure only; see oracle/__init__.py).

The paper's CPU executor loads and preprocesses each iteration's input batch
(section 3.4; "data preprocessing and data augmentation",
PAPER.md:1309-1312, section 5.3).  The workload's stage (reading Q27) is a
synthetic image pipeline, written here step by step from its definition:

  1. batch b = iter mod P of a pool of P * batch u8 images [rows][cols];
  2. sample r of the batch is pool row b * batch + r;
  3. it is flipped horizontally (each of its cols / img_w pixel rows reversed) when the
     low bit of output (row + 1) of splitmix64 seeded with ``seed`` is set;
  4. x = u8 / 255 in fp32 (one correctly rounded division); y = the row's label.

splitmix64 (Steele, Lea & Flood, OOPSLA 2014): state += 0x9E3779B97F4A7C15, output =
fin(state) with fin(z) = z ^= z >> 30, z *= 0xBF58476D1CE4E5B9, z ^= z >> 27,
z *= 0x94D049BB133111EB, z ^= z >> 31.

Pins (tests/test_oracle_feed.py): splitmix64 known-answer values for seed 0; x * 255 is
the u8 source exactly; a flipped sample is the mirror image of its source, unflipped
ones equal it; flips occur for about half the rows.
"""
from __future__ import annotations

from typing import Tuple

import numpy as np

GOLDEN = 0x9E3779B97F4A7C15
M64 = (1 << 64) - 1


def splitmix64(seed: int, n: int) -> int:
    """Output n (1-based) of splitmix64 seeded with ``seed``."""
    z = (seed + n * GOLDEN) & M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def u8_stage(images: np.ndarray, labels: np.ndarray, it: int, batch: int, img_w: int,
             seed: int) -> Tuple[np.ndarray, np.ndarray]:
    """Steps 1-4 of the module docstring: (x [batch][cols] f32, y [batch][1] i32)."""
    pool = images.shape[0] // batch
    b = it % pool
    cols = images.shape[1]
    x = np.empty((batch, cols), np.float32)
    y = np.empty((batch, 1), np.int32)
    for r in range(batch):
        row = b * batch + r
        src = images[row]
        if splitmix64(seed, row + 1) & 1:
            src = src.reshape(cols // img_w, img_w)[:, ::-1].reshape(cols)
        x[r] = src.astype(np.float32) / np.float32(255.0)
        y[r, 0] = labels.reshape(-1)[row]
    return x, y


def u8_pool(images: np.ndarray, labels: np.ndarray, batch: int, img_w: int,
            seed: int) -> Tuple[np.ndarray, np.ndarray]:
    """The stage's output for every batch of the pool, stacked ([P*batch][cols], [P*batch][1]):
    a FEED-op graph reading this pool sees exactly the host-fed inputs."""
    P = images.shape[0] // batch
    xs, ys = zip(*(u8_stage(images, labels, b, batch, img_w, seed) for b in range(P)))
    return np.concatenate(xs), np.concatenate(ys)
