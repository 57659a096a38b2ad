"""Pins for oracle/staging.py, parsed with ``struct`` independently of its writer.

- byte-exact golden fixture for a tiny hand-computed case (tests/golden/staging_tiny.json);
- every payload at a 256-B aligned offset, in ascending tensor id, back to back with
  round_up(nbytes, 256) strides; all other bytes zero; total as stated in the header;
- round trip pack -> unpack restores the tensors bit for bit; the empty live set.
"""
import json
import os
import struct

import numpy as np

from oracle import graph as OG, staging as S
from sf_inputs import graphs as G, data as D
from sf_inputs.ir import Graph, F32, I32, PARAM

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def test_golden_tiny_staging_bytes():
    gold = json.load(open(os.path.join(GOLD, "staging_tiny.json")))
    g = Graph("tiny")
    a = g.add("s", 1, 1, I32, PARAM)
    b = g.add("v", 1, 3, F32, PARAM)
    T = {a: np.array([[7]], np.int32), b: np.array([[1.0, 2.0, 3.0]], np.float32)}
    buf = S.pack(g, [a, b], T, gold["k"], gold["iter"])
    assert len(buf) == gold["total"]
    expect = bytearray(gold["total"])
    for r in gold["regions"]:
        raw = bytes.fromhex(r["hex"])
        expect[r["offset"]:r["offset"] + len(raw)] = raw
    assert buf == bytes(expect)


def _independent_check(g, ids, T, buf, k, it):
    magic, ver, n, kk, iters, total = struct.unpack_from("<4sIIIQQ", buf, 0)
    assert (magic, ver, n, kk, iters, total) == (b"SFST", 1, len(ids), k, it, len(buf))
    covered = np.zeros(len(buf), bool)
    covered[:32 + 24 * n] = True
    expect_off = -(-(32 + 24 * n) // 256) * 256
    for e, tid in enumerate(ids):
        t_id, dt, off, nb = struct.unpack_from("<IIQQ", buf, 32 + 24 * e)
        assert t_id == tid and dt == g.tensors[tid].dtype and nb == g.tensors[tid].nbytes
        assert off % 256 == 0 and off == expect_off
        assert buf[off:off + nb] == np.ascontiguousarray(T[tid]).tobytes()
        covered[off:off + nb] = True
        expect_off = off + -(-nb // 256) * 256
    assert expect_off == total
    pad = np.frombuffer(buf, np.uint8)[~covered]
    assert not pad.any()


def test_c1_every_cut_staging_layout():
    g = G.mlp_train()
    parts = OG.partition(g)
    rng = np.random.default_rng(0)
    T = {}
    for i, t in enumerate(g.tensors):
        if t.dtype == F32:
            T[i] = rng.standard_normal((t.rows, t.cols)).astype(np.float32)
        else:
            T[i] = rng.integers(-5, 5, (t.rows, t.cols)).astype(np.int32)
    for k in range(len(parts)):
        L = OG.live_set(g, parts, k)
        buf = S.pack(g, L, T, k, 42)
        _independent_check(g, L, T, buf, k, 42)
        back = {}
        kk, it = S.unpack(g, buf, back)
        assert (kk, it) == (k, 42) and sorted(back) == L
        for i in L:
            assert back[i].tobytes() == T[i].tobytes()


def test_resnet_cut0_staging_size():
    g = G.resnet50_forest(batch=1, spatial_div=8)
    L = OG.live_set(g, OG.partition(g), 0)
    st = D.init_state(g)
    buf = S.pack(g, L, st, 0, 0)
    _independent_check(g, L, st, buf, 0, 0)
    # 535 entries; all sizes are multiples of 256 except the 4-byte cursor (-> 256)
    # and fc bias + its momentum (4000 B -> 4096 each)
    assert len(buf) == -(-(32 + 24 * 535) // 256) * 256 + 204881216 + 256 + 2 * 96


def test_empty_live_set():
    g = Graph("e")
    buf = S.pack(g, [], {}, 0, 0)
    assert len(buf) == 256 and buf[:4] == b"SFST" and not any(buf[32:])
