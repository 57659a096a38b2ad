"""Pins for oracle/graph.py (partition, live sets) — independent of the oracle itself.

- C1 partition and live-set table: golden fixture from SURVEY.md 8(c) (+ data cursor).
- Brute force: for every cut k of several iterations, a run whose target device is
  poisoned and restored from L_k only equals the unpreempted run bitwise
  ("no work is lost"); a missing tensor would turn into NaN / -1.
- Minimality: dropping any non-persistent member of L_k breaks the result.
- Table 1 identity: cut-0 state of all-trainable VGG16 / VGG19
  = 2 x params x 4 B = the paper's MiB; Keras ResNet-50 census.
"""
import json
import os

import numpy as np
import pytest

from oracle import graph as OG, runner as R
from sf_inputs import graphs as G, data as D
from sf_inputs.ir import (OP_NAMES, PERSISTENT_KINDS, Graph, F32, I32, PARAM, ACT, INPUT,
                          DATASET, GEMM, BIAS_ACT, SCALAR_STATE, SGD_MOM, SLOT, GRAD, STEP_INC)

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _bitwise_equal(a, b):
    return a.dtype == b.dtype and a.shape == b.shape and a.tobytes() == b.tobytes()


def test_c1_partition_matches_survey():
    gold = json.load(open(os.path.join(GOLD, "c1_live_sets.json")))
    g = G.mlp_train()
    parts = OG.partition(g)
    assert [[OP_NAMES[g.ops[j].type] for j in range(a, b)] for a, b in parts] == gold["partition_ops"]


def test_c1_live_sets_golden():
    gold = json.load(open(os.path.join(GOLD, "c1_live_sets.json")))
    g = G.mlp_train()
    parts = OG.partition(g)
    for row in gold["survey_table"]:
        L = OG.live_set(g, parts, row["k"])
        inflight = sorted(g.tensors[i].name for i in L if g.tensors[i].kind not in PERSISTENT_KINDS)
        assert inflight == sorted(row["inflight"]), row
        assert OG.live_bytes(g, L) == row["bytes"] + gold["cursor_bytes"]
        assert len(L) == row["tensors"] + 1
        assert L == sorted(L)


CASES = [
    ("mlp232", lambda: G.mlp_train((2, 3, 2), batch=4, pool=3), 4),
    ("mlp4653", lambda: G.mlp_train((4, 6, 5, 3), batch=5, pool=2), 3),
    ("c1", lambda: G.mlp_train(), 2),
    ("resnet_prefix", lambda: G.resnet50_forest(batch=1, spatial_div=8, max_layers=5), 2),
    ("bert_tiny", lambda: G.bert_chain(layers=2, hidden=8, inter=16, vocab=11, tokens=6,
                                       positions=6), 2),
]


@pytest.mark.parametrize("name,mk,iters", CASES, ids=[c[0] for c in CASES])
def test_restore_from_live_set_every_cut_is_bitwise(name, mk, iters):
    g = mk()
    parts = OG.partition(g)
    st, ds = D.init_state(g), D.datasets(g)
    ref = R.run(g, iters, st, ds, keep_stagings=False)
    for it in range(iters):
        for k in range(len(parts)):
            for tgt in (1, R.HOST):
                got = R.run(g, iters, st, ds, schedule=[(it, k, tgt)], keep_stagings=False)
                assert got.device == (1 if tgt == 1 else 0)
                for i in ref.state:
                    assert _bitwise_equal(ref.state[i], got.state[i]), (it, k, g.tensors[i].name)
                for o1, o2 in zip(ref.outputs, got.outputs):
                    for kk in o1:
                        assert _bitwise_equal(o1[kk], o2[kk])


def test_many_preemptions_ping_pong_bitwise():
    g = G.mlp_train((5, 7, 3), batch=4, pool=3)
    parts = OG.partition(g)
    st, ds = D.init_state(g), D.datasets(g)
    ref = R.run(g, 6, st, ds)
    sched = D.preemption_schedule(6, len(parts), 12, targets=[1, 0, R.HOST])
    # targets must differ from the current device for a peer move; the oracle allows any
    got = R.run(g, 6, st, ds, schedule=sched, n_devices=2)
    for i in ref.state:
        assert _bitwise_equal(ref.state[i], got.state[i])


@pytest.mark.parametrize("name,mk,iters", CASES[:3], ids=[c[0] for c in CASES[:3]])
def test_live_set_minimal(name, mk, iters):
    g = mk()
    parts = OG.partition(g)
    st, ds = D.init_state(g), D.datasets(g)
    ref = R.run(g, 2, st, ds, keep_stagings=False)
    for k in range(len(parts)):
        L = OG.live_set(g, parts, k)
        for t in L:
            if g.tensors[t].kind in PERSISTENT_KINDS:
                continue
            got = R.run(g, 2, st, ds, schedule=[(1, k, 1)], omit=[t], keep_stagings=False)
            differs = any(not _bitwise_equal(ref.state[i], got.state[i]) for i in ref.state) or \
                any(not _bitwise_equal(a[n], b[n]) for a, b in zip(ref.outputs, got.outputs) for n in a)
            assert differs, (k, g.tensors[t].name)


def test_cut0_is_weights_only():
    """At the iteration boundary only persistent state is live (the paper's case, Q1)."""
    for g in (G.mlp_train(), G.resnet50_forest(batch=1, spatial_div=8), G.bert_chain(
            layers=2, hidden=8, inter=16, vocab=11, tokens=6, positions=6)):
        parts = OG.partition(g)
        L = OG.live_set(g, parts, 0)
        assert all(g.tensors[i].kind in PERSISTENT_KINDS for i in L)
        assert len(L) == len(g.ids_of_kind(*PERSISTENT_KINDS))


def test_table1_identity_vgg():
    gold = json.load(open(os.path.join(GOLD, "table1_state_sizes.json")))
    for row in gold["rows"][:2]:
        depth = 16 if row["model"] == "VGG16" else 19
        g = G.forest(G.vgg_layers(depth), batch=1)
        assert g.param_count() == row["keras_params"]
        parts = OG.partition(g)
        L = OG.live_set(g, parts, 0)
        state = OG.live_bytes(g, L) - 4  # minus the int32 cursor
        assert state == 2 * row["keras_params"] * 4
        assert round(state / 2 ** 20, 2) == row["mib"]


def test_resnet50_census():
    gold = json.load(open(os.path.join(GOLD, "table1_state_sizes.json")))["resnet50_keras_census"]
    g = G.resnet50_forest(batch=1)
    ids = g.ids_of_kind(PARAM, SLOT)
    sz = np.array([g.tensors[i].nbytes for i in ids])
    assert len(ids) == gold["tensors"] and sz.sum() == gold["bytes"]
    assert sz.min() == gold["min_bytes"] and np.median(sz) == gold["median_bytes"]
    assert sz.max() == gold["max_bytes"]
    assert (sz < 4096).sum() == gold["lt_4KiB"] and (sz < 65536).sum() == gold["lt_64KiB"]
    assert g.param_count() == 25636712


def test_bert_large_census():
    g = G.bert_chain()
    assert g.param_count() == 335141888
    assert len(g.ids_of_kind(PARAM)) == 391
    assert len(g.ids_of_kind(*PERSISTENT_KINDS)) == 391 * 3 + 1
    parts = OG.partition(g)
    assert OG.live_bytes(g, OG.live_set(g, parts, 0)) == 335141888 * 12 + 4


def test_max_ops_partition_keeps_update_whole():
    g = G.mlp_train()
    parts = OG.partition(g, "max_ops", 1)
    assert all(b - a == 1 for a, b in parts[:-1])
    assert parts[-1] == (12, 17)
    assert parts[0][0] == 0 and parts[-1][1] == len(g.ops)
    assert all(p[1] == q[0] for p, q in zip(parts, parts[1:]))


@pytest.mark.parametrize("U", [2, 3, 8])
def test_update_chunks_rule(U):
    g = G.resnet50_forest(batch=1, spatial_div=8)
    whole = OG.partition(g)
    parts = OG.partition(g, update_chunks=U)
    a, b = whole[-1]
    upd = [p for p in parts if p[0] >= a]
    assert parts[:len(whole) - 1] == whole[:-1]
    assert upd[0][0] == a and upd[-1][1] == b and len(upd) == U
    assert all(p[1] == q[0] for p, q in zip(upd, upd[1:]))
    w = lambda j: g.tensors[g.ops[j].outs[0]].nbytes if g.ops[j].type != STEP_INC else 0
    W = sum(w(j) for j in range(a, b))
    biggest = max(w(j) for j in range(a, b))
    for (x, y) in upd:
        assert sum(w(j) for j in range(x, y)) <= W / U + biggest


@pytest.mark.parametrize("mk,U", [(lambda: G.mlp_train((5, 7, 3), batch=4, pool=2), 3),
                                  (lambda: G.resnet50_forest(batch=1, spatial_div=8, max_layers=6), 4)])
def test_cut_inside_update_is_bitwise(mk, U):
    """Cutting between optimizer ops resumes with the remaining updates only."""
    g = mk()
    parts = OG.partition(g, update_chunks=U)
    st, ds = D.init_state(g), D.datasets(g)
    ref = R.run(g, 2, st, ds, parts=parts, keep_stagings=False)
    n_upd = sum(1 for p in parts if any(g.ops[j].type in (SGD_MOM, STEP_INC) for j in range(*p)))
    for k in range(len(parts) - n_upd + 1, len(parts)):
        got = R.run(g, 2, st, ds, parts=parts, schedule=[(1, k, 1)], keep_stagings=False)
        for i in ref.state:
            assert _bitwise_equal(ref.state[i], got.state[i]), (k, g.tensors[i].name)
        L = OG.live_set(g, parts, k)
        assert any(g.tensors[i].kind == GRAD for i in L)  # not-yet-applied gradients


def test_validate_rejects_bad_graphs():
    g = Graph("bad")
    a = g.add("a", 2, 3, F32, ACT)
    w = g.add("w", 3, 4, F32, PARAM)
    z = g.add("z", 2, 4, F32, ACT)
    g.op(GEMM, [a, w], [z])
    with pytest.raises(OG.GraphError):
        OG.validate(g)  # reads a before it is written
    g2 = Graph("bad2")
    x = g2.add("x", 2, 3, F32, INPUT)
    w = g2.add("w", 4, 4, F32, PARAM)
    z = g2.add("z", 2, 4, F32, ACT)
    g2.op(GEMM, [x, w], [z])
    with pytest.raises(OG.GraphError):
        OG.validate(g2)  # K mismatch
    g3 = Graph("bad3")
    d = g3.add("d", 1, 4, F32, DATASET)
    gg = g3.add("g", 1, 4, F32, INPUT)
    a3 = g3.add("a", 1, 4, F32, SLOT)
    g3.op(SGD_MOM, [gg], [d, a3], f=[0.1, 0.9])
    with pytest.raises(OG.GraphError):
        OG.validate(g3)  # writes a dataset
