"""Pins for oracle/feed.py (the workload's host input stage) and the lockstep invariant I6.

- splitmix64 known-answer values (Vigna's reference splitmix64.c, seed 0);
- x * 255 reproduces the u8 source exactly; a flipped sample is the mirror image of its
  source, an unflipped one equals it; about half the rows flip;
- the FEED-pool form (u8_pool) equals the per-iteration stage output;
- the runner's ``feeds`` hook with the stage equals the FEED-op graph over u8_pool;
- I6: hand-built lockstep traces pass, split / reordered blocks are rejected.
"""
import numpy as np
import pytest

from oracle import feed as FD, runner as R, schedule as SC
from sf_inputs import data as D, graphs as G


def test_splitmix64_known_answers():
    assert FD.splitmix64(0, 1) == 0xE220A8397B1DCDAF
    assert FD.splitmix64(0, 2) == 0x6E789E6AA1B965F4
    assert FD.splitmix64(0, 3) == 0x06C45D188009454F


def test_u8_stage_properties():
    imgs, labels = D.u8_images(64, 28 * 28, 10, seed=5)
    flips = 0
    for it in range(4):
        x, y = FD.u8_stage(imgs, labels, it, 16, 28, seed=9)
        assert x.dtype == np.float32 and x.shape == (16, 784) and y.shape == (16, 1)
        b = it % 4
        for r in range(16):
            src = imgs[b * 16 + r]
            back = np.rint(x[r].astype(np.float64) * 255.0)
            assert np.all(np.abs(x[r].astype(np.float64) * 255.0 - back) < 1e-4)
            back = back.astype(np.uint8)
            mirror = src.reshape(28, 28)[:, ::-1].reshape(-1)
            flipped = bool(FD.splitmix64(9, b * 16 + r + 1) & 1)
            assert np.array_equal(back, mirror if flipped else src)
            flips += flipped
            assert y[r, 0] == labels[b * 16 + r, 0]
    assert 16 <= flips <= 48  # ~half of 64 samples


def test_u8_pool_equals_stage_and_runner_feeds():
    imgs, labels = D.u8_images(32, 12, 3, seed=2)
    px, py = FD.u8_pool(imgs, labels, 8, 4, seed=1)
    for it in range(6):
        x, y = FD.u8_stage(imgs, labels, it, 8, 4, seed=1)
        b = it % 4
        assert np.array_equal(x, px[b * 8:(b + 1) * 8]) and np.array_equal(y, py[b * 8:(b + 1) * 8])
    gp = G.mlp_train((12, 5, 3), batch=8, pool=4)
    gh = G.mlp_train((12, 5, 3), batch=8, pool=4, host_fed=True)
    st = D.init_state(gp)
    ds = {gp.tid("X_pool"): px, gp.tid("Y_pool"): py}
    ref = R.run(gp, 6, st, ds, schedule=[(2, 1, R.HOST), (3, 0, 1)])
    sth = {gh.tid(gp.tensors[i].name): a for i, a in st.items()}
    xt, yt = gh.tid("x"), gh.tid("y")
    got = R.run(gh, 6, sth, {}, schedule=[(2, 1, R.HOST), (3, 0, 1)],
                feeds=lambda it: dict(zip((xt, yt), FD.u8_stage(imgs, labels, it, 8, 4, seed=1))))
    for i, a in ref.state.items():
        assert a.tobytes() == got.state[gh.tid(gp.tensors[i].name)].tobytes()


def _ev(job, it, t0, t1, k=0):
    return {"dev": 0, "job": job, "kind": "train", "iter": it, "k": k, "t0": t0, "t1": t1}


def test_lockstep_checker():
    ok = [_ev(5, 0, 0, 1), _ev(5, 0, 1, 2, 1), _ev(7, 0, 2, 3), _ev(7, 0, 3, 4, 1),
          _ev(5, 1, 4, 5), _ev(7, 1, 5, 6), _ev(9, 0, 6, 7)]
    SC.check_lockstep(ok[:-1], [5, 7])
    with pytest.raises(SC.InvariantError):  # member 7 ran iteration 0 before member 5 did
        SC.check_lockstep([_ev(7, 0, 0, 1), _ev(5, 0, 1, 2)], [5, 7])
    with pytest.raises(SC.InvariantError):  # member 5's iteration 0 split by member 7's
        SC.check_lockstep([_ev(5, 0, 0, 1), _ev(7, 0, 1, 2), _ev(5, 0, 2, 3, 1)], [5, 7])
    with pytest.raises(SC.InvariantError):  # member 5 ran ahead to iteration 1
        SC.check_lockstep([_ev(5, 0, 0, 1), _ev(5, 1, 1, 2), _ev(7, 0, 2, 3)], [5, 7])
    SC.check_lockstep(ok, [5, 7])  # other jobs' subgraphs are ignored
