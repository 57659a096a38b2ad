"""Pins for oracle/runner.py (trajectory, inference) and oracle/schedule.py (invariants).

runner: C1 trains (loss falls over 100 iterations — sanity, not parity); inference
vs a brute-force fp64 forward written with Python loops; the preempter running at the
cut does not perturb the trajectory.
schedule: hand-built traces violating I1..I4 are rejected; the discrete-event
model's traces satisfy all four; closed-form latencies of the model.
"""
import math

import numpy as np
import pytest

from oracle import runner as R, schedule as SC, graph as OG
from sf_inputs import graphs as G, data as D


def test_c1_loss_decreases():
    g = G.mlp_train()
    tr = R.run(g, 100, D.init_state(g), D.datasets(g), keep_stagings=False)
    losses = [float(o["loss"][0, 0]) for o in tr.outputs]
    assert abs(losses[0] - math.log(10)) < 0.5
    assert np.mean(losses[-10:]) < losses[0] - 0.1


def test_inference_brute_force():
    gi = G.mlp_infer((7, 5, 3))
    params = D.init_state(gi, seed=9)
    rng = np.random.default_rng(1)
    for i, t in enumerate(gi.tensors):
        if t.rows == 1 and t.kind == 0:
            params[i] = rng.standard_normal((1, t.cols)).astype(np.float32)
    x = D.infer_inputs(gi, 1)[0]
    got = R.run_inference(gi, params, x)
    W1, b1, W2, b2 = (params[gi.tid(n)] for n in ("W1", "b1", "W2", "b2"))
    h = [max(0.0, sum(float(x[0, k]) * float(W1[k, j]) for k in range(7)) + float(b1[0, j]))
         for j in range(5)]
    l = [sum(h[k] * float(W2[k, j]) for k in range(5)) + float(b2[0, j]) for j in range(3)]
    m = max(l)
    e = [math.exp(v - m) for v in l]
    p = [v / sum(e) for v in e]
    np.testing.assert_allclose(got[0], p, rtol=1e-6)


def test_preempter_at_cut_does_not_perturb():
    g = G.mlp_train((5, 7, 3), batch=4, pool=2)
    gi = G.mlp_infer((5, 7, 3))
    st, ds = D.init_state(g), D.datasets(g)
    ref = R.run(g, 3, st, ds)
    got = R.run(g, 3, st, ds, schedule=[(1, 2, R.HOST), (2, 3, 1)],
                inference=(gi, D.init_state(gi), D.infer_inputs(gi, 1)[0]))
    for i in ref.state:
        assert ref.state[i].tobytes() == got.state[i].tobytes()


def _ev(dev, job, kind, t0, t1, it=0, k=0, arrival=None):
    e = {"dev": dev, "job": job, "kind": kind, "iter": it, "k": k, "t0": t0, "t1": t1}
    if arrival is not None:
        e["arrival"] = arrival
    return e


def test_checker_rejects_corun():
    evs = [_ev(0, 0, "train", 0, 10), _ev(0, 1, "infer", 5, 7, arrival=4)]
    with pytest.raises(SC.InvariantError):
        SC.check_no_corun(evs)
    SC.check_no_corun([_ev(0, 0, "train", 0, 10), _ev(1, 1, "infer", 5, 7, arrival=4)])


def test_checker_device_ordered_overlap():
    """An early-launched request (dispatched while job 0's subgraph was still in flight,
    ordered after it on the device) may overlap that subgraph's host interval; a subgraph
    of the job dispatched after the request, or another job's, may not."""
    tr = _ev(0, 0, "train", 0, 10)
    tr["launch"] = 0
    r = _ev(0, 1 << 20, "infer", 5, 30, arrival=4)
    r["after"] = 0
    SC.check_no_corun([tr, r])
    late = dict(tr, t0=6, t1=12, launch=6, k=1)  # dispatched after the request
    with pytest.raises(SC.InvariantError):
        SC.check_no_corun([tr, r, late])
    other = dict(tr, job=2)
    with pytest.raises(SC.InvariantError):
        SC.check_no_corun([other, r])
    plain = dict(r)
    del plain["after"]
    with pytest.raises(SC.InvariantError):
        SC.check_no_corun([tr, plain])
    # a non-adjacent overlap (long subgraph, short one inside) is still found
    with pytest.raises(SC.InvariantError):
        SC.check_no_corun([_ev(0, 0, "train", 0, 100), _ev(0, 0, "train", 1, 2, k=1),
                           _ev(0, 3, "train", 50, 60)])


def test_checker_rejects_order_gap_and_duplicate():
    ok = [_ev(0, 0, "train", i, i + 1, it=i // 3, k=i % 3) for i in range(7)]
    SC.check_job_order(ok, {0: 3})
    gap = ok[:3] + ok[4:]
    with pytest.raises(SC.InvariantError):
        SC.check_job_order(gap, {0: 3})
    dup = ok[:4] + [dict(ok[3], t0=4.5, t1=4.9)] + ok[4:]
    with pytest.raises(SC.InvariantError):
        SC.check_job_order(dup, {0: 3})
    overlap = [dict(e) for e in ok]
    overlap[2]["t0"] = 1.5
    with pytest.raises(SC.InvariantError):
        SC.check_job_order(overlap, {0: 3})


def test_checker_rejects_long_wait_and_cut_rule():
    evs = [_ev(0, 0, "train", 0, 10), _ev(0, 0, "train", 10, 20, k=1),
           _ev(0, 1, "infer", 20, 21, arrival=5)]
    ok = [_ev(0, 0, "train", 0, 10), _ev(0, 1, "infer", 10, 11, arrival=5),
          _ev(0, 0, "train", 11, 21, k=1)]
    SC.check_preempt_latency(ok, 0)
    SC.check_cut_rule(ok)
    with pytest.raises(SC.InvariantError):
        SC.check_preempt_latency(evs, 0)  # waited 15 > longest subgraph 10
    evs2 = [_ev(0, 0, "train", 0, 4), _ev(0, 0, "train", 4, 8, k=1),
            _ev(0, 0, "train", 8, 12, k=2), _ev(0, 1, "infer", 12, 13, arrival=1)]
    with pytest.raises(SC.InvariantError):
        SC.check_preempt_latency(evs2, 0)
    with pytest.raises(SC.InvariantError):
        SC.check_cut_rule(evs)  # subgraph k=1 started at 10 after arrival 5


def test_preempt_latency_window_and_host_outliers():
    # two subgraphs of 10 in flight (window 2): a wait of 15 after the arrival is legal only
    # with window >= 2
    evs = [_ev(0, 0, "train", 0, 10), _ev(0, 0, "train", 10, 20, k=1),
           _ev(0, 1, "infer", 20, 21, arrival=5)]
    SC.check_preempt_latency(evs, 0, window=2)
    with pytest.raises(SC.InvariantError):
        SC.check_preempt_latency(evs, 0, window=1)
    # a request whose host dispatch decision (h0) came after ready + bound is a host outlier,
    # one dispatched in time but started late on the device is a violation
    late_dev = dict(_ev(0, 1, "infer", 40, 41, arrival=5), h0=6)
    late_host = dict(_ev(0, 1, "infer", 40, 41, arrival=5), h0=30)
    r = SC.preempt_latency_report([evs[0], late_dev], 1, window=1)
    assert len(r["violations"]) == 1 and not r["host_outliers"] and r["n"] == 1
    r = SC.preempt_latency_report([evs[0], late_host], 1, window=1)
    assert len(r["host_outliers"]) == 1 and not r["violations"]
    assert r["bound"][0] == 11 and r["waits"] == [35]
    # a request that recorded no device dependency (iter -1: nothing drained before it) is not
    # an I3 violation whatever its wait: it is dispatch / launch time
    no_dep = dict(_ev(0, 1, "infer", 40, 41, arrival=5), h0=6, iter=-1)
    r = SC.preempt_latency_report([evs[0], no_dep], 1, window=1)
    assert len(r["host_outliers"]) == 1 and not r["violations"]
    # the ready time is the previous request's end when requests queue back to back
    q = [_ev(0, 0, "train", 0, 10), _ev(0, 1, "infer", 10, 30, arrival=5),
         _ev(0, 2, "infer", 30, 31, arrival=6)]
    assert SC.preempt_latency_report(q, 0)["waits"] == [5, 0]


def test_device_view_uses_device_intervals():
    """Host intervals that overlap (a request observed before the subgraph's completion was
    observed) are disjoint on the device; a device overlap is still caught."""
    tr = dict(_ev(0, 0, "train", 0, 10), d0=2, d1=8)
    r = dict(_ev(0, 1 << 20, "infer", 5, 30, arrival=4), d0=9, d1=20, after=0)
    with pytest.raises(SC.InvariantError):
        SC.check_no_corun([tr, dict(r, after=None)])
    dv = SC.device_view([tr, r])
    assert (dv[0]["t0"], dv[0]["t1"], dv[0]["h0"]) == (2, 8, 0) and "after" not in dv[1]
    SC.check_no_corun(dv)
    with pytest.raises(SC.InvariantError):
        SC.check_no_corun(SC.device_view([tr, dict(r, d0=7)]))
    # events without a device interval pass through unchanged
    host = {"dev": -1, "job": 5, "kind": "host", "iter": 0, "k": -1, "t0": 1, "t1": 2}
    assert SC.device_view([host]) == [host]
    assert SC.device_view([dict(tr, d0=0)])[0]["t0"] == 0


def test_cut_rule_uses_dispatch_time():
    # S_1 dispatched (launch 9) before the arrival (10) but queued behind S_0 (t0 = 12):
    # allowed; a subgraph dispatched after the arrival is not
    ok = [_ev(0, 0, "train", 0, 12), dict(_ev(0, 0, "train", 12, 20, k=1), launch=9),
          _ev(0, 1, "infer", 20, 21, arrival=10)]
    SC.check_cut_rule(ok)
    bad = [_ev(0, 0, "train", 0, 12), dict(_ev(0, 0, "train", 12, 20, k=1), launch=11),
           _ev(0, 1, "infer", 20, 21, arrival=10)]
    with pytest.raises(SC.InvariantError):
        SC.check_cut_rule(bad)


def test_model_satisfies_invariants_host_and_peer():
    dur = [3.0, 1.0, 2.0, 0.5, 1.5]
    arr = list(D.poisson_arrivals(40, 0.2, seed=3))
    for tier in ("host", "peer"):
        evs = SC.simulate(dur, 30, arr, 0.7, tier=tier, swap_out=0.4, swap_in=0.4, gate=0.01)
        SC.check_all(evs, {0: len(dur)}, slack=0.02)
        trains = [e for e in evs if e["kind"] == "train"]
        assert len(trains) == 30 * len(dur)
        assert len([e for e in evs if e["kind"] == "infer"]) == 40


def test_model_closed_form_single_arrival():
    dur = [4.0, 4.0, 4.0]
    # arrival at 5 while S_1 runs [4, 8): served at 8 (cut k=2), done 9; host swap
    evs = SC.simulate(dur, 2, [5.0], 1.0, tier="host", swap_out=0.5, swap_in=2.0)
    inf = [e for e in evs if e["kind"] == "infer"][0]
    assert (inf["t0"], inf["t1"]) == (8.0, 9.0)
    nxt = [e for e in evs if e["kind"] == "train" and e["t0"] >= 8.0][0]
    assert (nxt["iter"], nxt["k"], nxt["t0"]) == (0, 2, 11.0)  # max(9, 8.5) + 2
    evs = SC.simulate(dur, 2, [5.0], 1.0, tier="peer", swap_out=0.5)
    nxt = [e for e in evs if e["kind"] == "train" and e["t0"] >= 8.0][0]
    assert (nxt["dev"], nxt["k"], nxt["t0"]) == (1, 2, 8.5)


# ---- I5: training priority (Fig. 7 scenario) ---------------

def test_priority_checker_rejects_lower_dispatch_and_late_start():
    prio = {0: 0, 1: 1}
    ok = [_ev(0, 0, "train", 0, 2), _ev(0, 0, "train", 2, 4, k=1),   # S_1 running at 3
          _ev(0, 1, "train", 4, 5), _ev(0, 1, "train", 5, 6, k=1),
          _ev(0, 0, "train", 6, 8, it=1)]
    SC.check_priority(ok, prio, {1: (0, 3)})
    SC.check_no_corun(ok)
    # a low-priority subgraph dispatched at 4.5 while job 1 is present on device 0
    bad = ok[:3] + [_ev(0, 0, "train", 4.5, 4.9, it=1)] + ok[3:4]
    with pytest.raises(SC.InvariantError):
        SC.check_priority(bad, prio, {1: (0, 3)})
    # ... but on another device (the peer it migrated to) it may run
    SC.check_priority(ok[:3] + [_ev(1, 0, "train", 4.5, 4.9, it=1)] + ok[3:4], prio, {1: (0, 3)})
    # job 1 waited 5 > one outstanding low subgraph (2) after submission
    late = [_ev(0, 0, "train", 0, 2), _ev(0, 0, "train", 2, 4, k=1),
            _ev(0, 1, "train", 8, 9), _ev(0, 1, "train", 9, 10, k=1)]
    with pytest.raises(SC.InvariantError):
        SC.check_priority(late, prio, {1: (0, 3)})
    SC.check_priority(late, prio, {1: (0, 3)}, window=3)
    # two lower-priority subgraphs dispatched before the submission still drained after it:
    # legal with an in-flight window of 2 only
    two = [_ev(0, 0, "train", 0, 2), dict(_ev(0, 0, "train", 2, 4, k=1), launch=1),
           dict(_ev(0, 0, "train", 4, 6, k=2), launch=2.5),
           _ev(0, 1, "train", 6, 7), _ev(0, 1, "train", 7, 8, k=1)]
    SC.check_priority(two, prio, {1: (0, 3)}, slack=10, window=2)
    with pytest.raises(SC.InvariantError):
        SC.check_priority(two, prio, {1: (0, 3)}, slack=10, window=1)


def test_priority_model_closed_form():
    lo, hi = [2.0, 2.0], [1.0, 1.0]
    # job 1 submitted at 3 while S_1 of job 0 runs [2, 4): cut at 4, job 1 runs [4, 8)
    evs = SC.simulate_priority(lo, 3, hi, 2, 3.0, tier="host", swap_out=0.5, swap_in=1.5)
    h = [e for e in evs if e["job"] == 1]
    assert (h[0]["t0"], h[-1]["t1"]) == (4.0, 8.0)
    nxt = [e for e in evs if e["job"] == 0 and e["t0"] >= 4.0][0]
    assert (nxt["dev"], nxt["iter"], nxt["k"], nxt["t0"]) == (0, 1, 0, 9.5)  # max(8, 4.5) + 1.5
    evs = SC.simulate_priority(lo, 3, hi, 2, 3.0, tier="peer", swap_out=0.5)
    nxt = [e for e in evs if e["job"] == 0 and e["t0"] >= 4.0][0]
    assert (nxt["dev"], nxt["iter"], nxt["k"], nxt["t0"]) == (1, 1, 0, 4.5)
    # migrate-back: the first job-0 boundary after 8 is 8.5 on device 1 -> device 0 at 9.0
    evs = SC.simulate_priority(lo, 4, hi, 2, 3.0, tier="peer", swap_out=0.5, home=True)
    back = [e for e in evs if e["job"] == 0 and e["t0"] >= 8.0]
    assert (back[0]["dev"], back[0]["t0"]) == (0, 9.0)


def test_priority_model_satisfies_invariants():
    lo, hi = [0.7, 1.3, 0.4, 2.1], [0.5, 0.9, 1.1]
    for tier, home in (("host", False), ("peer", False), ("peer", True)):
        for t_hi in (0.0, 3.3, 7.0, 100.0):
            evs = SC.simulate_priority(lo, 6, hi, 4, t_hi, tier=tier, swap_out=0.3,
                                       swap_in=0.3, home=home)
            SC.check_no_corun(evs)
            SC.check_job_order(evs, {0: len(lo), 1: len(hi)})
            SC.check_priority(evs, {0: 0, 1: 1}, {1: (0, t_hi)}, slack=1e-9)
            assert len([e for e in evs if e["job"] == 0]) == 6 * len(lo)
            assert len([e for e in evs if e["job"] == 1]) == 4 * len(hi)


def test_inference_weight_layouts_agree():
    """mlp_infer(wt=True) stores W_i as [N][K] (GEMM TB): with W^T it computes the same forward
    pass as the [K][N] layout (one rounding per op, so bit-identical)."""
    g0 = G.mlp_infer((9, 6, 4))
    g1 = G.mlp_infer((9, 6, 4), wt=True)
    p0 = D.init_state(g0, seed=2)
    p1 = {g1.tid(g0.tensors[i].name): (a.T.copy() if g0.tensors[i].name.startswith("W") else a)
          for i, a in p0.items()}
    x = D.infer_inputs(g0, 1)[0]
    assert R.run_inference(g0, p0, x).tobytes() == R.run_inference(g1, p1, x).tobytes()
