"""GPU tests of host input stages:

- interleaving: a job's CPU executor (the built-in u8 image stage)
  prefetches on its own thread; two host-fed jobs on one slot keep invariant I1 on the GPU
  while one job's host stage overlaps the other's subgraphs;
- the session-slicing baseline (host_stage_inline + iteration granularity)
  computes the same trajectory;
- input reuse: one shared feed, an immutable device copy per batch, the
  members in lockstep round-robin (I6), the host stage run once per batch.

Bars: a host-fed job's state is bit-identical to the same graph fed by FEED ops from the
oracle's u8_pool (the stage's output for every batch) and within 1e-4 of the oracle run with
the stage as its ``feeds`` hook; preempted runs (host, peer, cut 0) are bit-identical.
"""
import numpy as np
import pytest

from oracle import feed as FD, graph as OG, runner as R, schedule as SC
from sf_inputs import data as D, graphs as G

pytestmark = pytest.mark.gpu
TOL = 1e-4
HOST = -1
BATCH, POOL, IMG_W, SEED = 64, 8, 28, 21


def rel(a, b):
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    return float(np.abs(a - b).max() / max(np.abs(b).max(), 1e-30))


@pytest.fixture(scope="module")
def P():
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_middleware_wur0hdh21_b200 import runtime as RT, _abi as A
    return RT, A


def images(seed=D.SEED_DATA):
    return D.u8_images(POOL * BATCH, 784, 10, seed=seed)


def fed_graph(widths=(784, 256, 10)):
    return G.mlp_train(widths, batch=BATCH, pool=POOL, host_fed=True)


def pool_graph(widths=(784, 256, 10)):
    return G.mlp_train(widths, batch=BATCH, pool=POOL)


def run_pool(P, widths, iters, imgs, labels, seed_init=D.SEED_INIT):
    """Reference GPU run: FEED ops over the oracle's stage output (u8_pool)."""
    RT, _ = P
    g = pool_graph(widths)
    px, py = FD.u8_pool(imgs, labels, BATCH, IMG_W, SEED)
    st = D.init_state(g, seed=seed_init)
    with RT.Runtime([0]) as rt:
        gh = rt.register(g)
        gh.partition()
        gh.bind(0)
        gh.load(0, {**st, g.tid("X_pool"): px, g.tid("Y_pool"): py})
        j = rt.start_training(gh, 0, iters, 0)
        rt.wait_job(j, 120)
        return {g.tensors[i].name: gh.read(0, i) for i in st}


def setup_fed(rt, g, feed, slots=1, prio=0, seed_init=D.SEED_INIT):
    gh = rt.register(g, priority=prio)
    gh.partition()
    for s in range(slots):
        gh.bind(s, staging=True, host_staging=True)
    st = D.init_state(g, seed=seed_init)
    gh.load(0, st)
    gh.attach_feed(feed, [g.tid("x"), g.tid("y")])
    return gh, st


@pytest.mark.parametrize("mode", ["prefetch", "inline", "preempted"])
def test_host_fed_job_equals_feed_op_pool_and_oracle(P, mode):
    RT, A = P
    imgs, labels = images()
    iters = 20
    base = run_pool(P, (784, 256, 10), iters, imgs, labels)
    g = fed_graph()
    kw = dict(host_stage_inline=True, iteration_granularity=True) if mode == "inline" else {}
    slots = 2 if mode == "preempted" else 1
    n = len(OG.partition(g))
    sched = sorted([(3, k, HOST) for k in range(n)] + [(5, 0, 1), (6, 2, 0), (8, 0, HOST), (9, 3, 1)]) \
        if mode == "preempted" else []
    with RT.Runtime([0] * slots, poison=mode == "preempted", **kw) as rt:
        f = rt.u8_feed(imgs, labels, BATCH, IMG_W, SEED, depth=3)
        gh, st = setup_fed(rt, g, f, slots)
        j = rt.start_training(gh, 0, iters, HOST, schedule=sched)
        rt.wait_job(j, 120)
        info = rt.job_info(j)
        got = {g.tensors[i].name: gh.read(info["dev"], i) for i in st}
        trace = rt.trace()
    if mode == "preempted":
        assert info["n_preemptions"] == len(sched)
    for name, a in base.items():
        assert got[name].tobytes() == a.tobytes(), name
    hosts = [e for e in trace if e["kind"] == "host"]
    assert len(hosts) >= iters
    xt, yt = g.tid("x"), g.tid("y")
    ref = R.run(g, iters, st, {}, keep_stagings=False,
                feeds=lambda it: dict(zip((xt, yt), FD.u8_stage(imgs, labels, it, BATCH, IMG_W, SEED))))
    for i, a in ref.state.items():
        if a.dtype == np.float32:
            assert rel(got[g.tensors[i].name], a) <= TOL, g.tensors[i].name


def test_interleaved_host_fed_jobs(P):
    """Two host-fed jobs on one slot: I1 on the GPU, per-job order, bitwise vs solo runs; one
    job's host stage overlaps the other job's GPU subgraphs (the point of PAPER.md:816-826)."""
    RT, A = P
    imgs, labels = images()
    imgs2, labels2 = images(seed=99)
    iters = 30
    wa, wb = (784, 256, 10), (784, 512, 10)
    base_a = run_pool(P, wa, iters, imgs, labels)
    base_b = run_pool(P, wb, iters, imgs2, labels2, seed_init=7)
    with RT.Runtime([0], max_inflight=2) as rt:
        fa = rt.u8_feed(imgs, labels, BATCH, IMG_W, SEED)
        fb = rt.u8_feed(imgs2, labels2, BATCH, IMG_W, SEED)
        ga, sta = setup_fed(rt, fed_graph(wa), fa)
        gb, stb = setup_fed(rt, fed_graph(wb), fb, seed_init=7)
        ja = rt.start_training(ga, 0, iters, 0)
        jb = rt.start_training(gb, 0, iters, 0)
        rt.wait_job(ja, 120)
        rt.wait_job(jb, 120)
        got_a = {ga.graph.tensors[i].name: ga.read(0, i) for i in sta}
        got_b = {gb.graph.tensors[i].name: gb.read(0, i) for i in stb}
        trace = rt.trace()
    for got, base in ((got_a, base_a), (got_b, base_b)):
        for name, a in base.items():
            assert got[name].tobytes() == a.tobytes(), name
    trains = [e for e in trace if e["kind"] == "train"]
    SC.check_no_corun(trains)
    SC.check_job_order(trains, {ja: len(OG.partition(ga.graph)), jb: len(OG.partition(gb.graph))},
                       start={ja: (0, 0), jb: (0, 0)})
    # the CPU executors run while the GPU is occupied: host stages overlap
    # training subgraphs (the prefetch of iteration i+2 starts when S_0 of iteration i retired,
    # while S_1.. run); which job's subgraph it overlaps depends on timing
    hosts = [e for e in trace if e["kind"] == "host"]
    overlaps = sum(1 for h in hosts for t in trains if t["t0"] < h["t1"] and h["t0"] < t["t1"])
    assert overlaps > 0


def test_shared_feed_lockstep_input_reuse(P):
    """Input reuse: two different models share one feed; the stage runs once per batch,
    members alternate per batch (I6), each is bit-identical to its own FEED-pool run."""
    RT, A = P
    imgs, labels = images()
    iters = 16
    wa, wb = (784, 256, 10), (784, 128, 10)
    base_a = run_pool(P, wa, iters, imgs, labels)
    base_b = run_pool(P, wb, iters, imgs, labels, seed_init=11)
    with RT.Runtime([0], max_inflight=2, poison=True) as rt:
        f = rt.u8_feed(imgs, labels, BATCH, IMG_W, SEED, depth=2, shared=True, dev=0)
        ga, sta = setup_fed(rt, fed_graph(wa), f, slots=1)
        gb, stb = setup_fed(rt, fed_graph(wb), f, slots=1, seed_init=11)
        ja = rt.start_training(ga, 0, iters, HOST)
        jb = rt.start_training(gb, 0, iters, HOST, schedule=[(4, 2, HOST), (9, 0, HOST)])
        rt.wait_job(ja, 120)
        rt.wait_job(jb, 120)
        got_a = {ga.graph.tensors[i].name: ga.read(0, i) for i in sta}
        got_b = {gb.graph.tensors[i].name: gb.read(0, i) for i in stb}
        ib = rt.job_info(jb)
        trace = rt.trace()
    assert ib["n_preemptions"] == 2
    for got, base in ((got_a, base_a), (got_b, base_b)):
        for name, a in base.items():
            assert got[name].tobytes() == a.tobytes(), name
    trains = [e for e in trace if e["kind"] == "train"]
    SC.check_no_corun(trains)
    SC.check_lockstep(trains, [ja, jb])
    hosts = [e for e in trace if e["kind"] == "host"]
    assert iters <= len(hosts) <= iters + 2  # once per batch (+ <= depth prefetched past the end)
