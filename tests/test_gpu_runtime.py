"""GPU system tests of the preemption path through the C ABI (sf_* via the binding).

North_star bars:
  - migrated bytes bit-exact (cut-0 staging == oracle pack of the seeded state; mid-cut
    header / entries == oracle's, payloads within 1e-4 / exact for int32);
  - a GPU run preempted N times (host tier, peer tier ping-pong, poisoned released
    arenas) is bit-identical to the unpreempted GPU run;
  - GPU vs CPU oracle within relative 1e-4 (fp32) on the training trajectory and on
    inference;
  - the recorded schedule satisfies the paper's invariants (oracle/schedule.py).
Two logical slots on one physical B200 exercise the peer-store path (same kernel; a
different-GPU slot only changes the destination aperture to NVLink).
"""
import ctypes

import numpy as np
import pytest
import torch

from oracle import graph as OG, runner as R, schedule as SC, staging as S
from sf_inputs import data as D, graphs as G
from sf_inputs.ir import DATASET, F32, PERSISTENT_KINDS

pytestmark = pytest.mark.gpu
TOL = 1e-4
HOST = -1


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


def setup(P, g, slots=1, poison=False, host=True, auto=True, **kw):
    RT, A = P
    rt = RT.Runtime([0] * slots, poison=poison, auto_preempt=auto, **kw)
    gh = rt.register(g)
    gh.partition()
    st, ds = D.init_state(g), D.datasets(g)
    for s in range(slots):
        gh.bind(s, staging=True, host_staging=host)
        gh.load(s, ds)
    gh.load(0, st)
    return rt, gh, st, ds


def run_gpu(P, g, iters, schedule=(), slots=2, poison=False, **kw):
    rt, gh, st, ds = setup(P, g, slots=slots, poison=poison, **kw)
    job = rt.start_training(gh, 0, iters, HOST, schedule=schedule)
    rt.wait_job(job, 300)
    info = rt.job_info(job)
    dev = info["dev"]
    state = {i: gh.read(dev, i) for i in st}
    outs = {t.name: gh.read(dev, i) for i, t in enumerate(g.tensors) if t.kind == 8}
    trace = rt.trace()
    host_stg = gh.mem[0]["host_staging"]
    hs = host_stg.numpy().copy() if host_stg is not None else None
    rt.close()
    return state, outs, info, trace, hs


def assert_bitwise(a, b):
    for i in a:
        assert a[i].tobytes() == b[i].tobytes(), i


def test_c1_trajectory_vs_oracle(P):
    """20 iterations: longer fp32 ReLU trajectories cross kinks inside the fp32 error
    envelope (one mask flip at iteration 43 seen on B200, reading Q19); long
    horizons are covered by GPU-vs-GPU bit identity and by the ReLU-free C2 forest."""
    g = G.mlp_train()
    st, ds = D.init_state(g), D.datasets(g)
    state, outs, info, _, _ = run_gpu(P, g, 20, slots=1)
    ref = R.run(g, 20, st, ds, keep_stagings=False)
    for i in st:
        if st[i].dtype == np.float32:
            assert rel(state[i], ref.state[i]) <= TOL, g.tensors[i].name
        else:
            assert np.array_equal(state[i], ref.state[i])
    assert rel(outs["loss"], ref.outputs[-1]["loss"]) <= TOL


def test_c2_prefix_long_trajectory_vs_oracle(P):
    """The forest has no ReLU (smooth loss), so 30 iterations stay within 1e-4."""
    g = G.resnet50_forest(batch=1, spatial_div=4, max_layers=8)
    st, ds = D.init_state(g), D.datasets(g)
    state, outs, _, _, _ = run_gpu(P, g, 30, slots=1)
    ref = R.run(g, 30, st, ds, keep_stagings=False)
    for i in st:
        if st[i].dtype == np.float32:
            assert rel(state[i], ref.state[i]) <= TOL, g.tensors[i].name
    for name, v in outs.items():
        assert rel(v, ref.outputs[-1][name]) <= TOL, name


@pytest.mark.parametrize("W", [1, 2, 4])
def test_c1_preempted_at_every_cut_is_bit_identical(P, W):
    g = G.mlp_train()
    base, bo, _, _, _ = run_gpu(P, g, 60, max_inflight=W)
    n = len(OG.partition(g))
    sched = [(50, k, HOST) for k in range(n)] + [(52, k, 1 - (k % 2)) for k in range(1, n)]
    sched += [(55, 2, 1), (56, 4, 0), (57, 1, HOST), (58, 3, 1)]
    sched = sorted(sched)
    got, go, info, trace, _ = run_gpu(P, g, 60, schedule=sched, poison=True, max_inflight=W)
    assert info["n_preemptions"] >= 10
    assert_bitwise(base, got)
    assert bo["loss"].tobytes() == go["loss"].tobytes()
    SC.check_job_order([e for e in trace if e["kind"] == "train"], {0: n}, start={0: (0, 0)})


def test_random_schedule_ping_pong_resnet_prefix(P):
    g = G.resnet50_forest(batch=1, spatial_div=4, max_layers=12)
    n = len(OG.partition(g))
    sched = D.preemption_schedule(3, n, 15, targets=[1, 0, HOST], seed=11)
    base, _, _, _, _ = run_gpu(P, g, 3)
    got, _, info, _, _ = run_gpu(P, g, 3, schedule=sched, poison=True)
    assert info["n_preemptions"] >= 5, info
    print("preemptions", info["n_preemptions"], "re-parks", info["n_reparks"])
    assert_bitwise(base, got)
    ref = R.run(g, 3, D.init_state(g), D.datasets(g), keep_stagings=False)
    for i in ref.state:
        if ref.state[i].dtype == np.float32:
            assert rel(got[i], ref.state[i]) <= TOL, g.tensors[i].name


def test_update_chunk_cuts_bit_identical(P):
    g = G.resnet50_forest(batch=1, spatial_div=4, max_layers=10)
    RT, A = P

    def go(schedule):
        rt = RT.Runtime([0, 0], poison=True)
        gh = rt.register(g)
        gh.partition(update_chunks=4)
        st, ds = D.init_state(g), D.datasets(g)
        for s_ in (0, 1):
            gh.bind(s_, host_staging=True)
            gh.load(s_, ds)
        gh.load(0, st)
        job = rt.start_training(gh, 0, 2, HOST, schedule=schedule)
        rt.wait_job(job, 120)
        dev = rt.job_info(job)["dev"]
        out = {i: gh.read(dev, i) for i in st}
        n = gh.n_subgraphs
        rt.close()
        return out, n
    base, n = go(())
    got, _ = go([(0, n - 3, 1), (0, n - 2, HOST), (1, n - 1, 0)])
    assert_bitwise(base, got)


def test_cut0_staging_bytes_equal_oracle_pack(P):
    g = G.mlp_train()
    st, ds = D.init_state(g), D.datasets(g)
    _, _, _, _, hs = run_gpu(P, g, 1, schedule=[(0, 0, HOST)], slots=1)
    L = OG.live_set(g, OG.partition(g), 0)
    expect = S.pack(g, L, st, 0, 0)
    assert hs[:len(expect)].tobytes() == expect


def test_mid_cut_staging_header_and_payloads(P):
    g = G.mlp_train()
    st, ds = D.init_state(g), D.datasets(g)
    _, _, _, _, hs = run_gpu(P, g, 4, schedule=[(3, 3, HOST)], slots=1)
    ref = R.run(g, 4, st, ds, schedule=[(3, 3, R.HOST)])
    (_, _, _, buf) = ref.stagings[0]
    hdr, ents = S.parse(buf)
    ps = -(-(32 + 24 * len(ents)) // 256) * 256
    assert hs[:ps].tobytes() == buf[:ps]  # header + entries + zero pad: bit-exact
    gb = hs[:len(buf)].tobytes()
    for (tid, dt, off, nb) in ents:
        a = np.frombuffer(gb[off:off + nb], np.float32 if dt == F32 else np.int32)
        b = np.frombuffer(buf[off:off + nb], np.float32 if dt == F32 else np.int32)
        if dt == F32:
            assert rel(a, b) <= TOL, g.tensors[tid].name
        else:
            assert np.array_equal(a, b)
        pad = -(-nb // 256) * 256
        assert not any(gb[off + nb:off + pad])


def test_explicit_preempt_resume_peer_and_host(P):
    RT, A = P
    g = G.mlp_train()
    base, _, _, _, _ = run_gpu(P, g, 400)
    rt, gh, st, ds = setup(P, g, slots=2, poison=True)
    job = rt.start_training(gh, 0, 400, HOST)
    cut = rt.preempt(job, 1)
    assert cut["src_dev"] == 0 and cut["dst_dev"] == 1
    assert rt.job_info(job)["state_name"] in ("preempted", "migrating")
    with pytest.raises(A.SFError):
        rt.resume(job, 0)  # a peer-migrated job resumes on its target
    import time
    while rt.job_info(job)["state_name"] != "preempted":
        time.sleep(0.001)
    rt.resume(job, 1)
    cut2 = rt.preempt(job, HOST)
    while rt.job_info(job)["state_name"] != "preempted":
        time.sleep(0.001)
    rt.resume(job, 0)
    rt.wait_job(job, 120)
    info = rt.job_info(job)
    assert info["n_preemptions"] == 2 and info["dev"] == 0
    got = {i: gh.read(0, i) for i in st}
    for i in st:  # the ABI read (sf_read_tensor) sees the same bytes as the torch view
        assert rt.read_tensor(job, gh, i).tobytes() == got[i].tobytes()
    buf = ctypes.create_string_buffer(16)  # out-of-range tensor id: SF_EINVAL through the ABI
    assert A.lib().sf_read_tensor(rt.h, job, 10 ** 6, ctypes.cast(buf, ctypes.c_void_p), 16) == A.SF_EINVAL
    rt.close()
    assert_bitwise(base, got)


@pytest.mark.parametrize("W,early,gate", [(1, False, False), (2, False, False), (1, True, False),
                                          (2, True, False), (2, True, True)])
def test_inference_vs_oracle_and_auto_preemption_invariants(P, W, early, gate):
    """Auto-preemption by batch-1 requests: outputs vs the oracle, and the schedule
    invariants on the recorded trace.  With early_launch the chain is enqueued behind a
    device-side wait on the job's in-flight subgraphs; I1 then accepts the host-interval
    overlap only through that recorded dependency."""
    RT, A = P
    g = G.mlp_train()
    gi = G.mlp_infer()
    rt, gh, st, ds = setup(P, g, slots=1, max_inflight=W, early_launch=early, dispatch_spin_us=-1,
                           drain_gate=gate)
    ghi = rt.register(gi, priority=1)
    ghi.partition()
    ghi.bind(0, staging=False)
    sti = D.init_state(gi, seed=D.SEED_INFER)
    ghi.load(0, sti)
    # with the gate, enough requests that some land while a subgraph is queued behind the
    # running one (the hold path; where arrivals land is up to the OS scheduler)
    nreq = 60 if gate else 20
    xs = D.infer_inputs(gi, nreq)
    job = rt.start_training(gh, 0, 100000, HOST)
    import time
    outs, timings = [], []
    xin = torch.from_numpy(xs).cuda()
    out = torch.zeros(nreq, 1, 10, device="cuda")
    for r in range(nreq):
        time.sleep(0.002)
        req = rt.submit(ghi, 0, xin[r].data_ptr(), out[r].data_ptr())
        timings.append(rt.wait(req, 30))
    rt.stop_job(job)
    rt.wait_job(job, 60)
    info = rt.job_info(job)
    trace = rt.trace()
    n = gh.n_subgraphs
    rt.close()
    # a request that finds the device between two of the job's subgraphs (window 1 releases the
    # token at every boundary; the spinning dispatcher catches that gap) runs without a cut
    assert info["n_preemptions"] >= 8
    for r in range(nreq):
        assert rel(out[r].cpu().numpy(), R.run_inference(gi, sti, xs[r])) <= TOL
    assert sum(t["preempted_job"] == job for t in timings) >= 8
    evs = [dict(e, job=(1 if e["kind"] == "infer" else 0)) for e in trace]
    if early:
        assert sum("after" in e for e in evs) >= 10  # the early path was taken
    if not gate:  # host intervals (supersets) with the recorded device dependency; a subgraph
        SC.check_no_corun(evs)  # held by the drain gate spans later requests' host intervals
    # device intervals (GPU timeline, reading Q37): every train / infer event carries one
    dv = SC.device_view(evs)
    assert all(e["d0"] and e["d1"] >= e["d0"] for e in dv if e["kind"] in ("train", "infer"))
    SC.check_no_corun(dv)  # no "after" needed: the GPU never ran them together
    SC.check_job_order([e for e in dv if e["kind"] == "train"], {0: n}, start={0: (0, 0)})
    SC.check_cut_rule(dv)
    if gate:  # the queued subgraph was held behind (most) requests: only the running one drains
        held = sum(e["kind"] == "infer" and e["k"] == 1 for e in evs)
        # how often a request lands while a subgraph is queued behind the running one is up to
        # the OS scheduler here; test_drain_gate_holds_the_queued_subgraph forces the hold path
        print("drain gate held", held, "of", sum(e["kind"] == "infer" for e in evs))
    check_i3_device(dv, 1 if gate else W, early)


def check_i3_device(dv, W, early):
    """I3 on device intervals: wait <= W x longest subgraph + slack.  Slack: 20 us when the
    chain is enqueued behind the drain on the device (early launch: the GPU starts it the
    moment the dispatched subgraphs end); 50 us when the host launches it after observing the
    drain (event poll + token hand-off + first launch, Q32).  A request whose host
    dispatch decision itself came after ready + bound (the spinning dispatcher thread was
    descheduled) is a host outlier: at most max(2, 2%) of them, and never a device-side
    violation."""
    # the first request is a warm-up (first launches of the request kernels: lazy module load)
    first = min((e for e in dv if e["kind"] == "infer"), key=lambda e: e["arrival"])
    dv = [e for e in dv if e is not first]
    r = SC.preempt_latency_report(dv, slack=20e3 if early else 50e3, window=W)
    print("I3 bound us", {d: b / 1e3 for d, b in r["bound"].items()},
          "p50/max wait us", np.median(r["waits"]) / 1e3, max(r["waits"]) / 1e3,
          "host outliers", len(r["host_outliers"]))
    assert not r["violations"], [(e["arrival"], w) for e, w in r["violations"]]
    # host outliers are OS-scheduling events on the test box, not I3 violations (reading Q37):
    # two may land in a 20-request run (seen once in the round-2 refresh: 2 of 19)
    assert len(r["host_outliers"]) <= max(2, int(0.02 * r["n"]))


def test_error_paths(P):
    RT, A = P
    g = G.mlp_train()
    rt, gh, st, ds = setup(P, g, slots=2)
    job = rt.start_training(gh, 0, 50000, HOST)
    with pytest.raises(A.SFError) as e:
        rt.preempt(job, 0)
    assert e.value.status == A.SF_EINVAL
    with pytest.raises(A.SFError) as e:
        rt.resume(job, 1)
    assert e.value.status == A.SF_ESTATE
    rt.stop_job(job)
    rt.wait_job(job, 60)
    rt.close()
    # device budget: persistent state must fit
    rt = RT.Runtime([0], budget_bytes=1000)
    gh = rt.register(g)
    gh.partition()
    with pytest.raises(A.SFError) as e:
        gh.bind(0)
    assert e.value.status == A.SF_ENOMEM
    rt.close()
    # ops outside the fixed set are refused at registration
    from sf_inputs.ir import Graph, Op
    bad = G.mlp_train((2, 3, 2), batch=2, pool=1)
    bad.ops[3] = Op(42, bad.ops[3].ins, bad.ops[3].outs)
    rt = RT.Runtime([0])
    with pytest.raises(A.SFError) as e:
        rt.register(bad)
    assert e.value.status == A.SF_EUNSUPPORTED
    rt.close()


@pytest.mark.parametrize("U", [1, 3, 8])
def test_live_sets_match_oracle(P, U):
    RT, A = P
    rt = RT.Runtime([0])
    for g in (G.mlp_train(), G.resnet50_forest(batch=1, spatial_div=8),
              G.bert_chain(layers=2, hidden=8, inter=16, vocab=11, tokens=6, positions=6)):
        gh = rt.register(g)
        gh.partition(update_chunks=U)
        parts = OG.partition(g, update_chunks=U)
        assert gh.n_subgraphs == len(parts)
        for k in range(len(parts)):
            assert gh.subgraph_range(k) == parts[k]
            ids, nb = gh.live_set(k)
            L = OG.live_set(g, parts, k)
            assert ids == L and nb == OG.live_bytes(g, L)
            tot, offs = gh.staging_layout(k)
            eo, et = S.layout([g.tensors[i].nbytes for i in L])
            assert tot == et and offs == eo
    rt.close()


def _bert_mini(act="relu"):
    return G.bert_chain(layers=2, hidden=64, inter=128, vocab=301, tokens=32, positions=32, act=act)


@pytest.mark.parametrize("act", ["relu", "gelu"])
def test_c3_mini_vs_oracle_and_mid_cut_bitwise(P, act):
    """BERT-shaped chain with Adam (misaligned vocab 301 -> padded GEMM operands); with
    act="gelu" the FFN intermediate is GELU."""
    g = _bert_mini(act)
    st, ds = D.init_state(g), D.datasets(g)
    base, bo, _, _, _ = run_gpu(P, g, 3)
    ref = R.run(g, 3, st, ds, keep_stagings=False)
    for i in ref.state:
        if ref.state[i].dtype == np.float32:
            assert rel(base[i], ref.state[i]) <= TOL, g.tensors[i].name
        else:
            assert np.array_equal(base[i], ref.state[i])
    assert rel(bo["loss"], ref.outputs[-1]["loss"]) <= TOL
    cut = G.bert_mid_cut_phase(layers=2, after_layer=1)
    n = len(OG.partition(g))
    sched = [(0, cut, 1), (1, n - 1, HOST), (2, 3, 0)]
    got, go, info, _, _ = run_gpu(P, g, 3, schedule=sched, poison=True)
    assert info["n_preemptions"] == 3
    assert_bitwise(base, got)


@pytest.mark.slow
def test_c3_full_size_mid_cut_peer_bitwise_and_sampled_oracle(P):
    """BERT-large state (391 tensors x {w, m, v}, 4.02 GB) + activations at the layer-12 cut."""
    RT, A = P
    g = G.bert_chain()
    st, ds = D.init_state(g), D.datasets(g)
    cut = G.bert_mid_cut_phase()

    def go(schedule):
        rt = RT.Runtime([0, 0], poison=bool(schedule))
        gh = rt.register(g)
        info = gh.partition(update_chunks=8)
        for s_ in (0, 1):
            gh.bind(s_, staging=False, host_staging=False)
            gh.load(s_, ds)
        gh.load(0, st)
        job = rt.start_training(gh, 0, 1, 1, schedule=schedule)
        rt.wait_job(job, 600)
        ji = rt.job_info(job)
        dev = ji["dev"]
        out = {i: gh.read(dev, i) for i, t in enumerate(g.tensors) if t.kind in (0, 1, 2)}
        logits = gh.read(dev, g.tid("logits"))
        loss = gh.read(dev, g.tid("loss"))
        live = gh.live_set(cut)[1]
        rt.close()
        return out, logits, loss, ji, live, info

    base, logits, loss, _, live, info = go(())
    got, _, loss2, ji, _, _ = go([(0, cut, 1)])
    assert ji["n_preemptions"] == 1 and ji["dev"] == 1
    assert ji["migrated_bytes"] == live
    assert live > 4.0e9  # 4.02 GB of state + in-flight activations
    for i in base:
        assert base[i].tobytes() == got[i].tobytes(), g.tensors[i].name
    assert loss.tobytes() == loss2.tobytes()
    # sampled oracle: the forward chain is row-independent, so logits rows can be recomputed
    # one token at a time with the oracle's ops (fp64 accumulate, fp32 outputs)
    from oracle import ops as O
    from sf_inputs.ir import GEMM, BIAS_ACT, TA, TB
    rows = [0, 7, 255, 511]
    T = {i: a for i, a in st.items()}
    for r in rows:
        h = None
        for op in g.ops:
            if op.phase > G.bert_mid_cut_phase(after_layer=24):
                break
            if op.type == BIAS_ACT and h is None:  # x0 = pos + emb LN
                h = O.bias_act(T[op.ins[0]][r:r + 1], [T[b] for b in op.ins[1:]], False)
                continue
            if op.type == GEMM:
                z = O.gemm(h, T[op.ins[1]], None, op.flags)  # last GEMM: logits = h . word^T
            elif op.type == BIAS_ACT:
                h = O.bias_act(z, [T[b] for b in op.ins[1:]], True)
        assert rel(logits[r:r + 1], z) <= TOL, r
    # sampled post-update state: the head's word-embedding rows (the 128x256-tile TA dW GEMM
    # 30522x1024x512 through the padded-pitch path, then Adam at t = 1).  Its gradient
    # dword = dlogits^T . h_pool depends on forward quantities only, which are continuous in
    # rounding; gradients below a backward ReLU mask are not compared here, because a mask
    # decided on a pre-activation within fp32 rounding of 0 legitimately flips (Q19).
    ref_T = dict(st)
    ref_T.update(ds)
    shapes = {i: (t.rows, t.cols) for i, t in enumerate(g.tensors)}
    from sf_inputs.ir import SOFTMAX_CE
    for op in g.ops:
        O.apply_op(op, ref_T, shapes)
        if op.type == SOFTMAX_CE:
            break
    assert rel(loss, ref_T[g.tid("loss")]) <= TOL
    word, wm, wv = g.tid("word_embeddings"), g.tid("word_embeddings_m"), g.tid("word_embeddings_v")
    rng = np.random.default_rng(5)
    vs = sorted(set([0, 1, 127, 128, 255, 256, 30519, 30520, 30521]) |
                set(int(v) for v in rng.integers(0, 30522, 55)))
    gword = O.gemm(ref_T[g.tid("dlogits")][:, vs], ref_T[g.tid("pool_h")], None, TA)
    op_adam = next(op for op in g.ops if op.type == 8 and op.outs[0] == word)
    w1, m1, v1 = O.adam(st[word][vs], st[wm][vs], st[wv][vs], gword, st[g.tid("step")], *op_adam.f[:4])
    for name, got_t, ref_rows in (("w", base[word], w1), ("m", base[wm], m1), ("v", base[wv], v1)):
        assert rel(got_t[vs], ref_rows) <= TOL, name
    assert int(base[g.tid("step")][0, 0]) == 1


@pytest.mark.parametrize("host_mode,defer", [(1, 0), (1, 1), (0, 1)])
def test_host_modes_and_deferred_migration_bitwise(P, host_mode, defer):
    """Zero-copy host tier (pack straight into mapped pinned memory) and deferred migration
    give the same trajectory, bit for bit, as the unpreempted run."""
    g = G.mlp_train((784, 256, 10))
    base, _, _, _, _ = run_gpu(P, g, 30, slots=1)
    sched = [(5, k, HOST) for k in range(5)] + [(20, 2, HOST)]
    got, _, info, _, hs = run_gpu(P, g, 30, schedule=sched, slots=1, poison=True,
                                  host_mode=host_mode, defer_migration=bool(defer))
    assert info["n_preemptions"] == 6
    assert_bitwise(base, got)


@pytest.mark.parametrize("defer", [0, 1])
def test_duplex_host_round_trip_bitwise(P, defer):
    """Full-duplex host round trip (host_duplex): chunk c comes back H2D as soon as its D2H
    landed, with the device staging chunk poisoned in between and the released arena
    poisoned before the unpack.  A ~70 MB live set spans ~35 chunks.  The trajectory equals
    the unpreempted run bit for bit, and the parked pinned bytes equal those of a sequential
    (D2H, then H2D) round trip of the same schedule."""
    g = G.mlp_train((2048, 4096, 10), batch=64, pool=4)
    base, _, _, _, _ = run_gpu(P, g, 8, slots=1)
    sched = [(2, k, HOST) for k in range(5)] + [(5, 2, HOST)]
    got, _, info, _, hs = run_gpu(P, g, 8, schedule=sched, slots=1, poison=True,
                                  defer_migration=bool(defer), host_duplex=True)
    assert info["n_preemptions"] == 6
    assert_bitwise(base, got)
    _, _, info_s, _, hs_s = run_gpu(P, g, 8, schedule=sched, slots=1, poison=True,
                                    defer_migration=bool(defer), host_duplex=False)
    assert info_s["n_preemptions"] == 6
    assert hs.tobytes() == hs_s.tobytes()  # same parks in the same order: same pinned bytes


def _run_with_requests(P, g, gi, n_req, **kw):
    RT, A = P
    rt, gh, st, ds = setup(P, g, slots=1, **kw)
    ghi = rt.register(gi, priority=1)
    ghi.partition()
    ghi.bind(0, staging=False)
    ghi.load(0, D.init_state(gi, seed=D.SEED_INFER))
    job = rt.start_training(gh, 0, 100000, HOST)
    x = torch.from_numpy(D.infer_inputs(gi, 1)[0]).cuda()
    out = torch.zeros(1, 10, device="cuda")
    import time
    tms = []
    for _ in range(n_req):
        time.sleep(0.002)
        tms.append(rt.wait(rt.submit(ghi, 0, x.data_ptr(), out.data_ptr()), 30))
    rt.stop_job(job)
    rt.wait_job(job, 60)
    info = rt.job_info(job)
    trace = rt.trace()
    n = gh.n_subgraphs
    rt.close()
    return info, tms, trace, n


def test_iteration_granularity_cuts_only_at_iteration_boundaries(P):
    """Session time slicing baseline: requests wait for the iteration."""
    info, tms, trace, n = _run_with_requests(P, G.mlp_train(), G.mlp_infer(), 10,
                                             iteration_granularity=True)
    assert info["n_preemptions"] >= 5
    assert all(t["cut_k"] in (-1, 0) for t in tms)
    evs = [dict(e, job=(1 if e["kind"] == "infer" else 0)) for e in trace]
    SC.check_no_corun(evs)
    SC.check_job_order([e for e in evs if e["kind"] == "train"], {0: n}, start={0: (0, 0)})


def test_free_corun_baseline_never_preempts(P):
    """exclusive_gpu=0 (multi-threaded TF analogue)."""
    info, tms, trace, n = _run_with_requests(P, G.mlp_train(), G.mlp_infer(), 10, exclusive=False)
    assert info["n_preemptions"] == 0
    assert all(t["preempted_job"] == -1 for t in tms)


def test_remote_slot_errors(P):
    RT, A = P
    g = G.mlp_train()
    rt = RT.Runtime([0, -1])
    gh = rt.register(g)
    gh.partition()
    with pytest.raises(A.SFError) as e:
        gh.bind(1)  # remote slots are mapped, not bound
    assert e.value.status == A.SF_EINVAL
    with pytest.raises(A.SFError) as e:
        rt.import_arena(gh, 1, bytes(96))  # no local binding yet
    assert e.value.status in (A.SF_ESTATE, A.SF_EINVAL)
    gh.bind(0)
    blob = rt.export_arena(gh, 0)
    assert len(blob) == ctypes.sizeof(A.sf_ipc_arena) == 88
    with pytest.raises(A.SFError):
        rt.import_arena(gh, 0, blob)  # slot 0 is local
    rt.close()


_INFER_CHILD = r"""
import os, sys, numpy as np, torch
sys.path.insert(0, '.')
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime
from sf_inputs import data as D, graphs as G
g = G.mlp_train()
gi = G.mlp_infer((256, 512, 516, 128), name="infer_paths", wt=os.environ.get("WT") == "1")
rt = Runtime([0], dispatch_spin_us=int(sys.argv[2]))
gh = rt.register(g); gh.partition(); gh.bind(0, staging=True, host_staging=True)
gh.load(0, {**D.init_state(g), **D.datasets(g)})
ghi = rt.register(gi, 1); ghi.partition(); ghi.bind(0, staging=False)
ghi.load(0, D.init_state(gi, seed=D.SEED_INFER))
xs = D.infer_inputs(gi, 6)
job = rt.start_training(gh, 0, 100000, -1)
xin = torch.from_numpy(xs).cuda()
out = torch.zeros(6, 1, 128, device="cuda")
host_out = torch.zeros(6, 1, 128).pin_memory()
host_in = torch.from_numpy(xs).pin_memory()
for r in range(6):
    if r % 2:
        req = rt.submit(ghi, 0, host_in[r].data_ptr(), host_out[r].data_ptr())
        rt.wait(req, 60)
        out[r] = host_out[r].cuda()
    else:
        req = rt.submit(ghi, 0, xin[r].data_ptr(), out[r].data_ptr())
        rt.wait(req, 60)
rt.stop_job(job); rt.wait_job(job, 60); rt.close()
np.save(sys.argv[1], out.cpu().numpy())
"""


@pytest.mark.parametrize("env,spin", [({}, -1), ({"SF_GEMV_BLOCKED": "0"}, -1), ({"SF_CHAIN": "1"}, -1),
                                      ({"SF_CHAIN": "1", "SF_PDL": "0"}, 0),
                                      ({"SF_INFER_DIRECT": "0"}, 0), ({"SF_GEMV": "split"}, 2000),
                                      ({"SF_GEMV": "cluster", "SF_INFER_DIRECT": "0"}, -1),
                                      ({"WT": "1"}, -1), ({"WT": "1", "SF_INFER_DIRECT": "0"}, 0),
                                      ({"WT": "1", "SF_FUSE_SOFTMAX": "0", "SF_INFER_REDIRECT": "0",
                                        "SF_PDL": "0"}, 0),
                                      ({"SF_INFER_GRAPH": "1"}, -1), ({"SF_INFER_GRAPH": "1", "SF_CHAIN": "1"}, -1),
                                      ({"SF_INFER_GRAPH": "0"}, -1)],
                         ids=["default", "tma-gemv", "chain", "chain-nopdl", "graphs", "split-gemv", "cluster-gemv",
                              "rows", "rows-graphs", "rows-unfused", "req-graph", "req-graph-chain",
                              "direct-only"])
def test_inference_paths_vs_oracle(env, spin, tmp_path):
    """Every inference launch path (fused chain, PDL direct launches, captured graphs, the
    GEMV variants; device and pinned-host request buffers; spinning and blocking dispatcher)
    gives the oracle's forward pass while a training job is being preempted around it."""
    import os, subprocess, sys
    f = tmp_path / "out.npy"
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    subprocess.run([sys.executable, "-c", _INFER_CHILD, str(f), str(spin)], cwd=root,
                   env=dict(os.environ, **env), check=True, timeout=240)
    got = np.load(f)
    gi = G.mlp_infer((256, 512, 516, 128), name="infer_paths", wt=env.get("WT") == "1")
    sti = D.init_state(gi, seed=D.SEED_INFER)
    xs = D.infer_inputs(gi, 6)
    for r in range(6):
        assert rel(got[r], R.run_inference(gi, sti, xs[r])) <= TOL, (env, r)


@pytest.mark.parametrize("defer,duplex,early,gate", [(True, False, False, False), (False, False, False, False),
                                                    (True, True, False, False), (True, True, True, False),
                                                    (False, False, True, False), (True, True, True, True)])
def test_open_loop_requests_during_swap_in_are_bitwise(P, defer, duplex, early, gate):
    """Open-loop request stream (arrivals independent of the job's state): requests land
    while the parked state is being swapped back in, so the job is re-preempted before it
    ran anything (re-park without pack / D2H) or while its H2D + unpack is still in flight
    (the pack must wait for it).  With released arenas poisoned, any ordering mistake turns
    into NaN; the final state must equal the unpreempted GPU run bit for bit."""
    g = G.mlp_train((2048, 4096, 10), batch=64, pool=4)
    iters = 24 if early else 12  # early launch + duplex park less: run longer for enough cuts
    base = run_gpu(P, g, iters, slots=1)[0]
    RT, A = P
    rt, gh, st, ds = setup(P, g, slots=1, poison=True, defer_migration=defer, dispatch_spin_us=-1,
                           host_duplex=duplex, early_launch=early, max_inflight=2 if early else 1,
                           drain_gate=gate)
    gi = G.mlp_infer((256, 512, 12))
    ghi = rt.register(gi, priority=1)
    ghi.partition()
    ghi.bind(0, staging=False)
    ghi.load(0, D.init_state(gi, seed=D.SEED_INFER))
    x = torch.rand(1, 256, device="cuda")
    out = torch.empty(1, 12, device="cuda")
    job = rt.start_training(gh, 0, iters, HOST)
    rng = np.random.default_rng(7)
    import time
    reqs = []
    while rt.job_info(job)["state_name"] not in ("done", "failed") and len(reqs) < 4000:
        time.sleep(rng.exponential(3e-4))
        reqs.append(rt.submit(ghi, 0, x.data_ptr(), out.data_ptr()))
        if len(reqs) > 8:
            rt.wait(reqs[-9], 60)
    for r in reqs[-8:]:
        rt.wait(r, 60)
    rt.wait_job(job, 300)
    info = rt.job_info(job)
    got = {i: gh.read(0, i) for i in st}
    trace = [e for e in rt.trace() if e["kind"] in ("train", "infer")]
    rt.close()
    if not gate:
        SC.check_no_corun(trace)
    SC.check_no_corun(SC.device_view(trace))
    assert info["n_preemptions"] >= (3 if early else 5), info
    print("preemptions", info["n_preemptions"], "re-parks", info["n_reparks"])
    assert_bitwise(base, got)


# ---- copy-engine-only migration (SF_MIG_CE) ----------------------

def test_ce_migration_staging_bytes_equal_oracle_pack(P):
    """The CE host tier writes the same staging bytes as the pack kernel: the CPU writes
    header + zero padding, the copy engines the payloads (cut 0: exact oracle pack)."""
    RT, A = P
    g = G.mlp_train()
    st = D.init_state(g)
    _, _, _, _, hs = run_gpu(P, g, 1, schedule=[(0, 0, HOST)], slots=1,
                             migration_engine=A.SF_MIG_CE)
    L = OG.live_set(g, OG.partition(g), 0)
    expect = S.pack(g, L, st, 0, 0)
    assert hs[:len(expect)].tobytes() == expect
    # a mid cut after a different cut dirtied the staging: header + padding still exact
    ds = D.datasets(g)
    _, _, _, _, hs = run_gpu(P, g, 4, schedule=[(1, 4, HOST), (3, 3, HOST)], slots=1,
                             migration_engine=A.SF_MIG_CE)
    ref = R.run(g, 4, st, ds, schedule=[(1, 4, R.HOST), (3, 3, R.HOST)])
    buf = ref.stagings[-1][3]
    hdr, ents = S.parse(buf)
    ps = -(-(32 + 24 * len(ents)) // 256) * 256
    gb = hs[:len(buf)].tobytes()
    assert gb[:ps] == buf[:ps]
    for (tid, dt, off, nb) in ents:
        pad = -(-nb // 256) * 256
        assert not any(gb[off + nb:off + pad])


@pytest.mark.parametrize("W", [1, 2])
def test_ce_migration_host_and_peer_bitwise(P, W):
    """Copy-engine-only migration on both tiers, every cut, poisoned released arenas:
    bit-identical to the unpreempted run; resnet prefix (many small tensors) as well."""
    RT, A = P
    g = G.mlp_train()
    base, _, _, _, _ = run_gpu(P, g, 30, max_inflight=W)
    n = len(OG.partition(g))
    sched = sorted([(5, k, HOST) for k in range(n)] + [(8, k, 1 - (k % 2)) for k in range(1, n)]
                   + [(12, 0, 0), (15, 2, 1), (16, 3, HOST), (20, 1, 0)])
    got, _, info, _, _ = run_gpu(P, g, 30, schedule=sched, poison=True, max_inflight=W,
                                 migration_engine=A.SF_MIG_CE)
    assert info["n_preemptions"] >= 10
    assert_bitwise(base, got)
    gr = G.resnet50_forest(batch=1, spatial_div=4, max_layers=12)
    nr = len(OG.partition(gr))
    sched = D.preemption_schedule(3, nr, 10, targets=[1, 0, HOST], seed=5)
    base, _, _, _, _ = run_gpu(P, gr, 3)
    got, _, info, _, _ = run_gpu(P, gr, 3, schedule=sched, poison=True,
                                 migration_engine=A.SF_MIG_CE)
    assert info["n_preemptions"] >= 4
    assert_bitwise(base, got)


# ---- GELU layers ----------------------------------------------------

def test_gelu_mlp_trajectory_vs_oracle_and_preempted_bitwise(P):
    """A GELU MLP (u_i kept for the backward, so it is live across the cuts between the
    layer's forward and its backward): 20 iterations vs the oracle at 1e-4, and preempted at
    every cut (host + peer, poisoned arenas) bit-identical to the unpreempted GPU run."""
    g = G.mlp_train(act="gelu")
    st, ds = D.init_state(g), D.datasets(g)
    got, outs, _, _, _ = run_gpu(P, g, 20)
    ref = R.run(g, 20, st, ds, keep_stagings=False)
    for i in ref.state:
        if ref.state[i].dtype == np.float32:
            assert rel(got[i], ref.state[i]) <= TOL, g.tensors[i].name
    assert rel(outs["loss"], ref.outputs[-1]["loss"]) <= TOL
    n = len(OG.partition(g))
    u1 = g.tid("u1")
    assert any(u1 in OG.live_set(g, OG.partition(g), k) for k in range(n))
    sched = sorted([(5, k, HOST) for k in range(n)] + [(8, k, 1 - (k % 2)) for k in range(1, n)])
    base, _, _, _, _ = run_gpu(P, g, 12)
    got, _, info, _, _ = run_gpu(P, g, 12, schedule=sched, poison=True)
    assert info["n_preemptions"] >= 8
    assert_bitwise(base, got)


@pytest.mark.parametrize("early,gate", [(False, False), (True, False), (True, True)])
def test_requests_chase_peer_migrations_bitwise(P, early, gate):
    """Auto-preemption to a peer slot: requests are submitted to the slot the job runs on.
    The first one migrates the job to slot 1 through the peer-store walk (poisoned released
    arena); it stays there, so later requests cut it at a boundary and it
    yields in place.  With early_launch the chain waits on the device for the job's
    dispatched subgraphs.  Final state bit-identical to the unpreempted run; requests within
    1e-4 of the oracle; invariant 1 on the trace."""
    import time
    g = G.mlp_train((784, 512, 10), batch=64, pool=4)
    gi = G.mlp_infer()
    iters = 1500
    base = run_gpu(P, g, iters, slots=1)[0]
    RT, A = P
    rt, gh, st, ds = setup(P, g, slots=2, poison=True, early_launch=early, max_inflight=2,
                           dispatch_spin_us=-1, drain_gate=gate)
    ghi = rt.register(gi, priority=1)
    ghi.partition()
    sti = D.init_state(gi, seed=D.SEED_INFER)
    for s in range(2):
        ghi.bind(s, staging=False)
        ghi.load(s, sti)
    xs = D.infer_inputs(gi, 6)
    xin = torch.from_numpy(xs).cuda()
    out = torch.zeros(6, 1, 10, device="cuda")
    job = rt.start_training(gh, 0, iters, 1)
    tims = []
    for r in range(6):
        time.sleep(0.002)
        info = rt.job_info(job)
        if info["state_name"] != "running":
            break
        tims.append(rt.wait(rt.submit(ghi, info["dev"], xin[r].data_ptr(), out[r].data_ptr()), 30))
    rt.wait_job(job, 120)
    info = rt.job_info(job)
    got = {i: gh.read(info["dev"], i) for i in st}
    trace = [e for e in rt.trace() if e["kind"] in ("train", "infer")]
    rt.close()
    assert info["n_preemptions"] >= 1 and info["dev"] == 1, info
    assert_bitwise(base, got)
    assert len(tims) >= 3
    for r in range(len(tims)):
        assert rel(out[r].cpu().numpy(), R.run_inference(gi, sti, xs[r])) <= TOL
    if not gate:
        SC.check_no_corun(trace)
    SC.check_no_corun(SC.device_view(trace))


def test_device_clock_mapping_is_consistent(P):
    """Device intervals on the host clock (reading Q37): on an idle device a request's chain
    starts after its submission and within a launch of the host dispatch, and ends before the
    host observed its completion; repeated over ~1 s so several clock anchors are used."""
    import time
    RT, A = P
    gi = G.mlp_infer((2048, 4096, 4096, 1000), name="infer_mlp_29M")
    with RT.Runtime([0], dispatch_spin_us=-1) as rt:
        ghi = rt.register(gi, priority=1)
        ghi.partition()
        ghi.bind(0, staging=False)
        ghi.load(0, D.init_state(gi, seed=D.SEED_INFER))
        x = torch.rand(1, 2048, device="cuda")
        out = torch.empty(1, 1000, device="cuda")
        rows = []
        for i in range(60):
            time.sleep(0.02)
            tm = rt.wait(rt.submit(ghi, 0, x.data_ptr(), out.data_ptr()), 30)
            rows.append(tm)
        trace = [e for e in rt.trace() if e["kind"] == "infer"]
    rows, trace = rows[2:], trace[2:]  # warm-up launches
    lead = [(t["start_ns"] - t["arrival_ns"]) * 1e-3 for t in rows]
    tail = [(e["t1"] - e["d1"]) * 1e-3 for e in trace]
    print("start - submit us p50/min/max", np.median(lead), min(lead), max(lead),
          "| host completion - device end us p50/min", np.median(tail), min(tail))
    # the mapping is good to a few us (anchor bracket + one-sided host observation delay)
    assert min(lead) > -5.0 and np.median(lead) < 60.0
    assert min(tail) > -5.0 and np.median(tail) < 60.0
    for e in trace:
        assert e["d1"] >= e["d0"] and (e["d1"] - e["d0"]) * 1e-3 < 500


@pytest.mark.skipif(not torch.cuda.is_available() or torch.cuda.device_count() < 2,
                    reason="needs two physical GPUs (peer store over NVLink)")
@pytest.mark.parametrize("W", [1, 2])
def test_two_device_peer_migration_bit_identical(P, W):
    """Slots on two DISTINCT devices (cuda:0, cuda:1) in one process: the peer-store walk
    writes across NVLink, the cross-device event waits order unpack/resume, and a run
    preempted at every cut (both directions + host tier, poisoned arenas) is bit-identical
    to the unpreempted single-device run (§3.3, 'no work is lost')."""
    RT, A = P
    g = G.mlp_train()
    base, bo, _, _, _ = run_gpu(P, g, 60, slots=1, max_inflight=W)
    n = len(OG.partition(g))
    sched = [(50, k, 1 - (k % 2)) for k in range(n)] + [(53, k, HOST) for k in range(1, n)]
    sched += [(55, 2, 1), (56, 4, 0), (57, 1, 1)]
    rt = RT.Runtime([0, 1], poison=True, max_inflight=W)
    gh = rt.register(g)
    gh.partition()
    st, ds = D.init_state(g), D.datasets(g)
    for s in range(2):
        gh.bind(s, staging=True, host_staging=True)
        gh.load(s, ds)
    gh.load(0, st)
    job = rt.start_training(gh, 0, 60, HOST, schedule=sorted(sched))
    rt.wait_job(job, 300)
    info = rt.job_info(job)
    got = {i: gh.read(info["dev"], i) for i in st}
    rt.close()
    assert info["n_preemptions"] >= 10, info
    assert_bitwise(base, got)


def test_drain_gate_holds_the_queued_subgraph(P):
    """Drain gate (reading Q38), forced: subgraphs of ~0.5 ms (4096-wide MLP, batch
    4096) with a count-only window of 2, so a request arriving mid-subgraph always finds one
    subgraph running and one queued.  The queued one must be held (the request runs right after
    the running one: the trace marks it k = 1), the job migrates at its next boundary, and the
    final state is bit-identical to the run without requests."""
    RT, A = P
    g = G.mlp_train(widths=(4096, 4096, 4096, 10), batch=4096, pool=2)
    gi = G.mlp_infer()
    sti = D.init_state(gi, seed=D.SEED_INFER)
    xs = D.infer_inputs(gi, 6)
    results = []
    for with_requests in (False, True):
        rt, gh, st, ds = setup(P, g, slots=1, max_inflight=2, early_launch=True, dispatch_spin_us=-1,
                               drain_gate=True, inflight_budget_us=0)
        ghi = rt.register(gi, priority=1)
        ghi.partition()
        ghi.bind(0, staging=False)
        ghi.load(0, sti)
        job = rt.start_training(gh, 0, 60, HOST)  # ~3.7 ms per iteration alone
        out = torch.zeros(6, 1, 10, device="cuda")
        if with_requests:
            import time
            xin = torch.from_numpy(xs).cuda()
            time.sleep(0.005)
            for r in range(6):
                time.sleep(0.03)  # the job is back on the device (host round trip ~15 ms)
                rt.wait(rt.submit(ghi, 0, xin[r].data_ptr(), out[r].data_ptr()), 30)
        rt.wait_job(job, 120)
        info = rt.job_info(job)
        state = {i: gh.read(info["dev"], i) for i in st}
        trace = rt.trace()
        rt.close()
        results.append((state, info, trace, out.cpu().numpy()))
    (base, _, _, _), (got, info, trace, outs) = results
    assert_bitwise(base, got)
    infer = [e for e in trace if e["kind"] == "infer"]
    held = sum(e["k"] == 1 for e in infer)
    print("held", held, "of", len(infer), "preemptions", info["n_preemptions"])
    assert held >= 3, (held, len(infer))
    for r in range(6):
        assert rel(outs[r], R.run_inference(gi, sti, xs[r])) <= TOL
    dv = SC.device_view([dict(e, job=(1 if e["kind"] == "infer" else 0)) for e in trace])
    SC.check_no_corun(dv)


_C4_CHILD = r"""
import os, sys, numpy as np, torch
sys.path.insert(0, '.')
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime
from sf_inputs import data as D, graphs as G
gi = G.mlp_infer((2048, 4096, 4096, 1000), name="infer_mlp_29M")
xs = D.infer_inputs(gi, 4)
with Runtime([0], dispatch_spin_us=-1) as rt:
    ghi = rt.register(gi, 1); ghi.partition(); ghi.bind(0, staging=False)
    ghi.load(0, D.init_state(gi, seed=D.SEED_INFER))
    out = torch.zeros(4, 1, 1000, device="cuda")
    host_in = torch.from_numpy(xs).pin_memory()
    host_out = torch.zeros(4, 1, 1000).pin_memory()
    xin = torch.from_numpy(xs).cuda()
    for r in range(4):
        if r % 2:
            rt.wait(rt.submit(ghi, 0, host_in[r].data_ptr(), host_out[r].data_ptr()), 60)
            out[r] = host_out[r].cuda()
        else:
            rt.wait(rt.submit(ghi, 0, xin[r].data_ptr(), out[r].data_ptr()), 60)
np.save(sys.argv[1], out.cpu().numpy())
"""


@pytest.mark.parametrize("env", [{}, {"SF_GEMV_HEAD": "0"}, {"SF_GEMV_HEAD": "1"}, {"SF_INFER_GRAPH": "0"},
                                 {"SF_INFER_GRAPH": "1"}, {"SF_CHAIN": "1"}],
                         ids=["default", "cluster-all", "cluster-wide-layers", "direct-only", "graph-always",
                              "fold-chain"])
def test_c4_inference_model_vs_oracle(env, tmp_path):
    """The bench's preempter model (2048-4096-4096-1000 MLP + softmax) through
    the request path the bench times (blocked GEMVs; the cluster-free head over 8-column blocks;
    the captured request graph) against the oracle's forward pass, device and pinned-host
    request buffers alike."""
    import os, subprocess, sys
    f = tmp_path / "out.npy"
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    subprocess.run([sys.executable, "-c", _C4_CHILD, str(f)], cwd=root, env=dict(os.environ, **env),
                   check=True, timeout=240)
    got = np.load(f)
    gi = G.mlp_infer((2048, 4096, 4096, 1000), name="infer_mlp_29M")
    sti = D.init_state(gi, seed=D.SEED_INFER)
    xs = D.infer_inputs(gi, 4)
    for r in range(4):
        assert rel(got[r], R.run_inference(gi, sti, xs[r])) <= TOL, (env, r)
