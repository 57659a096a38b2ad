"""Process-per-GPU peer migration over CUDA IPC, on one B200 (two processes, one device).

Each process owns slot 0 (cuda:0) and maps the partner's arena as REMOTE slot 1; every
batch-1 request preempts the job into the partner's arena with the peer-store kernel and the
partner adopts it (pairs.run_pair_steps).  The final state after T iterations must be
bit-identical to an unpreempted single-process GPU run of T iterations.
"""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu

T_ITERS = 3000


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=2)
    from paper_conf_middleware_wur0hdh21_b200.pairs import PairLink, RuntimeOps, run_pair_steps
    from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime
    from sf_inputs import data as D, graphs as G
    g, gi = G.mlp_train(), G.mlp_infer()
    rt = Runtime([0, -1], poison=True)
    gh = rt.register(g)
    gh.partition()
    gh.bind(0, host_staging=False)
    gh.load(0, D.datasets(g))
    if rank == 0:
        gh.load(0, D.init_state(g))
    ghi = rt.register(gi, priority=1)
    ghi.partition()
    ghi.bind(0, staging=False)
    ghi.load(0, D.init_state(gi, seed=D.SEED_INFER))
    link = PairLink()
    gh_blob = rt.export_arena(gh, 0)
    rt.import_arena(gh, 1, link.exchange_bytes(gh_blob))
    xs = torch.from_numpy(D.infer_inputs(gi, 4)).cuda()
    outs = torch.zeros(4, 1, 10, device="cuda")
    ops = RuntimeOps(rt, gh, ghi, 0, 1, [x.data_ptr() for x in xs], [o.data_ptr() for o in outs],
                     sub_ms=0.05, rng=np.random.default_rng(rank), iters=T_ITERS)
    if link.starts_holding:
        ops.start()
    S = run_pair_steps(link, ops, steps=6, warmup=0)
    state = None
    if S["holding_at_end"]:  # rank 0 holds the job again after an even number of steps
        rt.wait_job(ops.job, 120)
        info = rt.job_info(ops.job)
        assert info["state_name"] == "done", info
        state = {i: gh.read(0, i) for i in D.init_state(g)}
    dist.barrier()
    rt.close()
    q.put((rank, S, state))
    dist.destroy_process_group()


def test_ipc_pair_ping_pong_bit_identical():
    import __graft_entry__
    __graft_entry__.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(2):
        r, S, state = q.get(timeout=300)
        res[r] = (S, state)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    S0, st0 = res[0]
    S1, _ = res[1]
    assert len(S0["lat"]) == 3 and len(S1["lat"]) == 3
    assert all(x > 0 for x in S0["p2r"] + S1["p2r"])
    # reference: the same job, unpreempted, one process
    from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime
    from sf_inputs import data as D, graphs as G
    g = G.mlp_train()
    with Runtime([0]) as rt:
        gh = rt.register(g)
        gh.partition()
        gh.bind(0, host_staging=True)
        gh.load(0, {**D.init_state(g), **D.datasets(g)})
        j = rt.start_training(gh, 0, T_ITERS, -1)
        rt.wait_job(j, 300)
        ref = {i: gh.read(0, i) for i in D.init_state(g)}
    for i in ref:
        assert ref[i].tobytes() == st0[i].tobytes(), g.tensors[i].name
