#!/usr/bin/env python
"""C5 (BASELINE.json config 5): migration sweep, 1 MB - 8 GB live sets x 4 size
mixes, concurrent GPU-pair migrations (0->1, 2->3, 4->5, 6->7 on 8 x B200) through NVSwitch.

One process per GPU (torchrun), pairs (2i, 2i+1) as in the N>1 bench:
each rank binds the synthetic state graph (every tensor PARAM, so cut 0's live set is the whole
list) to its own GPU and maps its partner's arena over CUDA IPC into a REMOTE slot.  For every
(size, mix, engine, direction), all senders start together behind a gloo barrier and move the
live set once into the partner's HBM (sf_probe_peer); the time is max over ranks of ...
per-rank durations; GB/s per pair and aggregate, against 900 GB/s per direction (nominal) and
770 GB/s (measured peer copy, B200_PROFILING.md).

  direction  uni  : even ranks send, odd ranks receive (4 concurrent one-way migrations)
             swap : both ranks of every pair send at once (bidirectional swap)
  engine     sm   : the peer-store descriptor walk (product path)
             ce_batch / ce_tensor / ce_single : copy-engine baselines (cudaMemcpyAsync per segment in
             2 MB groups, cudaMemcpyAsync per tensor = cudaMemcpyPeerAsync, one copy of the span)
             nccl : torch.distributed NCCL send / recv of one contiguous buffer of the same size
NVLink byte counters: run ONE rank's process under ncu (never a multi-rank command), e.g.
  ncu --metrics gpu__time_duration.sum,nvltx__bytes.sum,nvlrx__bytes.sum -k regex:mtcopy ...
(metric names as listed by `ncu --query-metrics`; unverified on the 1-GPU pool).

Launch: python -m torch.distributed.run --nnodes=1 --nproc-per-node 8 --master-addr 127.0.0.1 \
            --master-port 29511 scripts/bench_c5.py [--quick]
SF_BENCH_SAME_GPU=1 runs every rank on GPU 0 (functional check on a 1-GPU box: the "peer" is
the same HBM, so the numbers are NOT NVLink numbers and frac is null).
"""
import argparse
import json
import os
import sys
import time

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))
from bench_configs import sizes_for, state_graph  # noqa: E402

ENGINES = {"sm": 0, "ce_batch": 1, "ce_tensor": 2, "ce_single": 3}
NVL_NOMINAL, NVL_MEASURED = 900.0, 770.0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--quick", action="store_true", help="3 sizes, 2 mixes, 2 reps")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--out", default="gpurun_out/c5_sweep.jsonl")
    args = ap.parse_args()
    rank, world = int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    same = os.environ.get("SF_BENCH_SAME_GPU") == "1"
    if same:
        local = 0
    torch.cuda.set_device(local)
    if world < 2 or world % 2:
        raise SystemExit("bench_c5 needs an even number of ranks (GPU pairs)")
    dist.init_process_group("gloo" if same else "nccl",
                            **({} if same else {"device_id": torch.device("cuda", local)}))
    gloo = dist.new_group(backend="gloo") if not same else dist.group.WORLD
    import __graft_entry__
    if rank == 0:
        __graft_entry__.build()
    dist.barrier(group=gloo)
    __graft_entry__.build()
    from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime

    partner = rank ^ 1
    totals = [1 << 20, 4 << 20, 16 << 20, 64 << 20, 256 << 20, 1 << 30, 2 << 30, 4 << 30, 8 << 30]
    mixes = ["single", "resnet_hist", "uniform_1MB", "all_4KB"]
    reps = args.reps
    if args.quick:
        totals, mixes, reps = [1 << 20, 64 << 20, 1 << 30], ["single", "resnet_hist"], 2
    rows = []
    for mix in mixes:
        for tot in totals:
            if mix == "all_4KB" and tot > (512 << 20):
                continue  # 128k+ tensors: graph registration dominates (reading in DESIGN.md)
            sizes = sizes_for(tot, mix)
            g = state_graph(sizes)
            with Runtime([local, -1]) as rt:
                gh = rt.register(g)
                gh.partition()
                gh.bind(0, staging=False)
                objs = [None] * world
                dist.all_gather_object(objs, rt.export_arena(gh, 0), group=gloo)
                rt.import_arena(gh, 1, objs[partner])
                for direction in ("uni", "swap"):
                    sender = direction == "swap" or rank % 2 == 0
                    for eng, code in list(ENGINES.items()) + [("nccl", None)]:
                        ts, moved = [], 0
                        for r in range(reps + 1):
                            dist.barrier(group=gloo)
                            if eng == "nccl":
                                us, moved = nccl_once(tot, rank, partner, direction)
                            elif sender:
                                us, moved = rt.probe_peer(gh, 0, 1, 0, code)
                            else:
                                us = 0.0
                            if r > 0:
                                ts.append(us)
                        allv = [None] * world
                        dist.all_gather_object(allv, {"rank": rank, "sender": sender, "us": ts, "bytes": moved},
                                               group=gloo)
                        if rank == 0:
                            rows.append(summarise(allv, tot, mix, direction, eng, len(sizes), same))
                            print(json.dumps(rows[-1]), flush=True)
    if rank == 0:
        os.makedirs(os.path.dirname(args.out) or ".", exist_ok=True)
        with open(args.out, "w") as f:
            for r in rows:
                f.write(json.dumps(r) + "\n")
    dist.barrier(group=gloo)
    dist.destroy_process_group()


def nccl_once(nbytes, rank, partner, direction):
    """NCCL baseline: one contiguous buffer of the same size, send/recv within the pair."""
    buf = nccl_once.bufs.get(nbytes)
    if buf is None:
        nccl_once.bufs.clear()
        buf = nccl_once.bufs[nbytes] = (torch.empty(nbytes, dtype=torch.uint8, device="cuda"),
                                        torch.empty(nbytes, dtype=torch.uint8, device="cuda"))
    if os.environ.get("SF_BENCH_SAME_GPU") == "1":
        return 0.0, nbytes  # gloo cannot carry device tensors between ranks on one GPU
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    torch.cuda.synchronize()
    e0.record()
    ops = []
    if direction == "swap" or rank % 2 == 0:
        ops.append(dist.P2POp(dist.isend, buf[0], partner))
    if direction == "swap" or rank % 2 == 1:
        ops.append(dist.P2POp(dist.irecv, buf[1], partner))
    for w in dist.batch_isend_irecv(ops):
        w.wait()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3, nbytes


nccl_once.bufs = {}


def summarise(allv, tot, mix, direction, eng, n_tensors, same):
    senders = [a for a in allv if a["sender"] or eng == "nccl"]
    # per repetition: the slowest concurrent migration bounds the step (max over ranks)
    reps = len(senders[0]["us"]) if senders else 0
    step_us = [max(a["us"][r] for a in senders) for r in range(reps)] if reps else []
    moved = max(a["bytes"] for a in allv)
    per_pair = [moved / (np.median(a["us"]) * 1e-6) / 1e9 for a in senders if np.median(a["us"]) > 0]
    n_mig = len([a for a in allv if a["sender"]]) if eng != "nccl" else len(allv) // (1 if direction == "swap" else 2)
    agg = n_mig * moved / (np.median(step_us) * 1e-6) / 1e9 if step_us and np.median(step_us) > 0 else None
    med_pair = float(np.median(per_pair)) if per_pair else None
    return {"mix": mix, "live_bytes": int(moved), "requested_bytes": int(tot), "n_tensors": n_tensors,
            "direction": direction, "engine": eng, "n_migrations": n_mig,
            "step_us_median": float(np.median(step_us)) if step_us else None,
            "step_us_best": float(np.min(step_us)) if step_us else None,
            "per_migration_gbs_median": med_pair, "aggregate_gbs": agg,
            "frac_of_900": (med_pair / NVL_NOMINAL) if med_pair and not same else None,
            "frac_of_770_measured": (med_pair / NVL_MEASURED) if med_pair and not same else None,
            "same_gpu": same}


if __name__ == "__main__":
    main()
