#!/usr/bin/env python
"""Interleaving and input reuse (Figs. 8-10).

Two jobs share one B200 slot; each iteration starts with the built-in host stage (u8 image
decode + seeded flip, reading Q27) on a pool of synthetic 28x28 images.  Completion time of
N iterations of both jobs under:
  slicing      session-based time slicing (Gandiva-like baseline): the
               host stage runs inline while the job holds the device, one iteration per turn
               (host_stage_inline + iteration_granularity);
  interleave   SwitchFlow: each job's stage prefetches on its own thread and never holds the
               device; GPU subgraphs of the two jobs alternate at subgraph boundaries
               (Fig. 10);
  reuse        SwitchFlow input reuse: one shared feed (stage once per batch, immutable device
               copy) and the two models in lockstep round-robin (Figs. 8-9).
Workloads: "train" = MLP 784-1024-1024-10 training (SGD-momentum) and "infer" = the same
MLP's forward pass as a job (softmax outputs), batch 128 and 512.
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime  # noqa: E402
from sf_inputs import data as D, graphs as G  # noqa: E402
from sf_inputs.ir import BIAS_ACT, F32, GEMM, INPUT, LABEL, OUTPUT, PARAM, RELU, SOFTMAX, ACT, Graph  # noqa: E402

POOL, IMG_W, SEED = 8, 28, 21
WIDTHS = (784, 1024, 1024, 10)


def infer_job_graph(widths, batch):
    """Forward-only job: host-fed x (and an unused label, so the feed is the same) ->
    Linear+ReLU ... -> softmax probabilities."""
    g = Graph("infer_job")
    x = g.add("x", batch, widths[0], F32, INPUT)
    g.add("y", batch, 1, 1, LABEL)
    h = x
    for i in range(len(widths) - 1):
        W = g.add(f"W{i+1}", widths[i], widths[i + 1], F32, PARAM)
        b = g.add(f"b{i+1}", 1, widths[i + 1], F32, PARAM)
        z = g.add(f"z{i+1}", batch, widths[i + 1], F32, ACT)
        g.op(GEMM, [h, W], [z], phase=i)
        hn = g.add(f"h{i+1}", batch, widths[i + 1], F32, ACT)
        last = i == len(widths) - 2
        g.op(BIAS_ACT, [z, b], [hn], flags=0 if last else RELU, phase=i)
        h = hn
    p = g.add("probs", batch, widths[-1], F32, OUTPUT)
    g.op(SOFTMAX, [h], [p], phase=len(widths) - 2)
    return g


def graph(kind, batch):
    if kind == "train":
        return G.mlp_train(WIDTHS, batch=batch, pool=POOL, host_fed=True)
    return infer_job_graph(WIDTHS, batch)


def run(mode, kind, batch, iters):
    imgs, labels = D.u8_images(POOL * batch, 784, 10, seed=1)
    kw = dict(max_inflight=2)
    if mode == "slicing":
        kw.update(host_stage_inline=True, iteration_granularity=True)
    with Runtime([0], **kw) as rt:
        if mode == "reuse":
            f = rt.u8_feed(imgs, labels, batch, IMG_W, SEED, depth=2, shared=True, dev=0)
            feeds = [f, f]
        else:
            feeds = [rt.u8_feed(imgs, labels, batch, IMG_W, SEED, depth=2) for _ in range(2)]
        ghs = []
        for j in range(2):
            g = graph(kind, batch)
            gh = rt.register(g)
            gh.partition()
            gh.bind(0, staging=False)
            gh.load(0, D.init_state(g, seed=3 + j))
            gh.attach_feed(feeds[j], [g.tid("x"), g.tid("y")])
            ghs.append(gh)
        t0 = time.perf_counter()
        jobs = [rt.start_training(gh, 0, iters, 0) for gh in ghs]
        for j in jobs:
            rt.wait_job(j, 600)
        dt = time.perf_counter() - t0
        tr = rt.trace()
    hosts = [e for e in tr if e["kind"] == "host"]
    trains = [e for e in tr if e["kind"] == "train"]
    host_us = sum(e["t1"] - e["t0"] for e in hosts) / max(1, len(hosts)) * 1e-3
    gpu_busy = sum(e["t1"] - e["t0"] for e in trains) * 1e-9
    return {"mode": mode, "kind": kind, "batch": batch, "iters_per_job": iters,
            "seconds": dt, "iters_per_s": 2 * iters / dt, "host_stage_us_mean": host_us,
            "host_stages": len(hosts), "gpu_busy_frac": gpu_busy / dt,
            "host_stage_threads": 1 if mode == "reuse" else 2,
            "host_stage_cpu_s": sum(e["t1"] - e["t0"] for e in hosts) * 1e-9}


def main():
    iters = int(os.environ.get("FEED_ITERS", "200"))
    out = []
    for kind in ("infer", "train"):
        for batch in (128, 512):
            rows = {m: run(m, kind, batch, iters) for m in ("slicing", "interleave", "reuse")}
            for m in ("interleave", "reuse"):
                rows[m]["speedup_vs_slicing"] = rows["slicing"]["seconds"] / rows[m]["seconds"]
            for r in rows.values():
                print(json.dumps(r), flush=True)
                out.append(r)
    os.makedirs("gpurun_out", exist_ok=True)
    json.dump(out, open("gpurun_out/feeds.json", "w"), indent=1)


if __name__ == "__main__":
    main()
