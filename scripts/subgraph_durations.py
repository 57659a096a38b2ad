"""Per-subgraph device durations of the bench's training job (C2 forest, MAX_OPS=1, 8 update
chunks), window 1 so every trace interval is one subgraph alone: which subgraphs bound the
drain a preemption waits for.  Prints the longest subgraphs with their ops."""
import json, sys
import numpy as np
sys.path.insert(0, ".")
import bench
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime

g, gi = bench.build_workload(8, 1)
arrs, _ = bench.workload_arrays(g, gi, (8, 1))
with Runtime([0], max_inflight=1) as rt:
    gh = rt.register(g)
    gh.partition("max_ops", 1, update_chunks=8)
    gh.bind(0, staging=True, host_staging=True)
    gh.load(0, arrs)
    job = rt.start_training(gh, 0, 12, -1)
    rt.wait_job(job, 300)
    tr = [e for e in rt.trace() if e["kind"] == "train" and e["iter"] >= 2]
    ranges = [gh.subgraph_range(k) for k in range(gh.n_subgraphs)]
d = {}
for e in tr:
    t0, t1 = (e["d0"], e["d1"]) if e.get("d0") and e.get("d1") else (e["t0"], e["t1"])  # device interval
    d.setdefault(e["k"], []).append((t1 - t0) * 1e-3)
rows = sorted(((float(np.median(v)), k) for k, v in d.items()), reverse=True)
tot = sum(m for m, _ in rows)
print(json.dumps({"n_subgraphs": len(rows), "iteration_us_sum_of_medians": round(tot, 1),
                  "p50_us": round(float(np.median([m for m, _ in rows])), 1)}))
for m, k in rows[:15]:
    b, e_ = ranges[k]
    ops = [g.ops[j] for j in range(b, e_)]
    desc = ", ".join(f"{o.type}:{[tuple((g.tensors[t].rows, g.tensors[t].cols)) for t in o.ins[:2]]}" for o in ops)
    print(f"k={k:3d} {m:7.1f} us  {desc[:150]}")
