"""Debug: where the p99 comes from (per-subgraph durations, per-request breakdown)."""
import sys, json, numpy as np
sys.path.insert(0, ".")
import bench
class A: pass
args = A(); args.batch = 8; args.spatial_div = 1; args.world = 1; args.defer = 1; args.update_chunks = 8
import torch
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime
S = bench.run_arm(args, 0, 200, 10, host_io=False, measure=False)
lat = np.array(S["lat"]); pre = np.array(S["pre"]); ks = np.array(S["cut_k"])
inf = lat - pre
print("lat p50/p90/p99/max", np.percentile(lat, [50, 90, 99, 100]).round(3))
print("pre p50/p90/p99/max", np.percentile(pre, [50, 90, 99, 100]).round(3))
print("inf p50/p90/p99/max", np.percentile(inf, [50, 90, 99, 100]).round(3))
idx = np.argsort(-lat)[:8]
for i in idx: print(f"  lat {lat[i]:.3f} pre {pre[i]:.3f} inf {inf[i]:.3f} cut_k {ks[i]}")
# per-subgraph durations from a fresh runtime trace (no requests)
g, gi = bench.build_workload(8, 1)
from sf_inputs import data as D
rt = Runtime([0]); gh = rt.register(g); gh.partition(update_chunks=8); gh.bind(0, host_staging=True)
gh.load(0, bench.workload_arrays(g, gi, (8, 1))[0])
j = rt.start_training(gh, 0, 3, -1); rt.wait_job(j, 60)
tr = [e for e in rt.trace() if e["kind"] == "train" and e["iter"] == 2]
d = sorted(((e["t1"] - e["t0"]) / 1e3, e["k"]) for e in tr)[::-1]
print("longest subgraphs (us, k):", [(round(a), b) for a, b in d[:8]], "sum", round(sum(a for a, _ in d)))
rt.close()
