"""Inference-only latency (no training job): p50/p99 of submit->done for the C4 MLP."""
import json, sys, numpy as np, torch
sys.path.insert(0, ".")
import bench
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime
g, gi = bench.build_workload(8, 1)
arrs, arrs_i = bench.workload_arrays(g, gi, (8, 1))
import os
rt = Runtime([0], dispatch_spin_us=int(os.environ.get("SPIN", "0")))
ghi = rt.register(gi, 1); ghi.partition(); ghi.bind(0, staging=False); ghi.load(0, arrs_i)
x = torch.rand(1, 2048, device="cuda"); out = torch.empty(1, 1000, device="cuda")
lat, pre, dev = [], [], []
for i in range(int(sys.argv[1]) if len(sys.argv) > 1 else 300):
    r = rt.submit(ghi, 0, x.data_ptr(), out.data_ptr()); tm = rt.wait(r, 300)
    if i >= 20:
        lat.append((tm["end_ns"] - tm["arrival_ns"]) * 1e-6)
        pre.append((tm["start_ns"] - tm["arrival_ns"]) * 1e-6)
        dev.append(tm["device_us"] * 1e-3)
rt.close()
print(json.dumps({"p50_ms": float(np.median(lat)), "p99_ms": float(np.percentile(lat, 99)),
                  "min_ms": float(np.min(lat)), "wake_p50_ms": float(np.median(pre)),
                  "device_p50_ms": float(np.median(dev))}))
