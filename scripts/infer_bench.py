"""Inference-only latency (no training job): p50/p99 of submit->done for the C4 MLP."""
import json, sys, numpy as np, torch
sys.path.insert(0, ".")
import bench
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime
g, gi = bench.build_workload(8, 1)
arrs, arrs_i = bench.workload_arrays(g, gi, (8, 1))
import os
rt = Runtime([0], dispatch_spin_us=int(os.environ.get("SPIN", "0")),
             infer_l2_persist_bytes=int(float(os.environ.get("L2P_MB", "0")) * (1 << 20)))
ghi = rt.register(gi, 1); ghi.partition(); ghi.bind(0, staging=False); ghi.load(0, arrs_i)
x = torch.rand(1, 2048, device="cuda"); out = torch.empty(1, 1000, device="cuda")
lat, pre, dev, ho, lu = [], [], [], [], []
gap = float(os.environ.get("GAP_MS", "0")) * 1e-3
if os.environ.get("COPY"):  # background copy-engine traffic like a host-tier migration
    import threading
    dsrc = torch.empty(227 << 20, dtype=torch.uint8, device="cuda")
    hdst = torch.empty(227 << 20, dtype=torch.uint8).pin_memory()
    cs = torch.cuda.Stream()
    stop_copy = False
    cs2 = torch.cuda.Stream()
    dsrc2 = torch.empty_like(dsrc)
    hdst2 = torch.empty_like(hdst).pin_memory()
    def bg():
        while not globals()["stop_copy"]:
            mode = os.environ.get("COPY")
            if mode in ("h2d", "duplex"):
                with torch.cuda.stream(cs):
                    dsrc.copy_(hdst, non_blocking=True)
            if mode in ("d2h", "duplex"):
                with torch.cuda.stream(cs2):
                    hdst2.copy_(dsrc2, non_blocking=True)
            cs.synchronize()
            cs2.synchronize()
    th = threading.Thread(target=bg, daemon=True)
    th.start()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda") if os.environ.get("FLUSH") else None
rflush = torch.ones(512 << 20, dtype=torch.uint8, device="cuda") if os.environ.get("FLUSH") == "r" else None
import time
for i in range(int(sys.argv[1]) if len(sys.argv) > 1 else 300):
    if rflush is not None:  # clean cold L2: read-only sweep of 512 MB
        rflush.view(torch.int64).sum()
        torch.cuda.synchronize()
    elif flush is not None:  # dirty cold L2: 256 MB of writes
        flush.fill_(i & 255)
        torch.cuda.synchronize()
    if gap:
        t_end = time.perf_counter() + gap
        while time.perf_counter() < t_end:
            pass
    r = rt.submit(ghi, 0, x.data_ptr(), out.data_ptr()); tm = rt.wait(r, 300)
    if i >= 20:
        lat.append((tm["end_ns"] - tm["arrival_ns"]) * 1e-6)
        pre.append((tm["start_ns"] - tm["arrival_ns"]) * 1e-6)
        dev.append(tm["device_us"] * 1e-3)
        ho.append((tm["end_ns"] - tm["start_ns"]) * 1e-3 - tm["device_us"])
        lu.append(tm["launch_us"])
if os.environ.get("COPY"):
    stop_copy = True
    th.join()
rt.close()
print(json.dumps({"l2p_mb": os.environ.get("L2P_MB", "0"), "flush": os.environ.get("FLUSH"),
                  "max_persist_mb": torch.cuda.get_device_properties(0).persisting_l2_cache_max_size / 2**20
                  if hasattr(torch.cuda.get_device_properties(0), "persisting_l2_cache_max_size") else None,
                  "p50_ms": float(np.median(lat)), "p99_ms": float(np.percentile(lat, 99)),
                  "min_ms": float(np.min(lat)), "wake_p50_ms": float(np.median(pre)),
                  "device_p50_ms": float(np.median(dev)), "device_p99_ms": float(np.percentile(dev, 99)),
                  "copy": os.environ.get("COPY"), "spin": os.environ.get("SPIN", "0"),
                  "host_overhead_us_p50": float(np.median(ho)), "host_overhead_us_p99": float(np.percentile(ho, 99)),
                  "launch_us_p50": float(np.median(lu))}))
