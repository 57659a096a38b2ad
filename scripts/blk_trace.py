"""Per-layer device timeline of the blocked-GEMV inference chain (C4 MLP, batch 1) through the
runtime's request path, L2 dirtied (256 MB write) before each request: globaltimer marks per
layer {first/last CTA start, first/last return from griddepcontrol.wait, first/last CTA done
streaming, last CTA end} relative to the first CTA start of layer 0 (sf_debug_chain_trace)."""
import ctypes as C, json, os, sys
import numpy as np, torch
os.environ.setdefault("SF_CHAIN", "0")  # the per-layer GEMV chain (the fused kernel has its own trace)
os.environ.setdefault("SF_INFER_GRAPH", "0")  # direct launches: the captured graph has no trace pointer
sys.path.insert(0, ".")
import bench
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime
from paper_conf_middleware_wur0hdh21_b200._abi import lib

g, gi = bench.build_workload(8, 1)
arrs, arrs_i = bench.workload_arrays(g, gi, (8, 1))
rt = Runtime([0], dispatch_spin_us=-1)
ghi = rt.register(gi, 1); ghi.partition(); ghi.bind(0, staging=False); ghi.load(0, arrs_i)
host_io = os.environ.get("HOSTIO") == "1"
x = torch.rand(1, 2048, device="cuda"); out = torch.empty(1, 1000, device="cuda")
if host_io:
    x = x.cpu().pin_memory(); out = out.cpu().pin_memory()
tr = torch.zeros(3 * 8, dtype=torch.int64, device="cuda")
init = torch.zeros(3, 8, dtype=torch.int64)
init[:, [0, 2, 4]] = -1  # mins start at ~0ull
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
lib().sf_debug_chain_trace(C.c_void_p(tr.data_ptr()))
rows, dev = [], []
for i in range(int(sys.argv[1]) if len(sys.argv) > 1 else 60):
    if not os.environ.get("WARM"):
        flush.fill_(i & 255)
    tr.copy_(init.view(-1))
    torch.cuda.synchronize()
    t = rt.wait(rt.submit(ghi, 0, x.data_ptr(), out.data_ptr()), 30)
    torch.cuda.synchronize()
    v = tr.view(3, 8).cpu().numpy().view(np.uint64).astype(np.float64)
    if i >= 10:
        rows.append(v - v[0, 0])
        dev.append(t["device_us"])
lib().sf_debug_chain_trace(None)
rt.close()
m = np.median(np.stack(rows), axis=0) / 1e3
names = ["start_min", "start_max", "wait_min", "wait_max", "streamed_min", "streamed_max", "softmax_start", "end_max"]
for l in range(3):
    print(f"layer {l}: " + " ".join(f"{names[e]} {m[l, e]:6.2f}" for e in range(8) if e != 6 or l == 2))
print("device_us p50", float(np.median(dev)))
