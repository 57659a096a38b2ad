"""Phase timeline of the fused inference chain (C4 MLP, M=1) from per-CTA globaltimer marks."""
import ctypes as C, sys, numpy as np, torch
sys.path.insert(0, ".")
from paper_conf_middleware_wur0hdh21_b200 import ops as K
from paper_conf_middleware_wur0hdh21_b200._abi import lib
widths = [int(w) for w in (sys.argv[1] if len(sys.argv) > 1 else "2048,4096,4096,1000").split(",")]
n = len(widths) - 1
Ws = [torch.randn(widths[i], widths[i + 1], device="cuda") / widths[i] ** 0.5 for i in range(n)]
bs = [torch.randn(1, widths[i + 1], device="cuda") for i in range(n)]
hs = [torch.empty(1, widths[i + 1], device="cuda") for i in range(n)]
x = torch.randn(1, widths[0], device="cuda")
probs = torch.empty(1, widths[-1], device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
tr = torch.zeros(160 * 64, dtype=torch.int64, device="cuda")
lib().sf_debug_chain_trace(C.c_void_p(tr.data_ptr()))
res = []
for it in range(12):
    flush.fill_(it)
    tr.zero_()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    K.mlp_chain(x, Ws, bs, [i < n - 1 for i in range(n)], hs, probs)
    e1.record()
    torch.cuda.synchronize()
    res.append(e0.elapsed_time(e1) * 1e3)
lib().sf_debug_chain_trace(None)
t = tr.view(160, 8, 8)[:, :n + 1, :].cpu().numpy().astype(np.float64)
t0 = t[t > 0].min()
print("event-timed us (cold L2):", np.round(res[2:], 1))
# mlp_fold_kernel events: layer 0: 0 start, 1 x staged, 4 columns streamed + combined;
# layer l > 0: 0 start, 1 my rows streamed, 2 grid barrier passed, 3 reduced; done at [n][7]
names = ["start", "streamed" , "barrier", "reduced", "l0_done", "published", "tail_landed", "done"]
names0 = ["start", "x_staged", "x_synced", "-", "l0_combined", "l0_items_done", "-", "-"]
for l in range(n + 1):
    row = []
    for e in range(8):
        v = t[:, l, e]
        v = v[v > 0]
        if len(v):
            row.append(f"{(names0 if l == 0 else names)[e]} {np.median(v - t0) / 1e3:6.2f}/{np.max(v - t0) / 1e3:6.2f}")
    print(f"layer {l}: " + " | ".join(row))
