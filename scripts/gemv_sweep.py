"""Batch-1 GEMV time vs weight bytes (fixed-cost intercept), ours vs cuBLAS, warm and cold L2."""
import json, sys
import torch
sys.path.insert(0, ".")
from paper_conf_middleware_wur0hdh21_b200 import ops as K

flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")


def t_one(fn, cold, reps=30):
    ts = []
    for i in range(reps):
        if cold:
            flush.fill_(i & 255)
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record(); fn(); e1.record(); e1.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    ts.sort()
    return ts[len(ts) // 2]


rows = []
for Kd in (2048, 4096):
    for N in (256, 1024, 2048, 4096, 8192):
        W = torch.randn(Kd, N, device="cuda")
        b = torch.randn(1, N, device="cuda")
        x = torch.randn(1, Kd, device="cuda")
        y = torch.empty(1, N, device="cuda")
        ours = lambda: K.gemm_bias_act(x, W, y, [b], True)
        cub = lambda: torch.matmul(x, W)
        rd = lambda: torch.sum(W)
        r = {"K": Kd, "N": N, "MB": Kd * N * 4 / 2**20}
        for name, fn in (("ours", ours), ("cublas", cub), ("torch_sum_read", rd)):
            for cold in (False, True):
                r[f"{name}_{'cold' if cold else 'warm'}_us"] = t_one(fn, cold)
        rows.append(r)
        print(json.dumps(r), flush=True)
