"""GEMM microbench on the bench workload's forest shapes (CUDA events), vs oracle error."""
import os, sys, json, numpy as np, torch
sys.path.insert(0, ".")
from oracle import ops as O
from paper_conf_middleware_wur0hdh21_b200 import ops as K
from sf_inputs import graphs as G
from sf_inputs.ir import GEMM, TA, TB

def rel(a, b):
    a = np.asarray(a, np.float64); b = np.asarray(b, np.float64)
    return float(np.abs(a - b).max() / max(np.abs(b).max(), 1e-30))

g = G.resnet50_forest(batch=8)
shapes = {}
for o in g.ops:
    if o.type != GEMM: continue
    A, B = g.tensors[o.ins[0]], g.tensors[o.ins[1]]
    M, Kd = (A.cols, A.rows) if o.flags & TA else (A.rows, A.cols)
    N = B.rows if o.flags & TB else B.cols
    shapes[(M, N, Kd, o.flags)] = shapes.get((M, N, Kd, o.flags), 0) + 1
tot_flop = tot_t = 0.0
rng = np.random.default_rng(0)
rows = []
for (M, N, Kd, fl), cnt in sorted(shapes.items(), key=lambda x: -x[0][0]*x[0][1]*x[0][2]*x[1]):
    A = torch.randn((Kd, M) if fl & TA else (M, Kd), device="cuda")
    B = torch.randn((N, Kd) if fl & TB else (Kd, N), device="cuda")
    C = torch.empty(M, N, device="cuda")
    for _ in range(3): K.gemm(A, B, C, fl)
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(10): K.gemm(A, B, C, fl)
    e1.record(); torch.cuda.synchronize()
    t = e0.elapsed_time(e1) / 10 * 1e-3
    fl_ = 2.0 * M * N * Kd
    tot_flop += fl_ * cnt; tot_t += t * cnt
    rows.append((M, N, Kd, fl, cnt, t * 1e6, fl_ / t / 1e12))
err = []
for (M, N, Kd, fl) in [(1000, 64, 576, 0), (576, 64, 3000, TA), (300, 200, 100, TA | TB), (129, 65, 33, 0), (512, 300, 1024, TB)]:
    a = rng.standard_normal((Kd, M) if fl & TA else (M, Kd)).astype(np.float32)
    b = rng.standard_normal((N, Kd) if fl & TB else (Kd, N)).astype(np.float32)
    c = torch.zeros(M, N, device="cuda")
    K.gemm(torch.from_numpy(a).cuda(), torch.from_numpy(b).cuda(), c, fl)
    err.append(rel(c.cpu().numpy(), O.gemm(a, b, None, fl)))
print(json.dumps({"path": os.environ.get("SF_GEMM_PATH", "tma"), "rawhi": os.environ.get("SF_GEMM_RAWHI", "0"),
                  "step_gemm_ms": tot_t * 1e3, "tflops_algorithmic": tot_flop / tot_t / 1e12, "max_rel_err": max(err)}))
for r in rows[:8]:
    print("  M=%d N=%d K=%d flags=%d x%d  %.1f us  %.1f TFLOP/s" % r)
