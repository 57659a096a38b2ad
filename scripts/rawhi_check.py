"""Bitwise check: raw fp32 as the tf32 'hi' operand == explicitly truncated hi (HW truncation)."""
import os, sys, numpy as np, torch
sys.path.insert(0, ".")
from paper_conf_middleware_wur0hdh21_b200 import ops as K
rng = np.random.default_rng(5)
outs = []
for (M, N, Kd, fl) in [(300, 200, 100, 0), (1000, 64, 576, 0), (576, 64, 3000, 1), (512, 300, 1024, 2), (257, 129, 999, 3)]:
    a = (rng.standard_normal((Kd, M) if fl & 1 else (M, Kd)) * rng.choice([1e-3, 1, 1e3])).astype(np.float32)
    b = rng.standard_normal((N, Kd) if fl & 2 else (Kd, N)).astype(np.float32)
    c = torch.zeros(M, N, device="cuda")
    K.gemm(torch.from_numpy(a).cuda(), torch.from_numpy(b).cuda(), c, fl)
    outs.append(c.cpu().numpy())
np.savez(sys.argv[1], *outs)
