import sys, numpy as np, torch
sys.path.insert(0, ".")
from paper_conf_middleware_wur0hdh21_b200 import ops as K
for (M, N, Kd, fl) in [(128, 128, 32, 2), (128, 128, 32, 0), (128, 128, 32, 1), (128, 128, 32, 3), (64, 256, 784, 0)]:
    A = torch.ones((Kd, M) if fl & 1 else (M, Kd), device="cuda")
    B = torch.ones((N, Kd) if fl & 2 else (Kd, N), device="cuda")
    C = torch.full((M, N), -7.0, device="cuda")
    K.gemm(A, B, C, fl); torch.cuda.synchronize()
    c = C.cpu().numpy()
    print(M, N, Kd, fl, "min", c.min(), "max", c.max(), "c00", c[0, 0], "c[-1,-1]", c[-1, -1])
    A = torch.arange(M * Kd, device="cuda", dtype=torch.float32).reshape(A.shape) % 7
    B = torch.arange(N * Kd, device="cuda", dtype=torch.float32).reshape(B.shape) % 5
    K.gemm(A, B, C, fl); torch.cuda.synchronize()
    Ar = A.T if fl & 1 else A; Br = B.T if fl & 2 else B
    ref = (Ar.double() @ Br.double()).float()
    print("   err", float((C - ref).abs().max()), "ref max", float(ref.abs().max()))
