"""One GEMM shape through sf_op_gemm (for ncu captures): python scripts/gemm_one.py M N K flags [reps]."""
import sys, torch
sys.path.insert(0, ".")
from paper_conf_middleware_wur0hdh21_b200 import ops as K
M, N, Kd, fl = (int(x) for x in sys.argv[1:5])
reps = int(sys.argv[5]) if len(sys.argv) > 5 else 20
A = torch.rand((Kd, M) if fl & 1 else (M, Kd), device="cuda")
B = torch.rand((N, Kd) if fl & 2 else (Kd, N), device="cuda")
C = torch.empty(M, N, device="cuda")
for _ in range(3):
    K.gemm(A, B, C, fl)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
e0.record()
for _ in range(reps):
    K.gemm(A, B, C, fl)
e1.record(); e1.synchronize()
us = e0.elapsed_time(e1) * 1e3 / reps
byts = 4 * (M * Kd + Kd * N + M * N)
print(f"M={M} N={N} K={Kd} flags={fl}: {us:.1f} us, {2*M*N*Kd/us/1e6:.1f} TFLOP/s, {byts/us/1e3:.0f} GB/s (A+B+C once)")
