"""C3 (BERT-large chain, T = 512) GEMM shapes: time and algorithmic TFLOP/s (3xTF32)."""
import json, sys, torch
sys.path.insert(0, ".")
from paper_conf_middleware_wur0hdh21_b200 import ops as K
TA, TB = 1, 2
T, H, I, V = 512, 1024, 4096, 30522
shapes = [("qkvo fwd", T, H, H, 0), ("ffn_i fwd", T, I, H, 0), ("ffn_o fwd", T, H, I, 0),
          ("head fwd", T, V, H, TB), ("dW qkvo", H, H, T, TA), ("dW ffn_i", H, I, T, TA),
          ("dW ffn_o", I, H, T, TA), ("dX qkvo", T, H, H, TB), ("dX ffn_i", T, H, I, TB),
          ("dX ffn_o", T, I, H, TB), ("dword", V, H, T, TA), ("dhead_x", T, H, V, 0)]
for name, M, N, Kd, fl in shapes:
    A = torch.randn((Kd, M) if fl & TA else (M, Kd), device="cuda")
    B = torch.randn((N, Kd) if fl & TB else (Kd, N), device="cuda")
    C = torch.empty(M, N, device="cuda")
    for _ in range(3):
        K.gemm(A, B, C, fl)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    n = 20
    e0.record()
    for _ in range(n):
        K.gemm(A, B, C, fl)
    e1.record(); e1.synchronize()
    us = e0.elapsed_time(e1) * 1e3 / n
    print(json.dumps({"name": name, "M": M, "N": N, "K": Kd, "us": round(us, 1),
                      "tflops_alg": round(2 * M * N * Kd / us / 1e6, 1), "path": K.last_gemm_path()}), flush=True)
