"""Does the persisting L2 set-aside keep a 64 MB weight block resident across a 512 MB write
flush on this B200?  torch.sum over the block on a stream with / without an access-policy
window (cuda-python runtime bindings), cold (after the flush) and warm."""
import json, torch
from cuda.bindings import runtime as cr

dev = torch.cuda.current_device()
err, mx = cr.cudaDeviceGetAttribute(cr.cudaDeviceAttr.cudaDevAttrMaxPersistingL2CacheSize, dev)
err, mw = cr.cudaDeviceGetAttribute(cr.cudaDeviceAttr.cudaDevAttrMaxAccessPolicyWindowSize, dev)
err, l2 = cr.cudaDeviceGetAttribute(cr.cudaDeviceAttr.cudaDevAttrL2CacheSize, dev)
out = {"max_persisting_l2_mb": mx / 2**20, "max_window_mb": mw / 2**20, "l2_mb": l2 / 2**20}
W = torch.randn(16 << 20, device="cuda")  # 64 MB
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
s = torch.cuda.Stream()


def timed(fn, cold, reps=20):
    ts = []
    for i in range(reps):
        if cold:
            flush.fill_(i & 255)
            torch.cuda.synchronize()
        with torch.cuda.stream(s):
            e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
            e0.record(); fn(); e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    ts.sort()
    return ts[len(ts) // 2]


out["sum_cold_us"] = timed(lambda: W.sum(), True)
out["sum_warm_us"] = timed(lambda: W.sum(), False)
for setaside_mb in (48, 80):
    cr.cudaDeviceSetLimit(cr.cudaLimit.cudaLimitPersistingL2CacheSize, min(mx, setaside_mb << 20))
    win = cr.cudaAccessPolicyWindow()
    win.base_ptr = W.data_ptr()
    win.num_bytes = min(W.numel() * 4, mw)
    win.hitRatio = min(1.0, (setaside_mb << 20) / win.num_bytes)
    win.hitProp = cr.cudaAccessProperty.cudaAccessPropertyPersisting
    win.missProp = cr.cudaAccessProperty.cudaAccessPropertyStreaming
    attr = cr.cudaStreamAttrValue()
    attr.accessPolicyWindow = win
    r = cr.cudaStreamSetAttribute(s.cuda_stream, cr.cudaLaunchAttributeID.cudaLaunchAttributeAccessPolicyWindow, attr)
    out[f"setattr_{setaside_mb}"] = str(r[0])
    out[f"sum_cold_persist{setaside_mb}_us"] = timed(lambda: W.sum(), True)
    cr.cudaCtxResetPersistingL2Cache()
print(json.dumps(out))
