"""Small host round trips (C1: 1.6 MB live set): what one pinned D2H / H2D copy costs at this
size, alone, back to back on one stream, and as overlapped chunks on two streams (CUDA events)."""
import json, sys, torch
n = int(float(sys.argv[1]) if len(sys.argv) > 1 else 1.6e6) // 16 * 16
d = torch.empty(n, dtype=torch.uint8, device="cuda")
d2 = torch.empty_like(d)
h = torch.empty(n, dtype=torch.uint8).pin_memory()
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
def timed(fn, reps=50):
    ts = []
    for _ in range(reps):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    ts.sort()
    return round(ts[len(ts) // 2], 1)
def d2h(): h.copy_(d, non_blocking=True)
def h2d(): d2.copy_(h, non_blocking=True)
def seq(): d2h(); h2d()
def chunked(k):
    def f():
        cs = n // k
        cur = torch.cuda.current_stream()
        evs = []
        for i in range(k):
            with torch.cuda.stream(s1):
                s1.wait_stream(cur) if i == 0 else None
                h[i*cs:(i+1)*cs].copy_(d[i*cs:(i+1)*cs], non_blocking=True)
                e = torch.cuda.Event(); e.record(s1); evs.append(e)
        for i in range(k):
            with torch.cuda.stream(s2):
                s2.wait_event(evs[i])
                d2[i*cs:(i+1)*cs].copy_(h[i*cs:(i+1)*cs], non_blocking=True)
        cur.wait_stream(s2)
    return f
out = {"bytes": n, "d2h_us": timed(d2h), "h2d_us": timed(h2d), "d2h_then_h2d_us": timed(seq)}
for k in (2, 4, 8):
    out[f"chunked_{k}_us"] = timed(chunked(k))
out["gbs_d2h"] = round(n / out["d2h_us"] / 1e3, 1)
out["gbs_h2d"] = round(n / out["h2d_us"] / 1e3, 1)
print(json.dumps(out))
