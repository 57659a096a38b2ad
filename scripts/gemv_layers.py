"""Device time of batch-1 inference chains of various shapes through the runtime (request
path: TMA cluster GEMVs under PDL, fused epilogues), cold L2 (512 MB flush between requests).
Fits time = a + bytes / B to separate the fixed per-chain / per-layer cost from streaming."""
import json, os, sys
import numpy as np, torch
sys.path.insert(0, ".")
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime
from sf_inputs import data as D, graphs as G

flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
shapes = [(4096, 32), (4096, 1024), (4096, 4096), (2048, 4096), (4096, 1000), (4096, 8192),
          (2048, 4096, 4096), (2048, 4096, 4096, 1000), (1024, 1024, 1024, 1024, 1024)]
rows = []
for w in shapes:
    gi = G.mlp_infer(w, name="m", wt=os.environ.get("WT") == "1")
    with Runtime([0], dispatch_spin_us=-1) as rt:  # env SF_PDL / SF_INFER_DIRECT apply
        gh = rt.register(gi, 1)
        gh.partition()
        gh.bind(0, staging=False)
        gh.load(0, D.init_state(gi, seed=4))
        x = torch.rand(1, w[0], device="cuda")
        out = torch.empty(1, w[-1], device="cuda")
        dev, lau = [], []
        for i in range(60):
            flush.fill_(i & 255)
            torch.cuda.synchronize()
            t = rt.wait(rt.submit(gh, 0, x.data_ptr(), out.data_ptr()), 30)
            if i >= 10:
                dev.append(t["device_us"])
                lau.append(t["launch_us"])
    mb = sum(w[i] * w[i + 1] for i in range(len(w) - 1)) * 4 / 1e6
    r = {"widths": w, "layers": len(w) - 1, "MB": mb, "device_us_p50": float(np.median(dev)),
         "launch_us_p50": float(np.median(lau)),
         "gbs": mb * 1e6 / (np.median(dev) * 1e-6) / 1e9}
    rows.append(r)
    print(json.dumps(r), flush=True)
