import os, sys, torch
sys.path.insert(0, ".")
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime
from sf_inputs import data as D, graphs as G
w = tuple(int(v) for v in sys.argv[1].split(","))
gi = G.mlp_infer(w, name="m", wt=True)
with Runtime([0], dispatch_spin_us=int(os.environ.get("SPIN", "-1"))) as rt:
    gh = rt.register(gi, 1); gh.partition(); gh.bind(0, staging=False)
    gh.load(0, D.init_state(gi, seed=4))
    x = torch.rand(1, w[0], device="cuda"); out = torch.empty(1, w[-1], device="cuda")
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda") if os.environ.get("FLUSH") else None
    for i in range(int(os.environ.get("N", "3"))):
        if flush is not None:
            flush.fill_(i & 255)
            torch.cuda.synchronize()
        t = rt.wait(rt.submit(gh, 0, x.data_ptr(), out.data_ptr()), 30)
    print("ok", t["device_us"], out.sum().item())
