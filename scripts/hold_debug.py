"""Debug the forced drain-gate hold scenario (tests/test_gpu_runtime.py)."""
import sys, time
sys.path.insert(0, ".")
import numpy as np, torch
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime
from sf_inputs import data as D, graphs as G
g = G.mlp_train(widths=(4096, 4096, 4096, 10), batch=4096, pool=2)
gi = G.mlp_infer()
sti = D.init_state(gi, seed=D.SEED_INFER)
xs = D.infer_inputs(gi, 6)
st, ds = D.init_state(g), D.datasets(g)
import os
gate, early, budget = (int(v) for v in os.environ.get("CFG", "1,1,0").split(","))
print("gate", gate, "early", early, "budget", budget)
rt = Runtime([0], auto_preempt=True, max_inflight=2, early_launch=bool(early), dispatch_spin_us=-1,
             drain_gate=bool(gate), inflight_budget_us=budget)
gh = rt.register(g); gh.partition(); gh.bind(0, staging=True, host_staging=True); gh.load(0, ds); gh.load(0, st)
print("n_subgraphs", gh.n_subgraphs)
ghi = rt.register(gi, priority=1); ghi.partition(); ghi.bind(0, staging=False); ghi.load(0, sti)
t0 = time.perf_counter()
job = rt.start_training(gh, 0, 60, -1)
xin = torch.from_numpy(xs).cuda(); out = torch.zeros(6, 1, 10, device="cuda")
time.sleep(0.005)
for r in range(6):
    time.sleep(0.03)
    tm = rt.wait(rt.submit(ghi, 0, xin[r].data_ptr(), out[r].data_ptr()), 30)
    ji = rt.job_info(job)
    print(r, "t", round(time.perf_counter() - t0, 4), "preempted_job", tm.get("preempted_job"), "job state", ji["state"], "iter", ji["iter"], "k", ji["k"], "npre", ji["n_preemptions"])
rt.wait_job(job, 120)
print("job done at", round(time.perf_counter() - t0, 4))
tr = rt.trace()
tt = [e for e in tr if e["kind"] == "train"]
print("train events", len(tt), "mean dur us", np.mean([(e["t1"] - e["t0"]) / 1e3 for e in tt]))
print("infer events", [(e["k"], e.get("iter")) for e in tr if e["kind"] == "infer"])
rt.close()
