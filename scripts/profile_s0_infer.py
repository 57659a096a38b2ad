"""Run one training iteration (C2, batch 8) and one inference, for ncu kernel timing."""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import bench
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime
g, gi = bench.build_workload(8, 1)
arrs, arrs_i = bench.workload_arrays(g, gi, (8, 1))
rt = Runtime([0]); gh = rt.register(g); gh.partition(update_chunks=8); gh.bind(0, host_staging=True); gh.load(0, arrs)
ghi = rt.register(gi, 1); ghi.partition(); ghi.bind(0, staging=False); ghi.load(0, arrs_i)
j = rt.start_training(gh, 0, 1, -1); rt.wait_job(j, 60)
x = torch.rand(1, 2048, device="cuda"); out = torch.empty(1, 1000, device="cuda")
for _ in range(3):
    r = rt.submit(ghi, 0, x.data_ptr(), out.data_ptr()); rt.wait(r, 10)
rt.close()
