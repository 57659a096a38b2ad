"""The 'C5 cliff' (round-1 verdict): a single-tensor live set moved slot -> slot on one B200 by
the peer-store walk (engine 0) vs one copy-engine memcpy (engine 3), 1-8 GB; prints GB/s."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from bench_configs import sizes_for, state_graph  # noqa: E402
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime  # noqa: E402

for gb in (1, 2, 4, 6, 8):
    g = state_graph(sizes_for(gb << 30, "single"))
    with Runtime([0, 0]) as rt:
        gh = rt.register(g)
        gh.partition()
        gh.bind(0, staging=False)
        gh.bind(1, staging=False)
        row = {"gb": gb}
        for eng, name in ((0, "sm_walk"), (3, "ce_single")):
            ts = sorted(rt.probe_peer(gh, 0, 1, 0, eng)[0] for _ in range(5))
            nb = rt.probe_peer(gh, 0, 1, 0, eng)[1]
            row[name + "_gbs"] = round(2 * nb / (ts[2] * 1e-6) / 1e9, 1)  # read + write HBM bytes
        print(json.dumps(row), flush=True)
