"""Target for an ncu capture of the pack / unpack walks of the bench's cut 0 (535 tensors,
204.9 MB) through sf_probe_migration, L2 cold and dirty (a 2 x L2 write first), so the DRAM
bytes of one launch can be read next to its algorithmic 2 x 204.9 MB."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_middleware_wur0hdh21_b200.runtime import Runtime  # noqa: E402

g, _ = bench.build_workload(8, 1)
with Runtime([0]) as rt:
    gh = rt.register(g)
    gh.partition("max_ops", 1, update_chunks=8)
    gh.bind(0, staging=True)
    for mode in (2, 2, 2, 1, 1, 0, 0):
        print(mode, rt.probe_migration(gh, 0, 0, mode))
