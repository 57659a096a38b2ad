"""Pack / unpack of the C2 cut-0 live set (535 tensors, 204.9 MB) by the descriptor walk, warm /
clean-cold / dirty-cold L2 (bench.probe_pack): run once with SF_COPY_BULK=0 (16-B LDG/STG walk,
the default) and once with SF_COPY_BULK=1 (cp.async.bulk G->S->G ring) for DESIGN.md's kernel
table (round-2 verdict #8)."""
import json, os, subprocess, sys

if len(sys.argv) > 1 and sys.argv[1] == "child":
    sys.path.insert(0, ".")
    import argparse, bench
    a = argparse.Namespace(batch=8, spatial_div=1, max_ops=1, update_chunks=8)
    hbm = bench.hbm_peak()[0] if hasattr(bench, "hbm_peak") else 6542.4
    print(json.dumps(bench.probe_pack(a, 0, hbm)))
    sys.exit(0)
for bulk in ("0", "1"):
    env = dict(os.environ, SF_COPY_BULK=bulk)
    r = subprocess.run([sys.executable, __file__, "child"], env=env, capture_output=True, text=True)
    line = r.stdout.strip().splitlines()[-1] if r.stdout.strip() else r.stderr[-500:]
    print(json.dumps({"SF_COPY_BULK": bulk, "probe": json.loads(line) if line.startswith("{") else line}))
