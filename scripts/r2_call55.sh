#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c55_build.log 2>&1 || { tail -20 gpurun_out/r2c55_build.log; exit 1; }
for l in 0 79; do FLUSH=1 L2P_MB=$l timeout 300 python scripts/infer_bench.py 200 2>&1 | tail -1 | cut -c1-300; done
for l in 0 79 0 79; do SF_BENCH_WATCHDOG_S=400 timeout 600 python bench.py --no-baselines --no-cpu-baseline --l2-persist-mb $l > gpurun_out/r2c55_bench_$l.json 2>/dev/null
python - $l <<'PY'
import json, sys
d=json.loads(open(f"gpurun_out/r2c55_bench_{sys.argv[1]}.json").read().strip().splitlines()[-1])
print("l2p", sys.argv[1], {k: round(d.get(k), 4) for k in ("p50_ms","p99_ms","preempt_latency_p99_ms")}, "e2e p99", round(d["e2e"]["value"],4), "loss", round(d["training_throughput"]["loss_frac"],3), "solo", round(d["training_throughput"]["solo_it_per_s"],1), "inf frac", round(d["inference_roofline"]["frac"],3))
PY
done
