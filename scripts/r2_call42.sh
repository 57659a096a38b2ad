#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c42_build.log 2>&1 || { tail -20 gpurun_out/r2c42_build.log; exit 1; }
for rep in 1 2; do for gate in 1 0; do
SF_BENCH_WATCHDOG_S=600 timeout 900 python bench.py --steps 40 --no-baselines --no-cpu-baseline --gate $gate > gpurun_out/r2c42_g$gate.json 2>/dev/null
python - $gate <<'PY'
import json, sys
d=json.loads(open(f"gpurun_out/r2c42_g{sys.argv[1]}.json").read().strip().splitlines()[-1])
print("gate", sys.argv[1], {k: round(d.get(k), 4) for k in ("p50_ms","p99_ms","preempt_latency_p50_ms","preempt_latency_p99_ms","preempt_to_resume_p50_ms")}, "e2e p99", round(d["e2e"]["value"],4), "loss", round(d["training_throughput"]["loss_frac"],3), "n", d["n_requests"])
PY
done; done
