#!/bin/bash
# In-flight budget sweep at the bench config (gate off, 8 queues): preemption wait vs training
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/bud_build.log 2>&1 || { tail -20 gpurun_out/bud_build.log; exit 1; }
for b in 50 30 20 50 30 20; do SF_BENCH_WATCHDOG_S=400 timeout 600 python bench.py --no-baselines --no-cpu-baseline --inflight-budget-us $b > gpurun_out/bud_$b.json 2>/dev/null
python - $b <<'PY'
import json, sys
d=json.loads(open(f"gpurun_out/bud_{sys.argv[1]}.json").read().strip().splitlines()[-1])
b=d["arrivals"]["latency_breakdown_us"]
print("budget", sys.argv[1], {k: round(d.get(k), 4) for k in ("p50_ms","p99_ms","preempt_latency_p99_ms")}, "e2e p99", round(d["e2e"]["value"],4),
      "pre wait p99", b["preempting"]["wait_p99"], "nonpre wait/dev p99", b["not_preempting"]["wait_p99"], b["not_preempting"]["device_p99"],
      "solo", round(d["training_throughput"]["solo_it_per_s"]), "coloc", round(d["training_throughput"]["collocated_it_per_s"]))
PY
done
