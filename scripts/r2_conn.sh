#!/bin/bash
# Hardware work queues (CUDA_DEVICE_MAX_CONNECTIONS) with the gate off: do requests that land
# during a host round trip queue behind the parked job's copy / event-wait commands?
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/cn_build.log 2>&1 || { tail -20 gpurun_out/cn_build.log; exit 1; }
for c in 8 16 32 8 16; do CUDA_DEVICE_MAX_CONNECTIONS=$c SF_BENCH_WATCHDOG_S=400 timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/cn_$c.json 2>/dev/null
python - $c <<'PY'
import json, sys
d=json.loads(open(f"gpurun_out/cn_{sys.argv[1]}.json").read().strip().splitlines()[-1])
b=d["arrivals"]["latency_breakdown_us"]
print("conn", sys.argv[1], {k: round(d.get(k), 4) for k in ("p50_ms","p99_ms","preempt_latency_p99_ms")}, "e2e p99", round(d["e2e"]["value"],4),
      "nonpre wait p50/p99", b["not_preempting"]["wait_p50"], b["not_preempting"]["wait_p99"], "dev p50/p99", b["not_preempting"]["device_p50"], b["not_preempting"]["device_p99"],
      "pre wait p99", b["preempting"]["wait_p99"], "solo", round(d["training_throughput"]["solo_it_per_s"]))
PY
done
