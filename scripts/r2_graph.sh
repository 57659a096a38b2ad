#!/bin/bash
# One-graph request chain (SF_INFER_GRAPH=1) vs direct PDL launches: parity, request path, bench.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/rg_build.log 2>&1 || { tail -20 gpurun_out/rg_build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_runtime.py -q -k "inference_paths" 2>&1 | tail -2
for cp in d2h; do for v in 0 2; do
  echo "copy=$cp graph=$v $(SF_INFER_GRAPH=$v COPY=$cp FLUSH=1 timeout 300 python scripts/infer_bench.py 300 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print({k: round(d[k]*1e3 if k.endswith('ms') else d[k],2) for k in ('p50_ms','p99_ms','wake_p50_ms','device_p50_ms','device_p99_ms','launch_us_p50','host_overhead_us_p50')})")"
done; done
for v in 2 0 2 0; do SF_INFER_GRAPH=$v SF_BENCH_WATCHDOG_S=400 timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/rg_bench_$v.json 2>/dev/null
python - $v <<'PY'
import json, sys
d=json.loads(open(f"gpurun_out/rg_bench_{sys.argv[1]}.json").read().strip().splitlines()[-1])
b=d["arrivals"]["latency_breakdown_us"]
print("graph", sys.argv[1], {k: round(d.get(k), 4) for k in ("p50_ms","p99_ms","preempt_latency_p99_ms")}, "e2e p99", round(d["e2e"]["value"],4),
      "pre wait/dev p99", b["preempting"]["wait_p99"], b["preempting"]["device_p99"], "nonpre wait/dev p99", b["not_preempting"]["wait_p99"], b["not_preempting"]["device_p99"],
      "launch p50", b["preempting"]["launch_p50"], "solo", round(d["training_throughput"]["solo_it_per_s"]))
PY
done
