#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c41_build.log 2>&1 || { tail -20 gpurun_out/r2c41_build.log; exit 1; }
SF_BENCH_WATCHDOG_S=600 timeout 900 python bench.py > gpurun_out/r2c41_bench.json 2> gpurun_out/r2c41_bench.err; echo "bench exit $?"
python - <<'PY'
import json
d=json.loads(open("gpurun_out/r2c41_bench.json").read().strip().splitlines()[-1])
print({k: d[k] for k in ("value","ms_per_step","gpu_launches")})
print("roofline", d.get("roofline"))
print("e2e", d.get("e2e"))
print({k: d.get(k) for k in ("p50_ms","p99_ms","n_requests","preempt_latency_p50_ms","preempt_latency_p99_ms","preempt_to_resume_p50_ms","inference_roofline")})
print("tp", d.get("training_throughput"))
print("baselines", {k: (v.get("p99_ms") if isinstance(v, dict) else v) for k, v in (d.get("baselines") or {}).items()})
PY
