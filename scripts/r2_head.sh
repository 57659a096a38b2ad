#!/bin/bash
# Cluster-free head GEMV (SF_GEMV_HEAD, default on) vs the 8-CTA cluster head: parity, trace, A/B
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/hd_build.log 2>&1 || { tail -20 gpurun_out/hd_build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_runtime.py -q -k "c4_inference or inference_paths" 2>&1 | tail -2
for h in 2 1; do echo "head=$h"; SF_GEMV_HEAD=$h SF_INFER_GRAPH=0 timeout 300 python scripts/blk_trace.py 40 2>&1 | tail -4; done
for h in 2 1 2 1; do
  echo "head=$h $(SF_GEMV_HEAD=$h FLUSH=1 timeout 300 python scripts/infer_bench.py 300 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print({k: round(d[k]*1e3 if k.endswith('ms') else d[k],2) for k in ('p50_ms','p99_ms','device_p50_ms','device_p99_ms','launch_us_p50')})")"
done
for h in 2 1 2 1; do SF_GEMV_HEAD=$h SF_BENCH_WATCHDOG_S=400 timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/hd_bench_$h.json 2>/dev/null
python - $h <<'PY'
import json, sys
d=json.loads(open(f"gpurun_out/hd_bench_{sys.argv[1]}.json").read().strip().splitlines()[-1])
b=d["arrivals"]["latency_breakdown_us"]
print("head", sys.argv[1], {k: round(d.get(k), 4) for k in ("p50_ms","p99_ms","preempt_latency_p99_ms")}, "e2e p99", round(d["e2e"]["value"],4), "inf frac", round(d["inference_roofline"]["frac"],3),
      "pre dev p50/p99", b["preempting"]["device_p50"], b["preempting"]["device_p99"], "nonpre dev p99", b["not_preempting"]["device_p99"])
PY
done
