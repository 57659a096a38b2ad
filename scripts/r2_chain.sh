#!/bin/bash
# Fused inference chain (mlp_fold_kernel): parity, phase trace, request-path A/B vs the
# per-layer GEMV chain (SF_CHAIN=0), bench A/B.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/chain_build.log 2>&1 || { tail -20 gpurun_out/chain_build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "chain" > gpurun_out/chain_tests.log 2>&1; echo "chain tests exit $?"; tail -3 gpurun_out/chain_tests.log
timeout 900 python -m pytest tests/test_gpu_runtime.py -q -x -k "infer or request or smoke" > gpurun_out/chain_rt_tests.log 2>&1; echo "runtime tests exit $?"; tail -3 gpurun_out/chain_rt_tests.log
timeout 300 python scripts/chain_trace.py > gpurun_out/chain_trace.log 2>&1; echo "trace exit $?"; cat gpurun_out/chain_trace.log
for c in 0 1; do SF_CHAIN=$c FLUSH=1 timeout 300 python scripts/infer_bench.py 300 2>&1 | tail -1 | cut -c1-400; done
for c in 1 0 1 0; do SF_CHAIN=$c SF_BENCH_WATCHDOG_S=400 timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/chain_bench_$c.json 2>/dev/null
python - $c <<'PY'
import json, sys
d=json.loads(open(f"gpurun_out/chain_bench_{sys.argv[1]}.json").read().strip().splitlines()[-1])
b=d["arrivals"]["latency_breakdown_us"]["preempting"]
print("chain", sys.argv[1], {k: round(d.get(k), 4) for k in ("p50_ms","p99_ms","preempt_latency_p99_ms")}, "e2e p99", round(d["e2e"]["value"],4), "inf frac", round(d["inference_roofline"]["frac"],3), "dev p50/p99", b["device_p50"], b["device_p99"], "launch p50", b["launch_p50"])
PY
done
