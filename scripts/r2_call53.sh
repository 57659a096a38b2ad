#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c53_build.log 2>&1 || { tail -20 gpurun_out/r2c53_build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r2c53_tests.log 2>&1; echo "tests exit $?"; tail -2 gpurun_out/r2c53_tests.log
timeout 600 python scripts/subgraph_durations.py 2>&1 | tail -13 | head -5
for i in 1 2; do SF_BENCH_WATCHDOG_S=400 timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/r2c53_bench_$i.json 2> gpurun_out/r2c53_bench_$i.err; echo "bench $i exit $?"
python - $i <<'PY'
import json, sys
d=json.loads(open(f"gpurun_out/r2c53_bench_{sys.argv[1]}.json").read().strip().splitlines()[-1])
print({k: round(d.get(k), 4) for k in ("p50_ms","p99_ms","preempt_latency_p50_ms","preempt_latency_p99_ms","preempt_to_resume_p50_ms")}, "e2e p99", round(d["e2e"]["value"],4), "loss", round(d["training_throughput"]["loss_frac"],3), "solo it/s", round(d["training_throughput"]["solo_it_per_s"],1))
PY
done
