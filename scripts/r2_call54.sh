#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c54_build.log 2>&1 || { tail -20 gpurun_out/r2c54_build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r2c54_tests.log 2>&1; echo "tests exit $?"; tail -1 gpurun_out/r2c54_tests.log
for i in 1 2 3 4 5 6 7 8; do SF_BENCH_WATCHDOG_S=400 timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/r2c54_bench_$i.json 2> gpurun_out/r2c54_bench_$i.err; rc=$?
python - $i $rc <<'PY'
import json, sys
try:
    d=json.loads(open(f"gpurun_out/r2c54_bench_{sys.argv[1]}.json").read().strip().splitlines()[-1])
    print(sys.argv[1], {k: round(d.get(k), 4) for k in ("p50_ms","p99_ms","preempt_latency_p99_ms")}, "e2e p99", round(d["e2e"]["value"],4), "loss", round(d["training_throughput"]["loss_frac"],3), "valve", d.get("gate_valve"))
except Exception as ex:
    print(sys.argv[1], "rc", sys.argv[2], ex)
PY
done
