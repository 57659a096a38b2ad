#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/tab2_build.log 2>&1 || { tail -20 gpurun_out/tab2_build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_priority.py tests/test_gpu_c2_bench_config.py -q -x > gpurun_out/tab2_tests.log 2>&1; echo "tests exit $?"; tail -3 gpurun_out/tab2_tests.log
for cfg in "1 32" "0 8" "0 32" "1 8" "1 32" "0 8"; do set -- $cfg
CUDA_DEVICE_MAX_CONNECTIONS=$2 SF_BENCH_WATCHDOG_S=400 timeout 600 python bench.py --no-baselines --no-cpu-baseline --steps 10 --gate $1 > gpurun_out/tab2_$1_$2.json 2>/dev/null
python - $1 $2 <<'PY'
import json, sys
d=json.loads(open(f"gpurun_out/tab2_{sys.argv[1]}_{sys.argv[2]}.json").read().strip().splitlines()[-1])
t=d["training_throughput"]; b=d["arrivals"]["latency_breakdown_us"]["preempting"]
print("gate", sys.argv[1], "conn", sys.argv[2], "solo it/s", round(t["solo_it_per_s"],1), "coloc", round(t["collocated_it_per_s"],1), "iter ms", round(d["training_iteration_ms_median"],3), "sub ms", round(d["training_subgraph_ms_mean"],4), "p50", round(d["p50_ms"],4), "p99", round(d["p99_ms"],4), "pre p99", round(d["preempt_latency_p99_ms"],4), "wait p99", b["wait_p99"], "dev p50", b["device_p50"])
PY
done
