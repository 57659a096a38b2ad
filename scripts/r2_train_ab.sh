#!/bin/bash
# Solo training throughput of the bench job: drain gate on / off x CUDA_DEVICE_MAX_CONNECTIONS.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/tab_build.log 2>&1 || { tail -20 gpurun_out/tab_build.log; exit 1; }
for cfg in "1 32" "0 32" "1 8" "0 8" "1 32"; do set -- $cfg
CUDA_DEVICE_MAX_CONNECTIONS=$2 SF_BENCH_WATCHDOG_S=400 timeout 600 python bench.py --no-baselines --no-cpu-baseline --steps 6 --gate $1 > gpurun_out/tab_$1_$2.json 2>/dev/null
python - $1 $2 <<'PY'
import json, sys
d=json.loads(open(f"gpurun_out/tab_{sys.argv[1]}_{sys.argv[2]}.json").read().strip().splitlines()[-1])
t=d["training_throughput"]
print("gate", sys.argv[1], "conn", sys.argv[2], "solo it/s", round(t["solo_it_per_s"],1), "coloc it/s", round(t["collocated_it_per_s"],1), "iter ms", round(d["training_iteration_ms_median"],3), "sub ms mean", round(d["training_subgraph_ms_mean"],4), "p99", round(d["p99_ms"],4), "wait p99", d["arrivals"]["latency_breakdown_us"]["preempting"]["wait_p99"])
PY
done
timeout 300 python scripts/subgraph_durations.py 2>&1 | head -3
