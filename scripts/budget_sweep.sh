#!/bin/bash
# p99 latency / preemption latency / iteration time vs the in-flight budget and window.
for cfg in "--inflight-budget-us 15" "--inflight-budget-us 25" "--inflight-budget-us 35" "--inflight-budget-us 50" "--max-inflight 1"; do
  timeout 300 python bench.py --steps 1000 --no-baselines --no-cpu-baseline $cfg 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('$cfg', 'p99', round(d['p99_ms'],4), 'p50', round(d['p50_ms'],4), 'pre99', round(d['preempt_latency_p99_ms'],4), 'pre50', round(d['preempt_latency_p50_ms'],4), 'iter', round(d['training_iteration_ms_median'],3), 'e2e99', round(d['e2e']['value'],4))"
done
