#!/bin/bash
# p99 latency and its breakdown under bench.py variants (env / flags), 1000 requests each.
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() { timeout 300 env $1 python bench.py --steps 1000 --no-baselines --no-cpu-baseline $2 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); b=d['arrivals']['latency_breakdown_us']
print('$1 $2', 'p99', round(d['p99_ms'],4), 'p95', round(d['p95_ms'],4), 'p50', round(d['p50_ms'],4), 'pre99', round(d['preempt_latency_p99_ms'],4), 'chase99', round(d['chase']['p99_ms'],4), 'chase50', round(d['chase']['p50_ms'],4), 'p2r50', round(d['preempt_to_resume_p50_ms'],3), 'pack_gbs', round(d['migration']['pack_gbs']), 'e2e99', round(d['e2e']['value'],4), 'iter', round(d['training_iteration_ms_median'],3))
for k,v in b.items(): print('   ', k, v)"; }
for v in "$@"; do run "${v%%|*}" "${v#*|}"; done
