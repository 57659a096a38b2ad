python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
run() { timeout 300 env $2 python bench.py --steps 1000 --no-baselines --no-cpu-baseline --duplex $1 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('duplex $1 $2', 'p99', round(d['p99_ms'],4), 'p95', round(d['p95_ms'],4), 'p50', round(d['p50_ms'],4), 'pre99', round(d['preempt_latency_p99_ms'],4), 'p2r50', round(d['preempt_to_resume_p50_ms'],3), 'chase99', round(d['chase']['p99_ms'],4), 'chase_p2r50', round(d['chase']['preempt_to_resume_p50_ms'],3), 'e2e99', round(d['e2e']['value'],4), 'dev50', d['arrivals']['inference_device_us_p50'])"; }
run 0 X=0
run 1 X=0
run 1 SF_DUPLEX_QUIET=0
run 1 SF_DUPLEX_DEPTH=1
run 1 SF_DUPLEX_CHUNK_KB=1024
run 1 "SF_DUPLEX_CHUNK_KB=1024 SF_DUPLEX_DEPTH=1"
