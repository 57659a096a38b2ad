#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c3_build.log 2>&1 || { tail -20 gpurun_out/c3_build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "chain" 2>&1 | tail -1
timeout 300 python scripts/chain_trace.py 2>&1 | tail -5
for fl in 1 ""; do
for v in "SF_CHAIN=0" "SF_CHAIN=1" "SF_CHAIN_CARVE=0" "SF_CHAIN_CARVE=0 SF_CHAIN_TAIL=0"; do
  echo "flush=$fl $v $(env $v FLUSH=$fl timeout 300 python scripts/infer_bench.py 300 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print({k: round(d[k]*1e3 if k.endswith('ms') else d[k],2) for k in ('p50_ms','p99_ms','device_p50_ms','device_p99_ms','launch_us_p50')})")"
done; done
