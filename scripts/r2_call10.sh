#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c10_build.log 2>&1 || { tail -20 gpurun_out/r2c10_build.log; exit 1; }
for v in 1 0; do
  for f in none 1; do
    if [ $f = none ]; then SF_GEMV_BLOCKED=$v FLUSH= timeout 120 python scripts/infer_bench.py 300; else SF_GEMV_BLOCKED=$v FLUSH=$f timeout 120 python scripts/infer_bench.py 300; fi | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('blocked=$v flush=$f device p50/p99', round(d['device_p50_ms']*1e3,1), round(d['device_p99_ms']*1e3,1))"
  done
done
timeout 300 python -m pytest tests/test_gpu_runtime.py -q -x -k "inference_paths or inference_vs_oracle" 2>&1 | tail -2
