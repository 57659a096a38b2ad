#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c43_build.log 2>&1 || { tail -20 gpurun_out/r2c43_build.log; exit 1; }
timeout 300 python scripts/bench_configs.py c1 2>&1 | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read())
for r in d['c1']: print({k: (round(v,1) if isinstance(v,float) else v) for k,v in r.items()})"
timeout 600 python -m pytest tests/test_gpu_runtime.py -q -x --timeout=300 -k "duplex or swap or host" 2>&1 | tail -1
