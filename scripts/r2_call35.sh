#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c35_build.log 2>&1 || { tail -20 gpurun_out/r2c35_build.log; exit 1; }
timeout 300 python scripts/blk_trace.py 60
HOSTIO=1 timeout 300 python scripts/blk_trace.py 60
