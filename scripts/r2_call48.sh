#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c48_build.log 2>&1 || { tail -20 gpurun_out/r2c48_build.log; exit 1; }
timeout 600 python scripts/subgraph_durations.py 2>&1 | tail -20
