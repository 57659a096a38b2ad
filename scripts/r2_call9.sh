#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c9_build.log 2>&1 || { tail -20 gpurun_out/r2c9_build.log; exit 1; }
timeout 300 python -m pytest tests/test_gpu_runtime.py -q -x -k "clock_mapping or inference_vs_oracle" -s 2>&1 | grep -E "start - submit|I3|passed|failed|Error"
