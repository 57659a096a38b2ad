#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c32_build.log 2>&1 || { tail -20 gpurun_out/r2c32_build.log; exit 1; }
for m in 1 0; do for i in 1 2 3 4 5 6; do SF_GEMM_CLUSTER_RED=$m timeout 300 python -m pytest tests/test_gpu_runtime.py -q -x -k "test_open_loop_requests_during_swap_in_are_bitwise" 2>&1 | tail -1 | sed "s/^/clred=$m /"; done; done
