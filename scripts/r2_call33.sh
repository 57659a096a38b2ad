#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c33_build.log 2>&1 || { tail -20 gpurun_out/r2c33_build.log; exit 1; }
for i in 1 2 3 4 5 6 7 8; do timeout 300 python -m pytest tests/test_gpu_runtime.py -q -x -k "test_open_loop_requests_during_swap_in_are_bitwise" 2>&1 | tail -1; done
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/r2c33_tests.log 2>&1; tail -3 gpurun_out/r2c33_tests.log
