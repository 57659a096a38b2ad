#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c37_build.log 2>&1 || { tail -20 gpurun_out/r2c37_build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_c2_bench_config.py -q -x -k "infer or softmax or request" > gpurun_out/r2c37_tests.log 2>&1; tail -3 gpurun_out/r2c37_tests.log
