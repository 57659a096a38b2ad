#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c40_build.log 2>&1 || { tail -20 gpurun_out/r2c40_build.log; exit 1; }
for i in 1 2 3; do timeout 600 python -m pytest tests/test_gpu_c2_bench_config.py -q -x --timeout=300 2>&1 | tail -1; done
timeout 1800 python -m pytest tests -m gpu -q --timeout=300 > gpurun_out/r2c40_tests.log 2>&1; echo "tests exit $?"; tail -3 gpurun_out/r2c40_tests.log
