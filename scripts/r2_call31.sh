#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c31_build.log 2>&1 || { tail -20 gpurun_out/r2c31_build.log; exit 1; }
timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" 2>&1 | tail -2
SF_GEMM_MAXSPLIT=8 timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" 2>&1 | tail -2
timeout 120 python scripts/gemm_c3.py 2>&1 | grep tma | cut -c1-92
for m in 0 1; do echo "CLRED=$m"; SF_GEMM_CLUSTER_RED=$m timeout 600 python scripts/bench_configs.py c3 2>&1 | tail -1 | cut -c1-400; done
for m in 0 1; do echo "CLRED=$m"; SF_GEMM_CLUSTER_RED=$m timeout 120 python scripts/gemm_bench.py 2>&1 | tail -9; done
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r2c31_tests.log 2>&1; tail -3 gpurun_out/r2c31_tests.log
