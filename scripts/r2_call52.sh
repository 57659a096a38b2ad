#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c52_build.log 2>&1 || { tail -20 gpurun_out/r2c52_build.log; exit 1; }
SF_GEMM_MERGE_BN=128 timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" 2>&1 | tail -1
for m in 64 128; do echo "MERGE_BN=$m"; SF_GEMM_MERGE_BN=$m timeout 120 python scripts/gemm_bench.py 2>&1 | tail -9; SF_GEMM_MERGE_BN=$m timeout 120 python scripts/gemm_c3.py 2>&1 | grep tma | cut -c1-80; done
for m in 64 128; do echo "MERGE_BN=$m"; SF_GEMM_MERGE_BN=$m timeout 600 python scripts/bench_configs.py c3 2>&1 | tail -1 | cut -c200-400; done
