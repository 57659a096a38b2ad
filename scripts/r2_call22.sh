#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c22_build.log 2>&1 || { tail -20 gpurun_out/r2c22_build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" 2>&1 | tail -3
for cr in 0 1; do echo "CLUSTER_RED=$cr"; SF_GEMM_CLUSTER_RED=$cr timeout 300 python scripts/gemm_c3.py 2>&1 | cut -c1-150; done
for cr in 0 1; do echo "CLUSTER_RED=$cr"; SF_GEMM_CLUSTER_RED=$cr timeout 600 python scripts/bench_configs.py c3 2>&1 | tail -1 | cut -c1-400; done
for cr in 0 1; do echo "CLUSTER_RED=$cr"; SF_GEMM_CLUSTER_RED=$cr timeout 300 python scripts/gemm_bench.py 2>&1 | tail -4; done
