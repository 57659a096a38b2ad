#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c30_build.log 2>&1 || { tail -20 gpurun_out/r2c30_build.log; exit 1; }
timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" 2>&1 | tail -2
SF_GEMM_MAXSPLIT=8 timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" 2>&1 | tail -2
for m in 1 2; do for sh in "512 1024 1024 0" "1024 1024 512 1"; do echo "== mode $m $sh"; SF_GEMM_CLUSTER_RED=$m SF_GEMM_DEBUG=8 timeout 60 python scripts/gemm_one.py $sh 3 | grep "bid 37" | tail -1; done; done
for m in 0 1 2; do echo "MODE=$m"; SF_GEMM_CLUSTER_RED=$m timeout 120 python scripts/gemm_c3.py 2>&1 | grep '"splits": [2-8]' | cut -c1-92; done
for m in 0 1 2; do echo "MODE=$m"; SF_GEMM_CLUSTER_RED=$m timeout 600 python scripts/bench_configs.py c3 2>&1 | tail -1 | cut -c1-400; done
for m in 0 1 2; do echo "MODE=$m"; SF_GEMM_CLUSTER_RED=$m timeout 120 python scripts/gemm_bench.py 2>&1 | tail -9; done
