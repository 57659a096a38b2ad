#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c29_build.log 2>&1 || { tail -20 gpurun_out/r2c29_build.log; exit 1; }
timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" 2>&1 | tail -2
SF_GEMM_MAXSPLIT=8 timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" 2>&1 | tail -2
for sh in "512 1024 1024 0" "512 1024 4096 0" "1024 1024 512 1"; do echo "== $sh"; SF_GEMM_DEBUG=8 timeout 60 python scripts/gemm_one.py $sh 3 | grep "bid 37" | tail -1; done
for v in 0 1; do echo "ATM=$v"; SF_GEMM_ATM=$v timeout 120 python scripts/gemm_c3.py 2>&1 | grep tma | cut -c1-92; done
for v in 0 1; do echo "ATM=$v"; SF_GEMM_ATM=$v timeout 600 python scripts/bench_configs.py c3 2>&1 | tail -1 | cut -c1-400; done
for v in 0 1; do echo "ATM=$v"; SF_GEMM_ATM=$v timeout 120 python scripts/gemm_bench.py 2>&1 | tail -9; done
