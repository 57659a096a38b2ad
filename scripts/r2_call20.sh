#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c20_build.log 2>&1 || { tail -20 gpurun_out/r2c20_build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" 2>&1 | tail -3
for bk in 32 16; do echo "BK256=$bk"; SF_GEMM_BK256=$bk timeout 300 python scripts/gemm_c3.py 2>&1 | grep '"bn": 256' | cut -c1-110; done
for bk in 32 16; do echo "BK256=$bk"; SF_GEMM_BK256=$bk timeout 600 python scripts/bench_configs.py c3 2>&1 | tail -1 | cut -c1-400; done
