#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c51_build.log 2>&1 || { tail -20 gpurun_out/r2c51_build.log; exit 1; }
SF_GEMM_MERGE=2 timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" 2>&1 | tail -1
for m in 1 2; do echo "MERGE=$m"; SF_GEMM_MERGE=$m timeout 120 python scripts/gemm_bench.py 2>&1 | tail -9; done
for m in 1 2; do echo "MERGE=$m"; SF_GEMM_MERGE=$m timeout 600 python scripts/subgraph_durations.py 2>&1 | tail -13 | head -6; done
