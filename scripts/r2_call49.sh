#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c49_build.log 2>&1 || { tail -20 gpurun_out/r2c49_build.log; exit 1; }
timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" 2>&1 | tail -2
SF_GEMM_MAXSPLIT=8 timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" 2>&1 | tail -2
timeout 120 python scripts/gemm_bench.py 2>&1 | tail -9
timeout 600 python scripts/subgraph_durations.py 2>&1 | tail -12
