#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c27_build.log 2>&1 || { tail -20 gpurun_out/r2c27_build.log; exit 1; }
for mc in "2,1" "1,2" "2,2" "4,1"; do echo "MC=$mc"; SF_GEMM_MC=$mc timeout 180 python -m pytest tests/test_gpu_kernels.py -q -x -k "gemm" 2>&1 | tail -2; done
for mc in "1,1" "2,1" "1,2" "2,2" "4,1"; do echo "MC=$mc"; SF_GEMM_MC=$mc timeout 120 python scripts/gemm_c3.py 2>&1 | grep tma | cut -c1-92; done
for mc in "1,1" "2,1" "2,2"; do echo "MC=$mc"; SF_GEMM_MC=$mc timeout 120 python scripts/gemm_bench.py 2>&1 | tail -9; done
