#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c24_build.log 2>&1 || { tail -20 gpurun_out/r2c24_build.log; exit 1; }
timeout 600 ncu --set full --import-source on --clock-control none -k regex:gemm_tma -s 3 -c 1 -o gpurun_out/r2c24_qkvo -f python scripts/gemm_one.py 512 1024 1024 0 5 > /dev/null 2>&1; echo "ncu $?"
timeout 600 ncu --set full --import-source on --clock-control none -k regex:gemm_tma -s 3 -c 1 -o gpurun_out/r2c24_ffni -f python scripts/gemm_one.py 512 4096 1024 0 5 > /dev/null 2>&1; echo "ncu $?"
for d in 0 2 4 6; do echo "dbg=$d"; SF_GEMM_DEBUG=$d python scripts/gemm_one.py 512 1024 1024 0 50; SF_GEMM_DEBUG=$d python scripts/gemm_one.py 512 4096 1024 0 50; done
