#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c25_build.log 2>&1 || { tail -20 gpurun_out/r2c25_build.log; exit 1; }
for sh in "512 1024 1024 0" "512 4096 1024 0" "1024 4096 512 1" "512 1024 4096 0"; do echo "== $sh"; SF_GEMM_DEBUG=8 python scripts/gemm_one.py $sh 3 | tail -4; done
