#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c21_build.log 2>&1 || { tail -20 gpurun_out/r2c21_build.log; exit 1; }
for d in 0 2 4 6; do echo "dbg=$d"; SF_GEMM_DEBUG=$d python scripts/gemm_one.py 1024 4096 512 1 50; SF_GEMM_DEBUG=$d python scripts/gemm_one.py 1024 4096 2048 1 50; SF_GEMM_DEBUG=$d python scripts/gemm_one.py 512 4096 1024 0 50; done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 6000 --csv --log-file gpurun_out/r2c21_c3_launches.csv python scripts/bench_configs.py c3 > /dev/null 2>&1; echo "ncu exit $?"
python scripts/launch_shares.py gpurun_out/r2c21_c3_launches.csv
