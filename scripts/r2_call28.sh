#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c28_build.log 2>&1 || { tail -20 gpurun_out/r2c28_build.log; exit 1; }
for atm in 1 0; do
for sh in "512 4096 1024 0" "512 1024 1024 0" "1024 4096 512 1" "25088 64 576 0"; do echo "== ATM=$atm $sh"; SF_GEMM_ATM=$atm SF_GEMM_DEBUG=8 timeout 60 python scripts/gemm_one.py $sh 3 | grep "bid 37" | tail -1; done
for d in 10 12 14; do echo "== ATM=$atm dbg=$d 512 4096 1024"; SF_GEMM_ATM=$atm SF_GEMM_DEBUG=$d timeout 60 python scripts/gemm_one.py 512 4096 1024 0 3 | grep "bid 37" | tail -1; done
done
echo "== MC 2,1"; SF_GEMM_MC=2,1 SF_GEMM_DEBUG=8 timeout 60 python scripts/gemm_one.py 512 4096 1024 0 3 | grep "bid 37" | tail -1
