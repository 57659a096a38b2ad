#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c7_build.log 2>&1 || { tail -20 gpurun_out/r2c7_build.log; exit 1; }
SF_BENCH_WATCHDOG_S=100 SF_BENCH_SAME_GPU=1 timeout 160 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 2 --warmup 1 --requests-per-step 20 --gate 1 > gpurun_out/r2c7_pairs.json 2> gpurun_out/r2c7_pairs.err; echo "pairs exit $?"
grep -E "RuntimeError" gpurun_out/r2c7_pairs.err | head -5
