#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c8_build.log 2>&1 || { tail -20 gpurun_out/r2c8_build.log; exit 1; }
SF_BENCH_WATCHDOG_S=400 SF_BENCH_SAME_GPU=1 timeout 500 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 10 --warmup 2 > gpurun_out/r2c8_pairs.json 2> gpurun_out/r2c8_pairs.err; echo "pairs exit $?"; grep RuntimeError gpurun_out/r2c8_pairs.err | head -3
timeout 900 python bench.py > gpurun_out/r2c8_bench.json 2> gpurun_out/r2c8_bench.err; echo "bench exit $?"
