#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c5_build.log 2>&1 || { tail -20 gpurun_out/r2c5_build.log; exit 1; }
timeout 900 python bench.py > gpurun_out/r2c5_bench.json 2> gpurun_out/r2c5_bench.err; echo "bench exit $?"; tail -3 gpurun_out/r2c5_bench.err
SF_BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 4 --warmup 2 > gpurun_out/r2c5_pairs.json 2> gpurun_out/r2c5_pairs.err; echo "pairs exit $?"; tail -5 gpurun_out/r2c5_pairs.err
SF_BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29534 scripts/bench_c5.py --quick --out gpurun_out/r2c5_c5.jsonl > gpurun_out/r2c5_c5.log 2>&1; echo "c5 exit $?"; tail -5 gpurun_out/r2c5_c5.log
