#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
SF_BENCH_SAME_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29534 scripts/bench_c5.py --out gpurun_out/r2c17_c5.jsonl > gpurun_out/r2c17_c5.log 2>&1; echo "c5 exit $?"
SF_BENCH_WATCHDOG_S=500 SF_BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 > gpurun_out/r2c17_pairs.json 2> gpurun_out/r2c17_pairs.err; echo "pairs exit $?"
