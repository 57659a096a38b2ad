#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c6_build.log 2>&1 || { tail -20 gpurun_out/r2c6_build.log; exit 1; }
SF_BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 4 --warmup 2 > gpurun_out/r2c6_pairs.json 2> gpurun_out/r2c6_pairs.err; echo "pairs exit $?"; grep -E "RuntimeError|Error" gpurun_out/r2c6_pairs.err | head -5; cat gpurun_out/r2c6_pairs.json | head -c 1500
timeout 300 python -m pytest tests/test_gpu_runtime.py -q -x -k "inference_vs_oracle" -s 2>&1 | grep -E "I3|passed|failed"
