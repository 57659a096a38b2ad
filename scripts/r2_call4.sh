#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c4_build.log 2>&1 || { tail -20 gpurun_out/r2c4_build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_runtime.py -q -x -k "chain or inference or gate or open_loop or chase" -s > gpurun_out/r2c4_tests.log 2>&1; echo "tests exit $?"; tail -5 gpurun_out/r2c4_tests.log
for f in none r 1; do
  if [ $f = none ]; then FLUSH= timeout 120 python scripts/infer_bench.py 200; else FLUSH=$f timeout 120 python scripts/infer_bench.py 200; fi
done > gpurun_out/r2c4_infer.jsonl 2>&1
SF_CHAIN=0 FLUSH=1 timeout 120 python scripts/infer_bench.py 200 >> gpurun_out/r2c4_infer.jsonl 2>&1
cat gpurun_out/r2c4_infer.jsonl
timeout 120 python scripts/chain_trace.py > gpurun_out/r2c4_chain_trace.log 2>&1; tail -30 gpurun_out/r2c4_chain_trace.log
