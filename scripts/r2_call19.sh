#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c19_build.log 2>&1 || { tail -20 gpurun_out/r2c19_build.log; exit 1; }
SF_COPY_BULK=1 timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_runtime.py tests/test_gpu_c2_bench_config.py -q -rf -k "mtcopy or cut0 or mid_cut or every_cut or explicit_preempt or seeded or two_device" > gpurun_out/r2c19_bulk_tests.log 2>&1; tail -5 gpurun_out/r2c19_bulk_tests.log
for b in 0 1; do SF_COPY_BULK=$b timeout 300 python scripts/pack_probe_ncu.py 2>&1 | tail -3 | sed "s/^/bulk=$b /"; done
SF_COPY_BULK=1 timeout 300 python scripts/cliff_probe.py 2>&1 | head -4
SF_BENCH_WATCHDOG_S=500 SF_BENCH_SAME_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 > gpurun_out/r2c19_pairs.json 2> gpurun_out/r2c19_pairs.err; echo "pairs exit $?"
