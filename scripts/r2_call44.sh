#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c44_build.log 2>&1 || { tail -20 gpurun_out/r2c44_build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q --timeout=300 > gpurun_out/r2c44_tests.log 2>&1; echo "tests exit $?"; tail -3 gpurun_out/r2c44_tests.log
for i in 1 2; do timeout 600 python -m pytest tests/test_gpu_c2_bench_config.py tests/test_gpu_runtime.py -q --timeout=300 -k "open_loop or auto_preemption" 2>&1 | tail -1; done
SF_BENCH_WATCHDOG_S=600 timeout 900 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/r2c44_bench.json 2>/dev/null; echo "bench exit $?"; cut -c1-200 gpurun_out/r2c44_bench.json
