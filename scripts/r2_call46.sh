#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c46_build.log 2>&1 || { tail -20 gpurun_out/r2c46_build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q --timeout=300 > gpurun_out/r2c46_tests.log 2>&1; echo "tests exit $?"; tail -1 gpurun_out/r2c46_tests.log
for i in 1 2 3 4 5 6; do
SF_BENCH_WATCHDOG_S=400 timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/r2c46_bench_$i.json 2> gpurun_out/r2c46_bench_$i.err; echo "bench $i exit $?"; cut -c90-130 gpurun_out/r2c46_bench_$i.json
done
