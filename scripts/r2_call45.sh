#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c45_build.log 2>&1 || { tail -20 gpurun_out/r2c45_build.log; exit 1; }
for i in 1 2 3 4; do
SF_BENCH_WATCHDOG_S=400 timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/r2c45_bench_$i.json 2> gpurun_out/r2c45_bench_$i.err; echo "bench $i exit $?"; cut -c1-120 gpurun_out/r2c45_bench_$i.json
done
