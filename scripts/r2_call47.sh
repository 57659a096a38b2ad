#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c47_build.log 2>&1 || { tail -20 gpurun_out/r2c47_build.log; exit 1; }
for i in 1 2 3 4 5 6 7 8 9 10; do
SF_BENCH_WATCHDOG_S=400 timeout 600 python bench.py --no-baselines --no-cpu-baseline > gpurun_out/r2c47_bench_$i.json 2> gpurun_out/r2c47_bench_$i.err; rc=$?; echo "bench $i exit $rc $(cut -c90-120 gpurun_out/r2c47_bench_$i.json)"
if [ $rc -ne 0 ]; then tail -30 gpurun_out/r2c47_bench_$i.err; fi
done
