#!/bin/bash
# Full refresh under gpurun: tests, smoke, bench, ncu launch list, ncu full captures.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests.log 2>&1; echo "tests exit $?"; tail -3 gpurun_out/gpu_tests.log
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke exit $?"; tail -1 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench exit $?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 20 --warmup 3 --no-baselines --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mtcopy -s 2 -c 2 \
  -o gpurun_out/prof_pack python bench.py --steps 6 --warmup 3 --no-baselines --no-cpu-baseline > gpurun_out/ncu_pack.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemv_tma -s 3 -c 3 \
  -o gpurun_out/prof_gemv python bench.py --steps 6 --warmup 3 --no-baselines --no-cpu-baseline > gpurun_out/ncu_gemv.log 2>&1
ls gpurun_out
