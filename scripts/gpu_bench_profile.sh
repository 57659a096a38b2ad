#!/bin/bash
# bench + ncu launch list + full captures of the top kernels + per-config runs (under gpurun)
python -c "import __graft_entry__ as g; g.build()" 2> /dev/null
python bench.py --steps 200 --warmup 10 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench exit $?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 10 --warmup 3 --no-baselines --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mtcopy -s 2 -c 2 \
  -o gpurun_out/prof_pack python bench.py --steps 6 --warmup 3 --no-baselines --no-cpu-baseline > gpurun_out/ncu_pack.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tma -s 20 -c 2 \
  -o gpurun_out/prof_gemm python bench.py --steps 6 --warmup 3 --no-baselines --no-cpu-baseline > gpurun_out/ncu_gemm.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemv4 -s 2 -c 2 \
  -o gpurun_out/prof_gemv python bench.py --steps 6 --warmup 3 --no-baselines --no-cpu-baseline > gpurun_out/ncu_gemv.log 2>&1
timeout 900 python scripts/bench_configs.py c1 c3 c5 > gpurun_out/configs.log 2>&1; echo "configs exit $?"
ls gpurun_out
