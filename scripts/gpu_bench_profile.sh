#!/bin/bash
# bench + ncu launch list + one full capture of the pack kernel and the GEMM (run under gpurun)
set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null
python bench.py --steps 200 --warmup 10 > gpurun_out/bench.json 2> gpurun_out/bench.err
tail -c 3000 gpurun_out/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 10 --warmup 3 --no-baselines --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mtcopy -s 2 -c 2 \
  -o gpurun_out/prof_pack python bench.py --steps 6 --warmup 3 --no-baselines --no-cpu-baseline > gpurun_out/ncu_pack.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tma -s 20 -c 2 \
  -o gpurun_out/prof_gemm python bench.py --steps 6 --warmup 3 --no-baselines --no-cpu-baseline > gpurun_out/ncu_gemm.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemv4 -s 2 -c 2 \
  -o gpurun_out/prof_gemv python bench.py --steps 6 --warmup 3 --no-baselines --no-cpu-baseline > gpurun_out/ncu_gemv.log 2>&1
ls -la gpurun_out
