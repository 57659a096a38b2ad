#!/bin/bash
# Round-2 final refresh (after r2_refresh.sh's per-config measurements): tests, smoke, bench (ours
# + reference arm), the ncu launch list of the bench command, ncu --set full of the pack walk and
# the request GEMVs.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_build.log 2>&1 || { tail -20 gpurun_out/r02_build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r02_gpu_tests.log 2>&1; echo "tests exit $?"; tail -1 gpurun_out/r02_gpu_tests.log
timeout 180 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02_smoke.log 2>&1; echo "smoke exit $?"; tail -1 gpurun_out/r02_smoke.log
SF_BENCH_WATCHDOG_S=800 timeout 900 python bench.py > gpurun_out/r02_bench.json 2> gpurun_out/r02_bench.err; echo "bench exit $?"; cut -c1-200 gpurun_out/r02_bench.json
timeout 600 python bench.py --impl reference > gpurun_out/r02_bench_ref.json 2> gpurun_out/r02_bench_ref.err; echo "ref exit $?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 6000 --csv \
  --log-file gpurun_out/r02_launches.csv python bench.py --steps 3 --warmup 3 --no-baselines --no-cpu-baseline --min-requests 0 > gpurun_out/r02_ncu_bench.log 2>&1; echo "ncu list exit $?"
python scripts/launch_shares.py gpurun_out/r02_launches.csv > gpurun_out/r02_launch_shares.md
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mtcopy -s 2 -c 2 \
  -o gpurun_out/r02_prof_pack -f python bench.py --steps 3 --warmup 3 --no-baselines --no-cpu-baseline --min-requests 0 > gpurun_out/r02_ncu_pack.log 2>&1; echo "ncu pack exit $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemv_blk -s 6 -c 3 \
  -o gpurun_out/r02_prof_gemv -f python bench.py --steps 3 --warmup 3 --no-baselines --no-cpu-baseline --min-requests 0 > gpurun_out/r02_ncu_gemv.log 2>&1; echo "ncu gemv exit $?"
timeout 300 python scripts/blk_trace.py 40 > gpurun_out/r02_blk_trace_final.log 2>&1; tail -4 gpurun_out/r02_blk_trace_final.log
