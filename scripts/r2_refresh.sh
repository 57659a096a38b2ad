#!/bin/bash
# Round-2 final refresh under gpurun: tests, smoke, bench (ours + reference arm), per-config
# measurements, ncu launch list of the bench command, ncu --set full captures of the pack
# walk, the inference GEMV and the training GEMM.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_build.log 2>&1 || { tail -20 gpurun_out/r02_build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r02_gpu_tests.log 2>&1; echo "tests exit $?"; tail -1 gpurun_out/r02_gpu_tests.log
timeout 180 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02_smoke.log 2>&1; echo "smoke exit $?"; tail -1 gpurun_out/r02_smoke.log
SF_BENCH_WATCHDOG_S=800 timeout 900 python bench.py > gpurun_out/r02_bench.json 2> gpurun_out/r02_bench.err; echo "bench exit $?"; cut -c1-300 gpurun_out/r02_bench.json
timeout 600 python bench.py --impl reference > gpurun_out/r02_bench_ref.json 2> gpurun_out/r02_bench_ref.err; echo "ref exit $?"; cut -c1-200 gpurun_out/r02_bench_ref.json
timeout 600 python scripts/bench_configs.py c1 c3 > gpurun_out/r02_configs.log 2>&1; echo "configs exit $?"; cp gpurun_out/configs.json gpurun_out/r02_configs.json 2>/dev/null
timeout 300 python scripts/gemm_c3.py > gpurun_out/r02_gemm_c3.jsonl 2>&1
timeout 300 python scripts/gemm_bench.py > gpurun_out/r02_gemm_bench.log 2>&1
timeout 300 python scripts/blk_trace.py 60 > gpurun_out/r02_blk_trace.log 2>&1
timeout 300 python scripts/subgraph_durations.py > gpurun_out/r02_subgraph_durations.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 6000 --csv \
  --log-file gpurun_out/r02_launches.csv python bench.py --steps 3 --warmup 3 --no-baselines --no-cpu-baseline --min-requests 0 > gpurun_out/r02_ncu_bench.log 2>&1; echo "ncu list exit $?"
python scripts/launch_shares.py gpurun_out/r02_launches.csv > gpurun_out/r02_launch_shares.md
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mtcopy -s 2 -c 2 \
  -o gpurun_out/r02_prof_pack -f python bench.py --steps 3 --warmup 3 --no-baselines --no-cpu-baseline --min-requests 0 > gpurun_out/r02_ncu_pack.log 2>&1; echo "ncu pack exit $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemv_blk -s 6 -c 3 \
  -o gpurun_out/r02_prof_gemv -f python bench.py --steps 3 --warmup 3 --no-baselines --no-cpu-baseline --min-requests 0 > gpurun_out/r02_ncu_gemv.log 2>&1; echo "ncu gemv exit $?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tma -s 20 -c 4 \
  -o gpurun_out/r02_prof_gemm -f python bench.py --steps 3 --warmup 3 --no-baselines --no-cpu-baseline --min-requests 0 > gpurun_out/r02_ncu_gemm.log 2>&1; echo "ncu gemm exit $?"
ls gpurun_out | grep r02
