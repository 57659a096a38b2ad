#!/bin/bash
# Round 2: bench smoke of the new bench line + inference-chain state profiling.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c3_build.log 2>&1
timeout 900 python bench.py > gpurun_out/r2c3_bench.json 2> gpurun_out/r2c3_bench.err; echo "bench exit $?"
tail -3 gpurun_out/r2c3_bench.err
for f in none r 1; do
  if [ $f = none ]; then FLUSH= timeout 120 python scripts/infer_bench.py 200; else FLUSH=$f timeout 120 python scripts/infer_bench.py 200; fi
done > gpurun_out/r2c3_infer.jsonl 2>&1
timeout 600 ncu --cache-control none --clock-control none \
  --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_op_read.sum,lts__t_sectors_op_write.sum,sm__cycles_active.avg,gpc__cycles_elapsed.max \
  -k regex:gemv_tma --launch-skip 60 --launch-count 60 --csv --log-file gpurun_out/r2c3_ncu_gemv.csv \
  python bench.py --steps 2 --warmup 1 --no-baselines --no-cpu-baseline > gpurun_out/r2c3_ncu.log 2>&1
echo "ncu exit $?"
