#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 300 python -m pytest tests/test_gpu_kernels.py -q 2>&1 | tail -3
for mode in ${MODES:-legacy tma rawhi}; do
  if [ $mode = legacy ]; then export SF_GEMM_PATH=legacy; else unset SF_GEMM_PATH; fi
  if [ $mode = rawhi ]; then unset SF_GEMM_RAWHI; else export SF_GEMM_RAWHI=0; fi
  ncu --metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:gemm --csv --log-file gpurun_out/gemm_$mode.csv python scripts/gemm_bench.py > gpurun_out/gemm_$mode.log 2>&1
  head -3 gpurun_out/gemm_$mode.log
done
