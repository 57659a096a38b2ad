#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" 2> /dev/null
timeout 300 python -m pytest tests/test_gpu_kernels.py -q --timeout 60 -k gemm 2>&1 | tail -2
for mode in 0 1; do
  SF_GEMM_PERSISTENT=$mode ncu --metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:"gemm|splitk" --csv --log-file gpurun_out/gemm_p$mode.csv python scripts/gemm_bench.py > /dev/null 2>&1
done
