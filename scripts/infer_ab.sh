#!/bin/bash
# A/B of the inference GEMV path: latency (infer_bench) and per-kernel ncu durations.
for m in ${MODES:-1 0}; do SF_GEMV_CLUSTER=$m python scripts/infer_bench.py 2>/dev/null | tail -1; done
for m in ${MODES:-1 0}; do
  SF_GEMV_CLUSTER=$m ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum --clock-control none --csv \
    --log-file gpurun_out/infer_$m.csv python scripts/infer_bench.py 25 >/dev/null 2>&1
done
