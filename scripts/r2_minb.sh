#!/bin/bash
# Cluster-free GEMV CTAs per SM (compile-time SF_GEMV_MINB: 2 -> 96 registers, 3 -> 80)
for mb in 2 NOPRE 2 NOPRE; do
  rm -f paper_conf_middleware_wur0hdh21_b200/_build/kernels_gemv.o
  SF_NVCC_EXTRA=$([ $mb = NOPRE ] && echo -DSF_GEMV_NOPRE=1 || echo -DSF_GEMV_MINB=2) python -c "import __graft_entry__ as g; g.build()" > gpurun_out/mb_build.log 2>&1 || { tail -5 gpurun_out/mb_build.log; exit 1; }
  echo "minb=$mb trace: $(timeout 300 python scripts/blk_trace.py 40 2>&1 | tail -2 | tr '\n' ' ' | cut -c1-260)"
  echo "minb=$mb $(FLUSH=1 timeout 300 python scripts/infer_bench.py 300 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print({k: round(d[k]*1e3 if k.endswith('ms') else d[k],2) for k in ('p50_ms','p99_ms','device_p50_ms','device_p99_ms')})")"
done
timeout 300 python -m pytest tests/test_gpu_runtime.py -q -k "c4_inference" 2>&1 | tail -1
