#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/wk_build.log 2>&1 || { tail -20 gpurun_out/wk_build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "copy or mtcopy or walk" 2>&1 | tail -1
for u in 8 16; do for b in 1 2 3; do
  SF_COPY_UNROLL=$u SF_COPY_BPS=$b timeout 300 python scripts/pack_walk_ab.py 2>&1 | head -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read())['probe']; print('unroll', $u, 'bps', $b, {k: (round(v['pack_gbs']), round(v['unpack_gbs'])) for k, v in d.items() if isinstance(v, dict)})"
done; done
