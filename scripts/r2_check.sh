#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/chk_build.log 2>&1 || { tail -20 gpurun_out/chk_build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/chk_tests.log 2>&1; echo "tests exit $?"; tail -2 gpurun_out/chk_tests.log
timeout 300 python -m pytest tests/test_gpu_runtime.py -q -s -k "holds_the_queued" 2>&1 | grep -E "held|passed|failed"
timeout 300 python scripts/bench_configs.py c1 2>/dev/null | grep '"c1"' | python -c "
import json,sys
d=json.loads(sys.stdin.read())['c1']
for dx in (False, True):
    r=[x for x in d if x['host_duplex']==dx]
    print('duplex', dx, 'p2r_us', [round(x['preempt_to_resume_us']) for x in r], 'xfer_us', [round(x['d2h_h2d_us']) for x in r], 'pack', [round(x['pack_us'],1) for x in r], 'unpack', [round(x['unpack_us'],1) for x in r])
"
