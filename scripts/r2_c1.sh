#!/bin/bash
# C1 host round trip vs duplex chunk size (reading Q31; round-2 verdict #8)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c1_build.log 2>&1 || { tail -20 gpurun_out/c1_build.log; exit 1; }
for ck in "" 1024 512 256 128; do
  if [ -n "$ck" ]; then export SF_DUPLEX_CHUNK_KB=$ck; else unset SF_DUPLEX_CHUNK_KB; fi
  timeout 300 python scripts/bench_configs.py c1 2>/dev/null | grep '"c1"' | python -c "
import json,sys
d=json.loads(sys.stdin.read())['c1']
for dx in (False, True):
    r=[x for x in d if x['host_duplex']==dx]
    print('chunk_kb', '${ck:-2048}', 'duplex', dx, 'p2r_us', [round(x['preempt_to_resume_us']) for x in r], 'xfer_us', [round(x['d2h_h2d_us']) for x in r], 'live_MB', [round(x['live_bytes']/1e6,2) for x in r])
"
done
