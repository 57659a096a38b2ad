#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for v in 1 0; do
SF_GEMV_BLOCKED=$v FLUSH=1 timeout 300 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,launch__grid_size,launch__occupancy_limit_registers,sm__cycles_active.avg -k regex:"gemv" -s 30 -c 3 --csv python scripts/infer_bench.py 40 > gpurun_out/r2c11_ncu_$v.csv 2>/dev/null
python - <<PY
import csv
rows=[r for r in csv.reader(open('gpurun_out/r2c11_ncu_$v.csv')) if len(r)>10]
h=rows[0]; out={}
for r in rows[1:]:
    d=dict(zip(h,r)); out.setdefault((d['ID'],d['Kernel Name'][:34]),{})[d['Metric Name']]=d['Metric Value']
for k,v in out.items(): print('$v', k, v)
PY
done
