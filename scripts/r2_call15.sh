#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python scripts/cliff_probe.py > gpurun_out/r2c15_cliff.jsonl 2>&1; cat gpurun_out/r2c15_cliff.jsonl
timeout 300 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_op_read.sum,lts__t_sectors_op_write.sum -k regex:mtcopy --csv python scripts/pack_probe_ncu.py > gpurun_out/r2c15_pack_ncu.csv 2>&1; echo "ncu exit $?"
