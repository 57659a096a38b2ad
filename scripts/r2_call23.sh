#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c23_build.log 2>&1 || { tail -20 gpurun_out/r2c23_build.log; exit 1; }
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r2c23_tests.log 2>&1; tail -3 gpurun_out/r2c23_tests.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 6000 --csv --log-file gpurun_out/r2c23_c3_launches.csv python scripts/bench_configs.py c3 > /dev/null 2>&1; echo "ncu exit $?"
python scripts/launch_shares.py gpurun_out/r2c23_c3_launches.csv
