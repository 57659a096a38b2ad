#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c13_build.log 2>&1 || { tail -20 gpurun_out/r2c13_build.log; exit 1; }
timeout 900 python bench.py > gpurun_out/r2c13_bench.json 2> gpurun_out/r2c13_bench.err; echo "bench exit $?"
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/r2c13_tests.log 2>&1; echo "tests exit $?"; tail -3 gpurun_out/r2c13_tests.log
