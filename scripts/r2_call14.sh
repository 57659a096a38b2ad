#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c14_build.log 2>&1 || { tail -20 gpurun_out/r2c14_build.log; exit 1; }
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/r2c14_tests.log 2>&1; echo "tests exit $?"; tail -5 gpurun_out/r2c14_tests.log
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
