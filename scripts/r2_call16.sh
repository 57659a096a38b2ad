#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python scripts/cliff_probe.py 2>&1
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -k mtcopy 2>&1 | tail -1
