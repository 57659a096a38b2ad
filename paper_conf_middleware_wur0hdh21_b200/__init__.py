"""SwitchFlow subgraph-granularity preemption, B200-native (sm_100a).

The product path is libswitchflow_b200.so (CUDA kernels + C++ runtime, include/sf.h);
this package only binds it.  See DESIGN.md.
"""
import os as _os

# The runtime keeps several streams per device (training, request, migration, clock) and the
# drain gate parks the training stream on a memory wait; with the default 8 hardware work
# queues, streams beyond that share a queue and a parked one can hold up its queue-mate.
# Effective only if set before the process creates its CUDA context (bench.py and the tests
# import this package first).
_os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

from ._abi import LIB_PATH, SFError, lib  # noqa: E402,F401

__all__ = ["LIB_PATH", "SFError", "lib"]
