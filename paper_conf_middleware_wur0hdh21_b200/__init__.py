"""SwitchFlow subgraph-granularity preemption, B200-native (sm_100a).

The product path is libswitchflow_b200.so (CUDA kernels + C++ runtime, include/sf.h);
this package only binds it.  See DESIGN.md.
"""
# With the drain gate (sf_config.drain_gate, off by default) the training stream parks on a
# memory wait; with the default 8 hardware work queues, streams beyond that share a queue and a
# parked one can hold up its queue-mate (the runtime's 5 ms valve then releases it).  Callers
# that turn the gate on should set CUDA_DEVICE_MAX_CONNECTIONS=32 before their CUDA context
# exists (bench.py --gate 1 and the tests do); without the gate the default 8 queues measured
# faster (bench: solo training 187 vs 142 iterations/s, reading Q38).

from ._abi import LIB_PATH, SFError, lib  # noqa: E402,F401

__all__ = ["LIB_PATH", "SFError", "lib"]
