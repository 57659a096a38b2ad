"""SwitchFlow subgraph-granularity preemption, B200-native (sm_100a).

The product path is libswitchflow_b200.so (CUDA kernels + C++ runtime, include/sf.h);
this package only binds it.  See DESIGN.md.
"""
from ._abi import LIB_PATH, SFError, lib  # noqa: F401

__all__ = ["LIB_PATH", "SFError", "lib"]
