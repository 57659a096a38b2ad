"""SwitchFlow subgraph-preemption ORACLE — TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct CPU implementation (numpy, fp64 accumulation, one
rounding to fp32 per op output) of what the B200 hot path computes:

* ops.py       — the fixed op set (GEMM, bias+ReLU and its backward, column sum,
                 softmax-cross-entropy, softmax, SGD-momentum, Adam, feed, step).
* graph.py     — graph validation, PER_LAYER_PHASE / MAX_OPS partition into
                 subgraphs, live set L_k at every cut.
* staging.py   — the staging format and pack / unpack of a live set.
* runner.py    — sequential execution of the partitioned graph for T iterations
                 under a preemption schedule with simulated devices whose arenas are
                 poisoned before unpack; batch-1 inference.
* feed.py      — the workload's host input stage (u8 image decode + seeded flip).
* schedule.py  — discrete-event schedule simulation and the invariant checker
                 (no two models' subgraphs overlap on a device; per-job order; stop
                 latency bounded by the in-flight subgraph).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import anything under ``oracle/``.  It shares no code
with ``paper_conf_middleware_wur0hdh21_b200`` (the CUDA path); the only common
import is ``sf_inputs`` (seeded workload graphs and data, no method arithmetic).

Parity status per function is stated in each module header; DESIGN.md section 3
lists the pins.
"""
