"""ctypes declarations of include/sf.h (argument marshalling only).

Every name here is the C symbol of the same name in libswitchflow_b200.so.  Loading
fails loudly when the library is missing: there is no CPU fallback.
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libswitchflow_b200.so")

SF_OK = 0
SF_EINVAL = -1
SF_ENOMEM = -2
SF_ESTATE = -3
SF_EBUSY = -4
SF_ECUDA = -5
SF_ETIMEOUT = -6
SF_EUNSUPPORTED = -7
SF_TARGET_HOST = -1
SF_HOST_CE = 0
SF_HOST_ZC = 1
SF_MIG_SM = 0
SF_MIG_CE = 1
SF_PART_PER_LAYER_PHASE = 0
SF_PART_MAX_OPS = 1
JOB_STATES = {0: "running", 1: "stopping", 2: "migrating", 3: "preempted", 4: "done", 5: "failed",
              6: "migrated_out"}
EV_TRAIN, EV_INFER, EV_MIGRATE, EV_HOST = 0, 1, 2, 3
INFER_JOB_FLAG = 1 << 20


class sf_tensor_desc(C.Structure):
    _fields_ = [("rows", C.c_int32), ("cols", C.c_int32), ("dtype", C.c_int32), ("kind", C.c_int32)]


class sf_op_desc(C.Structure):
    _fields_ = [("type", C.c_int32), ("n_in", C.c_int32), ("in_", C.c_int32 * 6),
                ("n_out", C.c_int32), ("out", C.c_int32 * 3), ("flags", C.c_int32),
                ("phase", C.c_int32), ("f", C.c_float * 4)]


class sf_graph_desc(C.Structure):
    _fields_ = [("name", C.c_char_p), ("n_tensors", C.c_uint32),
                ("tensors", C.POINTER(sf_tensor_desc)), ("n_ops", C.c_uint32),
                ("ops", C.POINTER(sf_op_desc))]


class sf_config(C.Structure):
    _fields_ = [("n_devices", C.c_int32), ("cuda_ordinals", C.POINTER(C.c_int32)),
                ("exclusive_gpu", C.c_int32), ("auto_preempt", C.c_int32),
                ("iteration_granularity", C.c_int32), ("host_mode", C.c_int32),
                ("poison_released", C.c_int32), ("trace_capacity", C.c_int32),
                ("max_inflight", C.c_int32), ("defer_migration", C.c_int32),
                ("device_budget_bytes", C.c_uint64), ("dispatch_spin_us", C.c_int32),
                ("inflight_budget_us", C.c_int32), ("migrate_home", C.c_int32),
                ("migration_engine", C.c_int32), ("host_stage_inline", C.c_int32),
                ("host_duplex", C.c_int32), ("infer_l2_persist_bytes", C.c_uint64),
                ("early_launch", C.c_int32), ("drain_gate", C.c_int32)]


class sf_partition_opts(C.Structure):
    _fields_ = [("policy", C.c_int32), ("max_ops", C.c_int32), ("update_chunks", C.c_int32)]


class sf_partition_info(C.Structure):
    _fields_ = [("n_subgraphs", C.c_int32), ("arena_bytes", C.c_uint64),
                ("staging_bytes", C.c_uint64), ("persistent_bytes", C.c_uint64),
                ("max_live_bytes", C.c_uint64)]


class sf_job_info(C.Structure):
    _fields_ = [("state", C.c_int32), ("dev", C.c_int32), ("iter", C.c_int64), ("k", C.c_int32),
                ("n_preemptions", C.c_int32), ("migrated_bytes", C.c_uint64),
                ("last_pack_us", C.c_double), ("last_xfer_us", C.c_double),
                ("last_unpack_us", C.c_double), ("last_stop_ns", C.c_uint64),
                ("last_resume_ns", C.c_uint64), ("n_reparks", C.c_int64),
                ("submit_ns", C.c_uint64), ("priority", C.c_int32), ("home", C.c_int32)]


class sf_cut_info(C.Structure):
    _fields_ = [("iter", C.c_int64), ("k", C.c_int32), ("n_tensors", C.c_int32),
                ("live_bytes", C.c_uint64), ("t_req_ns", C.c_uint64), ("t_stop_ns", C.c_uint64),
                ("src_dev", C.c_int32), ("dst_dev", C.c_int32)]


class sf_timing(C.Structure):
    _fields_ = [("arrival_ns", C.c_uint64), ("start_ns", C.c_uint64), ("end_ns", C.c_uint64),
                ("dev", C.c_int32), ("preempted_job", C.c_int32), ("cut_iter", C.c_int64),
                ("cut_k", C.c_int32), ("device_us", C.c_float),
                ("launch_us", C.c_float), ("dispatch_us", C.c_float)]


class sf_trace_event(C.Structure):
    _fields_ = [("dev", C.c_int32), ("job", C.c_int32), ("kind", C.c_int32), ("k", C.c_int32),
                ("iter", C.c_int64), ("t0_ns", C.c_uint64), ("t1_ns", C.c_uint64),
                ("arrival_ns", C.c_uint64), ("d0_ns", C.c_uint64), ("d1_ns", C.c_uint64)]


class sf_cut_request(C.Structure):
    _fields_ = [("iter", C.c_int64), ("k", C.c_int32), ("target", C.c_int32)]


class sf_ipc_arena(C.Structure):
    _fields_ = [("handle", C.c_uint8 * 64), ("offset", C.c_uint64), ("arena_bytes", C.c_uint64),
                ("cuda_ordinal", C.c_int32), ("pad", C.c_int32)]


class sf_feed_desc(C.Structure):
    _fields_ = [("fn", C.c_void_p), ("user", C.c_void_p), ("n", C.c_int32),
                ("bytes", C.POINTER(C.c_uint64)), ("depth", C.c_int32), ("shared", C.c_int32),
                ("dev", C.c_int32), ("pad", C.c_int32)]


class sf_u8_stage(C.Structure):
    _fields_ = [("images", C.c_void_p), ("labels", C.c_void_p), ("pool_rows", C.c_int64),
                ("batch", C.c_int32), ("cols", C.c_int32), ("img_w", C.c_int32),
                ("seed", C.c_uint32)]


class sf_gemm_path(C.Structure):
    _fields_ = [("kind", C.c_int32), ("bn", C.c_int32), ("splits", C.c_int32), ("a_mn", C.c_int32),
                ("b_mn", C.c_int32), ("pad", C.c_int32)]


class sf_migration_probe(C.Structure):
    _fields_ = [("pack_us", C.c_double), ("unpack_us", C.c_double), ("live_bytes", C.c_uint64),
                ("staging_bytes", C.c_uint64)]


class sf_slot_info(C.Structure):
    _fields_ = [("owner", C.c_int32), ("queued", C.c_int32), ("gate_held", C.c_int32), ("pad", C.c_int32),
                ("gate_value", C.c_uint32), ("gate_arrived", C.c_uint32), ("next_ticket", C.c_uint32),
                ("gate_valve", C.c_uint32)]


class sf_copy_desc(C.Structure):
    _fields_ = [("src", C.c_void_p), ("dst", C.c_void_p), ("nbytes", C.c_uint64),
                ("span", C.c_uint64)]


_P = C.POINTER
_vp = C.c_void_p
_st = C.c_int32
# name: (restype, argtypes) — mirrors include/sf.h one to one
PROTOTYPES = {
    "sf_create": (_st, [_P(sf_config), _P(_vp)]),
    "sf_destroy": (None, [_vp]),
    "sf_last_error": (C.c_char_p, []),
    "sf_abi_version": (C.c_int32, []),
    "sf_register_graph": (_st, [_vp, _P(sf_graph_desc), C.c_int32, _P(C.c_uint32)]),
    "sf_partition": (_st, [_vp, C.c_uint32, _P(sf_partition_opts), _P(sf_partition_info)]),
    "sf_subgraph_range": (_st, [_vp, C.c_uint32, C.c_int32, _P(C.c_int32), _P(C.c_int32)]),
    "sf_live_set": (_st, [_vp, C.c_uint32, C.c_int32, _P(C.c_uint32), C.c_uint32,
                          _P(C.c_uint32), _P(C.c_uint64)]),
    "sf_tensor_offset": (_st, [_vp, C.c_uint32, C.c_uint32, _P(C.c_uint64)]),
    "sf_staging_layout": (_st, [_vp, C.c_uint32, C.c_int32, _P(C.c_uint64), _P(C.c_uint64),
                                C.c_uint32]),
    "sf_bind": (_st, [_vp, C.c_uint32, C.c_int32, _vp, _vp, _vp]),
    "sf_start_training": (_st, [_vp, C.c_uint32, C.c_int32, C.c_int64, C.c_int32,
                                _P(sf_cut_request), C.c_int32, _P(C.c_uint32)]),
    "sf_preempt": (_st, [_vp, C.c_uint32, C.c_int32, _P(sf_cut_info)]),
    "sf_export_arena": (_st, [_vp, C.c_uint32, C.c_int32, _P(sf_ipc_arena)]),
    "sf_import_arena": (_st, [_vp, C.c_uint32, C.c_int32, _P(sf_ipc_arena)]),
    "sf_adopt_job": (_st, [_vp, C.c_uint32, C.c_int32, C.c_int64, C.c_int64, C.c_int32, C.c_int32,
                           _P(C.c_uint32)]),
    "sf_resume": (_st, [_vp, C.c_uint32, C.c_int32]),
    "sf_create_feed": (_st, [_vp, _P(sf_feed_desc), _P(C.c_uint32)]),
    "sf_attach_feed": (_st, [_vp, C.c_uint32, C.c_uint32, _P(C.c_uint32)]),
    "sf_stage_u8_normalize": (C.c_int32, [_vp, C.c_int64, _P(_vp), _P(C.c_uint64), C.c_int32]),
    "sf_job_query": (_st, [_vp, C.c_uint32, _P(sf_job_info)]),
    "sf_wait_job": (_st, [_vp, C.c_uint32, C.c_int64]),
    "sf_read_tensor": (_st, [_vp, C.c_uint32, C.c_uint32, _vp, C.c_size_t]),
    "sf_stop_job": (_st, [_vp, C.c_uint32]),
    "sf_submit_inference": (_st, [_vp, C.c_uint32, C.c_int32, _vp, _vp, C.c_uint64,
                                  _P(C.c_uint64)]),
    "sf_wait": (_st, [_vp, C.c_uint64, C.c_int64, _P(sf_timing)]),
    "sf_get_trace": (_st, [_vp, _P(sf_trace_event), C.c_size_t, _P(C.c_size_t)]),
    "sf_now_ns": (C.c_uint64, []),
    "sf_op_mtcopy": (_st, [_P(sf_copy_desc), C.c_int32, C.c_int64, _vp]),
    "sf_op_gemm": (_st, [_vp, _vp, _vp, C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.c_int32,
                         C.c_int32, C.c_int32, _vp]),
    "sf_op_gemm_bias_act": (_st, [_vp, _vp, _vp, C.c_int32, C.c_int32, C.c_int32, C.c_int32,
                                  C.c_int32, C.c_int32, C.c_int32, _vp, _vp, _vp, C.c_int32, _vp]),
    "sf_debug_chain_trace": (_st, [_vp]),
    "sf_op_mlp_chain": (_st, [_vp, C.c_int32, C.c_int32, _P(C.c_int32), _P(_vp), _P(_vp),
                              _P(C.c_int32), _P(_vp), _vp, _vp]),
    "sf_op_bias_act": (_st, [_vp, _vp, _vp, _vp, _vp, C.c_int32, C.c_int32, C.c_int32, _vp]),
    "sf_op_bias_act_bwd": (_st, [_vp, _vp, _vp, _vp, C.c_int32, C.c_int32, _vp]),
    "sf_op_gelu_bwd": (_st, [_vp, _vp, _vp, _vp, C.c_int32, C.c_int32, _vp]),
    "sf_op_colsum": (_st, [_vp, _vp, C.c_int32, C.c_int32, _vp]),
    "sf_op_softmax_ce": (_st, [_vp, _vp, _vp, _vp, C.c_int32, C.c_int32, _vp]),
    "sf_op_softmax": (_st, [_vp, _vp, C.c_int32, C.c_int32, _vp]),
    "sf_op_sgd_mom": (_st, [_vp, _vp, _vp, C.c_int64, C.c_float, C.c_float, _vp]),
    "sf_op_adam": (_st, [_vp, _vp, _vp, _vp, _vp, C.c_int64, C.c_float, C.c_float, C.c_float,
                         C.c_float, _vp]),
    "sf_op_fill": (_st, [_vp, C.c_uint64, C.c_int32, _vp]),
    "sf_last_gemm_path": (_st, [_P(sf_gemm_path)]),
    "sf_slot_query": (_st, [_vp, C.c_int32, _P(sf_slot_info)]),
    "sf_refresh_constants": (_st, [_vp, C.c_uint32, C.c_int32]),
    "sf_probe_peer": (_st, [_vp, C.c_uint32, C.c_int32, C.c_int32, C.c_int32, C.c_int32,
                            _P(C.c_double), _P(C.c_uint64)]),
    "sf_probe_migration": (_st, [_vp, C.c_uint32, C.c_int32, C.c_int32, C.c_int32,
                                 _P(sf_migration_probe)]),
    "sf_kernel_launches": (C.c_uint64, []),
}

_lib = None


def lib() -> C.CDLL:
    """Load libswitchflow_b200.so (built by build.py / __graft_entry__.build()).

    Raises if it is missing: the CUDA path has no fallback.
    """
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} not built: run `python -c 'import __graft_entry__ as g; "
                               "g.build()'` (the CUDA extension is required; no CPU fallback)")
        L = C.CDLL(LIB_PATH)
        for name, (res, args) in PROTOTYPES.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


class SFError(RuntimeError):
    def __init__(self, status: int, what: str):
        msg = lib().sf_last_error()
        super().__init__(f"{what} failed with status {status}: {msg.decode() if msg else ''}")
        self.status = status


def check(status: int, what: str) -> None:
    if status != SF_OK:
        raise SFError(status, what)
