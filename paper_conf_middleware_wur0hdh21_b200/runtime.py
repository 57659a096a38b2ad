"""Thin Python binding over the C ABI (include/sf.h): marshalling + torch plumbing only.

Every computation of the hot path (subgraph ops, pack / unpack / peer store, the
scheduler) runs inside libswitchflow_b200.so; PyTorch only allocates device memory
(arenas, staging), pinned host memory and reads results back for the caller.
"""
from __future__ import annotations

import ctypes as C
from typing import Dict, List, Optional, Sequence

import numpy as np
import torch

from . import _abi as A
from ._abi import check, lib

F32, I32 = 0, 1
_TORCH_DTYPE = {F32: torch.float32, I32: torch.int32}
_NP_DTYPE = {F32: np.float32, I32: np.int32}


def graph_desc(g):
    """Marshal an sf_inputs.ir.Graph into ctypes arrays (kept alive by the caller)."""
    T = (A.sf_tensor_desc * len(g.tensors))()
    for i, t in enumerate(g.tensors):
        T[i].rows, T[i].cols, T[i].dtype, T[i].kind = t.rows, t.cols, t.dtype, t.kind
    O = (A.sf_op_desc * len(g.ops))()
    for j, o in enumerate(g.ops):
        d = O[j]
        d.type = o.type
        d.n_in = len(o.ins)
        for i, x in enumerate(o.ins):
            d.in_[i] = x
        d.n_out = len(o.outs)
        for i, x in enumerate(o.outs):
            d.out[i] = x
        d.flags = o.flags
        d.phase = o.phase
        for i, x in enumerate(o.f[:4]):
            d.f[i] = x
    name = g.name.encode()
    desc = A.sf_graph_desc(name, len(g.tensors), T, len(g.ops), O)
    return desc, (T, O, name)


class GraphHandle:
    def __init__(self, rt: "Runtime", gid: int, graph, priority: int):
        self.rt, self.gid, self.graph, self.priority = rt, gid, graph, priority
        self.info: Optional[A.sf_partition_info] = None
        self.mem: Dict[int, dict] = {}

    # ---- partition / analysis ---------------------------------------------------------
    def partition(self, policy: str = "phase", max_ops: int = 0,
                  update_chunks: int = 1) -> A.sf_partition_info:
        o = A.sf_partition_opts(A.SF_PART_PER_LAYER_PHASE if policy == "phase" else A.SF_PART_MAX_OPS,
                                max_ops, update_chunks)
        info = A.sf_partition_info()
        check(lib().sf_partition(self.rt.h, self.gid, C.byref(o), C.byref(info)), "sf_partition")
        self.info = info
        return info

    @property
    def n_subgraphs(self) -> int:
        return self.info.n_subgraphs

    def subgraph_range(self, k: int):
        b, e = C.c_int32(), C.c_int32()
        check(lib().sf_subgraph_range(self.rt.h, self.gid, k, C.byref(b), C.byref(e)), "sf_subgraph_range")
        return b.value, e.value

    def live_set(self, k: int):
        n, nb = C.c_uint32(), C.c_uint64()
        check(lib().sf_live_set(self.rt.h, self.gid, k, None, 0, C.byref(n), C.byref(nb)), "sf_live_set")
        ids = (C.c_uint32 * max(1, n.value))()
        check(lib().sf_live_set(self.rt.h, self.gid, k, ids, n.value, C.byref(n), C.byref(nb)),
              "sf_live_set")
        return [ids[i] for i in range(n.value)], nb.value

    def offset(self, tid: int) -> int:
        o = C.c_uint64()
        check(lib().sf_tensor_offset(self.rt.h, self.gid, tid, C.byref(o)), "sf_tensor_offset")
        return o.value

    def staging_layout(self, k: int):
        ids, _ = self.live_set(k)
        offs = (C.c_uint64 * max(1, len(ids)))()
        tot = C.c_uint64()
        check(lib().sf_staging_layout(self.rt.h, self.gid, k, C.byref(tot), offs, len(ids)),
              "sf_staging_layout")
        return tot.value, [offs[i] for i in range(len(ids))]

    # ---- memory -------------------------------------------------------------------------
    def bind(self, slot: int, staging: bool = True, host_staging: bool = False) -> None:
        """Allocate this slot's arena (+ device / pinned host staging) with torch and bind."""
        if self.rt.ordinals[slot] < 0:  # REMOTE slot: the C call reports the error
            check(lib().sf_bind(self.rt.h, self.gid, slot, None, None, None), "sf_bind")
        dev = torch.device("cuda", self.rt.ordinals[slot])
        arena = torch.empty(self.info.arena_bytes, dtype=torch.uint8, device=dev)
        stg = torch.empty(self.info.staging_bytes, dtype=torch.uint8, device=dev) if staging else None
        hst = (torch.empty(self.info.staging_bytes, dtype=torch.uint8, pin_memory=True)
               if host_staging else None)
        check(lib().sf_bind(self.rt.h, self.gid, slot, C.c_void_p(arena.data_ptr()),
                            C.c_void_p(stg.data_ptr()) if stg is not None else None,
                            C.c_void_p(hst.data_ptr()) if hst is not None else None), "sf_bind")
        self.mem[slot] = {"arena": arena, "staging": stg, "host_staging": hst}

    def view(self, slot: int, tid: int) -> torch.Tensor:
        """torch view of tensor ``tid`` inside the slot's arena."""
        t = self.graph.tensors[tid]
        off = self.offset(tid)
        raw = self.mem[slot]["arena"][off:off + t.nbytes]
        return raw.view(_TORCH_DTYPE[t.dtype]).view(t.rows, t.cols)

    def load(self, slot: int, arrays: Dict[int, np.ndarray]) -> None:
        for tid, a in arrays.items():
            self.view(slot, tid).copy_(torch.from_numpy(np.ascontiguousarray(a)))
        torch.cuda.synchronize(self.rt.ordinals[slot])
        if self.priority > 0:  # inference weights: rebuild their blocked copies now
            self.refresh_constants(slot)

    def read(self, slot: int, tid: int) -> np.ndarray:
        torch.cuda.synchronize(self.rt.ordinals[slot])
        return self.view(slot, tid).cpu().numpy()

    def arena_bytes(self, slot: int) -> torch.Tensor:
        return self.mem[slot]["arena"]

    def refresh_constants(self, slot: int) -> None:
        """Rebuild the blocked inference-weight copies at the next request (sf_refresh_constants)."""
        check(lib().sf_refresh_constants(self.rt.h, self.gid, slot), "sf_refresh_constants")

    def attach_feed(self, feed: int, tensor_ids: Sequence[int]) -> None:
        """Feed these INPUT / LABEL tensors from host feed ``feed`` (sf_attach_feed)."""
        arr = (C.c_uint32 * len(tensor_ids))(*tensor_ids)
        check(lib().sf_attach_feed(self.rt.h, self.gid, feed, arr), "sf_attach_feed")


class Runtime:
    """One sf_runtime: logical device slots mapped onto CUDA devices."""

    def __init__(self, ordinals: Sequence[int] = (0,), exclusive: bool = True,
                 auto_preempt: bool = True, iteration_granularity: bool = False,
                 host_mode: int = A.SF_HOST_CE, poison: bool = False, budget_bytes: int = 0,
                 trace_capacity: int = 0, defer_migration: bool = False, max_inflight: int = 1,
                 dispatch_spin_us: int = 0, inflight_budget_us: int = 0,
                 migrate_home: bool = False, migration_engine: int = 0,
                 host_stage_inline: bool = False, infer_l2_persist_bytes: int = 0,
                 host_duplex: bool = False, early_launch: bool = False, drain_gate: bool = False):
        self.ordinals = list(ordinals)
        arr = (C.c_int32 * len(self.ordinals))(*self.ordinals)
        cfg = A.sf_config(len(self.ordinals), arr, int(exclusive), int(auto_preempt),
                          int(iteration_granularity), host_mode, int(poison), trace_capacity,
                          max_inflight, int(defer_migration), budget_bytes, dispatch_spin_us,
                          inflight_budget_us, int(migrate_home), migration_engine,
                          int(host_stage_inline), int(host_duplex), infer_l2_persist_bytes,
                          int(early_launch), int(drain_gate))
        h = C.c_void_p()
        check(lib().sf_create(C.byref(cfg), C.byref(h)), "sf_create")
        self.h = h
        self.graphs: List[GraphHandle] = []
        self._keep: list = []  # host-stage user data referenced by the library

    def close(self) -> None:
        if self.h:
            lib().sf_destroy(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def register(self, g, priority: int = 0) -> GraphHandle:
        desc, keep = graph_desc(g)
        gid = C.c_uint32()
        check(lib().sf_register_graph(self.h, C.byref(desc), priority, C.byref(gid)),
              "sf_register_graph")
        gh = GraphHandle(self, gid.value, g, priority)
        self.graphs.append(gh)
        return gh

    # ---- host input stages (sf_create_feed) ---------------------------------------------------
    def create_feed(self, fn_ptr: int, user_ptr: int, nbytes: Sequence[int], depth: int = 2,
                    shared: bool = False, dev: int = 0) -> int:
        b = (C.c_uint64 * len(nbytes))(*nbytes)
        d = A.sf_feed_desc(fn_ptr, user_ptr, len(nbytes), b, depth, int(shared), dev, 0)
        f = C.c_uint32()
        check(lib().sf_create_feed(self.h, C.byref(d), C.byref(f)), "sf_create_feed")
        return f.value

    def u8_feed(self, images: np.ndarray, labels: np.ndarray, batch: int, img_w: int, seed: int,
                depth: int = 2, shared: bool = False, dev: int = 0) -> int:
        """Feed driven by the built-in host stage sf_stage_u8_normalize (x f32, y i32)."""
        images = np.ascontiguousarray(images, dtype=np.uint8)
        labels = np.ascontiguousarray(labels, dtype=np.int32).reshape(-1)
        st = A.sf_u8_stage(images.ctypes.data, labels.ctypes.data, images.shape[0], batch,
                           images.shape[1], img_w, seed)
        self._keep += [images, labels, st]
        fn = C.cast(lib().sf_stage_u8_normalize, C.c_void_p).value
        return self.create_feed(fn, C.addressof(st), [batch * images.shape[1] * 4, batch * 4],
                                depth, shared, dev)

    # ---- jobs -----------------------------------------------------------------------------
    def start_training(self, gh: GraphHandle, slot: int, iters: int, auto_target: int,
                       schedule: Sequence = ()) -> int:
        """schedule: [(iter, k, target)] deterministic preemptions (ascending)."""
        arr = (A.sf_cut_request * max(1, len(schedule)))()
        for i, (it, k, tgt) in enumerate(schedule):
            arr[i].iter, arr[i].k, arr[i].target = it, k, tgt
        j = C.c_uint32()
        check(lib().sf_start_training(self.h, gh.gid, slot, iters, auto_target, arr, len(schedule),
                                      C.byref(j)), "sf_start_training")
        return j.value

    def adopt_job(self, gh: GraphHandle, slot: int, iters: int, it: int, k: int,
                  auto_target: int) -> int:
        """Continue a job whose cut-(it, k) state a partner peer-stored into this slot."""
        j = C.c_uint32()
        check(lib().sf_adopt_job(self.h, gh.gid, slot, iters, it, k, auto_target, C.byref(j)),
              "sf_adopt_job")
        return j.value

    def export_arena(self, gh: GraphHandle, slot: int) -> bytes:
        a = A.sf_ipc_arena()
        check(lib().sf_export_arena(self.h, gh.gid, slot, C.byref(a)), "sf_export_arena")
        return bytes(C.string_at(C.addressof(a), C.sizeof(a)))

    def import_arena(self, gh: GraphHandle, slot: int, blob: bytes) -> None:
        a = A.sf_ipc_arena.from_buffer_copy(blob)
        check(lib().sf_import_arena(self.h, gh.gid, slot, C.byref(a)), "sf_import_arena")

    def preempt(self, job: int, target: int) -> dict:
        c = A.sf_cut_info()
        check(lib().sf_preempt(self.h, job, target, C.byref(c)), "sf_preempt")
        return {f: getattr(c, f) for f, _ in A.sf_cut_info._fields_}

    def resume(self, job: int, slot: int) -> None:
        check(lib().sf_resume(self.h, job, slot), "sf_resume")

    def job_info(self, job: int) -> dict:
        i = A.sf_job_info()
        check(lib().sf_job_query(self.h, job, C.byref(i)), "sf_job_query")
        d = {f: getattr(i, f) for f, _ in A.sf_job_info._fields_}
        d["state_name"] = A.JOB_STATES.get(d["state"], "?")
        return d

    def read_tensor(self, job: int, gh: GraphHandle, tid: int) -> np.ndarray:
        """A job's tensor from the arena of the slot it occupies (sf_read_tensor, blocking)."""
        t = gh.graph.tensors[tid]
        out = np.empty((t.rows, t.cols), dtype=_NP_DTYPE[t.dtype])
        check(lib().sf_read_tensor(self.h, job, tid, C.c_void_p(out.ctypes.data), out.nbytes),
              "sf_read_tensor")
        return out

    def wait_job(self, job: int, timeout_s: float = -1) -> None:
        check(lib().sf_wait_job(self.h, job, int(timeout_s * 1e9) if timeout_s >= 0 else -1),
              "sf_wait_job")

    def stop_job(self, job: int) -> None:
        check(lib().sf_stop_job(self.h, job), "sf_stop_job")

    # ---- inference ------------------------------------------------------------------------
    def submit(self, gh: GraphHandle, slot: int, in_ptr: int, out_ptr: int,
               arrival_ns: int = 0) -> int:
        r = C.c_uint64()
        check(lib().sf_submit_inference(self.h, gh.gid, slot, C.c_void_p(in_ptr), C.c_void_p(out_ptr),
                                        arrival_ns, C.byref(r)), "sf_submit_inference")
        return r.value

    def wait(self, req: int, timeout_s: float = -1) -> dict:
        t = A.sf_timing()
        check(lib().sf_wait(self.h, req, int(timeout_s * 1e9) if timeout_s >= 0 else -1, C.byref(t)),
              "sf_wait")
        return {f: getattr(t, f) for f, _ in A.sf_timing._fields_}

    def probe_migration(self, gh: GraphHandle, slot: int, k: int, l2: int = 0) -> dict:
        """Kernel-only pack / unpack durations of cut k (sf_probe_migration; l2: 0 warm,
        1 cold clean, 2 cold dirty)."""
        o = A.sf_migration_probe()
        check(lib().sf_probe_migration(self.h, gh.gid, slot, k, l2, C.byref(o)), "sf_probe_migration")
        return {f: getattr(o, f) for f, _ in A.sf_migration_probe._fields_}

    def probe_peer(self, gh: GraphHandle, src: int, dst: int, k: int = 0, engine: int = 0):
        """Move cut k's live set src -> dst once (sf_probe_peer); returns (us, bytes)."""
        us, nb = C.c_double(), C.c_uint64()
        check(lib().sf_probe_peer(self.h, gh.gid, src, dst, k, engine, C.byref(us), C.byref(nb)),
              "sf_probe_peer")
        return us.value, nb.value

    def slot_info(self, slot: int) -> dict:
        """Scheduler state of a slot (sf_slot_query; diagnostics)."""
        o = A.sf_slot_info()
        check(lib().sf_slot_query(self.h, slot, C.byref(o)), "sf_slot_query")
        return {f: getattr(o, f) for f, _ in A.sf_slot_info._fields_ if not f.startswith("pad")}

    def poll(self, req: int) -> Optional[dict]:
        """Non-blocking sf_wait: the request's timing once done, else None."""
        t = A.sf_timing()
        st = lib().sf_wait(self.h, req, 0, C.byref(t))
        if st == A.SF_ETIMEOUT:
            return None
        check(st, "sf_wait")
        return {f: getattr(t, f) for f, _ in A.sf_timing._fields_}

    def trace(self) -> List[dict]:
        n = C.c_size_t()
        check(lib().sf_get_trace(self.h, None, 0, C.byref(n)), "sf_get_trace")
        buf = (A.sf_trace_event * max(1, n.value))()
        check(lib().sf_get_trace(self.h, buf, n.value, C.byref(n)), "sf_get_trace")
        out = []
        for i in range(n.value):
            e = buf[i]
            kind = {A.EV_TRAIN: "train", A.EV_INFER: "infer", A.EV_HOST: "host"}.get(e.kind, "migrate")
            d = {"dev": e.dev, "job": e.job, "kind": kind, "iter": e.iter, "k": e.k,
                 "t0": e.t0_ns, "t1": e.t1_ns, "d0": e.d0_ns, "d1": e.d1_ns}
            if kind == "infer":
                d["arrival"] = e.arrival_ns
                if e.iter >= 0:
                    d["after"] = e.iter  # device-ordered after that job's dispatched subgraphs
            elif kind == "train":
                d["launch"] = e.arrival_ns
            out.append(d)
        return out


def now_ns() -> int:
    return lib().sf_now_ns()


def kernel_launches() -> int:
    return lib().sf_kernel_launches()
