"""Python binding of libstg — the B200 (sm_100a) hot path of STGraph.

Argument marshalling only: every step of the path runs in libstg's CUDA
kernels (csrc/).  Functions keep the C-ABI names of include/stg.h.  PyTorch is
used for device memory and streams; there is NO CPU fallback — importing this
package fails loudly when libstg.so is missing, and every call raises StgError
on a non-OK status.
"""
from __future__ import annotations

import atexit
import ctypes
import os
import sys

import numpy as np
import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libstg.so")

STG_SELF_LOOPS = 1 << 0
STG_EDGE_IDS = 1 << 1
STG_VALIDATE = 1 << 2
STG_NORM_DGL_BOTH = 1 << 3
STG_NAIVE = 1 << 4
STG_PART_IN, STG_PART_OUT, STG_PART_EID = 1 << 0, 1 << 1, 1 << 2

STATUS = {0: "STG_OK", 1: "STG_ERR_INVALID_ARG", 2: "STG_ERR_OUT_OF_RANGE", 3: "STG_ERR_NO_MEMORY",
          4: "STG_ERR_CUDA", 5: "STG_ERR_NCCL", 6: "STG_ERR_STATE"}


class StgError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__("%s: %s" % (STATUS.get(status, status), msg))
        self.status = status


if not os.path.exists(LIB_PATH):
    raise ImportError("libstg.so not built (%s); run __graft_entry__.build()" % LIB_PATH)

_P = ctypes.c_void_p
_i32, _i64, _u32, _f32 = ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32, ctypes.c_float


class stg_dist(ctypes.Structure):
    _fields_ = [("rank", _i32), ("world", _i32), ("row_begin", _i32), ("row_end", _i32)]


class stg_csr_view(ctypes.Structure):
    _fields_ = [("num_nodes", _i32), ("row_begin", _i32), ("row_end", _i32), ("timestamp", _i32),
                ("num_edges", _i64),
                ("in_rowptr", _P), ("in_col", _P),
                ("out_rowptr", _P), ("out_col", _P),
                ("out_eid", _P),
                ("in_deg", _P), ("out_deg", _P), ("in_ids", _P), ("out_ids", _P),
                ("norm_src", _P), ("norm_dst", _P),
                ("in_sched", _P), ("out_sched", _P),
                ("workspace", _P)]


STG_MAX_PEERS = 8


class stg_peer_rows(ctypes.Structure):
    _fields_ = [("world", _i32), ("bounds", ctypes.POINTER(_i32)), ("blocks", ctypes.POINTER(_P)), ("ld", _i64)]


class stg_ipc_handle(ctypes.Structure):
    _fields_ = [("reserved", ctypes.c_ubyte * 64)]


class stg_tgcn_params(ctypes.Structure):
    _fields_ = [("F", _i32), ("H", _i32), ("W", _P), ("b", _P), ("L", _P), ("l", _P)]


class stg_tgcn_grads(ctypes.Structure):
    _fields_ = [("W", _P), ("b", _P), ("L", _P), ("l", _P)]


class stg_tgcn2_params(ctypes.Structure):
    _fields_ = [("F", _i32), ("H", _i32), ("Wg", _P), ("bg", _P), ("Wc", _P), ("bc", _P)]


class stg_tgcn2_grads(ctypes.Structure):
    _fields_ = [("Wg", _P), ("bg", _P), ("Wc", _P), ("bc", _P)]


_lib = ctypes.CDLL(LIB_PATH)


def _decl(name, argtypes, restype=_i32):
    f = getattr(_lib, name)
    f.argtypes = argtypes
    f.restype = restype
    return f


_decl("stg_last_error", [], ctypes.c_char_p)
_decl("stg_version", [], _i32)
_decl("stg_kernel_launch_count", [], _i64)
_decl("stg_memcpy", [_P, _P, ctypes.c_size_t, _i32, _P])
_decl("stg_static_graph_create", [_i32, _i64, _P, _P, _u32, _P, _P, ctypes.POINTER(_P)])
_decl("stg_graph_view", [_P, ctypes.POINTER(stg_csr_view)])
_decl("stg_graph_destroy", [_P], None)
_decl("stg_dtdg_create", [_i32, _i32, _i64, _P, _P, _P, _P, _P, _P, _P, _P, _u32, _P, _P, ctypes.POINTER(_P)])
_decl("stg_dtdg_get_snapshot", [_P, _i32, _P, ctypes.POINTER(stg_csr_view)])
_decl("stg_dtdg_get_backward_snapshot", [_P, _i32, _P, ctypes.POINTER(stg_csr_view)])
_decl("stg_dtdg_get_snapshot_parts", [_P, _i32, _i32, _u32, _P, ctypes.POINTER(stg_csr_view)])
_decl("stg_dtdg_num_edges", [_P, _i32], _i64)
_decl("stg_dtdg_num_timestamps", [_P], _i32)
_decl("stg_dtdg_num_deltas", [_P, _i32, _i32], _i64)
_decl("stg_dtdg_destroy", [_P], None)
_decl("stg_dtdg_memory", [_P, ctypes.POINTER(_i64), ctypes.POINTER(_i64), ctypes.POINTER(_i64)])
_decl("stg_gcn_aggregate_fwd", [ctypes.POINTER(stg_csr_view), _i32, _P, _i64, _P, _i64, _P])
_decl("stg_gcn_aggregate_bwd", [ctypes.POINTER(stg_csr_view), _i32, _P, _i64, _P, _i64, _P])
_decl("stg_gcn_aggregate_ex", [ctypes.POINTER(stg_csr_view), _i32, _i32, _P, _i64, _P, _i64, _P, _P, _P, _P])
_decl("stg_state_stack_create", [_i64, ctypes.POINTER(_P)])
_decl("stg_state_stack_depth", [_P], _i32)
_decl("stg_state_stack_destroy", [_P], None)
_decl("stg_tgcn_step", [ctypes.POINTER(stg_csr_view), ctypes.POINTER(stg_tgcn_params), _P, _P, _P, _P, _P])
_decl("stg_tgcn_step_backward", [ctypes.POINTER(stg_csr_view), ctypes.POINTER(stg_tgcn_params), _P, _P, _P,
                                 ctypes.POINTER(stg_tgcn_grads), _P, _P])
_decl("stg_mse_head", [_i32, _i32, _P, _P, _P, _P, _P, _P, _i32, _P, _P, _P])
_decl("stg_mse_head_ex", [_i32, _i32, _i32, _P, _P, _P, _P, _P, _P, _i32, _P, _P, _P])
_decl("stg_sgd_update", [_P, _P, _i64, _f32, _P])
_decl("stg_tgcn_train_sequence", [_P, _P, _i32, _i32, ctypes.POINTER(stg_tgcn_params), _P, _P,
                                  ctypes.POINTER(_P), ctypes.POINTER(_P), _P, _P, _P,
                                  ctypes.POINTER(stg_tgcn_grads), _P, _P, _P, _P, _P])
_decl("stg_tgcn_train_sequence_ev", [_P, _P, _i32, _i32, ctypes.POINTER(stg_tgcn_params), _P, _P,
                                     ctypes.POINTER(_P), ctypes.POINTER(_P), _P, _P, _P,
                                     ctypes.POINTER(stg_tgcn_grads), _P, _P, _P, _P, ctypes.POINTER(_P), _P])
_decl("stg_tgcn_train_sequence_batched", [_P, _i32, ctypes.POINTER(stg_tgcn_params), _P, _P, ctypes.POINTER(_P),
                                          ctypes.POINTER(_P), _P, _P, ctypes.POINTER(stg_tgcn_grads), _P, _P, _P, _P,
                                          _P])
_decl("stg_partition_rows", [_i32, _P, _i32, ctypes.POINTER(_i32), _P])
_decl("stg_profile_enable", [_i32])
_decl("stg_set_pipeline", [_i32])
_decl("stg_set_conv_order", [_i32])
_decl("stg_debug_tc_gemm", [_i32, _i32, _i32, _i32, _i32, _P, _P, _P, _P])
_decl("stg_debug_sum_parts", [_P, _i32, _i32, _P, _i32, _P])
_decl("stg_aggregate_set_strategy", [_i32])
_decl("stg_aggregate_set_param", [_i32, _i64])
_decl("stg_profile_read", [_i32, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(_i64), _i32])
_decl("stg_gcn_aggregate_weighted", [ctypes.POINTER(stg_csr_view), _i32, _i32, _P, _P, _i64, _P, _i64, _P, _P, _P,
                                     _P])
_decl("stg_gcn_weighted_norm", [ctypes.POINTER(stg_csr_view), _P, _P, _P])
_decl("stg_tgcn2_step", [ctypes.POINTER(stg_csr_view), ctypes.POINTER(stg_tgcn2_params), _P, _P, _P, _P, _P])
_decl("stg_tgcn2_step_backward", [ctypes.POINTER(stg_csr_view), ctypes.POINTER(stg_tgcn2_params), _P, _P, _P,
                                  ctypes.POINTER(stg_tgcn2_grads), _P, _P])
_decl("stg_tgcn2_peer_fwd", [_i32, ctypes.POINTER(stg_csr_view), ctypes.POINTER(stg_tgcn2_params), _P, _P,
                             ctypes.POINTER(stg_peer_rows), _P, _P, _P, _P])
_decl("stg_tgcn2_peer_bwd", [_i32, ctypes.POINTER(stg_csr_view), ctypes.POINTER(stg_tgcn2_params), _P, _P, _P,
                             ctypes.POINTER(stg_tgcn2_grads), _i32, _i32, ctypes.POINTER(_i32), ctypes.POINTER(_P), _P,
                             _P, _P])
_decl("stg_peer_alloc", [_i64, ctypes.POINTER(_P), ctypes.POINTER(stg_ipc_handle)])
_decl("stg_peer_free", [_P])
_decl("stg_peer_open", [ctypes.POINTER(stg_ipc_handle), ctypes.POINTER(_P)])
_decl("stg_peer_close", [_P])
_decl("stg_allgather_rows", [ctypes.POINTER(stg_peer_rows), _i32, _P, _i64, _P])
_decl("stg_gcn_aggregate_peer", [ctypes.POINTER(stg_csr_view), _i32, ctypes.POINTER(stg_peer_rows), _P, _i64, _P, _P,
                                 _P, _P])
_decl("stg_reduce_scatter_rows", [_i32, ctypes.POINTER(_i32), ctypes.POINTER(_P), _i64, _i32, _i32, _P, _i64, _P])
_decl("stg_tgcn_project", [ctypes.POINTER(stg_csr_view), ctypes.POINTER(stg_tgcn_params), _P, _P, _P])
_decl("stg_tgcn_step_peer", [ctypes.POINTER(stg_csr_view), ctypes.POINTER(stg_tgcn_params),
                             ctypes.POINTER(stg_peer_rows), _P, _P, _P, _P])
_decl("stg_tgcn_step_backward_peer", [ctypes.POINTER(stg_csr_view), ctypes.POINTER(stg_tgcn_params), _P, _P,
                                      ctypes.POINTER(stg_tgcn_grads), _P, _P, _P])
_decl("stg_tgcn_dw", [ctypes.POINTER(stg_tgcn_params), _i32, _P, _P, ctypes.POINTER(stg_tgcn_grads), _P, _P])


class stg_peer_exchange(ctypes.Structure):
    _fields_ = [("world", _i32), ("rank", _i32), ("bounds", ctypes.POINTER(_i32)),
                ("P", (_P * 8) * 2), ("dP", (_P * 8) * 2), ("flags", _P * 8),
                ("fwd_count", ctypes.c_uint32), ("bwd_count", ctypes.c_uint32)]


_decl("stg_tgcn_train_sequence_peer", [_P, _i32, _i32, ctypes.POINTER(stg_tgcn_params), _P, _P, _P, _P, _P, _P, _P,
                                       _P, ctypes.POINTER(stg_tgcn_grads), _P, _P, _P, _P,
                                       ctypes.POINTER(stg_peer_exchange), _P])

ABI_SYMBOLS = [
    "stg_last_error", "stg_version", "stg_kernel_launch_count", "stg_set_allocator", "stg_allocator_detach",
    "stg_memcpy",
    "stg_static_graph_create", "stg_graph_view", "stg_graph_destroy",
    "stg_dtdg_create", "stg_dtdg_get_snapshot", "stg_dtdg_get_backward_snapshot", "stg_dtdg_get_snapshot_parts",
    "stg_dtdg_num_edges",
    "stg_dtdg_num_timestamps", "stg_dtdg_num_deltas", "stg_dtdg_destroy", "stg_dtdg_memory",
    "stg_gcn_aggregate_fwd", "stg_gcn_aggregate_bwd", "stg_gcn_aggregate_ex",
    "stg_state_stack_create", "stg_state_stack_depth", "stg_state_stack_destroy",
    "stg_tgcn_step", "stg_tgcn_step_backward", "stg_mse_head", "stg_mse_head_ex", "stg_sgd_update", "stg_tgcn_train_sequence",
    "stg_tgcn_train_sequence_batched", "stg_tgcn_train_sequence_ev",
    "stg_partition_rows", "stg_profile_enable", "stg_profile_read", "stg_debug_tc_gemm", "stg_debug_sum_parts", "stg_set_pipeline", "stg_set_conv_order", "stg_aggregate_set_strategy",
    "stg_aggregate_set_param",
    "stg_gcn_aggregate_weighted", "stg_gcn_weighted_norm", "stg_tgcn2_step", "stg_tgcn2_step_backward",
    "stg_peer_alloc", "stg_peer_free", "stg_peer_open", "stg_peer_close", "stg_allgather_rows",
    "stg_gcn_aggregate_peer", "stg_reduce_scatter_rows", "stg_tgcn_project", "stg_tgcn_step_peer",
    "stg_tgcn_step_backward_peer", "stg_tgcn_dw", "stg_tgcn_train_sequence_peer", "stg_tgcn2_peer_fwd", "stg_tgcn2_peer_bwd",
]

# ---------------------------------------------------------------- allocator hook
# Library-owned device memory (snapshot slots, deltas, state stack, scratch) from
# PyTorch's caching allocator (include/stg.h stg_set_allocator), so torch's memory
# statistics cover it and freed blocks return to torch's pool.
_ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
_FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p)
_lib.stg_set_allocator.argtypes = [_ALLOC_FN, _FREE_FN, ctypes.c_void_p]
_lib.stg_set_allocator.restype = _i32
_hook_stats = {"alloc": 0, "free": 0, "bytes": 0}
_exiting = [False]


def _at_exit():
    # objects still alive are left to the process teardown, and the library forgets
    # its torch blocks: torch's allocator must not be called back during finalisation
    # (static library state is destroyed after the interpreter)
    _exiting[0] = True
    _lib.stg_allocator_detach()


atexit.register(_at_exit)


def _torch_alloc(nbytes, stream, ctx):
    try:
        p = torch.cuda.caching_allocator_alloc(int(nbytes), device=torch.cuda.current_device(),
                                               stream=int(stream or 0))
    except Exception:                      # out of memory: the library reports STG_ERR_NO_MEMORY
        return None
    _hook_stats["alloc"] += 1
    _hook_stats["bytes"] += int(nbytes)
    return p


def _torch_free(ptr, stream, ctx):
    _hook_stats["free"] += 1
    torch.cuda.caching_allocator_delete(int(ptr))


_hooks = (_ALLOC_FN(_torch_alloc), _FREE_FN(_torch_free))


def use_torch_allocator(on: bool = True):
    """Route libstg's device allocations through torch's caching allocator (default at
    import unless STG_TORCH_ALLOCATOR=0), or back to cudaMalloc (on=False)."""
    if on:
        _check(_lib.stg_set_allocator(_hooks[0], _hooks[1], None))
    else:
        _check(_lib.stg_set_allocator(_ALLOC_FN(0), _FREE_FN(0), None))


def allocator_stats() -> dict:
    """Calls of the torch allocator hook so far (alloc / free counts, bytes requested)."""
    return dict(_hook_stats)


PHASES = ["agg_fwd", "agg_bwd", "snapshot", "xw", "gru_fwd", "gru_bwd", "dw", "head", "dl", "snap_step",
          "snap_transpose"]


def stg_set_pipeline(on: bool):
    """Training-sequence schedule: True = three-stream pipeline, False = one stream (exact phase split)."""
    _check(_lib.stg_set_pipeline(int(bool(on))))


def stg_set_conv_order(order: int):
    """0 = linear-first Â(XW) + b (default), 1 = aggregate-first (ÂX)W + b (NEXT-1)."""
    _check(_lib.stg_set_conv_order(int(order)))


def stg_profile_enable(on: bool = True):
    _check(_lib.stg_profile_enable(int(on)))


def stg_profile_read(reset: bool = True) -> dict:
    """{phase: (total_ms, count)} for every profiled phase (synchronises on the events)."""
    out = {}
    for i, name in enumerate(PHASES):
        ms = ctypes.c_double(0.0)
        n = _i64(0)
        _check(_lib.stg_profile_read(i, ctypes.byref(ms), ctypes.byref(n), int(reset)))
        out[name] = (ms.value, n.value)
    return out


def _check(status: int):
    if status != 0:
        raise StgError(status, _lib.stg_last_error().decode(errors="replace"))


def _stream(stream=None):
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def _ptr(t, dt=torch.float32):
    """Device pointer of a contiguous CUDA tensor of dtype `dt` (float32 features
    and parameters, int32 ids): anything else would reach the kernels as raw bytes."""
    if t is None:
        return None
    if not t.is_cuda:
        raise StgError(1, "expected a CUDA tensor")
    if not t.is_contiguous():
        raise StgError(1, "expected a contiguous tensor")
    if t.dtype != dt:
        raise StgError(1, "expected a %s tensor, got %s" % (dt, t.dtype))
    return ctypes.c_void_p(t.data_ptr())


def _ptrs(ts):
    """Host array of device pointers of float32 CUDA tensors (per-timestamp inputs)."""
    return (_P * len(ts))(*[_ptr(t).value for t in ts])


def _dev_i32(a):
    if isinstance(a, torch.Tensor):
        return a.to(device="cuda", dtype=torch.int32).contiguous()
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.int32)).cuda()


def kernel_launch_count() -> int:
    return int(_lib.stg_kernel_launch_count())


def version() -> int:
    return int(_lib.stg_version())


# ---------------------------------------------------------------- graphs
class Graph:
    """Owner of a stg_graph* (static graph)."""

    def __init__(self, handle, keep=()):
        self.handle = handle
        self._keep = keep

    def view(self) -> stg_csr_view:
        return stg_graph_view(self)

    def close(self):
        if self.handle:
            _lib.stg_graph_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            if _exiting[0] or sys.is_finalizing():   # (the allocator hook calls back into torch)
                return
            self.close()
        except Exception:
            pass


class Dtdg:
    """Owner of a stg_dtdg* (discrete-time dynamic graph)."""

    def __init__(self, handle):
        self.handle = handle

    @property
    def T(self) -> int:
        return int(_lib.stg_dtdg_num_timestamps(self.handle))

    def num_edges(self, t: int) -> int:
        return int(_lib.stg_dtdg_num_edges(self.handle, t))

    def num_deltas(self, t: int, deletes: bool) -> int:
        return int(_lib.stg_dtdg_num_deltas(self.handle, t, int(deletes)))

    def memory(self) -> dict:
        """Device bytes: normalised deltas, snapshot cache, materialised snapshots (STG_NAIVE)."""
        a, b, c = _i64(0), _i64(0), _i64(0)
        _check(_lib.stg_dtdg_memory(self.handle, ctypes.byref(a), ctypes.byref(b), ctypes.byref(c)))
        return {"deltas": a.value, "cache": b.value, "materialised": c.value}

    def close(self):
        if self.handle:
            _lib.stg_dtdg_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            if _exiting[0] or sys.is_finalizing():   # (the allocator hook calls back into torch)
                return
            self.close()
        except Exception:
            pass


def _dist(dist):
    """dist = None (whole graph) or (rank, world, row_begin, row_end) -> stg_dist* (SURVEY §8(e))."""
    if dist is None:
        return None
    r, w, b, e = (int(x) for x in dist)
    return ctypes.byref(stg_dist(r, w, b, e))


def _order_inputs(stream, *ts):
    """The id arrays were staged on the current stream: order the library's stream
    after those copies and keep the caching allocator from reusing them early."""
    if stream is None or stream == torch.cuda.current_stream():
        return
    stream.wait_stream(torch.cuda.current_stream())
    for t in ts:
        t.record_stream(stream)


def stg_static_graph_create(V: int, src, dst, flags: int = 0, stream=None, dist=None) -> Graph:
    s, d = _dev_i32(src), _dev_i32(dst)
    _order_inputs(stream, s, d)
    out = ctypes.c_void_p()
    _check(_lib.stg_static_graph_create(V, s.numel(), _ptr(s, torch.int32), _ptr(d, torch.int32), flags, _dist(dist), _stream(stream),
                                        ctypes.byref(out)))
    return Graph(out)


def stg_graph_view(g: Graph) -> stg_csr_view:
    v = stg_csr_view()
    _check(_lib.stg_graph_view(g.handle, ctypes.byref(v)))
    return v


def stg_dtdg_create(V: int, T: int, src0, dst0, add_off, add_src, add_dst, del_off, del_src, del_dst,
                    flags: int = 0, stream=None, dist=None) -> Dtdg:
    s0, d0 = _dev_i32(src0), _dev_i32(dst0)
    a_s, a_d = _dev_i32(add_src), _dev_i32(add_dst)
    r_s, r_d = _dev_i32(del_src), _dev_i32(del_dst)
    _order_inputs(stream, s0, d0, a_s, a_d, r_s, r_d)
    ao = np.ascontiguousarray(add_off, dtype=np.int64)
    do = np.ascontiguousarray(del_off, dtype=np.int64)
    if ao.size != T + 1 or do.size != T + 1:
        raise StgError(1, "offset arrays must have T+1 entries")
    out = ctypes.c_void_p()
    _check(_lib.stg_dtdg_create(V, T, s0.numel(), _ptr(s0, torch.int32), _ptr(d0, torch.int32),
                                ao.ctypes.data_as(_P), _ptr(a_s, torch.int32) if a_s.numel() else None,
                                _ptr(a_d, torch.int32) if a_d.numel() else None,
                                do.ctypes.data_as(_P), _ptr(r_s, torch.int32) if r_s.numel() else None,
                                _ptr(r_d, torch.int32) if r_d.numel() else None,
                                flags, _dist(dist), _stream(stream), ctypes.byref(out)))
    torch.cuda.current_stream().synchronize()
    return Dtdg(out)


def stg_dtdg_get_snapshot(d: Dtdg, t: int, stream=None) -> stg_csr_view:
    v = stg_csr_view()
    _check(_lib.stg_dtdg_get_snapshot(d.handle, t, _stream(stream), ctypes.byref(v)))
    return v


def stg_dtdg_get_snapshot_parts(d: Dtdg, t: int, parts: int, backward: bool = False, stream=None) -> stg_csr_view:
    """Get-Graph / Get-Backward-Graph of only the CSR parts in `parts` (STG_PART_*)."""
    v = stg_csr_view()
    _check(_lib.stg_dtdg_get_snapshot_parts(d.handle, t, int(backward), parts, _stream(stream), ctypes.byref(v)))
    return v


def stg_dtdg_get_backward_snapshot(d: Dtdg, t: int, stream=None) -> stg_csr_view:
    v = stg_csr_view()
    _check(_lib.stg_dtdg_get_backward_snapshot(d.handle, t, _stream(stream), ctypes.byref(v)))
    return v


def view_arrays(v: stg_csr_view, stream=None) -> dict:
    """Copies of the view's arrays as CUDA tensors (for tests / inspection)."""
    V, E = v.num_nodes, v.num_edges
    R = v.row_end - v.row_begin
    spec = {"in_rowptr": (R + 1, torch.int32), "in_col": (E, torch.int32),
            "out_rowptr": (V + 1, torch.int32), "out_col": (E, torch.int32),
            "out_eid": (E, torch.int32), "in_deg": (V, torch.int32), "out_deg": (V, torch.int32),
            "in_ids": (V, torch.int32), "out_ids": (V, torch.int32), "norm_src": (V, torch.float32),
            "norm_dst": (V, torch.float32)}
    out = {}
    for k, (n, dt) in spec.items():
        p = getattr(v, k)
        if not p:
            continue
        t = torch.empty(n, dtype=dt, device="cuda")
        if n:
            _check(_lib.stg_memcpy(ctypes.c_void_p(t.data_ptr()), ctypes.c_void_p(p), t.numel() * t.element_size(),
                                   0, _stream(stream)))
        out[k] = t
    for k in ("in_sched", "out_sched"):
        p = getattr(v, k)
        if p:
            hdr = torch.empty(2, dtype=torch.int32, device="cuda")
            _check(_lib.stg_memcpy(ctypes.c_void_p(hdr.data_ptr()), ctypes.c_void_p(p), 8, 0, _stream(stream)))
            out[k] = hdr
    # COO row ids implied by the row pointers (derived here; the library keeps none)
    for k, rp, base in (("in_row", "in_rowptr", v.row_begin), ("out_row", "out_rowptr", 0)):
        if rp in out:
            n = out[rp].numel() - 1
            out[k] = torch.repeat_interleave(torch.arange(base, base + n, device="cuda", dtype=torch.int32),
                                             torch.diff(out[rp]).long())
    return out


# ---------------------------------------------------------------- aggregation
def _out2d(x, rows, W, out):
    if out is None:
        out = torch.empty((rows, W), dtype=torch.float32, device=x.device)
    return out


def stg_gcn_aggregate_fwd(v: stg_csr_view, x: torch.Tensor, y: torch.Tensor = None, stream=None):
    W = x.shape[1]
    y = _out2d(x, v.row_end - v.row_begin, W, y)
    _check(_lib.stg_gcn_aggregate_fwd(ctypes.byref(v), W, _ptr(x), x.stride(0), _ptr(y), y.stride(0),
                                      _stream(stream)))
    return y


def stg_gcn_aggregate_bwd(v: stg_csr_view, gy: torch.Tensor, gx: torch.Tensor = None, stream=None):
    W = gy.shape[1]
    gx = _out2d(gy, v.num_nodes, W, gx)
    _check(_lib.stg_gcn_aggregate_bwd(ctypes.byref(v), W, _ptr(gy), gy.stride(0), _ptr(gx), gx.stride(0),
                                      _stream(stream)))
    return gx


def stg_gcn_aggregate_ex(v: stg_csr_view, backward: bool, x: torch.Tensor, out: torch.Tensor = None,
                         scale_row=None, scale_col=None, bias=None, stream=None):
    W = x.shape[1]
    rows = v.num_nodes if backward else v.row_end - v.row_begin
    out = _out2d(x, rows, W, out)
    _check(_lib.stg_gcn_aggregate_ex(ctypes.byref(v), int(backward), W, _ptr(x), x.stride(0), _ptr(out),
                                     out.stride(0), _ptr(scale_row), _ptr(scale_col), _ptr(bias), _stream(stream)))
    return out


def stg_gcn_aggregate_weighted(v: stg_csr_view, backward: bool, ew: torch.Tensor, x: torch.Tensor,
                               out: torch.Tensor = None, scale_row=None, scale_col=None, bias=None, stream=None):
    """Edge-weighted aggregation; ew [E] in in-CSR order (edge label = in-CSR position)."""
    W = x.shape[1]
    rows = v.num_nodes if backward else v.row_end - v.row_begin
    out = _out2d(x, rows, W, out)
    _check(_lib.stg_gcn_aggregate_weighted(ctypes.byref(v), int(backward), W, _ptr(ew), _ptr(x), x.stride(0),
                                           _ptr(out), out.stride(0), _ptr(scale_row), _ptr(scale_col), _ptr(bias),
                                           _stream(stream)))
    return out


def stg_gcn_weighted_norm(v: stg_csr_view, ew: torch.Tensor, norm: torch.Tensor = None, stream=None):
    if norm is None:
        norm = torch.empty(v.row_end - v.row_begin, dtype=torch.float32, device="cuda")
    _check(_lib.stg_gcn_weighted_norm(ctypes.byref(v), _ptr(ew), _ptr(norm), _stream(stream)))
    return norm


# ---------------------------------------------------------------- TGCN
class StateStack:
    def __init__(self, capacity_bytes: int):
        h = ctypes.c_void_p()
        _check(_lib.stg_state_stack_create(int(capacity_bytes), ctypes.byref(h)))
        self.handle = h

    @property
    def depth(self) -> int:
        return int(_lib.stg_state_stack_depth(self.handle))

    def close(self):
        if self.handle:
            _lib.stg_state_stack_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            if _exiting[0] or sys.is_finalizing():   # (the allocator hook calls back into torch)
                return
            self.close()
        except Exception:
            pass


def stg_state_stack_create(capacity_bytes: int) -> StateStack:
    return StateStack(capacity_bytes)


def make_params(p: dict) -> stg_tgcn_params:
    F, H3 = p["W"].shape
    return stg_tgcn_params(F, H3 // 3, _ptr(p["W"]), _ptr(p["b"]), _ptr(p["L"]), _ptr(p["l"]))


def make_grads(g: dict) -> stg_tgcn_grads:
    return stg_tgcn_grads(_ptr(g["W"]), _ptr(g["b"]), _ptr(g["L"]), _ptr(g["l"]))


def stg_tgcn_step(v: stg_csr_view, params: dict, X, H_prev, H_next=None, stack: StateStack = None, stream=None):
    if H_next is None:
        H_next = torch.empty_like(H_prev)
    P = make_params(params)
    _check(_lib.stg_tgcn_step(ctypes.byref(v), ctypes.byref(P), _ptr(X), _ptr(H_prev), _ptr(H_next),
                              stack.handle if stack else None, _stream(stream)))
    return H_next


def stg_tgcn_step_backward(v: stg_csr_view, params: dict, X, dH_next, grads: dict, stack: StateStack,
                           dH_prev=None, stream=None):
    if dH_prev is None:
        dH_prev = torch.empty_like(dH_next)
    P = make_params(params)
    G = make_grads(grads)
    _check(_lib.stg_tgcn_step_backward(ctypes.byref(v), ctypes.byref(P), _ptr(X), _ptr(dH_next), _ptr(dH_prev),
                                       ctypes.byref(G), stack.handle, _stream(stream)))
    return dH_prev


def make_params2(p: dict) -> stg_tgcn2_params:
    K, H2 = p["Wg"].shape
    H = H2 // 2
    return stg_tgcn2_params(K - H, H, _ptr(p["Wg"]), _ptr(p["bg"]), _ptr(p["Wc"]), _ptr(p["bc"]))


def stg_tgcn2_step(v: stg_csr_view, params: dict, X, H_prev, H_next=None, stack: StateStack = None, stream=None):
    """Original T-GCN cell (NEXT-2): GCN over [X, H]."""
    if H_next is None:
        H_next = torch.empty_like(H_prev)
    P = make_params2(params)
    _check(_lib.stg_tgcn2_step(ctypes.byref(v), ctypes.byref(P), _ptr(X), _ptr(H_prev), _ptr(H_next),
                               stack.handle if stack else None, _stream(stream)))
    return H_next


def stg_tgcn2_step_backward(v: stg_csr_view, params: dict, X, dH_next, grads: dict, stack: StateStack,
                            dH_prev=None, stream=None):
    if dH_prev is None:
        dH_prev = torch.empty_like(dH_next)
    P = make_params2(params)
    G = stg_tgcn2_grads(_ptr(grads["Wg"]), _ptr(grads["bg"]), _ptr(grads["Wc"]), _ptr(grads["bc"]))
    _check(_lib.stg_tgcn2_step_backward(ctypes.byref(v), ctypes.byref(P), _ptr(X), _ptr(dH_next), _ptr(dH_prev),
                                        ctypes.byref(G), stack.handle, _stream(stream)))
    return dH_prev


def stg_mse_head(Hn, y, w_o, b_o, loss_accum=None, dH=None, accumulate=False, dw_o=None, db_o=None, stream=None,
                 V_total=None):
    V, H = Hn.shape
    _check(_lib.stg_mse_head_ex(V, V if V_total is None else int(V_total), H, _ptr(Hn), _ptr(y), _ptr(w_o),
                                _ptr(b_o), _ptr(loss_accum), _ptr(dH), int(accumulate), _ptr(dw_o), _ptr(db_o),
                                _stream(stream)))


def stg_sgd_update(p: torch.Tensor, g: torch.Tensor, lr: float, stream=None):
    _check(_lib.stg_sgd_update(_ptr(p), _ptr(g), p.numel(), float(lr), _stream(stream)))


def stg_tgcn_train_sequence_batched(graph, S: int, params: dict, w_o, b_o, Xs, Ys, H0, H_seq, grads: dict, dw_o,
                                    db_o, loss_accum, stack: StateStack, stream=None):
    """Sequence-batched Algorithm 1 over a static graph (NEXT-1): same maths, per-sequence kernels."""
    P = make_params(params)
    G = make_grads(grads)
    xp = _ptrs(Xs)
    yp = _ptrs(Ys)
    _check(_lib.stg_tgcn_train_sequence_batched(graph.handle, S, ctypes.byref(P), _ptr(w_o), _ptr(b_o), xp, yp,
                                                _ptr(H0), _ptr(H_seq), ctypes.byref(G), _ptr(dw_o), _ptr(db_o),
                                                _ptr(loss_accum), stack.handle, _stream(stream)))


def stg_tgcn_train_sequence(source, t0: int, S: int, params: dict, w_o, b_o, Xs, Ys, H0, H_seq, G_work,
                            grads: dict, dw_o, db_o, loss_accum, stack: StateStack, stream=None, xy_ready=None):
    """Algorithm 1 over one sequence; `source` is a Graph or a Dtdg.  xy_ready: optional list of
    torch.cuda.Event, one per timestamp, recorded after X_t / y_t were written."""
    P = make_params(params)
    G = make_grads(grads)
    xp = _ptrs(Xs)
    yp = _ptrs(Ys)
    graph = source.handle if isinstance(source, Graph) else None
    dtdg = source.handle if isinstance(source, Dtdg) else None
    ev = None
    if xy_ready is not None:
        ev = (_P * S)(*[e.cuda_event if e is not None else None for e in xy_ready])
    _check(_lib.stg_tgcn_train_sequence_ev(graph, dtdg, t0, S, ctypes.byref(P), _ptr(w_o), _ptr(b_o), xp, yp,
                                           _ptr(H0), _ptr(H_seq), _ptr(G_work), ctypes.byref(G), _ptr(dw_o),
                                           _ptr(db_o), _ptr(loss_accum), stack.handle, ev, _stream(stream)))


def stg_partition_rows(V: int, in_rowptr: torch.Tensor, world: int, stream=None) -> list:
    b = (_i32 * (world + 1))()
    _check(_lib.stg_partition_rows(V, _ptr(in_rowptr, torch.int32), world, b, _stream(stream)))
    return list(b)


def stg_debug_tc_gemm(mode: int, A: torch.Tensor, B: torch.Tensor, stream=None) -> torch.Tensor:
    """mode 0: A[M,K]·B[K,N]; mode 1: Aᵀ·B with A[R,128], B[R,N] (tcgen05 3xTF32);
    mode 2: as 0 with A in tensor memory; mode 3: one unsplit tf32 pass of A·B;
    mode 4: as 1 with TMA-loaded MN-major (SWIZZLE_128B_BASE32B) operands."""
    if mode not in (1, 4):
        M, K = A.shape
        N = B.shape[1]
        C = torch.empty(M, N, device=A.device)
        _check(_lib.stg_debug_tc_gemm(mode, M, N, K, 0, _ptr(A), _ptr(B), _ptr(C), _stream(stream)))
    else:
        R = A.shape[0]
        N = B.shape[1]
        C = torch.empty(128, N, device=A.device)
        _check(_lib.stg_debug_tc_gemm(mode, 128, N, 0, R, _ptr(A), _ptr(B), _ptr(C), _stream(stream)))
    return C


def stg_debug_sum_parts(part: torch.Tensor, variant: int, stream=None) -> torch.Tensor:
    """Fixed-order Σ over the rows of part [nb, n] (the Σ AᵀB partial sums): variant 0 serial, 1 parallel."""
    nb, n = part.shape
    tot = torch.empty(n, device=part.device)
    _check(_lib.stg_debug_sum_parts(_ptr(part), nb, n, _ptr(tot), int(variant), _stream(stream)))
    return tot


def stg_aggregate_set_strategy(strategy: int):
    """2 = edge stream (default), 1 = pipelined row items, 0 = row items (include/stg.h)."""
    _check(_lib.stg_aggregate_set_strategy(int(strategy)))


AGG_ROWS_IN_FLIGHT, AGG_MIN_BLOCKS, AGG_STREAM_WMIN = 0, 1, 2


def stg_aggregate_set_param(key: int, value: int):
    """Edge-stream tunables (include/stg.h): 0 rows in flight, 1 min blocks/SM, 2 min width."""
    _check(_lib.stg_aggregate_set_param(int(key), int(value)))


# ---------------------------------------------------------------- sharded mode (peer memory)
class PeerBuffer:
    """A CUDA-IPC-visible fp32 [rows, cols] buffer owned by libstg (stg_peer_alloc),
    exposed to torch through __cuda_array_interface__ (no copy)."""

    def __init__(self, rows: int, cols: int):
        self.rows, self.cols = int(rows), int(cols)
        self.handle = stg_ipc_handle()
        p = ctypes.c_void_p()
        _check(_lib.stg_peer_alloc(max(1, self.rows * self.cols * 4), ctypes.byref(p), ctypes.byref(self.handle)))
        self.ptr = p.value
        self.__cuda_array_interface__ = {"shape": (self.rows, self.cols), "typestr": "<f4",
                                         "data": (self.ptr, False), "version": 2, "strides": None}
        self.tensor = torch.as_tensor(self, device="cuda")

    def handle_bytes(self) -> bytes:
        return bytes(self.handle.reserved)

    def close(self):
        if self.ptr:
            self.tensor = None
            _lib.stg_peer_free(ctypes.c_void_p(self.ptr))
            self.ptr = None

    def __del__(self):
        try:
            if _exiting[0] or sys.is_finalizing():   # (the allocator hook calls back into torch)
                return
            self.close()
        except Exception:
            pass


def stg_peer_open(handle: bytes) -> int:
    """Map another process's PeerBuffer (its handle_bytes()); returns the device pointer."""
    h = stg_ipc_handle()
    ctypes.memmove(h.reserved, handle, 64)
    p = ctypes.c_void_p()
    _check(_lib.stg_peer_open(ctypes.byref(h), ctypes.byref(p)))
    return p.value


def stg_peer_close(ptr: int):
    _check(_lib.stg_peer_close(ctypes.c_void_p(ptr)))


class PeerRows:
    """stg_peer_rows: block k = rows [bounds[k], bounds[k+1]) at device pointer ptrs[k] (ld floats)."""

    def __init__(self, bounds, ptrs, ld: int):
        world = len(bounds) - 1
        if len(ptrs) != world or not 1 <= world <= STG_MAX_PEERS:
            raise StgError(1, "PeerRows: need 1 <= world <= %d blocks" % STG_MAX_PEERS)
        self._b = (_i32 * (world + 1))(*[int(x) for x in bounds])
        self._p = (_P * world)(*[int(p) if p else None for p in ptrs])
        self.c = stg_peer_rows(world, self._b, self._p, int(ld))


def _row_ptr(t):
    return t.data_ptr() if isinstance(t, torch.Tensor) else int(t)


def stg_allgather_rows(rows: PeerRows, W: int, full: torch.Tensor, stream=None) -> torch.Tensor:
    _check(_lib.stg_allgather_rows(ctypes.byref(rows.c), int(W), _ptr(full), full.stride(0), _stream(stream)))
    return full


def stg_gcn_aggregate_peer(v: stg_csr_view, rows: PeerRows, W: int, out: torch.Tensor = None, scale_row=None,
                           scale_col=None, bias=None, stream=None) -> torch.Tensor:
    if out is None:
        out = torch.empty((v.row_end - v.row_begin, W), dtype=torch.float32, device="cuda")
    _check(_lib.stg_gcn_aggregate_peer(ctypes.byref(v), int(W), ctypes.byref(rows.c), _ptr(out), out.stride(0),
                                       _ptr(scale_row), _ptr(scale_col), _ptr(bias), _stream(stream)))
    return out


def stg_reduce_scatter_rows(bounds, partials, ld: int, rank: int, W: int, out: torch.Tensor, stream=None):
    world = len(bounds) - 1
    b = (_i32 * (world + 1))(*[int(x) for x in bounds])
    pp = (_P * world)(*[_row_ptr(p) for p in partials])
    _check(_lib.stg_reduce_scatter_rows(world, b, pp, int(ld), int(rank), int(W), _ptr(out), out.stride(0),
                                        _stream(stream)))
    return out


def stg_tgcn_project(v: stg_csr_view, params: dict, X_loc, P_loc, stream=None):
    P = make_params(params)
    _check(_lib.stg_tgcn_project(ctypes.byref(v), ctypes.byref(P), _ptr(X_loc), ctypes.c_void_p(_row_ptr(P_loc)),
                                 _stream(stream)))


def stg_tgcn_step_peer(v: stg_csr_view, params: dict, rows: PeerRows, H_prev, H_next, stack: StateStack = None,
                       stream=None):
    P = make_params(params)
    _check(_lib.stg_tgcn_step_peer(ctypes.byref(v), ctypes.byref(P), ctypes.byref(rows.c), _ptr(H_prev),
                                   _ptr(H_next), stack.handle if stack else None, _stream(stream)))
    return H_next


def stg_tgcn_step_backward_peer(v: stg_csr_view, params: dict, dH_next, dH_prev, grads: dict, dP_part,
                                stack: StateStack, stream=None):
    P = make_params(params)
    G = make_grads(grads)
    _check(_lib.stg_tgcn_step_backward_peer(ctypes.byref(v), ctypes.byref(P), _ptr(dH_next), _ptr(dH_prev),
                                            ctypes.byref(G), ctypes.c_void_p(_row_ptr(dP_part)), stack.handle,
                                            _stream(stream)))
    return dH_prev


def stg_tgcn_dw(params: dict, X_loc, dP_loc, grads: dict, stack: StateStack, stream=None):
    P = make_params(params)
    G = make_grads(grads)
    R = X_loc.shape[0]
    _check(_lib.stg_tgcn_dw(ctypes.byref(P), int(R), _ptr(X_loc), ctypes.c_void_p(_row_ptr(dP_loc)),
                            ctypes.byref(G), stack.handle, _stream(stream)))


def stg_tgcn_train_sequence_peer(dtdg, t0: int, params: dict, w_o, b_o, X_loc, Y_loc, H0, H_seq, G_work, dP_loc,
                                 grads: dict, dw_o, db_o, loss_accum, stack, px: "stg_peer_exchange", stream=None):
    """Sharded-mode Algorithm 1 for one sequence inside the library (device-side exchange flags)."""
    P = make_params(params)
    G = make_grads(grads)
    S = len(X_loc)
    _check(_lib.stg_tgcn_train_sequence_peer(dtdg.handle, int(t0), S, ctypes.byref(P), _ptr(w_o), _ptr(b_o),
                                             _ptrs(X_loc), _ptrs(Y_loc), _ptr(H0), _ptr(H_seq), _ptr(G_work),
                                             _ptr(dP_loc), ctypes.byref(G), _ptr(dw_o), _ptr(db_o),
                                             _ptr(loss_accum), stack.handle, ctypes.byref(px), _stream(stream)))


def stg_tgcn2_peer_fwd(phase: int, v: stg_csr_view, params: dict, X_loc, H_loc, rows: PeerRows = None, Z_loc=None,
                       H_next=None, stack: StateStack = None, stream=None):
    """One phase of the sharded original T-GCN forward (include/stg.h)."""
    P = make_params2(params)
    _check(_lib.stg_tgcn2_peer_fwd(int(phase), ctypes.byref(v), ctypes.byref(P), _ptr(X_loc), _ptr(H_loc),
                                   ctypes.byref(rows.c) if rows is not None else None,
                                   ctypes.c_void_p(_row_ptr(Z_loc)) if Z_loc is not None else None,
                                   _ptr(H_next) if H_next is not None else None, stack.handle, _stream(stream)))


def stg_tgcn2_peer_bwd(phase: int, v: stg_csr_view, params: dict, X_loc, dH_next, dH_prev, grads: dict, rank: int,
                       bounds, parts, part_out, stack: StateStack, stream=None):
    """One phase of the sharded original T-GCN backward (include/stg.h)."""
    P = make_params2(params)
    G = stg_tgcn2_grads(_ptr(grads["Wg"]), _ptr(grads["bg"]), _ptr(grads["Wc"]), _ptr(grads["bc"]))
    world = len(bounds) - 1
    b = (_i32 * (world + 1))(*[int(x) for x in bounds])
    pp = (_P * world)(*[_row_ptr(x) for x in parts]) if parts is not None else None
    _check(_lib.stg_tgcn2_peer_bwd(int(phase), ctypes.byref(v), ctypes.byref(P), _ptr(X_loc),
                                   _ptr(dH_next) if dH_next is not None else None, _ptr(dH_prev), ctypes.byref(G),
                                   int(rank), world, b, pp,
                                   ctypes.c_void_p(_row_ptr(part_out)) if part_out is not None else None,
                                   stack.handle, _stream(stream)))


if os.environ.get("STG_TORCH_ALLOCATOR", "1") != "0" and torch.cuda.is_available():
    use_torch_allocator(True)
