"""ctypes binding of libagraph.so (include/agraph.h) — argument marshalling only.

Every step of the hot path runs in the library's CUDA kernels; this module only converts numpy
arrays / torch tensors to pointers and C structs.  There is no CPU fallback: if the shared
library is missing or no sm_100 device is present, calls raise.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field
from typing import Optional

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("AGRAPH_LIB") or os.path.join(HERE, "libagraph.so")  # override: experiment builds
INF = 0xFFFFFFFF

# enums (include/agraph.h)
UNORDERED, ORDERED = 0, 1
MAP_AUTO, MAP_THREAD, MAP_WARP, MAP_CTA, MAP_HYBRID = 0, 1, 2, 3, 4
WS_AUTO, WS_BITMAP, WS_QUEUE = 0, 1, 2
POLICY_PAPER, POLICY_TUNED = 0, 1
LAYOUT_AUTO, LAYOUT_IDENTITY, LAYOUT_DEGREE = 0, 1, 2
WINDOW_AUTO = 0xFFFFFFFF
WINDOW_ADAPTIVE = 0xFFFFFFFE
STATUS = {0: "AG_OK", 1: "AG_ERR_INVALID_ARG", 2: "AG_ERR_BAD_CSR", 3: "AG_ERR_SRC_RANGE", 4: "AG_ERR_NO_WEIGHTS",
          5: "AG_ERR_OVERFLOW", 6: "AG_ERR_OOM", 7: "AG_ERR_CUDA", 8: "AG_ERR_NCCL", 9: "AG_ERR_UNSUPPORTED",
          10: "AG_ERR_NO_DEVICE"}
MAP_LETTER = {MAP_THREAD: "T", MAP_WARP: "W", MAP_CTA: "B", MAP_HYBRID: "H"}
WS_NAME = {WS_BITMAP: "BM", WS_QUEUE: "QU"}


def variant(mapping: int, workset: int) -> int:
    return mapping * 4 + workset


def variant_name(v: int) -> str:
    return f"{MAP_LETTER.get(v >> 2, '?')}_{WS_NAME.get(v & 3, '?')}"


class AgError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{STATUS.get(code, code)}: {msg}")
        self.code = code
        self.status = STATUS.get(code, str(code))


class Policy(ctypes.Structure):
    _fields_ = [("struct_size", ctypes.c_uint32), ("order", ctypes.c_uint32), ("mapping", ctypes.c_uint32),
                ("workset", ctypes.c_uint32), ("kind", ctypes.c_uint32), ("t1_avg_degree", ctypes.c_uint32),
                ("t2_ws", ctypes.c_uint64), ("t3_ppm", ctypes.c_uint32), ("sample_every", ctypes.c_uint32),
                ("delta", ctypes.c_uint32), ("thread_tpb", ctypes.c_uint32), ("cta_group", ctypes.c_uint32),
                ("sssp_window", ctypes.c_uint32), ("sssp_hub_window", ctypes.c_uint32), ("free_ppm", ctypes.c_uint32),
                ("small_ws", ctypes.c_uint32)]


class GraphInfo(ctypes.Structure):
    _fields_ = [("num_vertices", ctypes.c_uint32), ("min_deg", ctypes.c_uint32), ("max_deg", ctypes.c_uint32),
                ("num_edges", ctypes.c_uint64), ("deg_sum", ctypes.c_uint64), ("isolated", ctypes.c_uint32),
                ("weighted", ctypes.c_uint32), ("device", ctypes.c_int32), ("num_sms", ctypes.c_uint32),
                ("offset_bytes", ctypes.c_uint32), ("layout", ctypes.c_uint32), ("max_weight", ctypes.c_uint32),
                ("reserved2", ctypes.c_uint32)]


class RunStats(ctypes.Structure):
    _fields_ = [("struct_size", ctypes.c_uint32), ("iterations", ctypes.c_uint32),
                ("vertices_expanded", ctypes.c_uint64), ("edges_inspected", ctypes.c_uint64),
                ("reached", ctypes.c_uint64), ("reached_edges", ctypes.c_uint64), ("device_ms", ctypes.c_float),
                ("trace_cap", ctypes.c_uint32), ("trace_len", ctypes.c_uint32), ("reserved", ctypes.c_uint32),
                ("trace_ws", ctypes.POINTER(ctypes.c_uint32)), ("trace_edges", ctypes.POINTER(ctypes.c_uint64)),
                ("trace_variant", ctypes.POINTER(ctypes.c_uint8)), ("trace_ns", ctypes.POINTER(ctypes.c_uint64))]


EXPORTS = ["ag_policy_default", "ag_select", "ag_graph_load_csr", "ag_graph_load_csr_ex", "ag_graph_info_get",
           "ag_graph_free", "ag_bfs", "ag_sssp", "ag_cc", "ag_graph_check", "ag_dist_unique_id", "ag_dist_init",
           "ag_dist_init_local", "ag_dist_free", "ag_dist_owned_range", "ag_dist_graph_load_csr",
           "ag_dist_graph_load_local", "ag_dist_bfs", "ag_dist_bfs_group", "ag_dist_sssp", "ag_dist_sssp_group", "ag_set_allocator", "ag_status_string",
           "ag_last_error", "ag_abi_version", "ag_kernel_launches"]

_lib = None


def lib():
    """Load libagraph.so (built by ``python -m paper_conf_ipps_lib13_b200.build``)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise AgError(10, f"{LIB_PATH} not built; run python -m paper_conf_ipps_lib13_b200.build")
    if "AG_NCCL_LIB" not in os.environ:  # the library dlopens NCCL on first multi-GPU use
        try:
            import nvidia.nccl as _n
            cand = os.path.join(list(_n.__path__)[0], "lib", "libnccl.so.2")
            if os.path.exists(cand):
                os.environ["AG_NCCL_LIB"] = cand
        except Exception:
            pass
    L = ctypes.CDLL(LIB_PATH)
    vp, u32, u64, i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
    L.ag_policy_default.argtypes = [ctypes.POINTER(Policy), i32]
    L.ag_select.argtypes = [ctypes.POINTER(Policy), ctypes.POINTER(GraphInfo), u64, u64]
    L.ag_select.restype = ctypes.c_uint8
    L.ag_graph_load_csr.argtypes = [u32, u64, vp, vp, vp, i32, ctypes.POINTER(vp)]
    L.ag_graph_load_csr_ex.argtypes = [u32, u64, vp, vp, vp, i32, u32, ctypes.POINTER(vp)]
    L.ag_graph_info_get.argtypes = [vp, ctypes.POINTER(GraphInfo)]
    L.ag_graph_free.argtypes = [vp]
    L.ag_graph_check.argtypes = [vp]
    for f in (L.ag_bfs, L.ag_sssp):
        f.argtypes = [vp, u32, vp, vp, ctypes.POINTER(Policy), ctypes.POINTER(RunStats), vp]
    L.ag_cc.argtypes = [vp, vp, ctypes.POINTER(Policy), ctypes.POINTER(RunStats), vp]
    L.ag_dist_unique_id.argtypes = [vp]
    L.ag_dist_init.argtypes = [i32, i32, vp, i32, ctypes.POINTER(vp)]
    L.ag_dist_free.argtypes = [vp]
    L.ag_dist_owned_range.argtypes = [u32, i32, i32, ctypes.POINTER(u32), ctypes.POINTER(u32)]
    L.ag_dist_graph_load_csr.argtypes = [vp, u32, u64, vp, vp, vp, ctypes.POINTER(vp)]
    L.ag_dist_bfs.argtypes = [vp, u32, vp, vp, ctypes.POINTER(Policy), ctypes.POINTER(RunStats), vp]
    L.ag_dist_init_local.argtypes = [i32, i32, vp]
    L.ag_dist_graph_load_local.argtypes = [vp, u32, u64, vp, vp, vp, ctypes.POINTER(vp)]
    L.ag_dist_bfs_group.argtypes = [vp, i32, u32, vp, vp, ctypes.POINTER(RunStats), vp]
    L.ag_dist_sssp.argtypes = [vp, u32, vp, vp, ctypes.POINTER(Policy), ctypes.POINTER(RunStats), vp]
    L.ag_dist_sssp_group.argtypes = [vp, i32, u32, vp, vp, ctypes.POINTER(RunStats), vp]
    L.ag_status_string.restype = ctypes.c_char_p
    L.ag_status_string.argtypes = [i32]
    L.ag_last_error.restype = ctypes.c_char_p
    L.ag_abi_version.restype = u32
    L.ag_kernel_launches.restype = u64
    _lib = L
    return L


def _check(rc: int):
    if rc != 0:
        raise AgError(rc, lib().ag_last_error().decode())


def _ptr(a) -> Optional[int]:
    """Pointer of a numpy array or torch tensor (contiguous), or None."""
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        assert a.flags.c_contiguous
        return a.ctypes.data
    if hasattr(a, "data_ptr"):
        assert a.is_contiguous()
        return a.data_ptr()
    raise TypeError(type(a))


def policy_default(device: int = 0, **overrides) -> Policy:
    p = Policy()
    _check(lib().ag_policy_default(ctypes.byref(p), device))
    for k, v in overrides.items():
        setattr(p, k, v)
    return p


def select(policy: Policy, info: GraphInfo, ws_size: int, ws_edges: int = 0) -> int:
    return int(lib().ag_select(ctypes.byref(policy), ctypes.byref(info), ws_size, ws_edges))


def kernel_launches() -> int:
    return int(lib().ag_kernel_launches())


@dataclass
class Stats:
    iterations: int
    vertices_expanded: int
    edges_inspected: int
    reached: int
    reached_edges: int
    device_ms: float
    trace_ws: np.ndarray = field(default_factory=lambda: np.zeros(0, np.uint32))
    trace_edges: np.ndarray = field(default_factory=lambda: np.zeros(0, np.uint64))
    trace_variant: np.ndarray = field(default_factory=lambda: np.zeros(0, np.uint8))
    trace_us: np.ndarray = field(default_factory=lambda: np.zeros(0, np.float64))  # per-iteration device time


class Graph:
    """A graph loaded into device memory (ag_graph_load_csr)."""

    def __init__(self, V: int, row_ptr, col, w=None, device: int = 0, layout: int = LAYOUT_AUTO):
        h = ctypes.c_void_p()
        E = int(row_ptr[-1]) if isinstance(row_ptr, np.ndarray) else int(row_ptr[-1].item())
        _check(lib().ag_graph_load_csr_ex(V, E, _ptr(row_ptr), _ptr(col), _ptr(w), device, layout, ctypes.byref(h)))
        self.h = h
        self.V, self.E, self.device = V, E, device
        self.info = GraphInfo()
        _check(lib().ag_graph_info_get(self.h, ctypes.byref(self.info)))

    @classmethod
    def from_csr(cls, g, device: int = 0, weighted: bool = True, layout: int = LAYOUT_AUTO):
        return cls(g.V, g.row_ptr, g.col, g.w if weighted else None, device, layout)

    def free(self):
        if self.h:
            _check(lib().ag_graph_free(self.h))
            self.h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass

    def _run(self, fn, src, out, parents, policy, stats, trace_cap, stream):
        if out is None:
            out = np.empty(self.V, dtype=np.uint32)
        st = None
        tr = None
        if stats:
            st = RunStats()
            st.struct_size = ctypes.sizeof(RunStats)
            if trace_cap:
                tr = (np.zeros(trace_cap, np.uint32), np.zeros(trace_cap, np.uint64), np.zeros(trace_cap, np.uint8),
                      np.zeros(trace_cap + 1, np.uint64))
                st.trace_cap = trace_cap
                st.trace_ws = tr[0].ctypes.data_as(ctypes.POINTER(ctypes.c_uint32))
                st.trace_edges = tr[1].ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))
                st.trace_variant = tr[2].ctypes.data_as(ctypes.POINTER(ctypes.c_uint8))
                st.trace_ns = tr[3].ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))
        rc = fn(self.h, int(src), _ptr(out), _ptr(parents), ctypes.byref(policy) if policy is not None else None,
                ctypes.byref(st) if st is not None else None, ctypes.c_void_p(stream or 0))
        _check(rc)
        res = None
        if st is not None:
            n = st.trace_len
            res = Stats(st.iterations, st.vertices_expanded, st.edges_inspected, st.reached, st.reached_edges,
                        st.device_ms)
            if tr is not None:
                res.trace_ws, res.trace_edges, res.trace_variant = tr[0][:n], tr[1][:n], tr[2][:n]
                if n == st.iterations:
                    res.trace_us = np.diff(tr[3][:n + 1].astype(np.float64)) / 1e3
        return out, parents, res

    def bfs(self, src: int, levels=None, parents=None, policy: Optional[Policy] = None, stats: bool = False,
            trace_cap: int = 0, stream: Optional[int] = None):
        """ag_bfs; returns (levels, parents, Stats|None)."""
        return self._run(lib().ag_bfs, src, levels, parents, policy, stats, trace_cap, stream)

    def sssp(self, src: int, dist=None, parents=None, policy: Optional[Policy] = None, stats: bool = False,
             trace_cap: int = 0, stream: Optional[int] = None):
        """ag_sssp; returns (dist, parents, Stats|None)."""
        return self._run(lib().ag_sssp, src, dist, parents, policy, stats, trace_cap, stream)

    def cc(self, labels=None, policy: Optional[Policy] = None, stats: bool = False, trace_cap: int = 0,
           stream: Optional[int] = None):
        """ag_cc (min-label components, R23); returns (labels, None, Stats|None)."""
        def fn(h, _src, out, _par, pol, st, strm):
            return lib().ag_cc(h, out, pol, st, strm)
        return self._run(fn, 0, labels, None, policy, stats, trace_cap, stream)

    def check(self):
        _check(lib().ag_graph_check(self.h))


# ---------------------------------------------------------------------------------------------
# multi-GPU (1-D destination partition)
# ---------------------------------------------------------------------------------------------
def owned_range(V: int, rank: int, world: int):
    b, e = ctypes.c_uint32(), ctypes.c_uint32()
    _check(lib().ag_dist_owned_range(V, rank, world, ctypes.byref(b), ctypes.byref(e)))
    return b.value, e.value


def dist_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib().ag_dist_unique_id(buf))
    return buf.raw


class Comm:
    """One rank's communicator: NCCL (ag_dist_init) or a member of a virtual group."""

    def __init__(self, handle, rank: int, world: int, device: int):
        self.h, self.rank, self.world, self.device = handle, rank, world, device

    @classmethod
    def nccl(cls, rank: int, world: int, unique_id: bytes, device: int):
        h = ctypes.c_void_p()
        idbuf = ctypes.create_string_buffer(unique_id, 128)
        _check(lib().ag_dist_init(rank, world, idbuf, device, ctypes.byref(h)))
        return cls(h, rank, world, device)

    def free(self):
        if self.h:
            _check(lib().ag_dist_free(self.h))
            self.h = None


def local_group(world: int, device: int = 0):
    """`world` virtual ranks in this process on one GPU (all-gather = device copy)."""
    arr = (ctypes.c_void_p * world)()
    _check(lib().ag_dist_init_local(world, device, arr))
    return [Comm(ctypes.c_void_p(arr[r]), r, world, device) for r in range(world)]


class DistGraph(Graph):
    """This rank's part of a 1-D destination-partitioned graph."""

    def __init__(self, comm: Comm, V: int, row_ptr, col, w=None, local: bool = False):
        h = ctypes.c_void_p()
        E = int(row_ptr[-1]) if isinstance(row_ptr, np.ndarray) else int(row_ptr[-1].item())
        fn = lib().ag_dist_graph_load_local if local else lib().ag_dist_graph_load_csr
        _check(fn(comm.h, V, E, _ptr(row_ptr), _ptr(col), _ptr(w), ctypes.byref(h)))
        self.h, self.V, self.E, self.device, self.comm = h, V, E, comm.device, comm
        self.own = owned_range(V, comm.rank, comm.world)
        self.info = GraphInfo()
        _check(lib().ag_graph_info_get(self.h, ctypes.byref(self.info)))

    def bfs(self, src: int, levels=None, parents=None, policy=None, stats: bool = False, trace_cap: int = 0,
            stream=None):
        """ag_dist_bfs (collective over the NCCL communicator): returns this rank's owned slices."""
        n = self.own[1] - self.own[0]
        if levels is None:
            levels = np.empty(n, np.uint32)
        st, tr = _mkstats(stats, trace_cap)
        _check(lib().ag_dist_bfs(self.h, int(src), _ptr(levels), _ptr(parents),
                                 ctypes.byref(policy) if policy is not None else None,
                                 ctypes.byref(st) if st is not None else None, ctypes.c_void_p(stream or 0)))
        return levels, parents, _stats_out(st, tr)


    def sssp(self, src: int, dist=None, parents=None, policy=None, stats: bool = False, trace_cap: int = 0,
             stream=None):
        """ag_dist_sssp (collective over the NCCL communicator): returns this rank's owned slices."""
        n = self.own[1] - self.own[0]
        if dist is None:
            dist = np.empty(n, np.uint32)
        st, tr = _mkstats(stats, trace_cap)
        _check(lib().ag_dist_sssp(self.h, int(src), _ptr(dist), _ptr(parents),
                                  ctypes.byref(policy) if policy is not None else None,
                                  ctypes.byref(st) if st is not None else None, ctypes.c_void_p(stream or 0)))
        return dist, parents, _stats_out(st, tr)


def dist_sssp_group(parts, src: int, parents: bool = False, stats: bool = False, trace_cap: int = 0):
    """Lock-step SSSP over the ranks of a virtual group; returns (dist, parents|None, Stats) in
    GLOBAL vertex order (owned slices concatenated)."""
    P = len(parts)
    dv = [np.empty(p.own[1] - p.own[0], np.uint32) for p in parts]
    pa = [np.empty(p.own[1] - p.own[0], np.uint32) for p in parts] if parents else None
    hs = (ctypes.c_void_p * P)(*[p.h.value for p in parts])
    dvp = (ctypes.c_void_p * P)(*[a.ctypes.data for a in dv])
    pap = (ctypes.c_void_p * P)(*[a.ctypes.data for a in pa]) if parents else None
    st, tr = _mkstats(stats, trace_cap)
    _check(lib().ag_dist_sssp_group(hs, P, int(src), dvp, pap, ctypes.byref(st) if st is not None else None, None))
    return np.concatenate(dv), (np.concatenate(pa) if parents else None), _stats_out(st, tr)


def dist_bfs_group(parts, src: int, parents: bool = False, stats: bool = False, trace_cap: int = 0):
    """Lock-step BFS over the ranks of a virtual group; returns (levels, parents|None, Stats) in
    GLOBAL vertex order (owned slices concatenated)."""
    P = len(parts)
    lv = [np.empty(p.own[1] - p.own[0], np.uint32) for p in parts]
    pa = [np.empty(p.own[1] - p.own[0], np.uint32) for p in parts] if parents else None
    hs = (ctypes.c_void_p * P)(*[p.h.value for p in parts])
    lvp = (ctypes.c_void_p * P)(*[a.ctypes.data for a in lv])
    pap = (ctypes.c_void_p * P)(*[a.ctypes.data for a in pa]) if parents else None
    st, tr = _mkstats(stats, trace_cap)
    _check(lib().ag_dist_bfs_group(hs, P, int(src), lvp, pap, ctypes.byref(st) if st is not None else None, None))
    return np.concatenate(lv), (np.concatenate(pa) if parents else None), _stats_out(st, tr)


def _mkstats(stats, trace_cap):
    if not stats:
        return None, None
    st = RunStats()
    st.struct_size = ctypes.sizeof(RunStats)
    tr = None
    if trace_cap:
        tr = (np.zeros(trace_cap, np.uint32), np.zeros(trace_cap, np.uint64), np.zeros(trace_cap, np.uint8),
              np.zeros(trace_cap + 1, np.uint64))
        st.trace_cap = trace_cap
        st.trace_ws = tr[0].ctypes.data_as(ctypes.POINTER(ctypes.c_uint32))
    return st, tr


def _stats_out(st, tr):
    if st is None:
        return None
    res = Stats(st.iterations, st.vertices_expanded, st.edges_inspected, st.reached, st.reached_edges, st.device_ms)
    if tr is not None:
        res.trace_ws = tr[0][: st.trace_len]
    return res


# ---------------------------------------------------------------------------------------------
# device allocator hook (ag_set_allocator): route the library's device allocations through the
# PyTorch caching allocator, so repeated graph loads reuse memory instead of cudaMalloc/cudaFree
# ---------------------------------------------------------------------------------------------
_ALLOC_T = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p)
_FREE_T = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p)
_alloc_refs = None


def use_torch_allocator(enable: bool = True):
    global _alloc_refs
    L = lib()
    L.ag_set_allocator.argtypes = [_ALLOC_T, _FREE_T, ctypes.c_void_p]
    if not enable:
        _check(L.ag_set_allocator(_ALLOC_T(0), _FREE_T(0), None))
        return   # (the callbacks stay referenced: buffers allocated through them are freed through them)
    import torch

    def _alloc(nbytes, dev, stream, ctx):
        try:
            return torch.cuda.caching_allocator_alloc(int(nbytes), int(dev))
        except Exception:
            return 0

    def _free(ptr, nbytes, dev, stream, ctx):
        torch.cuda.caching_allocator_delete(int(ptr))

    refs = (_ALLOC_T(_alloc), _FREE_T(_free))
    _alloc_refs = (_alloc_refs or []) + [refs]
    _check(L.ag_set_allocator(refs[0], refs[1], None))
