"""C-ABI boundary checks that need no GPU (-m "not gpu"): the library loads, exports every symbol
include/agraph.h declares, and its host-only entry points behave."""
import ctypes
import os
import re

import pytest

from paper_conf_ipps_lib13_b200 import agraph as A
from paper_conf_ipps_lib13_b200 import build as B

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "agraph.h")


@pytest.fixture(scope="module")
def L():
    B.build()
    return A.lib()


def declared_symbols():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(ag_[a-z_0-9]+)\s*\(", src)) - {"ag_graph_s", "ag_comm_s"})


def test_header_declares_the_boundary():
    syms = declared_symbols()
    for s in ["ag_graph_load_csr", "ag_bfs", "ag_sssp", "ag_select", "ag_policy_default", "ag_dist_bfs"]:
        assert s in syms
    assert set(A.EXPORTS) == set(syms)


def test_library_exports_every_declared_symbol(L):
    for s in declared_symbols():
        assert hasattr(L, s), s


def test_status_strings_and_version(L):
    assert L.ag_abi_version() == 1
    for code, name in A.STATUS.items():
        assert L.ag_status_string(code).decode() == name


def test_no_device_is_reported_not_crashed(L):
    import torch
    if torch.cuda.is_available():
        pytest.skip("has a GPU")
    with pytest.raises(A.AgError) as e:
        A.policy_default(0)
    assert e.value.status == "AG_ERR_NO_DEVICE"
    import numpy as np
    with pytest.raises(A.AgError) as e:
        A.Graph(3, np.array([0, 1, 2, 2], np.uint64), np.array([1, 2], np.uint32))
    assert e.value.status == "AG_ERR_NO_DEVICE"


def test_dist_owned_range_partitions(L):
    for V, world in [(1, 1), (1000, 3), (4194304, 8), (67108864, 8), (5000, 8), (1 << 20, 2)]:
        prev = 0
        for r in range(world):
            b, e = ctypes.c_uint32(), ctypes.c_uint32()
            assert L.ag_dist_owned_range(V, r, world, ctypes.byref(b), ctypes.byref(e)) == 0
            assert b.value == prev and e.value >= b.value
            assert b.value % 1024 == 0 or b.value == V        # whole 1024-bit bitmap slices
            prev = e.value
        assert prev == V
    b, e = ctypes.c_uint32(), ctypes.c_uint32()
    assert L.ag_dist_owned_range(10, 2, 2, ctypes.byref(b), ctypes.byref(e)) == 1  # rank out of range


def test_select_rejects_bad_policy(L):
    p = A.Policy()
    p.struct_size = 3
    info = A.GraphInfo()
    assert A.select(p, info, 10, 0) == 0


def _paper_policy(T1=32, T2=2688, t3_ppm=100000):
    p = A.Policy()
    p.struct_size = ctypes.sizeof(A.Policy)
    p.kind = A.POLICY_PAPER
    p.t1_avg_degree, p.t2_ws, p.t3_ppm = T1, T2, t3_ppm
    p.sample_every, p.delta, p.thread_tpb = 1, 1, 192
    return p


def test_ag_select_matches_fig11_oracle(L):
    """The library's decision maker (host copy of the device rule) == oracle/selector.py (Fig. 11)."""
    from oracle import selector
    p = _paper_policy(t3_ppm=100000)   # T3 = 10% of V = 10,000 for V = 100,000
    info = A.GraphInfo()
    for ws in [0, 1, 2687, 2688, 5000, 9999, 10000, 10001, 99999]:
        for E in [100000, 3199999, 3200000, 7390000]:
            info.num_vertices, info.num_edges = 100000, E
            m, w = selector.paper_select(ws, 100000, E, T1=32, T2=2688, T3=10000)
            v = A.select(p, info, ws, 0)
            assert A.variant_name(v) == f"{m}_{w}", (ws, E, A.variant_name(v))


def test_ag_select_forced_axes(L):
    p = _paper_policy()
    info = A.GraphInfo()
    info.num_vertices, info.num_edges = 1000, 5000
    p.mapping, p.workset = A.MAP_WARP, A.WS_BITMAP
    assert A.select(p, info, 1, 0) == A.variant(A.MAP_WARP, A.WS_BITMAP)
    p.mapping, p.workset = A.MAP_AUTO, A.WS_QUEUE
    assert A.select(p, info, 10**6, 0) == A.variant(A.MAP_THREAD, A.WS_QUEUE)


def _tuned_policy(order=0):
    p = _paper_policy()
    p.kind = A.POLICY_TUNED
    p.order = order
    return p


def test_ag_select_tuned_rule(L):
    """The tuned decision maker (common.cuh select_variant) as a pure function of (|WS|,
    m_F, graph): thread mapping only for small, low-degree working sets of a graph without long lists;
    the bitmap only for a dense ordered-SSSP pending set (>= V/32); the hybrid queue otherwise."""
    info = A.GraphInfo()
    info.num_vertices, info.num_edges, info.max_deg = 1 << 20, 8 << 20, 40     # ER-like: max degree 40
    p = _tuned_policy()
    T, H, QU, BM = A.MAP_THREAD, A.MAP_HYBRID, A.WS_QUEUE, A.WS_BITMAP
    assert A.select(p, info, 1000, 4000) == A.variant(T, QU)           # small, avg degree 4 (grid-like)
    assert A.select(p, info, 1000, 6000) == A.variant(T, QU)           # m_F = 6 |WS|: still low
    assert A.select(p, info, 1000, 6001) == A.variant(H, QU)           # above: load-balanced (ER's 8)
    assert A.select(p, info, 65535, 4 * 65535) == A.variant(T, QU)
    assert A.select(p, info, 65536, 4 * 65536) == A.variant(H, QU)     # big working set
    info.max_deg = 65                                                   # one long list: straggler risk
    assert A.select(p, info, 1000, 4000) == A.variant(H, QU)
    # unordered: never the bitmap, however dense
    assert A.select(p, info, 1 << 20, 8 << 20) == A.variant(H, QU)
    # ordered SSSP pending set: bitmap from V/32 on
    po = _tuned_policy(order=A.ORDERED)
    V32 = (1 << 20) // 32
    assert A.select(po, info, V32 - 1, 8 * V32) == A.variant(H, QU)
    assert A.select(po, info, V32, 8 * V32) == A.variant(H, BM)
