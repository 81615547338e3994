"""CPU oracle for the adaptive BFS/SSSP hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  It
shares no code with the CUDA path (``paper_conf_ipps_lib13_b200``) and neither
imports the other; the only shared module is ``aggen`` (seeded inputs).

Contents (each function cites the passage it follows):

* ``bfs``       — FIFO-queue BFS, ``agoracle.c:oracle_bfs`` (Fig. 4,
                  16.s24; 14.s19; 26.s21).
* ``dijkstra``  — binary-heap Dijkstra, ``agoracle.c:oracle_dijkstra``
                  (Fig. 5, 18.s28; 14.s20; 22.s10; 26.s36).
* ``cc``        — min-label connected components, ``agoracle.c:oracle_cc``
                  (label[v] = min{u : u reaches v}; PAPER.md:10.s9, 12.s13;
                  SURVEY.md §8(f) NEXT-4; R23).
* ``validate``  — shortest-path certificate.
* ``reached``   — V_r, E_r for the byte model.
* ``selector``  — Fig. 11 decision maker (24.s34-42), see ``oracle/selector.py``.
* derived unique quantities: ordered-BFS iteration count = ecc(src)+1 and
  per-level working-set sizes (16.s43, 26.s33); Delta=1 ordered-SSSP iteration
  count = number of distinct finite distances (28.s8, R9).

Pins (tests/test_oracle.py, -m "not gpu"): closed forms, brute force
(Floyd-Warshall, Bellman-Ford written in the tests), Fig. 7 CSR example,
edge/tightness invariants, symmetry and triangle inequalities, union-find
component sizes.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from . import selector  # noqa: F401  (re-export)

INF = 0xFFFFFFFF

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "agoracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile liboracle.so (gcc -O3, serial) if missing or stale."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-shared", "-fPIC", _SRC, "-o", tmp])
        os.replace(tmp, _LIB)
    return _LIB


def _L():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        vp, u32 = ctypes.c_void_p, ctypes.c_uint32
        _lib.oracle_bfs.argtypes = [u32, vp, vp, u32, vp, vp]
        _lib.oracle_dijkstra.argtypes = [u32, vp, vp, vp, u32, vp, vp]
        _lib.oracle_validate.argtypes = [u32, vp, vp, vp, u32, vp, vp, vp]
        _lib.oracle_reached.argtypes = [u32, vp, vp, vp, vp]
        _lib.oracle_reached.restype = None
        _lib.oracle_cc.argtypes = [u32, vp, vp, vp]
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data


def _chk(g):
    assert g.row_ptr.dtype == np.uint64 and g.col.dtype == np.uint32
    assert g.row_ptr.flags.c_contiguous and g.col.flags.c_contiguous


def bfs(g, src: int, want_parents: bool = True):
    """(level, parent) — uint32[V] each, INF = 0xFFFFFFFF for unreached."""
    _chk(g)
    level = np.empty(g.V, dtype=np.uint32)
    parent = np.empty(g.V, dtype=np.uint32) if want_parents else None
    rc = _L().oracle_bfs(g.V, _p(g.row_ptr), _p(g.col), int(src), _p(level), _p(parent))
    if rc != 0:
        raise ValueError(f"oracle_bfs rc={rc}")
    return level, parent


class OverflowError32(ArithmeticError):
    pass


def dijkstra(g, src: int, want_parents: bool = True):
    """(dist, parent) — uint32[V]; raises OverflowError32 if a finite distance > 0xFFFFFFFE."""
    _chk(g)
    assert g.w is not None and g.w.dtype == np.uint32
    dist = np.empty(g.V, dtype=np.uint32)
    parent = np.empty(g.V, dtype=np.uint32) if want_parents else None
    rc = _L().oracle_dijkstra(g.V, _p(g.row_ptr), _p(g.col), _p(g.w), int(src), _p(dist), _p(parent))
    if rc == 1:
        raise OverflowError32("finite distance exceeds 0xFFFFFFFE")
    if rc != 0:
        raise ValueError(f"oracle_dijkstra rc={rc}")
    return dist, parent


VALIDATE_MSG = {0: "ok", 1: "out[src] != 0", 2: "edge inequality violated", 3: "bad parent",
                4: "parent edge not tight", 5: "unreached vertex has a parent", 6: "parent[src] != src"}


def validate(g, src: int, out: np.ndarray, parent=None, weighted: bool = False):
    """Certificate check; returns (code, bad_vertex).  code 0 = valid."""
    _chk(g)
    out = np.ascontiguousarray(out, dtype=np.uint32)
    parent = None if parent is None else np.ascontiguousarray(parent, dtype=np.uint32)
    bad = ctypes.c_uint32(0)
    rc = _L().oracle_validate(g.V, _p(g.row_ptr), _p(g.col), _p(g.w) if weighted else None, int(src),
                              _p(out), _p(parent), ctypes.addressof(bad))
    return rc, bad.value


def cc(g):
    """label uint32[V]: label[v] = min{u : u reaches v along out-edges} (R23); on a
    symmetric graph the smallest vertex id of v's connected component."""
    _chk(g)
    label = np.empty(g.V, dtype=np.uint32)
    rc = _L().oracle_cc(g.V, _p(g.row_ptr), _p(g.col), _p(label))
    if rc != 0:
        raise ValueError(f"oracle_cc rc={rc}")
    return label


def reached(g, out: np.ndarray):
    """(V_r, E_r): reached vertices and CSR entries whose source is reached."""
    out = np.ascontiguousarray(out, dtype=np.uint32)
    a, b = ctypes.c_uint64(0), ctypes.c_uint64(0)
    _L().oracle_reached(g.V, _p(g.row_ptr), _p(out), ctypes.addressof(a), ctypes.addressof(b))
    return a.value, b.value


# --------------------------------------------------------------------------
# derived unique quantities (definitions written out)
# --------------------------------------------------------------------------
def bfs_level_sizes(level: np.ndarray) -> np.ndarray:
    """|WS| at each level-synchronous iteration: #{v : level[v] == L} for L = 0..ecc.
    Ordered BFS processes each node exactly once, level by level (16.s43, 18.s8);
    unordered GPU BFS proceeds level by level too (26.s33)."""
    fin = level[level != INF].astype(np.int64)
    return np.bincount(fin) if len(fin) else np.zeros(0, dtype=np.int64)


def bfs_iterations(level: np.ndarray) -> int:
    """ecc(src) + 1 (R11)."""
    return len(bfs_level_sizes(level))


def bfs_level_edges(g, level: np.ndarray) -> np.ndarray:
    """Sum of out-degrees of the vertices at each level (m_F of each iteration)."""
    fin = level != INF
    deg = np.diff(g.row_ptr).astype(np.int64)
    return np.bincount(level[fin].astype(np.int64), weights=deg[fin]).astype(np.int64) if fin.any() \
        else np.zeros(0, dtype=np.int64)


def ordered_sssp_iterations(dist: np.ndarray, delta: int = 1) -> int:
    """Delta=1 ordered SSSP settles all pending vertices at the current minimum
    distance per iteration (28.s8, R9): #distinct finite distances."""
    fin = dist[dist != INF]
    assert delta == 1
    return int(len(np.unique(fin)))
