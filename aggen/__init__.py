"""aggen — seeded synthetic graph inputs shared by the oracle and the CUDA path.

Holds none of the method's arithmetic (no traversal, no levels/distances, no
selector): only CSR construction.  The recipe of each workload is stated in
DESIGN.md §3 and SURVEY.md §8(d):

* ``rmat(scale, ef, seed)`` — Graph500 Kronecker A,B,C,D = .57,.19,.19,.05,
  keyed random relabelling, symmetrised, self-loops dropped, duplicates merged
  (configs C1 = scale 12, C2 = scale 22, C5 = scale 26; BASELINE.json configs).
* ``grid(W, H, keep)`` — 4-neighbour grid, row-major ids; ``keep < 1`` bond-
  percolates it (C3 = 4096x4096, C3' keep = 0.6 ~ CO-road's avg degree 2.4,
  PAPER.md:12.s38).
* ``er(n, m)`` — Erdos-Renyi G(n, m) with uniform endpoints (C4: n = 2^25, m = 4n).
* ``weights(g, seed, wmax)`` — symmetric integer weights in [1, wmax]
  (reading R7).
* tiny closed-form families and seeded random multigraphs for the tests.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "aggen.c")
_LIB = os.path.join(_HERE, "libaggen.so")


def build(force: bool = False) -> str:
    """Compile libaggen.so with gcc (-O3 -fopenmp) if missing or stale."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-march=x86-64-v2", "-fopenmp", "-shared", "-fPIC",
                               _SRC, "-o", tmp])
        os.replace(tmp, _LIB)
    return _LIB


class _CSR(ctypes.Structure):
    _fields_ = [("V", ctypes.c_uint32), ("E", ctypes.c_uint64),
                ("row_ptr", ctypes.POINTER(ctypes.c_uint64)), ("col", ctypes.POINTER(ctypes.c_uint32))]


_lib = None


def _L():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        u32, u64, i32 = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
        _lib.aggen_rmat.argtypes = [u32, u32, u64, u32, u32, u32, i32, ctypes.POINTER(_CSR)]
        _lib.aggen_er.argtypes = [u32, u64, u64, ctypes.POINTER(_CSR)]
        _lib.aggen_grid.argtypes = [u32, u32, u32, u64, ctypes.POINTER(_CSR)]
        _lib.aggen_weights.argtypes = [u32, ctypes.c_void_p, ctypes.c_void_p, u64, u32, ctypes.c_void_p]
        _lib.aggen_weights.restype = None
        _lib.aggen_sources.argtypes = [u32, ctypes.c_void_p, u64, u32, ctypes.c_void_p]
        _lib.aggen_free.argtypes = [ctypes.POINTER(_CSR)]
        _lib.aggen_free.restype = None
        _lib.aggen_set_owned.argtypes = [u32, u32]
        _lib.aggen_set_owned.restype = None
    return _lib


@dataclass
class Graph:
    """A CSR graph: out-edges of u are col[row_ptr[u]:row_ptr[u+1]] (PAPER.md:20.s16-29)."""
    V: int
    row_ptr: np.ndarray          # uint64[V+1]
    col: np.ndarray              # uint32[E]
    w: Optional[np.ndarray] = None  # uint32[E] or None
    name: str = ""

    @property
    def E(self) -> int:
        return int(self.row_ptr[-1])

    def degrees(self) -> np.ndarray:
        return np.diff(self.row_ptr).astype(np.int64)


def _take(c: _CSR, name: str) -> Graph:
    V, E = int(c.V), int(c.E)
    rp = np.ctypeslib.as_array(c.row_ptr, shape=(V + 1,)).copy()
    col = np.ctypeslib.as_array(c.col, shape=(max(E, 1),))[:E].copy()
    _L().aggen_free(ctypes.byref(c))
    return Graph(V, rp, col, None, name)


def rmat(scale: int, edgefactor: int = 16, seed: int = 1, a: float = 0.57, b: float = 0.19,
         c: float = 0.19, permute: bool = True) -> Graph:
    cs = _CSR()
    rc = _L().aggen_rmat(scale, edgefactor, seed, int(round(a * 1e6)), int(round(b * 1e6)),
                         int(round(c * 1e6)), int(permute), ctypes.byref(cs))
    if rc != 0:
        raise RuntimeError(f"aggen_rmat failed ({rc})")
    return _take(cs, f"rmat{scale}_ef{edgefactor}_s{seed}")


def rmat_part(scale: int, edgefactor: int, seed: int, own_b: int, own_e: int) -> Graph:
    """The CSR entries of rmat(scale, edgefactor, seed) whose DESTINATION is in [own_b, own_e) (rows over
    all V): exactly one rank's part of the 1-D destination partition, generated without the rest."""
    _L().aggen_set_owned(own_b, own_e)
    try:
        return rmat(scale, edgefactor, seed)
    finally:
        _L().aggen_set_owned(0, 0xFFFFFFFF)


def er(n: int, m: int, seed: int = 1) -> Graph:
    cs = _CSR()
    if _L().aggen_er(n, m, seed, ctypes.byref(cs)) != 0:
        raise RuntimeError("aggen_er failed")
    return _take(cs, f"er{n}_m{m}_s{seed}")


def grid(W: int, H: int, keep: float = 1.0, seed: int = 1) -> Graph:
    cs = _CSR()
    if _L().aggen_grid(W, H, min(1000000, int(round(keep * 1e6))), seed, ctypes.byref(cs)) != 0:
        raise RuntimeError("aggen_grid failed")
    return _take(cs, f"grid{W}x{H}_k{keep}_s{seed}")


def weights(g: Graph, seed: int = 2, wmax: int = 100) -> np.ndarray:
    """Symmetric weights 1 + splitmix64(seed ^ pack(min,max)) % wmax (R7).
    ``wmax == 0`` gives the constant weight ``seed`` (closed-form grid pins)."""
    w = np.empty(max(g.E, 1), dtype=np.uint32)
    _L().aggen_weights(g.V, g.row_ptr.ctypes.data, g.col.ctypes.data, seed, wmax, w.ctypes.data)
    return w[: g.E]


def with_weights(g: Graph, seed: int = 2, wmax: int = 100) -> Graph:
    g.w = weights(g, seed, wmax)
    return g


def sources(g: Graph, count: int, seed: int = 3) -> np.ndarray:
    """`count` seeded sources with out-degree >= 1."""
    out = np.zeros(count, dtype=np.uint32)
    got = _L().aggen_sources(g.V, g.row_ptr.ctypes.data, seed, count, out.ctypes.data)
    return out[:got]


# ---------------------------------------------------------------------------
# small graphs built in numpy (directed edge lists -> CSR)
# ---------------------------------------------------------------------------
def csr_from_edges(V: int, src, dst, w=None, symmetrize: bool = False, dedup: bool = False,
                   drop_self: bool = False, sort_rows: bool = True, name: str = "") -> Graph:
    src = np.asarray(src, dtype=np.int64)
    dst = np.asarray(dst, dtype=np.int64)
    wt = None if w is None else np.asarray(w, dtype=np.int64)
    if symmetrize:
        src, dst = np.concatenate([src, dst]), np.concatenate([dst, src])
        if wt is not None:
            wt = np.concatenate([wt, wt])
    if drop_self:
        keep = src != dst
        src, dst = src[keep], dst[keep]
        if wt is not None:
            wt = wt[keep]
    if sort_rows:
        order = np.lexsort((dst, src))
    else:
        order = np.argsort(src, kind="stable")
    src, dst = src[order], dst[order]
    if wt is not None:
        wt = wt[order]
    if dedup and len(src):
        keep = np.ones(len(src), dtype=bool)
        keep[1:] = (src[1:] != src[:-1]) | (dst[1:] != dst[:-1])
        src, dst = src[keep], dst[keep]
        if wt is not None:
            wt = wt[keep]
    counts = np.bincount(src, minlength=V) if len(src) else np.zeros(V, dtype=np.int64)
    rp = np.zeros(V + 1, dtype=np.uint64)
    rp[1:] = np.cumsum(counts)
    return Graph(V, rp, dst.astype(np.uint32), None if wt is None else wt.astype(np.uint32), name)


def path(n: int) -> Graph:
    i = np.arange(n - 1)
    return csr_from_edges(n, i, i + 1, symmetrize=True, name=f"path{n}")


def directed_cycle(n: int) -> Graph:
    i = np.arange(n)
    return csr_from_edges(n, i, (i + 1) % n, name=f"dcycle{n}")


def star(n: int) -> Graph:
    i = np.arange(1, n)
    return csr_from_edges(n, np.zeros(n - 1, dtype=np.int64), i, symmetrize=True, name=f"star{n}")


def complete(n: int) -> Graph:
    u, v = np.meshgrid(np.arange(n), np.arange(n), indexing="ij")
    m = u != v
    return csr_from_edges(n, u[m], v[m], name=f"K{n}")


def binary_tree(n: int) -> Graph:
    """Complete binary tree in heap order: children of i are 2i+1, 2i+2."""
    c = np.arange(1, n)
    return csr_from_edges(n, (c - 1) // 2, c, symmetrize=True, name=f"btree{n}")


def random_graph(V: int, M: int, seed: int, wmax: int = 100, directed: bool = True,
                 self_loops: bool = True, multi: bool = True, sort_rows: bool = True) -> Graph:
    """Seeded random (multi)graph with weights, for property tests on tiny inputs."""
    rng = np.random.default_rng(seed)
    src = rng.integers(0, V, size=M)
    dst = rng.integers(0, V, size=M)
    if not self_loops:
        keep = src != dst
        src, dst = src[keep], dst[keep]
    w = rng.integers(1, wmax + 1, size=len(src))
    g = csr_from_edges(V, src, dst, w, symmetrize=not directed, dedup=not multi,
                       sort_rows=sort_rows, name=f"rand{V}_{M}_s{seed}")
    return g


# ---------------------------------------------------------------------------
# BASELINE.json configs
# ---------------------------------------------------------------------------
def config(name: str, weighted: bool = True) -> Graph:
    """C1..C5 recipes.  Seeds: graph 1, weights 2 (sources use seed 3)."""
    if name == "C1":
        g = rmat(12, 16, seed=1)
    elif name == "C2":
        g = rmat(22, 16, seed=1)
    elif name == "C3":
        g = grid(4096, 4096, 1.0, seed=1)
    elif name == "C3p":
        g = grid(4096, 4096, 0.6, seed=1)
    elif name == "C4":
        g = er(1 << 25, 4 << 25, seed=1)
    elif name == "C5":
        g = rmat(26, 16, seed=1)
    elif name.startswith("rmat"):
        g = rmat(int(name[4:]), 16, seed=1)
    elif name.startswith("path"):     # per-iteration latency floor (one vertex per level)
        g = path(int(name[4:]))
    else:
        raise KeyError(name)
    g.name = name
    if weighted:
        with_weights(g, seed=2, wmax=100)
    return g
