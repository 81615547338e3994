"""Input generators: shape and determinism of the synthetic workloads."""
import os
import subprocess
import sys

import numpy as np

import aggen


def _check_simple_symmetric(g):
    deg = np.diff(g.row_ptr).astype(np.int64)
    src = np.repeat(np.arange(g.V), deg)
    assert np.all(g.col < g.V)
    assert not np.any(src == g.col)                          # no self loops (R6)
    # rows strictly ascending => sorted and deduplicated
    same_row = src[1:] == src[:-1]
    assert np.all(g.col[1:][same_row] > g.col[:-1][same_row])
    key = src * g.V + g.col.astype(np.int64)
    rkey = g.col.astype(np.int64) * g.V + src
    assert np.array_equal(np.sort(key), np.sort(rkey))      # symmetric (R5)


def test_rmat_shape_and_determinism():
    g = aggen.rmat(12, 16, seed=1)
    _check_simple_symmetric(g)
    assert g.V == 4096 and 90_000 < g.E < 100_000            # 96,444 for their RNG
    iso = float(np.mean(np.diff(g.row_ptr) == 0))
    assert 0.12 < iso < 0.25                                 # ~18% isolated
    g2 = aggen.rmat(12, 16, seed=1)
    assert np.array_equal(g.row_ptr, g2.row_ptr) and np.array_equal(g.col, g2.col)
    g3 = aggen.rmat(12, 16, seed=2)
    assert not np.array_equal(g.col[:1000], g3.col[:1000])


def test_rmat_thread_count_independent():
    code = ("import aggen,hashlib;g=aggen.rmat(11,16,seed=5);"
            "print(hashlib.sha256(g.row_ptr.tobytes()+g.col.tobytes()).hexdigest())")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    outs = []
    for t in ("1", "3"):
        env = dict(os.environ, OMP_NUM_THREADS=t, PYTHONPATH=root)
        outs.append(subprocess.check_output([sys.executable, "-c", code], env=env, cwd=root).strip())
    assert outs[0] == outs[1]


def test_grid_and_percolation():
    g = aggen.grid(64, 32)
    _check_simple_symmetric(g)
    assert g.E == 2 * (32 * 63 + 31 * 64)
    p = aggen.grid(256, 256, keep=0.6, seed=3)
    _check_simple_symmetric(p)
    full = 2 * 2 * 256 * 255 / 65536                      # avg degree of the unpercolated 256^2 grid
    assert abs(p.E / p.V - 0.6 * full) < 0.05             # ~2.4 = CO-road (PAPER.md:12.s38)
    assert np.diff(p.row_ptr).max() <= 4


def test_er_shape():
    g = aggen.er(1 << 14, 4 << 14, seed=1)
    _check_simple_symmetric(g)
    assert 7.8 < g.E / g.V <= 8.0


def test_weights_symmetric_and_range():
    g = aggen.rmat(10, 16, seed=1)
    w = aggen.weights(g, seed=2, wmax=100)
    assert w.min() >= 1 and w.max() <= 100
    deg = np.diff(g.row_ptr).astype(np.int64)
    src = np.repeat(np.arange(g.V), deg)
    d = dict(zip(zip(src.tolist(), g.col.tolist()), w.tolist()))
    assert all(d[(v, u)] == wt for (u, v), wt in d.items())
    c = aggen.weights(g, seed=9, wmax=0)
    assert np.all(c == 9)


def test_sources_have_edges():
    g = aggen.rmat(12, 16, seed=1)
    s = aggen.sources(g, 64, seed=3)
    assert len(s) == 64 and np.all(np.diff(g.row_ptr)[s] > 0)
