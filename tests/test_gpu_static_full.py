"""Every static variant at full size (-m gpu): the paper's X4/X5 static study (PAPER.md:26.s20-25)
times each (order x mapping x working set) variant on each graph, and DESIGN.md §8b's static-vs-
adaptive table does the same on B200 — so each of those runs is result-checked here, element by
element against the oracle, on the full-size configs (one source each) before any time is trusted.

Covered per config: BFS {ordered, unordered} x {T, W, B, H} x {bitmap, queue} + both adaptive
policies; unordered SSSP over the same 8 (mapping x working set) variants + both adaptive policies;
ordered SSSP over the same variants at delta = 1 (the paper's Dijkstra batches, 28.s8) and at the
bucket width delta = 64.  Levels / distances bit-exact; parents by the certificate validator.
"""
import pytest

import aggen
import oracle

from . import test_gpu_parity as P
from .test_gpu_parity import MAPS, WSS, check_bfs, check_sssp, pol

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

_CACHE = {}


@pytest.fixture(scope="module", autouse=True)
def _lib():
    from paper_conf_ipps_lib13_b200 import agraph, build
    build.build()
    P.A = agraph
    yield


def _setup(cfg):
    if cfg not in _CACHE:
        from paper_conf_ipps_lib13_b200 import agraph as A
        g = aggen.config(cfg)
        G = A.Graph.from_csr(g)
        s = int(aggen.sources(g, 1, seed=17)[0])
        lv = oracle.bfs(g, s, want_parents=False)[0]
        d = oracle.dijkstra(g, s, want_parents=False)[0]
        _CACHE.clear()
        _CACHE[cfg] = (g, G, s, lv, d)
    return _CACHE[cfg]


def _variants(order, **kw):
    out = [pol(order, m, w, **kw) for m in MAPS for w in WSS]
    out += [pol(order, 0, 0, kind=0, **kw), pol(order, 0, 0, kind=1, **kw)]
    return out


@pytest.mark.parametrize("cfg", ["C2", "C3p", "C4"])
@pytest.mark.parametrize("order", [0, 1])
def test_full_size_bfs_every_variant(cfg, order):
    g, G, s, lv, _ = _setup(cfg)
    for p in _variants(order):
        check_bfs(g, G, s, p, expect_level=lv)


@pytest.mark.parametrize("cfg", ["C2", "C3p", "C4"])
def test_full_size_unordered_sssp_every_variant(cfg):
    g, G, s, _, d = _setup(cfg)
    for p in _variants(0):
        check_sssp(g, G, s, p, expect_dist=d)


@pytest.mark.parametrize("cfg", ["C2", "C3p", "C4"])
@pytest.mark.parametrize("delta", [1, 64])
def test_full_size_ordered_sssp_every_variant(cfg, delta):
    g, G, s, _, d = _setup(cfg)
    for p in _variants(1, delta=delta):
        check_sssp(g, G, s, p, expect_dist=d)
