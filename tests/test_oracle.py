"""Pins of the CPU oracle against what the paper and mathematics fix (-m "not gpu").

Each test names the pin: closed forms, brute force, paper worked example
(Fig. 7), literal transcriptions of Fig. 4/5, invariants, symmetry.
"""
import os

import numpy as np
import pytest

import aggen
import oracle
from oracle import selector
from tests import bruteforce as bf

INF = oracle.INF
GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _read_fig7():
    d = {}
    for line in open(os.path.join(GOLD, "fig7_csr.txt")):
        if line.startswith("#") or not line.strip():
            continue
        k, *vals = line.split()
        d[k] = [int(x) for x in vals]
    V = d["V"][0]
    return aggen.Graph(V, np.array(d["node"], dtype=np.uint64), np.array(d["edge"], dtype=np.uint32))


# ---------------------------------------------------------------- Fig. 7
def test_fig7_csr_worked_example():
    """PAPER.md:20.s24-29: neighbours of node 2 are edge[node[2]:node[3]] = edge[4:6] = {22, 38}."""
    g = _read_fig7()
    assert len(g.row_ptr) == g.V + 1                       # "extra element" (20.s29)
    assert (int(g.row_ptr[2]), int(g.row_ptr[3])) == (4, 6)
    assert list(g.col[4:6]) == [22, 38]
    level, parent = oracle.bfs(g, 2)
    assert set(np.nonzero(level == 1)[0].tolist()) == {22, 38}
    assert parent[22] == 2 and parent[38] == 2 and level[2] == 0


# ---------------------------------------------------------------- closed forms
@pytest.mark.parametrize("n,src", [(1, 0), (2, 1), (17, 0), (17, 9), (1000, 999)])
def test_path_closed_form(n, src):
    g = aggen.path(n)
    level, _ = oracle.bfs(g, src)
    assert np.array_equal(level, np.abs(np.arange(n) - src).astype(np.uint32))


@pytest.mark.parametrize("n,src", [(5, 0), (64, 13)])
def test_directed_cycle_closed_form(n, src):
    g = aggen.directed_cycle(n)
    level, _ = oracle.bfs(g, src)
    assert np.array_equal(level, ((np.arange(n) - src) % n).astype(np.uint32))


def test_star_closed_form():
    g = aggen.star(50)
    level, _ = oracle.bfs(g, 0)
    assert level[0] == 0 and np.all(level[1:] == 1)
    level, _ = oracle.bfs(g, 7)
    exp = np.full(50, 2, dtype=np.uint32)
    exp[0], exp[7] = 1, 0
    assert np.array_equal(level, exp)


def test_complete_and_tree_closed_form():
    g = aggen.complete(12)
    level, _ = oracle.bfs(g, 5)
    exp = np.ones(12, dtype=np.uint32)
    exp[5] = 0
    assert np.array_equal(level, exp)
    n = 1023
    g = aggen.binary_tree(n)
    level, _ = oracle.bfs(g, 0)
    assert np.array_equal(level, np.floor(np.log2(np.arange(n) + 1)).astype(np.uint32))


@pytest.mark.parametrize("W,H,sx,sy", [(1, 1, 0, 0), (7, 5, 0, 0), (64, 48, 63, 47), (33, 40, 10, 22)])
def test_grid_manhattan(W, H, sx, sy):
    """4-neighbour grid: level = |x - sx| + |y - sy|; constant weight c: c * that."""
    g = aggen.grid(W, H)
    y, x = np.divmod(np.arange(W * H), W)
    man = (np.abs(x - sx) + np.abs(y - sy)).astype(np.uint32)
    level, _ = oracle.bfs(g, sy * W + sx)
    assert np.array_equal(level, man)
    g.w = aggen.weights(g, seed=7, wmax=0)  # constant weight 7
    dist, _ = oracle.dijkstra(g, sy * W + sx)
    assert np.array_equal(dist, 7 * man)


def test_weighted_path_prefix_sums():
    g = aggen.path(200)
    aggen.with_weights(g, seed=5, wmax=100)
    dist, _ = oracle.dijkstra(g, 0)
    # path edges i<->i+1: weight of (i, i+1) is the entry in row i pointing to i+1
    step = [int(g.w[e]) for i in range(199) for e in range(int(g.row_ptr[i]), int(g.row_ptr[i + 1]))
            if g.col[e] == i + 1]
    assert np.array_equal(dist, np.concatenate([[0], np.cumsum(step)]).astype(np.uint32))


def test_disconnected_is_inf():
    g = aggen.csr_from_edges(6, [0, 1, 3], [1, 2, 4], w=[5, 5, 5], symmetrize=True)
    level, parent = oracle.bfs(g, 0)
    assert list(level) == [0, 1, 2, INF, INF, INF]
    assert parent[3] == INF and parent[5] == INF and parent[0] == 0
    dist, _ = oracle.dijkstra(g, 3)
    assert list(dist) == [INF, INF, INF, 0, 5, INF]


def test_unit_weight_sssp_equals_bfs():
    g = aggen.rmat(10, 8, seed=4)
    g.w = aggen.weights(g, seed=1, wmax=0)  # all ones
    for s in aggen.sources(g, 4):
        level, _ = oracle.bfs(g, s)
        dist, _ = oracle.dijkstra(g, s)
        assert np.array_equal(level, dist)


# ---------------------------------------------------------------- brute force
@pytest.mark.parametrize("seed", range(12))
def test_bruteforce_floyd_warshall(seed):
    """Directed multigraphs with self-loops and isolated vertices vs Floyd-Warshall."""
    rng = np.random.default_rng(seed)
    V = int(rng.integers(1, 60))
    M = int(rng.integers(0, 4 * V))
    g = aggen.random_graph(V, M, seed=seed, wmax=int(rng.integers(1, 100)), sort_rows=bool(seed % 2))
    D = bf.floyd_warshall(g, weighted=True)
    Du = bf.floyd_warshall(g, weighted=False)
    for s in range(min(V, 6)):
        dist, par = oracle.dijkstra(g, s)
        assert np.array_equal(dist, bf.to_u32(D[s]))
        level, lpar = oracle.bfs(g, s)
        assert np.array_equal(level, bf.to_u32(Du[s]))
        assert oracle.validate(g, s, dist, par, weighted=True)[0] == 0
        assert oracle.validate(g, s, level, lpar, weighted=False)[0] == 0


def test_bruteforce_bellman_ford_c1():
    """Config C1 (R-MAT s12 ef16, weights 1..100) vs synchronous Bellman-Ford."""
    g = aggen.config("C1")
    for s in aggen.sources(g, 4):
        dist, _ = oracle.dijkstra(g, s)
        bfd, _ = bf.bellman_ford(g, s, weighted=True)
        assert np.array_equal(dist, bfd)
        level, _ = oracle.bfs(g, s)
        bfl, rounds = bf.bellman_ford(g, s, weighted=False)
        assert np.array_equal(level, bfl)
        assert oracle.bfs_iterations(level) == rounds  # ecc rounds to settle + 1 confirming round


@pytest.mark.parametrize("seed", range(6))
def test_literal_fig4_fig5(seed):
    """Oracle == literal Fig. 4 / Fig. 5 transcriptions, ordered and unordered."""
    g = aggen.random_graph(80, 300, seed=100 + seed, wmax=20)
    for s in (0, 17, 79):
        level, _ = oracle.bfs(g, s)
        assert np.array_equal(level, bf.fig4_bfs(g, s, ordered=True))
        assert np.array_equal(level, bf.fig4_bfs(g, s, ordered=False))
        dist, _ = oracle.dijkstra(g, s)
        d_o, iters = bf.fig5_sssp(g, s, ordered=True)
        d_u, _ = bf.fig5_sssp(g, s, ordered=False)
        assert np.array_equal(dist, d_o) and np.array_equal(dist, d_u)
        assert oracle.ordered_sssp_iterations(dist) == iters


# ---------------------------------------------------------------- invariants
def test_invariants_and_symmetry_c1():
    g = aggen.config("C1")
    srcs = aggen.sources(g, 3)
    comp = bf.components(g)
    comp_e = bf.component_edge_entries(g)
    D = {}
    for s in srcs:
        dist, par = oracle.dijkstra(g, s)
        level, lpar = oracle.bfs(g, s)
        assert oracle.validate(g, s, dist, par, weighted=True)[0] == 0
        assert oracle.validate(g, s, level, lpar)[0] == 0
        Vr, Er = oracle.reached(g, dist)
        assert Vr == comp[s]                       # union-find component size
        assert Er == comp_e[s]                     # edge-list entries leaving s's union-find component
        assert np.array_equal(level != INF, dist != INF)
        D[int(s)] = dist.astype(np.int64)
    a, b, c = [int(x) for x in srcs]
    assert D[a][b] == D[b][a] and D[a][c] == D[c][a]  # symmetric weights, symmetric graph
    fin = (D[a] != INF) & (D[b] != INF)
    assert np.all(np.abs(D[a][fin] - D[b][fin]) <= D[a][b])  # triangle inequality


def test_validator_rejects_corruption():
    g = aggen.config("C1")
    s = int(aggen.sources(g, 1)[0])
    dist, par = oracle.dijkstra(g, s)
    v = int(np.nonzero((dist != INF) & (np.arange(g.V) != s))[0][5])
    bad = dist.copy(); bad[v] += 1
    assert oracle.validate(g, s, bad, par, weighted=True)[0] in (2, 4)
    bad = dist.copy(); bad[v] -= 1
    assert oracle.validate(g, s, bad, par, weighted=True)[0] in (2, 4)
    bp = par.copy(); bp[v] = v
    assert oracle.validate(g, s, dist, bp, weighted=True)[0] in (3, 4)
    bad = dist.copy(); bad[s] = 1
    assert oracle.validate(g, s, bad, par, weighted=True)[0] == 1


def test_validator_rejects_parent_corruption_codes_5_and_6():
    """Certificate rule 4: an unreached vertex must have parent INF (code 5) and the
    source must be its own parent (code 6, Graph500 convention) — each corruption alone is rejected
    with its own code, and the uncorrupted certificate passes."""
    g = aggen.csr_from_edges(6, [0, 1, 1, 3], [1, 0, 2, 4], w=[2, 2, 5, 1])   # 3 -> 4 and 5 unreachable from 0
    for weighted in (False, True):
        out, par = (oracle.dijkstra(g, 0) if weighted else oracle.bfs(g, 0))
        assert list(out[[3, 4, 5]]) == [INF] * 3 and oracle.validate(g, 0, out, par, weighted)[0] == 0
        bp = par.copy(); bp[4] = 3                    # unreached vertex 4 claims the real edge (3, 4)
        assert oracle.validate(g, 0, out, bp, weighted) == (5, 4)
        bp = par.copy(); bp[5] = 0
        assert oracle.validate(g, 0, out, bp, weighted) == (5, 5)
        bp = par.copy(); bp[0] = 1                    # the source's parent is not itself
        assert oracle.validate(g, 0, out, bp, weighted) == (6, 0)
        bp = par.copy(); bp[0] = INF
        assert oracle.validate(g, 0, out, bp, weighted) == (6, 0)


def test_bfs_level_sizes_definition():
    g = aggen.binary_tree(127)
    level, _ = oracle.bfs(g, 0)
    assert list(oracle.bfs_level_sizes(level)) == [1, 2, 4, 8, 16, 32, 64]
    assert oracle.bfs_iterations(level) == 7
    assert list(oracle.bfs_level_edges(g, level)) == [2, 6, 12, 24, 48, 96, 64]


def test_overflow_detected():
    g = aggen.path(4)
    g.w = np.full(g.E, 0x7FFFFFFF, dtype=np.uint32)
    g3 = aggen.path(3)
    g3.w = np.full(g3.E, 0x7FFFFFFF, dtype=np.uint32)
    dist, _ = oracle.dijkstra(g3, 0)
    assert dist[2] == 0xFFFFFFFE                 # largest finite value is representable
    with pytest.raises(oracle.OverflowError32):  # 3 * (2^31 - 1) > 0xFFFFFFFE
        oracle.dijkstra(g, 0)


# ---------------------------------------------------------------- selector (Fig. 11)
def test_fig11_truth_table():
    rows = [l.split() for l in open(os.path.join(GOLD, "fig11_regions.txt"))
            if l.strip() and not l.startswith("#")]
    assert len(rows) >= 10
    for ws, V, E, m, w in rows:
        assert selector.paper_select(int(ws), int(V), int(E), T1=32, T2=2688, T3=10000) == (m, w), (ws, V, E)


def test_selector_paper_constants():
    assert selector.t2_default(192, 14) == 2688          # 28.s27
    assert selector.t3_from_ppm(100, 10000) == 1 and selector.t3_from_ppm(1000, 130000) == 130
    # block size = multiple of 32 closest to average out-degree (26.s28)
    assert selector.block_size(434102, 2 * 16036720) == 64   # CiteSeer avg 73.9 (12.s38) -> 64
    assert selector.block_size(100, 4800) == 64          # avg 48: tie between 32/64 -> up
    assert selector.block_size(100, 100) == 32 and selector.block_size(1, 10**6) == 1024


# ---------------------------------------------------------------- min-label CC (NEXT-4)
def test_cc_closed_forms():
    """label[v] = min{u : u reaches v} (R23): closed forms."""
    assert np.array_equal(oracle.cc(aggen.path(17)), np.zeros(17, np.uint32))
    assert np.array_equal(oracle.cc(aggen.directed_cycle(9)), np.zeros(9, np.uint32))
    assert np.array_equal(oracle.cc(aggen.star(30)), np.zeros(30, np.uint32))
    fwd = aggen.csr_from_edges(4, [0, 1, 2], [1, 2, 3])            # 0 -> 1 -> 2 -> 3
    assert list(oracle.cc(fwd)) == [0, 0, 0, 0]
    bwd = aggen.csr_from_edges(4, [3, 2, 1], [2, 1, 0])            # 3 -> 2 -> 1 -> 0
    assert list(oracle.cc(bwd)) == [0, 1, 2, 3]
    dis = aggen.csr_from_edges(7, [0, 1, 4, 6], [1, 2, 3, 5], symmetrize=True)
    assert list(oracle.cc(dis)) == [0, 0, 0, 3, 3, 5, 5]
    loops = aggen.csr_from_edges(3, [1, 1, 2], [1, 1, 2])          # self-loops only
    assert list(oracle.cc(loops)) == [0, 1, 2]


@pytest.mark.parametrize("seed", range(10))
def test_cc_bruteforce_reachability(seed):
    """Directed multigraphs with self-loops and isolated vertices vs the transitive closure."""
    rng = np.random.default_rng(500 + seed)
    V = int(rng.integers(1, 70))
    M = int(rng.integers(0, 3 * V))
    g = aggen.random_graph(V, M, seed=500 + seed, wmax=5, sort_rows=bool(seed % 2))
    lab = oracle.cc(g)
    assert np.array_equal(lab, bf.reach_min_label(g))
    assert np.array_equal(lab, bf.jacobi_min_label(g)[0])


def test_cc_c1_components():
    """C1 (symmetric): labels == union-find set minima; one label per component; sizes agree."""
    g = aggen.config("C1", weighted=False)
    lab = oracle.cc(g)
    assert np.array_equal(lab, bf.uf_min_label(g))
    assert np.array_equal(lab, bf.jacobi_min_label(g)[0])
    assert np.all(lab <= np.arange(g.V))                     # a vertex reaches itself
    assert np.all(lab[lab] == lab)                           # a label is its own label
    sizes = np.bincount(lab, minlength=g.V)[lab]
    assert np.array_equal(sizes, bf.components(g))
