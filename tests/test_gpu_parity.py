"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, bit-exact (-m gpu).

Levels and distances are unique and compared element by element (memcmp); parents are
legitimately nondeterministic and are checked with the oracle's certificate validator
(SURVEY.md §8(c)).  Every variant of the three axes is exercised: {ordered, unordered} x
{thread, warp, CTA, hybrid} x {bitmap, queue}, plus the adaptive selector (paper and tuned).
"""
import numpy as np
import pytest

import aggen
import oracle
from oracle import selector

pytestmark = pytest.mark.gpu

A = None


@pytest.fixture(scope="module", autouse=True)
def _lib():
    global A
    from paper_conf_ipps_lib13_b200 import agraph, build
    build.build()
    A = agraph
    yield


INF = oracle.INF
MAPS = [1, 2, 3, 4]            # T, W, B(CTA), H
WSS = [1, 2]                   # BM, QU


def pol(order=0, mapping=0, workset=0, kind=1, **kw):
    p = A.policy_default(0)
    p.order, p.mapping, p.workset, p.kind = order, mapping, workset, kind
    for k, v in kw.items():
        setattr(p, k, v)
    return p


def all_policies():
    out = []
    for order in (0, 1):
        for m in MAPS:
            for w in WSS:
                out.append(pol(order, m, w))
        out.append(pol(order, 0, 0, kind=0))   # paper adaptive
        out.append(pol(order, 0, 0, kind=1))   # tuned adaptive
    return out


def pname(p):
    return f"{'O' if p.order else 'U'}_{'auto' if not p.mapping else A.MAP_LETTER[p.mapping]}_" \
           f"{'auto' if not p.workset else A.WS_NAME[p.workset]}_{'paper' if p.kind == 0 else 'tuned'}"


def check_bfs(g, G, s, p, expect_level=None, want_parents=True):
    lv, par = oracle.bfs(g, s) if expect_level is None else (expect_level, None)
    parents = np.empty(g.V, np.uint32) if want_parents else None
    out, _, st = G.bfs(s, parents=parents, policy=p, stats=True, trace_cap=1 << 16)
    assert np.array_equal(out, lv), f"BFS levels differ ({pname(p)}, src {s}): " \
        f"{np.count_nonzero(out != lv)} mismatches"
    if want_parents:
        code, bad = oracle.validate(g, s, out, parents, weighted=False)
        assert code == 0, f"BFS parent certificate failed: {oracle.VALIDATE_MSG[code]} at {bad} ({pname(p)})"
    Vr, Er = oracle.reached(g, lv)
    assert (st.reached, st.reached_edges) == (Vr, Er)
    # level-synchronous: ordered AND unordered BFS expand each reached vertex exactly once (16.s43, 26.s33)
    assert st.vertices_expanded == Vr and st.edges_inspected == Er
    assert st.iterations == oracle.bfs_iterations(lv)
    assert list(st.trace_ws) == list(oracle.bfs_level_sizes(lv))
    assert list(st.trace_edges) == list(oracle.bfs_level_edges(g, lv))
    return st


def check_sssp(g, G, s, p, expect_dist=None):
    d = oracle.dijkstra(g, s, want_parents=False)[0] if expect_dist is None else expect_dist
    parents = np.empty(g.V, np.uint32)
    out, _, st = G.sssp(s, parents=parents, policy=p, stats=True)
    assert np.array_equal(out, d), f"SSSP dist differ ({pname(p)}, src {s}): {np.count_nonzero(out != d)} mismatches"
    code, bad = oracle.validate(g, s, out, parents, weighted=True)
    assert code == 0, f"SSSP parent certificate failed: {oracle.VALIDATE_MSG[code]} at {bad} ({pname(p)})"
    Vr, Er = oracle.reached(g, d)
    assert (st.reached, st.reached_edges) == (Vr, Er)
    if p.order == 1 and p.delta == 1:
        # Dijkstra batches: each vertex settled exactly once (18.s2); one iteration per distinct distance (28.s8)
        assert st.vertices_expanded == Vr and st.edges_inspected == Er
        assert st.iterations == oracle.ordered_sssp_iterations(d)
    else:
        assert st.vertices_expanded >= Vr and st.edges_inspected >= Er
    # no parents requested: the tuned kernels keep the distance-only u32 state instead of the packed word
    out2, _, st2 = G.sssp(s, policy=p, stats=True)
    assert np.array_equal(out2, d), f"SSSP dist (no parents) differ ({pname(p)}, src {s}): " \
        f"{np.count_nonzero(out2 != d)} mismatches"
    assert (st2.reached, st2.reached_edges) == (Vr, Er)
    return st


# ------------------------------------------------------------------------------------------------
@pytest.mark.parametrize("layout", [0, 2])
@pytest.mark.parametrize("seed", range(8))
def test_tiny_random_all_variants(seed, layout):
    rng = np.random.default_rng(seed)
    V = int(rng.integers(1, 300))
    g = aggen.random_graph(V, int(rng.integers(0, 6 * V + 1)), seed=seed, wmax=int(rng.integers(1, 100)),
                           sort_rows=bool(seed % 2))
    G = A.Graph.from_csr(g, layout=layout)
    assert G.info.layout in (1, 2) and (layout == 0 or G.info.layout == layout)
    srcs = sorted(set([0, V - 1, int(rng.integers(0, V))]))
    for p in all_policies():
        for s in srcs:
            check_bfs(g, G, s, p)
            check_sssp(g, G, s, p)


@pytest.mark.parametrize("window", [0, 1, 7, 50, 300, 0xFFFFFFFF])
def test_unordered_sssp_window(window):
    """The deferral window reorders unordered SSSP but never changes the distances."""
    for g in (aggen.config("C1"), aggen.with_weights(aggen.grid(60, 50), seed=9, wmax=100),
              aggen.with_weights(aggen.er(5000, 20000, seed=4), seed=5, wmax=100)):
        G = A.Graph.from_csr(g)
        for s in aggen.sources(g, 2):
            for m in (0, 1, 4):
                check_sssp(g, G, s, pol(0, m, 2 if m else 0, sssp_window=window))
                check_sssp(g, G, s, pol(0, m, 2 if m else 0, sssp_window=window, sssp_hub_window=1 + window % 5))


@pytest.mark.parametrize("free_ppm", [0, 1, 3906, 250000, 1000000])
def test_free_output_threshold(free_ppm):
    """Free-output iterations (raw next bitmap by fire-and-forget reductions, compacted by the next
    iteration) at every threshold: never, always, the default, and in between."""
    graphs = [aggen.config("C1"), aggen.with_weights(aggen.grid(60, 50), seed=9, wmax=100),
              aggen.with_weights(aggen.er(5000, 20000, seed=4), seed=5, wmax=100),
              aggen.with_weights(aggen.star(20000)), aggen.random_graph(300, 1500, seed=3)]
    for g in graphs:
        for layout in (0, 1):
            G = A.Graph.from_csr(g, layout=layout)
            for s in sorted(set(int(x) for x in aggen.sources(g, 2)) | {0}):
                for order in (0, 1):
                    check_bfs(g, G, s, pol(order, free_ppm=free_ppm), want_parents=False)
                    check_bfs(g, G, s, pol(order, free_ppm=free_ppm))
                check_sssp(g, G, s, pol(0, free_ppm=free_ppm))
                check_sssp(g, G, s, pol(0, free_ppm=free_ppm, sssp_window=0, sssp_hub_window=0))


@pytest.mark.parametrize("delta", [1, 7, 100, 1000])
def test_ordered_sssp_delta(delta):
    g = aggen.config("C1")
    G = A.Graph.from_csr(g)
    for s in aggen.sources(g, 3):
        for w in WSS:
            check_sssp(g, G, s, pol(1, 4, w, delta=delta))
            check_sssp(g, G, s, pol(1, 1, w, delta=delta))


def test_c1_all_sources_adaptive():
    """C1 (R-MAT s12 ef16): all 64 sources, BFS + SSSP, adaptive tuned and paper policies."""
    g = aggen.config("C1")
    G = A.Graph.from_csr(g)
    for s in aggen.sources(g, 64):
        for kind in (0, 1):
            check_bfs(g, G, s, pol(0, kind=kind))
            check_sssp(g, G, s, pol(0, kind=kind))


@pytest.mark.parametrize("layout", [1, 2])
def test_c1_all_static_variants(layout):
    g = aggen.config("C1")
    G = A.Graph.from_csr(g, layout=layout)
    for s in aggen.sources(g, 4, seed=11):
        for p in all_policies():
            check_bfs(g, G, s, p)
            check_sssp(g, G, s, p)


def test_paper_policy_trace_matches_fig11():
    """The per-iteration variant chosen on device == Fig. 11 applied to the oracle's level sizes."""
    g = aggen.rmat(16, 16, seed=1)
    G = A.Graph.from_csr(g, weighted=False)
    p = pol(0, kind=0)
    T3 = selector.t3_from_ppm(g.V, p.t3_ppm)
    for s in aggen.sources(g, 3):
        st = check_bfs(g, G, s, p)
        lv, _ = oracle.bfs(g, s)
        exp = [selector.paper_select(int(n), g.V, g.E, T1=p.t1_avg_degree, T2=p.t2_ws, T3=T3)
               for n in oracle.bfs_level_sizes(lv)]
        got = [tuple(A.variant_name(int(v)).split("_")) for v in st.trace_variant]
        assert got == exp


def test_closed_form_grid_and_path():
    W, H = 300, 200
    g = aggen.grid(W, H)
    g.w = aggen.weights(g, seed=3, wmax=0)
    G = A.Graph.from_csr(g)
    y, x = np.divmod(np.arange(W * H), W)
    for sx, sy in [(0, 0), (299, 199), (123, 45)]:
        man = (np.abs(x - sx) + np.abs(y - sy)).astype(np.uint32)
        for p in (pol(0), pol(1), pol(0, 1, 2), pol(0, 1, 1)):
            out, _, _ = G.bfs(sy * W + sx, policy=p)
            assert np.array_equal(out, man)
            out, _, _ = G.sssp(sy * W + sx, policy=p)
            assert np.array_equal(out, 3 * man)
    g = aggen.path(5000)
    G = A.Graph.from_csr(g, weighted=False)
    out, _, st = G.bfs(17, policy=pol(0), stats=True)
    assert np.array_equal(out, np.abs(np.arange(5000) - 17).astype(np.uint32)) and st.iterations == 4983


@pytest.mark.parametrize("layout", [1, 2])
def test_hubs_and_star(layout):
    """Degree >> HUB_DEG exercises hub splitting (hybrid) and long CTA loops (paper variants)."""
    n = 300_000
    g = aggen.star(n)
    aggen.with_weights(g, seed=4, wmax=100)
    G = A.Graph.from_csr(g, layout=layout)
    for p in [pol(0), pol(1), pol(0, 4, 2), pol(0, 4, 1), pol(0, 1, 2), pol(0, 3, 1), pol(1, 4, 2)]:
        for s in (0, 5):
            check_bfs(g, G, s, p)
            check_sssp(g, G, s, p)


def test_edge_cases_and_errors():
    g1 = aggen.csr_from_edges(1, [], [], w=[])
    G = A.Graph.from_csr(g1)
    out, _, st = G.bfs(0, stats=True)
    assert list(out) == [0] and st.iterations == 1
    out, par, _ = G.sssp(0, parents=np.empty(1, np.uint32))
    assert list(out) == [0] and list(par) == [0]
    with pytest.raises(A.AgError) as e:
        G.bfs(1)
    assert e.value.status == "AG_ERR_SRC_RANGE"
    # isolated source
    g = aggen.csr_from_edges(5, [1, 2], [2, 3], w=[1, 1])
    G = A.Graph.from_csr(g)
    out, par, _ = G.bfs(0, parents=np.empty(5, np.uint32))
    assert list(out) == [0, INF, INF, INF, INF] and list(par) == [0, INF, INF, INF, INF]
    # SSSP without weights
    Gu = A.Graph.from_csr(g, weighted=False)
    with pytest.raises(A.AgError) as e:
        Gu.sssp(0)
    assert e.value.status == "AG_ERR_NO_WEIGHTS"
    # bad CSR
    for rp, col, w in [([1, 1, 2], [0, 1], None), ([0, 2, 1], [0, 1], None), ([0, 1, 2], [0, 5], None),
                       ([0, 1, 2], [0, 1], [1, 0]), ([0, 1, 2], [0, 1], [1, 1 << 31])]:
        with pytest.raises(A.AgError) as e:
            A.Graph(2, np.array(rp, np.uint64), np.array(col, np.uint32), None if w is None else np.array(w, np.uint32))
        assert e.value.status == "AG_ERR_BAD_CSR"
    # overflow: path with huge weights
    g = aggen.path(4)
    g.w = np.full(g.E, 0x7FFFFFFF, np.uint32)
    G = A.Graph.from_csr(g)
    for order in (0, 1):
        with pytest.raises(A.AgError) as e:
            G.sssp(0, policy=pol(order))
        assert e.value.status == "AG_ERR_OVERFLOW"
    g3 = aggen.path(3)
    g3.w = np.full(g3.E, 0x7FFFFFFF, np.uint32)
    out, _, _ = A.Graph.from_csr(g3).sssp(0)
    assert list(out) == [0, 0x7FFFFFFF, 0xFFFFFFFE]


def test_device_buffers_and_async():
    import torch
    g = aggen.config("C1")
    G = A.Graph.from_csr(g)
    s = int(aggen.sources(g, 1)[0])
    lv, _ = oracle.bfs(g, s)
    d, _ = oracle.dijkstra(g, s)
    out = torch.empty(g.V, dtype=torch.int32, device="cuda")
    par = torch.empty(g.V, dtype=torch.int32, device="cuda")
    stream = torch.cuda.current_stream().cuda_stream
    G.bfs(s, levels=out, parents=par, stream=stream)        # enqueued only
    G.check()
    assert np.array_equal(out.cpu().numpy().view(np.uint32), lv)
    assert oracle.validate(g, s, out.cpu().numpy().view(np.uint32), par.cpu().numpy().view(np.uint32))[0] == 0
    G.sssp(s, dist=out, parents=par, stream=stream)
    G.check()
    assert np.array_equal(out.cpu().numpy().view(np.uint32), d)
    # device-resident CSR input
    t_rp = torch.from_numpy(g.row_ptr.view(np.int64)).cuda()
    t_col = torch.from_numpy(g.col.view(np.int32)).cuda()
    t_w = torch.from_numpy(g.w.view(np.int32)).cuda()
    G2 = A.Graph(g.V, t_rp, t_col, t_w)
    out2, _, _ = G2.sssp(s)
    assert np.array_equal(out2, d)


# ------------------------------------------------------------------------------------------------
# full-size configs (BASELINE.json), in the launch configuration bench.py times
# ------------------------------------------------------------------------------------------------
@pytest.mark.parametrize("cfg", ["C2", "C3", "C3p", "C4"])
def test_full_size_configs(cfg):
    g = aggen.config(cfg)
    G = A.Graph.from_csr(g)
    assert G.info.layout == (2 if cfg == "C2" else 1)   # inspector: skewed degrees -> degree layout
    srcs = [0] if cfg.startswith("C3") else []
    srcs += [int(s) for s in aggen.sources(g, 2)]
    for s in srcs:
        check_bfs(g, G, s, pol(0))
        check_bfs(g, G, s, pol(0), want_parents=False)   # bench.py's call: free-output iterations
        check_sssp(g, G, s, pol(0))
        if cfg == "C2":
            check_bfs(g, G, s, pol(0, kind=0))
            check_bfs(g, G, s, pol(1))
    if cfg in ("C3", "C3p"):
        check_sssp(g, G, srcs[-1], pol(1, delta=1 if cfg == "C3p" else 64))


def test_torch_allocator_hook():
    """ag_set_allocator routes every device buffer through the PyTorch caching allocator."""
    import torch
    g = aggen.config("C1")
    s = int(aggen.sources(g, 1)[0])
    lv, _ = oracle.bfs(g, s)
    d, _ = oracle.dijkstra(g, s)
    A.use_torch_allocator(True)
    try:
        before = torch.cuda.memory_allocated()
        G = A.Graph.from_csr(g)
        out, _, _ = G.bfs(s)
        assert np.array_equal(out, lv)
        out, _, _ = G.sssp(s)
        assert np.array_equal(out, d)
        assert torch.cuda.memory_allocated() > before      # the library's buffers live in torch's pool
        G.free()
        assert torch.cuda.memory_allocated() == before
    finally:
        A.use_torch_allocator(False)


# ------------------------------------------------------------------------------------------------
# small-frontier mode (tuned kernels on graphs without hub tasks): iterations with |WS| < small_ws run
# on one CTA per SM while the rest park; thresholds forced low so the group shrinks and grows many
# times inside one traversal (policy field small_ws)
# ------------------------------------------------------------------------------------------------
@pytest.mark.parametrize("small_ws", [1, 8, 100, 5000, 0xFFFFFFFF])
def test_small_frontier_mode_transitions(small_ws):
    graphs = [aggen.config("C1"), aggen.with_weights(aggen.grid(60, 50), seed=9, wmax=100),
              aggen.with_weights(aggen.er(5000, 20000, seed=4), seed=5, wmax=100),
              aggen.random_graph(3000, 9000, seed=12)]
    for g in graphs:
        for layout in (1, 2):
            G = A.Graph.from_csr(g, layout=layout)
            lab = oracle.cc(g)
            for s in sorted(set(int(x) for x in aggen.sources(g, 2)) | {0}):
                check_bfs(g, G, s, pol(0, small_ws=small_ws), want_parents=False)
                check_bfs(g, G, s, pol(0, small_ws=small_ws))
                check_bfs(g, G, s, pol(1, small_ws=small_ws))
                check_sssp(g, G, s, pol(0, small_ws=small_ws))
                check_sssp(g, G, s, pol(0, small_ws=small_ws, free_ppm=1000000))
                check_sssp(g, G, s, pol(1, delta=4, small_ws=small_ws))
            assert np.array_equal(G.cc(policy=pol(0, small_ws=small_ws))[0], lab)
            assert np.array_equal(G.cc(policy=pol(0, small_ws=small_ws, free_ppm=1000000))[0], lab)


def test_ordered_sssp_bitmap_tier():
    """The tuned policy switches the ordered-SSSP pending set between the bitmap (>= V/32 pending) and
    the queue per iteration (select_variant); both representations and every switch must give the
    Dijkstra distances."""
    for g in (aggen.with_weights(aggen.er(20000, 100000, seed=4), seed=5, wmax=100),
              aggen.config("C1"), aggen.with_weights(aggen.grid(80, 60), seed=9, wmax=100)):
        G = A.Graph.from_csr(g)
        for s in aggen.sources(g, 2):
            for delta in (1, 16):
                st = check_sssp(g, G, int(s), pol(1, delta=delta))
                assert st.iterations >= 1
            out, _, st = G.sssp(int(s), policy=pol(1), stats=True, trace_cap=1 << 16)
            v = set(int(x) & 3 for x in st.trace_variant)
            if g.V == 20000:
                assert v == {1, 2}, v   # both tiers used on the ER graph


@pytest.mark.parametrize("cfg", ["C3", "C4"])
def test_default_policy_full_size_no_parents(cfg):
    """bench.py's calls on the latency-bound grid and on ER (free output, no parents)."""
    g = aggen.config(cfg)
    G = A.Graph.from_csr(g)
    for s in [int(x) for x in aggen.sources(g, 1)]:
        check_bfs(g, G, s, pol(0), want_parents=False)
        check_sssp(g, G, s, pol(0))


# ------------------------------------------------------------------------------------------------
# pipelined graph load: several 16M-edge chunks, host and device inputs, both layouts, rows that span
# chunk boundaries (hubs), and CSR errors found in a LATER chunk (after earlier chunks were processed)
# ------------------------------------------------------------------------------------------------
def test_pipelined_load_multichunk_host_and_device():
    import torch
    g = aggen.with_weights(aggen.rmat(20, 20, seed=7), seed=8, wmax=100)   # E ~ 38M: 3 chunks, hub rows span them
    assert g.E > 2 * (1 << 24)
    s = int(aggen.sources(g, 1, seed=5)[0])
    lv, _ = oracle.bfs(g, s, want_parents=False)
    d, _ = oracle.dijkstra(g, s, want_parents=False)
    lab = oracle.cc(g)
    t_rp = torch.from_numpy(g.row_ptr.view(np.int64)).cuda()
    t_col = torch.from_numpy(g.col.view(np.int32)).cuda()
    t_w = torch.from_numpy(g.w.view(np.int32)).cuda()
    for layout in (1, 2):
        for dev in (False, True):
            G = A.Graph(g.V, t_rp, t_col, t_w, layout=layout) if dev else A.Graph.from_csr(g, layout=layout)
            assert G.info.layout == layout and G.info.max_weight == int(g.w.max())
            assert G.info.max_deg == int(np.diff(g.row_ptr).max())
            assert np.array_equal(G.bfs(s)[0], lv)
            assert np.array_equal(G.sssp(s)[0], d)
            assert np.array_equal(G.cc()[0], lab)
            G.free()


@pytest.mark.parametrize("where", ["first", "last"])
@pytest.mark.parametrize("layout", [1, 2])
def test_pipelined_load_errors_in_any_chunk(where, layout):
    g = aggen.with_weights(aggen.rmat(20, 20, seed=7), seed=8, wmax=100)
    pos = 5 if where == "first" else g.E - 3
    col = g.col.copy()
    col[pos] = g.V                  # out-of-range neighbour
    with pytest.raises(A.AgError) as e:
        A.Graph(g.V, g.row_ptr, col, g.w, layout=layout)
    assert e.value.status == "AG_ERR_BAD_CSR"
    w = g.w.copy()
    w[pos] = 0                      # zero weight
    with pytest.raises(A.AgError) as e:
        A.Graph(g.V, g.row_ptr, g.col, w, layout=layout)
    assert e.value.status == "AG_ERR_BAD_CSR"
    # the library is still usable after rejected loads
    G = A.Graph.from_csr(g, layout=layout)
    s = int(aggen.sources(g, 1, seed=5)[0])
    assert np.array_equal(G.bfs(s)[0], oracle.bfs(g, s, want_parents=False)[0])


def test_pipelined_load_degree_layout_edge_cases():
    """Forced degree layout with no edges, with trailing isolated vertices, and unweighted."""
    g0 = aggen.csr_from_edges(70, [], [], w=[])
    G = A.Graph.from_csr(g0, layout=2)
    assert list(G.bfs(3)[0]) == [INF] * 3 + [0] + [INF] * 66
    assert np.array_equal(G.cc()[0], np.arange(70, dtype=np.uint32))
    g = aggen.csr_from_edges(100, [0, 0, 1, 5], [1, 5, 2, 0], w=[3, 4, 5, 6])   # 6..99 isolated
    for weighted in (True, False):
        G = A.Graph.from_csr(g, layout=2, weighted=weighted)
        assert np.array_equal(G.bfs(0)[0], oracle.bfs(g, 0)[0])
        if weighted:
            assert np.array_equal(G.sssp(0)[0], oracle.dijkstra(g, 0)[0])
        assert np.array_equal(G.cc()[0], oracle.cc(g))


def test_allocator_hook_switched_between_load_and_free():
    """A buffer always goes back to the allocator it came from, whatever the hook is at free time."""
    import sys

    import torch
    errs = []
    old = sys.unraisablehook
    sys.unraisablehook = errs.append
    try:
        g = aggen.config("C1")
        s = int(aggen.sources(g, 1)[0])
        G1 = A.Graph.from_csr(g)                 # cudaMalloc
        G1.bfs(s)
        A.use_torch_allocator(True)
        G2 = A.Graph.from_csr(g)                 # PyTorch caching allocator
        G2.sssp(s)
        G1.free()                                # -> cudaFree, not the torch hook
        before = torch.cuda.memory_allocated()
        A.use_torch_allocator(False)
        G2.free()                                # -> back to torch although the hook is off
        assert torch.cuda.memory_allocated() < before
    finally:
        A.use_torch_allocator(False)
        sys.unraisablehook = old
    assert not errs, errs


def test_failed_call_does_not_desynchronise_launch_parity():
    """A call rejected before launch (ordered CC) must not break the next traversals on the handle:
    the small-frontier mode's virtual-CTA counters are double-buffered by a DEVICE launch counter,
    so the host can never consume a parity without a launch."""
    g = aggen.config("C1")
    G = A.Graph.from_csr(g)
    lab = oracle.cc(g)
    s = int(aggen.sources(g, 1)[0])
    lv, _ = oracle.bfs(g, s, want_parents=False)
    assert np.array_equal(G.cc()[0], lab)
    for _ in range(3):
        with pytest.raises(A.AgError) as e:
            G.cc(policy=pol(1))
        assert e.value.status == "AG_ERR_UNSUPPORTED"
        assert np.array_equal(G.cc()[0], lab)
        assert np.array_equal(G.bfs(s)[0], lv)


def test_deferred_overflow_is_sticky_across_queries():
    """An overflow of an EARLIER enqueued SSSP is still reported by ag_graph_check after later
    queries on the same handle were enqueued, and the check clears it."""
    import torch
    g = aggen.path(4)
    g.w = np.full(g.E, 0x7FFFFFFF, np.uint32)     # 0 -> 3 is 3 * (2^31 - 1) > 0xFFFFFFFE
    G = A.Graph.from_csr(g)
    out = torch.empty(g.V, dtype=torch.int32, device="cuda")
    stream = torch.cuda.current_stream().cuda_stream
    G.sssp(0, dist=out, stream=stream)             # overflows
    G.sssp(3, dist=out, stream=stream)             # from the other end: also overflows
    G.sssp(1, dist=out, stream=stream)             # 1 -> 3 = 2 * (2^31 - 1) = 0xFFFFFFFE: fine
    with pytest.raises(A.AgError) as e:
        G.check()
    assert e.value.status == "AG_ERR_OVERFLOW"
    G.check()                                      # cleared
    assert list(out.cpu().numpy().view(np.uint32)) == [0x7FFFFFFF, 0, 0x7FFFFFFF, 0xFFFFFFFE]
    G.sssp(0, dist=out, stream=stream)
    G.sssp(1, dist=out, stream=stream)
    with pytest.raises(A.AgError) as e:           # the earlier overflow survives the later good query
        G.check()
    assert e.value.status == "AG_ERR_OVERFLOW"
    # the same with parents requested (packed (dist, parent) state instead of the distance-only one)
    par = torch.empty(g.V, dtype=torch.int32, device="cuda")
    G.sssp(0, dist=out, parents=par, stream=stream)
    G.sssp(1, dist=out, parents=par, stream=stream)
    with pytest.raises(A.AgError) as e:
        G.check()
    assert e.value.status == "AG_ERR_OVERFLOW"
    G.sssp(1, dist=out, parents=par, stream=stream)
    G.check()


@pytest.mark.parametrize("mode", ["window", "delta"])
def test_adaptive_order_axis(mode):
    """NEXT-3: the SSSP order axis adapted per iteration from the measured re-expansion ratio — the
    unordered deferral window (sssp_window = AG_WINDOW_ADAPTIVE) or the ordered bucket width
    (delta = 0) — reorders the work but never changes the distances."""
    graphs = [aggen.config("C1"), aggen.with_weights(aggen.grid(60, 50), seed=9, wmax=100),
              aggen.with_weights(aggen.er(5000, 20000, seed=4), seed=5, wmax=100),
              aggen.random_graph(2000, 12000, seed=21, wmax=1000),
              aggen.with_weights(aggen.star(20000))]
    for g in graphs:
        for layout in (1, 2):
            G = A.Graph.from_csr(g, layout=layout)
            for s in sorted(set(int(x) for x in aggen.sources(g, 2)) | {0}):
                if mode == "window":
                    check_sssp(g, G, s, pol(0, sssp_window=A.WINDOW_ADAPTIVE))
                    check_sssp(g, G, s, pol(0, sssp_window=A.WINDOW_ADAPTIVE, free_ppm=1000000))
                    check_sssp(g, G, s, pol(0, 1, 2, sssp_window=A.WINDOW_ADAPTIVE))
                else:
                    check_sssp(g, G, s, pol(1, delta=0))
                    check_sssp(g, G, s, pol(1, 4, 1, delta=0))
                    check_sssp(g, G, s, pol(1, 1, 2, delta=0))


@pytest.mark.parametrize("cfg", ["C3p", "C4"])
def test_adaptive_order_axis_full_size(cfg):
    g = aggen.config(cfg)
    G = A.Graph.from_csr(g)
    s = int(aggen.sources(g, 1, seed=5)[0])
    d = oracle.dijkstra(g, s, want_parents=False)[0]
    check_sssp(g, G, s, pol(0, sssp_window=A.WINDOW_ADAPTIVE), expect_dist=d)
    check_sssp(g, G, s, pol(1, delta=0), expect_dist=d)
