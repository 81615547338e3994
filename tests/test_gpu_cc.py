"""GPU parity of min-label connected components (ag_cc; R23)
against the CPU oracle (oracle.cc), bit-exact (-m gpu).

labels[v] = min{u : u reaches v along out-edges} is unique, so it is compared element by element
for every mapping x working-set variant, both selector policies, both device layouts, the
free-output thresholds, the tiny families, directed multigraphs, and the full-size configs.
"""
import numpy as np
import pytest

import aggen
import oracle

pytestmark = pytest.mark.gpu

A = None


@pytest.fixture(scope="module", autouse=True)
def _lib():
    global A
    from paper_conf_ipps_lib13_b200 import agraph, build
    build.build()
    A = agraph
    yield


def pol(mapping=0, workset=0, kind=1, **kw):
    p = A.policy_default(0)
    p.mapping, p.workset, p.kind = mapping, workset, kind
    for k, v in kw.items():
        setattr(p, k, v)
    return p


def variants():
    out = [pol(m, w) for m in (1, 2, 3, 4) for w in (1, 2)]
    out += [pol(kind=0), pol(kind=1), pol(free_ppm=0), pol(free_ppm=1), pol(free_ppm=1000000)]
    return out


def check(g, G, p, expect=None):
    lab = oracle.cc(g) if expect is None else expect
    out, _, st = G.cc(policy=p, stats=True)
    bad = np.nonzero(out != lab)[0]
    assert bad.size == 0, f"V={g.V} first bad v={bad[:5]} got {out[bad[:5]]} want {lab[bad[:5]]}"
    assert st.reached == g.V and st.iterations >= 1
    return st


@pytest.mark.parametrize("layout", [1, 2])
@pytest.mark.parametrize("seed", range(8))
def test_cc_tiny_random_all_variants(seed, layout):
    """Directed multigraphs with self-loops and isolated vertices, every variant."""
    rng = np.random.default_rng(900 + seed)
    V = int(rng.integers(1, 400))
    g = aggen.random_graph(V, int(rng.integers(0, 4 * V + 1)), seed=900 + seed, wmax=3, sort_rows=bool(seed % 2))
    G = A.Graph.from_csr(g, layout=layout)
    lab = oracle.cc(g)
    for p in variants():
        check(g, G, p, lab)


def test_cc_families_closed_forms():
    fams = [aggen.path(1000), aggen.directed_cycle(777), aggen.star(20000), aggen.complete(40),
            aggen.binary_tree(4095), aggen.grid(70, 30)]
    for g in fams:
        for layout in (1, 2):
            G = A.Graph.from_csr(g, weighted=False, layout=layout)
            check(g, G, pol(), np.zeros(g.V, np.uint32))       # connected: every label is 0
    # disjoint union with reversed ids: components {0..9}, {10..19}, ... label = block minimum
    src, dst = [], []
    for b in range(50):
        for i in range(9):
            src.append(b * 10 + 9 - i)
            dst.append(b * 10 + 8 - i)
    g = aggen.csr_from_edges(500, src, dst, symmetrize=True)
    G = A.Graph.from_csr(g, weighted=False)
    check(g, G, pol(), (np.arange(500) // 10 * 10).astype(np.uint32))
    # directed chain pointing DOWN in id: nobody smaller reaches v, labels = ids
    g = aggen.csr_from_edges(300, list(range(299, 0, -1)), list(range(298, -1, -1)))
    G = A.Graph.from_csr(g, weighted=False)
    check(g, G, pol(), np.arange(300, dtype=np.uint32))


@pytest.mark.parametrize("layout", [1, 2])
def test_cc_c1_and_ragged(layout):
    """C1 (R-MAT s12, ~18% isolated vertices) and ragged V (not a multiple of 32 / of a tile)."""
    for g in (aggen.config("C1", weighted=False), aggen.rmat(11, 4, seed=5), aggen.er(12345, 9000, seed=2),
              aggen.random_graph(1000 * 32 + 7, 20000, seed=8, wmax=1)):
        G = A.Graph.from_csr(g, weighted=False, layout=layout)
        for p in variants():
            check(g, G, p)


def test_cc_errors():
    g = aggen.config("C1", weighted=False)
    G = A.Graph.from_csr(g, weighted=False)
    p = pol()
    p.order = 1
    with pytest.raises(A.AgError) as e:
        G.cc(policy=p)
    assert e.value.code == 9   # AG_ERR_UNSUPPORTED
    assert np.array_equal(G.cc()[0], oracle.cc(g))   # handle still usable


@pytest.mark.parametrize("cfg", ["C2", "C4"])
def test_cc_full_size(cfg):
    """Full-size configs in the default (tuned adaptive) launch configuration."""
    g = aggen.config(cfg, weighted=False)
    G = A.Graph.from_csr(g, weighted=False)
    lab = oracle.cc(g)
    check(g, G, pol(), lab)
    check(g, G, pol(free_ppm=0), lab)
