"""Multi-GPU path (1-D destination partition + per-level frontier-bitmap all-gather).

No box here has more than one GPU, so the path is checked three ways:
  (i)  -m gpu: P virtual ranks on ONE GPU (ag_dist_init_local; all-gather = device copy) and a
       real NCCL communicator of world 1, bit-exact vs the oracle;
  (ii) -m "not gpu": world-size-2 gloo processes run the partitioned level-synchronous algorithm
       on CPU (owned ranges from the library's host function, parts from the generator, bitmap
       exchange by torch.distributed.all_gather) and must reproduce the global oracle;
  (iii) the generator's per-rank parts union to the global graph.
"""
import os

import numpy as np
import pytest

import aggen
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


# ------------------------------------------------------------------------------------------------
# CPU: partitioned algorithm over gloo (world 2)
# ------------------------------------------------------------------------------------------------
def _partitioned_bfs_worker(rank, world, port, scale, src, out_q):
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_lib13_b200 import agraph as A
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    V = 1 << scale
    b, e = A.owned_range(V, rank, world)
    part = aggen.rmat_part(scale, 16, 1, b, e)          # this rank's destination-owned entries
    S = A.owned_range(V, 0, world)[1]                    # slice size (bits); padded global bitmap
    level = np.full(V, oracle.INF, np.uint32)
    front = np.zeros(S * world, bool)
    front[src] = True
    level[src] = 0
    visited = np.zeros(V, bool)
    visited[src] = True
    L = 0
    while True:
        nxt = np.zeros(S * world, bool)
        for u in np.nonzero(front[:V])[0]:
            for v in part.col[part.row_ptr[u]:part.row_ptr[u + 1]]:
                assert b <= v < e                        # only owned destinations are stored
                if not visited[v]:
                    visited[v] = True
                    level[v] = L + 1
                    nxt[v] = True
        mine = torch.from_numpy(nxt[rank * S:(rank + 1) * S].copy())
        gathered = [torch.zeros(S, dtype=torch.bool) for _ in range(world)]
        dist.all_gather(gathered, mine)
        front = torch.cat(gathered).numpy()
        L += 1
        if not front.any():
            break
    out_q.put((rank, b, e, level[b:e].copy(), L))
    # NCCL bootstrap: rank 0 creates the unique id, broadcast over the CPU group
    try:
        uid = A.dist_unique_id() if rank == 0 else bytes(128)
        t = torch.frombuffer(bytearray(uid), dtype=torch.uint8).clone()
        dist.broadcast(t, 0)
        out_q.put(("uid", rank, bytes(t.numpy())))
    except A.AgError:
        out_q.put(("uid", rank, None))
    dist.destroy_process_group()


def test_partitioned_algorithm_gloo_world2():
    import socket

    import torch.multiprocessing as mp
    scale, world = 10, 2
    g = aggen.rmat(scale, 16, seed=1)
    src = int(aggen.sources(g, 1)[0])
    ref, _ = oracle.bfs(g, src)
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_partitioned_bfs_worker, args=(r, world, port, scale, src, q)) for r in range(world)]
    for p in procs:
        p.start()
    res, uids = {}, {}
    for _ in range(2 * world):
        item = q.get(timeout=300)
        if item[0] == "uid":
            uids[item[1]] = item[2]
        else:
            res[item[0]] = item
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    level = np.concatenate([res[r][3] for r in range(world)])
    assert np.array_equal(level, ref)
    assert res[0][4] == oracle.bfs_iterations(ref)
    if uids[0] is not None:
        assert uids[0] == uids[1] and len(uids[0]) == 128   # every rank got rank 0's NCCL id


def test_generator_parts_union_to_global():
    g = aggen.rmat(11, 16, seed=3)
    from paper_conf_ipps_lib13_b200 import agraph as A
    for world in (2, 3, 8):
        parts = [aggen.rmat_part(11, 16, 3, *A.owned_range(g.V, r, world)) for r in range(world)]
        assert sum(p.E for p in parts) == g.E
        deg = sum(np.diff(p.row_ptr) for p in parts)
        assert np.array_equal(deg, np.diff(g.row_ptr))


# ------------------------------------------------------------------------------------------------
# GPU: virtual ranks on one device, and a real NCCL communicator of world 1
# ------------------------------------------------------------------------------------------------
def _graphs():
    yield aggen.config("C1", weighted=False)
    yield aggen.random_graph(700, 3000, seed=5)          # directed multigraph
    yield aggen.grid(120, 90)
    yield aggen.star(20000)                              # hub >= HUB_DEG


@pytest.mark.gpu
@pytest.mark.parametrize("world", [1, 2, 3, 5])
def test_virtual_group_matches_oracle(world):
    from paper_conf_ipps_lib13_b200 import agraph as A
    for g in _graphs():
        comms = A.local_group(world, 0)
        parts = [A.DistGraph(c, g.V, g.row_ptr, g.col) for c in comms]
        for src in sorted(set([0, g.V - 1, int(aggen.sources(g, 1)[0])])):
            ref, _ = oracle.bfs(g, src)
            lv, par, st = A.dist_bfs_group(parts, src, parents=True, stats=True, trace_cap=1 << 14)
            assert np.array_equal(lv, ref), (g.name, world, src)
            assert oracle.validate(g, src, lv, par)[0] == 0
            assert st.iterations == oracle.bfs_iterations(ref)
            assert list(st.trace_ws) == list(oracle.bfs_level_sizes(ref))
            assert st.vertices_expanded == world * oracle.reached(g, ref)[0]  # every rank expands the frontier
            assert st.edges_inspected == oracle.reached(g, ref)[1]            # edges split by destination
        for p in parts:
            p.free()
        for c in comms:
            c.free()


@pytest.mark.gpu
def test_virtual_group_local_parts():
    """Parts built per rank by the generator (ag_dist_graph_load_local) == global oracle."""
    from paper_conf_ipps_lib13_b200 import agraph as A
    scale, world = 14, 4
    g = aggen.rmat(scale, 16, seed=1)
    comms = A.local_group(world, 0)
    parts = []
    for c in comms:
        b, e = A.owned_range(g.V, c.rank, world)
        pg = aggen.rmat_part(scale, 16, 1, b, e)
        parts.append(A.DistGraph(c, g.V, pg.row_ptr, pg.col, local=True))
    for src in aggen.sources(g, 3):
        ref, _ = oracle.bfs(g, int(src))
        lv, _, _ = A.dist_bfs_group(parts, int(src))
        assert np.array_equal(lv, ref)
    # a part holding a foreign destination is rejected
    bad = aggen.rmat_part(scale, 16, 1, 0, g.V)
    with pytest.raises(A.AgError) as e:
        A.DistGraph(comms[1], g.V, bad.row_ptr, bad.col, local=True)
    assert e.value.status == "AG_ERR_BAD_CSR"


@pytest.mark.gpu
def test_nccl_world1():
    from paper_conf_ipps_lib13_b200 import agraph as A
    g = aggen.config("C1", weighted=False)
    uid = A.dist_unique_id()
    comm = A.Comm.nccl(0, 1, uid, 0)
    part = A.DistGraph(comm, g.V, g.row_ptr, g.col)
    for src in aggen.sources(g, 2):
        ref, _ = oracle.bfs(g, int(src))
        lv, _, st = part.bfs(int(src), stats=True)
        assert np.array_equal(lv, ref) and st.iterations == oracle.bfs_iterations(ref)
    part.free()
    comm.free()


# ------------------------------------------------------------------------------------------------
# Multi-GPU SSSP: same partition, list exchange of (vertex, distance)
# ------------------------------------------------------------------------------------------------
def _partitioned_sssp_worker(rank, world, port, scale, src, out_q):
    """The distributed unordered SSSP of ag_dist_sssp on CPU: every rank relaxes the gathered global
    list of (u, dist u) over its destination-owned part; the improved owned vertices join the rank's
    pending set, from which the OWNER sends every non-hub (in-degree < 64) vertex and every hub below
    hi = (global minimum pending distance of the last exchange) + hub window, holding the other hubs
    back; all_gather of (sent, held back, min pending), then of the (v, dist) lists padded to the
    largest count; done when nothing is sent or held back anywhere."""
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_lib13_b200 import agraph as A
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    V = 1 << scale
    b, e = A.owned_range(V, rank, world)
    part = aggen.rmat_part(scale, 16, 1, b, e)
    w = aggen.weights(part, seed=2, wmax=100)
    d = np.full(V, oracle.INF, np.int64)
    if b <= src < e:
        d[src] = 0
    indeg = np.bincount(part.col.astype(np.int64) - b, minlength=max(e - b, 1))
    hw = max(1, int(w.max()) // 50) if len(w) else 1
    hi = hw
    pending = set()
    lst = [(src, 0)]
    rounds = 0
    while True:
        for u, du in lst:
            for k in range(part.row_ptr[u], part.row_ptr[u + 1]):
                v = int(part.col[k])
                assert b <= v < e
                nd = du + int(w[k])
                if nd < d[v]:
                    d[v] = nd
                    pending.add(v)
        lmin = min((int(d[v]) for v in pending), default=oracle.INF)
        mine = sorted(v for v in pending if indeg[v - b] < 64 or d[v] < hi)
        pending -= set(mine)
        cnt = torch.tensor([len(mine), len(pending), lmin], dtype=torch.int64)
        counts = [torch.zeros(3, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(counts, cnt)
        maxc = int(max(c[0].item() for c in counts))
        held = sum(int(c[1].item()) for c in counts)
        lo = min(int(c[2].item()) for c in counts)
        hi = lo + hw if lo != oracle.INF else 1 << 62
        rounds += 1
        if maxc == 0 and held == 0:
            break
        if maxc == 0:
            lst = []
            continue
        buf = torch.full((maxc, 2), -1, dtype=torch.int64)
        for i, v in enumerate(mine):
            buf[i, 0], buf[i, 1] = v, int(d[v])
        bufs = [torch.zeros((maxc, 2), dtype=torch.int64) for _ in range(world)]
        dist.all_gather(bufs, buf)
        lst = [(int(v), int(dv)) for t in bufs for v, dv in t.tolist() if v >= 0]
    out_q.put((rank, b, e, d[b:e].astype(np.uint64).copy(), rounds))
    dist.destroy_process_group()


def test_partitioned_sssp_gloo_world2():
    import socket

    import torch.multiprocessing as mp
    scale, world = 9, 2
    g = aggen.with_weights(aggen.rmat(scale, 16, seed=1), seed=2, wmax=100)
    src = int(aggen.sources(g, 1)[0])
    ref, _ = oracle.dijkstra(g, src)
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_partitioned_sssp_worker, args=(r, world, port, scale, src, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        item = q.get(timeout=300)
        res[item[0]] = item
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    d = np.concatenate([res[r][3] for r in range(world)])
    d = np.where(d == np.uint64(oracle.INF), oracle.INF, d).astype(np.uint32)
    assert np.array_equal(d, ref)
    assert res[0][4] == res[1][4]                       # every rank sees the same termination round


def _wgraphs():
    yield aggen.config("C1")
    yield aggen.random_graph(700, 3000, seed=5)          # directed multigraph with self-loops
    yield aggen.with_weights(aggen.grid(120, 90))
    yield aggen.with_weights(aggen.star(20000))          # hub >= HUB_DEG


@pytest.mark.gpu
@pytest.mark.parametrize("world", [1, 2, 3, 5])
def test_virtual_group_sssp_matches_oracle(world):
    from paper_conf_ipps_lib13_b200 import agraph as A
    for g in _wgraphs():
        comms = A.local_group(world, 0)
        parts = [A.DistGraph(c, g.V, g.row_ptr, g.col, g.w) for c in comms]
        for src in sorted(set([0, g.V - 1, int(aggen.sources(g, 1)[0])])):
            ref, _ = oracle.dijkstra(g, src)
            d, par, st = A.dist_sssp_group(parts, src, parents=True, stats=True, trace_cap=1 << 14)
            assert np.array_equal(d, ref), (g.name, world, src)
            assert oracle.validate(g, src, d, par, weighted=True)[0] == 0
            assert st.trace_ws[0] == 1 and st.iterations >= 1
        for p in parts:
            p.free()
        for c in comms:
            c.free()


@pytest.mark.gpu
def test_virtual_group_sssp_local_parts_and_errors():
    from paper_conf_ipps_lib13_b200 import agraph as A
    scale, world = 14, 4
    g = aggen.with_weights(aggen.rmat(scale, 16, seed=1), seed=2, wmax=100)
    comms = A.local_group(world, 0)
    parts = []
    for c in comms:
        b, e = A.owned_range(g.V, c.rank, world)
        pg = aggen.rmat_part(scale, 16, 1, b, e)
        parts.append(A.DistGraph(c, g.V, pg.row_ptr, pg.col, aggen.weights(pg, seed=2, wmax=100), local=True))
    for src in aggen.sources(g, 3):
        ref, _ = oracle.dijkstra(g, int(src))
        d, _, _ = A.dist_sssp_group(parts, int(src))
        assert np.array_equal(d, ref)
    # unweighted parts cannot run SSSP
    uw = [A.DistGraph(c, g.V, g.row_ptr, g.col) for c in A.local_group(2, 0)]
    with pytest.raises(A.AgError) as e:
        A.dist_sssp_group(uw, 0)
    assert e.value.status == "AG_ERR_NO_WEIGHTS"


@pytest.mark.gpu
def test_nccl_world1_sssp():
    from paper_conf_ipps_lib13_b200 import agraph as A
    g = aggen.config("C1")
    uid = A.dist_unique_id()
    comm = A.Comm.nccl(0, 1, uid, 0)
    part = A.DistGraph(comm, g.V, g.row_ptr, g.col, g.w)
    for src in aggen.sources(g, 2):
        ref, _ = oracle.dijkstra(g, int(src))
        d, _, st = part.sssp(int(src), stats=True)
        assert np.array_equal(d, ref)
    part.free()
    comm.free()


@pytest.mark.gpu
def test_c5_full_size_world8_virtual_group():
    """C5 at full size (R-MAT scale 26, 2.1B CSR entries) partitioned 1-D over 8 ranks on one GPU: the
    partition, kernels and exchange protocol of the 8-GPU bench (the all-gathers are device copies).
    BFS levels are compared with
    the oracle element by element; SSSP distances with parents must pass the shortest-path certificate
    (edge inequalities + a tight parent edge for every reached vertex = exact distances)."""
    import torch
    from paper_conf_ipps_lib13_b200 import agraph as A
    world = 8
    g = aggen.config("C5")
    # the global CSR goes to the device once; every rank keeps its destination-owned part of it
    t = [torch.from_numpy(x.view(np.int64 if x.dtype == np.uint64 else np.int32)).cuda() for x in (g.row_ptr, g.col, g.w)]
    comms = A.local_group(world, 0)
    parts = [A.DistGraph(c, g.V, t[0], t[1], t[2]) for c in comms]
    del t
    torch.cuda.empty_cache()
    src = int(aggen.sources(g, 1, seed=3)[0])
    lv, _, _ = A.dist_bfs_group(parts, src)
    ref, _ = oracle.bfs(g, src, want_parents=False)
    assert np.array_equal(lv, ref)
    d, par, _ = A.dist_sssp_group(parts, src, parents=True)
    assert np.array_equal(d != oracle.INF, ref != oracle.INF)
    assert oracle.validate(g, src, d, par, weighted=True)[0] == 0
    for p in parts:
        p.free()
    for c in comms:
        c.free()
