// traverse.cuh — the device-resident adaptive traversal (hot path rows a2-a7 of SURVEY.md §8).
//
// ONE cooperative kernel per query runs the paper's whole host loop (Fig. 8, PAPER.md:20.s21:
// "while working set is not empty: CUDA_computation; CUDA_workingset_generation") on the device:
//
//   phase 0  init (a2): level/dist = INF, src = 0, WS = {src}                       (Fig. 4 l.3-4)
//   loop     (a7) while |WS| > 0, separated by a software grid barrier:
//     a3  every CTA evaluates the decision maker on (|WS|, E, V)   (Fig. 11, 24.s34-42)
//     a5' (ordered SSSP only, when switching bitmap -> queue) O(V/32) warp-scan compaction
//     a4  expansion with the selected (mapping, workset) variant:             (Fig. 9 22.s1-5)
//           BFS ordered    : visited-claim, "if (m.level == INF)"              (Fig. 4 l.8)
//           BFS unordered  : atomicMin(level), "if (m.level > level)"          (Fig. 4 l.8')
//           SSSP unordered : packed 64-bit atomicMin((dist<<32)|parent)        (Fig. 5 l.6-9)
//           SSSP ordered   : bucket [lo, lo+delta) of the pending set; lo = findmin by block
//                            reduction + atomicMin fused into the pass         (Fig. 5; 22.s9-11)
//     a5  the next working set is written as the update vector = next-frontier bitmap (atomicOr,
//         20.s39-40) AND as a queue by warp-aggregated atomic append (22.s18), so either
//         representation is ready for the next iteration without an extra pass.
//
// Mappings (axis ii), all over "tiles" of BS working-set elements (BS queue entries, or BS
// consecutive vertex ids of the bitmap — thread per node id as in Fig. 9 line 1/2):
//   T  thread per element, the thread visits all neighbours                  (Fig. 9 line 4)
//   W  warp per element, lanes visit neighbours (block mapping at 32 threads, 24.s15)
//   B  group of `cta_group` threads per element (26.s28), threads visit neighbours (Fig. 9 l.4')
//   H  per element by degree: <32 edge-parallel via CTA scan, <BS warp, <HUB_DEG CTA,
//      >= HUB_DEG split into chunks drained by all CTAs (18.s43-44 "intermediate solutions").
#pragma once

#include "common.cuh"

namespace ag {

template <typename Off>
struct TravArgs {
    const Off *rp;
    const uint32_t *col;
    const uint32_t *w;
    uint32_t V;
    uint32_t nwords;
    uint32_t *level;            // BFS level array (V)
    uint32_t *parent;           // BFS parent array (V) or nullptr
    unsigned long long *P;      // SSSP packed state (V)
    uint32_t *vis;              // BFS ordered: visited bitmap
    uint32_t *bm[3];            // rotating frontier bitmaps (SSSP ordered: bm[0] = pending bitmap)
    uint32_t *q[3];             // rotating queues (capacity V)
    uint32_t *hub;              // hybrid hub-chunk tasks, 4 words each
    uint32_t hub_cap;
    Ctl *ctl;
    uint32_t *dist_out;         // SSSP outputs (V) — may alias nothing
    uint32_t *parent_out;
    uint32_t *trace_ws;
    unsigned long long *trace_edges;
    uint8_t *trace_var;
    uint32_t trace_cap;
    DevPolicy pol;
    uint32_t src;
    uint32_t nblocks;
    uint32_t epoch;
    uint32_t max_iters;
    uint32_t has_hubs;
};

template <typename Off>
struct __align__(16) TileSmem {
    Off beg[BS];
    uint32_t u[BS];
    uint32_t uval[BS];
    uint32_t deg[BS];
    uint32_t scan[BS + 1];
    uint32_t big[BS];
    unsigned long long red64[2][WARPS_PER_CTA];
    uint32_t red32[2][WARPS_PER_CTA];
    int redi[WARPS_PER_CTA];
    uint32_t nbig;
    uint32_t tile;
    uint32_t task;
    uint32_t status;
};

// ------------------------------------------------------------------------------------------------
// Per-iteration operations of one algorithm (gate = which WS elements are expanded; visit = the
// per-edge update).  Per-thread counters are reduced once per CTA at the end of the iteration.
// ------------------------------------------------------------------------------------------------
template <int ALG, int ORD, typename Off>
struct Ops {
    const TravArgs<Off> &a;
    uint32_t it;
    uint64_t hi;            // SSSP ordered: exclusive bound lo + delta of the current bucket
    uint32_t *bm_next;      // next-frontier bitmap (SSSP ordered: the pending bitmap)
    uint32_t *q_next;
    unsigned *qlen_next;
    bool append_next;
    unsigned long long ne, nv;
    uint32_t vmin;
    int dpend;
    bool ovf;

    __device__ Ops(const TravArgs<Off> &a_, uint32_t it_, uint64_t hi_, bool append_)
        : a(a_), it(it_), hi(hi_), append_next(append_), ne(0), nv(0), vmin(INF), dpend(0), ovf(false) {
        const uint32_t sn = (it_ + 1) % 3;
        bm_next = (ALG == ALG_SSSP && ORD == ORD_O) ? a_.bm[0] : a_.bm[sn];
        q_next = a_.q[sn];
        qlen_next = &a_.ctl->q_len[sn];
    }

    // Is working-set element u expanded in this iteration?  Fills its adjacency range and value.
    __device__ __forceinline__ bool gate(uint32_t u, Off &beg, uint32_t &deg, uint32_t &uval) {
        bool ex = true;
        if constexpr (ALG == ALG_BFS) {
            uval = it;  // the frontier of iteration it is exactly level it (level-synchronous, 26.s33)
        } else {
            uint32_t t = (uint32_t)(ld_relaxed64(&a.P[u]) >> 32);
            uval = t;
            if constexpr (ORD == ORD_O) {
                if ((uint64_t)t < hi) {  // in the current bucket: claim (settle) it
                    const uint32_t m = 1u << (u & 31);
                    uint32_t old = atomicAnd(&a.bm[0][u >> 5], ~m);
                    ex = (old & m) != 0;
                    if (ex) dpend -= 1;
                } else {  // pending survivor: stays in the working set, feeds findmin (22.s11)
                    ex = false;
                    vmin = min(vmin, t);
                }
                if (append_next) warp_append(q_next, qlen_next, !ex && (uint64_t)t >= hi, u);
            }
        }
        if (ex) {
            beg = a.rp[u];
            Off end = a.rp[u + 1];
            deg = (uint32_t)(end - beg);
            nv += 1;
            ne += deg;
        } else {
            deg = 0;
        }
        return ex;
    }

    // Per-edge update for edge (u -> v, wt) from a frontier element with value uval.
    __device__ __forceinline__ void visit(uint32_t u, uint32_t uval, uint32_t v, uint32_t wt) {
        const uint32_t m = 1u << (v & 31);
        bool nw = false;
        if constexpr (ALG == ALG_BFS) {
            const uint32_t nl = uval + 1;
            if constexpr (ORD == ORD_O) {
                uint32_t *wp = a.vis + (v >> 5);
                if (!(*wp & m)) {                          // m.level == INF ?  (L1-cached status)
                    if (!(atomicOr(wp, m) & m)) {          // claim: first visit wins
                        nw = true;
                        a.level[v] = nl;
                        if (a.parent) a.parent[v] = u;
                        red_or(a.bm[(it + 1) % 3] + (v >> 5), m);
                    }
                }
            } else {
                if (a.level[v] > nl) {                     // m.level > level ?
                    if (atomicMin(&a.level[v], nl) > nl) {
                        nw = true;
                        if (a.parent) a.parent[v] = u;
                        red_or(bm_next + (v >> 5), m);
                    }
                }
            }
            warp_append(q_next, qlen_next, nw, v);
        } else {
            const uint64_t nd = (uint64_t)uval + wt;   // d = n.distance + w(n,m)   (Fig. 5 l.6)
            if (nd > MAX_FINITE) {
                ovf = true;
            } else {
                unsigned long long cur = a.P[v];
                if ((cur >> 32) > nd) {                    // d < m.distance            (Fig. 5 l.7)
                    unsigned long long old = atomicMin(&a.P[v], (nd << 32) | u);
                    if ((old >> 32) > nd) {                // we lowered it             (Fig. 5 l.8)
                        uint32_t ob = atomicOr(bm_next + (v >> 5), m);
                        nw = !(ob & m);                    // ws.add(m), deduplicated   (Fig. 5 l.9)
                        if constexpr (ORD == ORD_O) {
                            vmin = min(vmin, (uint32_t)nd);
                            if (nw) dpend += 1;
                        }
                    }
                }
            }
            if (ORD == ORD_U || append_next) warp_append(q_next, qlen_next, nw, v);
        }
    }

    __device__ __forceinline__ void edge(uint32_t u, uint32_t uval, Off e) {
        uint32_t v = ld_stream(a.col + e);
        uint32_t wt = (ALG == ALG_SSSP) ? ld_stream(a.w + e) : 1u;
        visit(u, uval, v, wt);
    }

    // thread-mapped neighbour loop with 4 independent loads in flight
    __device__ __forceinline__ void edges_thread(uint32_t u, uint32_t uval, Off beg, uint32_t deg) {
        Off e = beg, end = beg + deg;
        for (; e + 4 <= end; e += 4) {
            uint32_t v0 = ld_stream(a.col + e), v1 = ld_stream(a.col + e + 1);
            uint32_t v2 = ld_stream(a.col + e + 2), v3 = ld_stream(a.col + e + 3);
            uint32_t w0 = 1, w1 = 1, w2 = 1, w3 = 1;
            if constexpr (ALG == ALG_SSSP) {
                w0 = ld_stream(a.w + e); w1 = ld_stream(a.w + e + 1);
                w2 = ld_stream(a.w + e + 2); w3 = ld_stream(a.w + e + 3);
            }
            visit(u, uval, v0, w0);
            visit(u, uval, v1, w1);
            visit(u, uval, v2, w2);
            visit(u, uval, v3, w3);
        }
        for (; e < end; ++e) edge(u, uval, e);
    }

    // cooperative neighbour loop: `lane` of `width` threads
    __device__ __forceinline__ void edges_coop(uint32_t u, uint32_t uval, Off beg, uint32_t deg,
                                               uint32_t lane, uint32_t width) {
        for (uint32_t k = lane; k < deg; k += width) edge(u, uval, beg + k);
    }
};

// ------------------------------------------------------------------------------------------------
template <int ALG, int ORD, typename Off>
__device__ __forceinline__ void block_reduce_flush(Ops<ALG, ORD, Off> &ops, TileSmem<Off> &sm, Ctl *ctl,
                                                   uint32_t slot) {
    const unsigned lane = lane_id(), wid = threadIdx.x >> 5;
    unsigned long long ne = warp_sum(ops.ne), nv = warp_sum(ops.nv);
    uint32_t vmin = warp_min(ops.vmin);
    int dp = warp_sum(ops.dpend);
    unsigned ovf = __any_sync(0xffffffffu, ops.ovf);
    if (lane == 0) {
        sm.red64[0][wid] = ne;
        sm.red64[1][wid] = nv;
        sm.red32[0][wid] = vmin;
        sm.red32[1][wid] = ovf;
        sm.redi[wid] = dp;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long se = 0, sv = 0;
        uint32_t mn = INF, ov = 0;
        int sd = 0;
        for (int i = 0; i < WARPS_PER_CTA; ++i) {
            se += sm.red64[0][i];
            sv += sm.red64[1][i];
            mn = min(mn, sm.red32[0][i]);
            ov |= sm.red32[1][i];
            sd += sm.redi[i];
        }
        if (se) atomicAdd(&ctl->it_edges[slot], se);
        if (sv) atomicAdd(&ctl->it_verts[slot], sv);
        if (ALG == ALG_SSSP && ORD == ORD_O) {
            if (mn != INF) atomicMin(&ctl->next_min[(slot + 1) % 3], mn);
            if (sd) atomicAdd(&ctl->pend_count, (unsigned)sd);
        }
        if (ov) ctl->overflow = 1;
    }
    // (the following grid barrier begins with __syncthreads)
}

// ------------------------------------------------------------------------------------------------
// One tile: thread tid holds working-set element (valid, u).  Applies the mapping.
// ------------------------------------------------------------------------------------------------
template <int ALG, int ORD, typename Off>
__device__ __forceinline__ void process_tile(Ops<ALG, ORD, Off> &ops, TileSmem<Off> &sm, uint32_t map,
                                             bool valid, uint32_t u, uint32_t group, bool hubs, uint32_t slot,
                                             uint32_t tag) {
    const TravArgs<Off> &a = ops.a;
    Off beg = 0;
    uint32_t deg = 0, uval = 0;
    bool ex = valid && ops.gate(u, beg, deg, uval);
    if (!ex) deg = 0;
    const uint32_t tid = threadIdx.x, lane = lane_id();

    if (map == MAP_T) {
        if (ex) ops.edges_thread(u, uval, beg, deg);
        return;
    }
    if (map == MAP_W || (map == MAP_B && group == 32)) {
        unsigned m = __ballot_sync(0xffffffffu, ex && deg > 0);
        while (m) {
            const int j = __ffs(m) - 1;
            m &= m - 1;
            uint32_t uj = __shfl_sync(0xffffffffu, u, j);
            uint32_t vj = __shfl_sync(0xffffffffu, uval, j);
            uint32_t dj = __shfl_sync(0xffffffffu, deg, j);
            Off bj = (Off)__shfl_sync(0xffffffffu, (unsigned long long)beg, j);
            ops.edges_coop(uj, vj, bj, dj, lane, 32);
        }
        return;
    }
    if (map == MAP_B) {
        sm.u[tid] = u;
        sm.uval[tid] = uval;
        sm.deg[tid] = deg;
        sm.beg[tid] = beg;
        __syncthreads();
        const uint32_t ng = BS / group, g = tid / group, gl = tid % group;
        if (g < ng) {
            for (uint32_t i = g; i < (uint32_t)BS; i += ng) {
                uint32_t d = sm.deg[i];
                if (d) ops.edges_coop(sm.u[i], sm.uval[i], sm.beg[i], d, gl, group);
            }
        }
        __syncthreads();
        return;
    }
    // ---- MAP_H: per-element degree classes
    const bool is_hub = hubs && deg >= HUB_DEG;
    const bool is_big = !is_hub && deg >= (uint32_t)BS;
    const bool is_mid = deg >= 32 && deg < (uint32_t)BS;
    const uint32_t small = (deg < 32) ? deg : 0;
    if (is_hub) {  // split into HUB_CHUNK-edge tasks for all CTAs (drained after the tile loop)
        const uint32_t nch = (deg + HUB_CHUNK - 1) / HUB_CHUNK;
        uint32_t base = atomicAdd(&a.ctl->hub_tail[slot], nch);
        // capacity hub_cap >= E/HUB_CHUNK + E/HUB_DEG + 16 covers any frontier (each vertex is at most
        // once per iteration in it); the guard only protects memory.
        for (uint32_t k = 0; k < nch; ++k) {
            uint32_t idx = base + k;
            if (idx < a.hub_cap) {
                uint32_t *tk = a.hub + 4ull * idx;
                tk[0] = u;
                tk[1] = uval;
                tk[2] = k;
                __threadfence();
                st_release(tk + 3, tag);
            } else {
                a.ctl->aborted = 2;
            }
        }
    }
    const bool big_path = is_big;
    // CTA-wide exclusive scan of the small degrees
    uint32_t x = small;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= (unsigned)o) x += y;
    }
    if (lane == 31) sm.red32[0][tid >> 5] = x;
    if (tid == 0) sm.nbig = 0;
    __syncthreads();
    if (tid < 32) {
        uint32_t wv = (tid < (unsigned)WARPS_PER_CTA) ? sm.red32[0][tid] : 0, wx = wv;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint32_t y = __shfl_up_sync(0xffffffffu, wx, o);
            if (tid >= (unsigned)o) wx += y;
        }
        if (tid < (unsigned)WARPS_PER_CTA) sm.red32[1][tid] = wx - wv;  // exclusive warp offsets
    }
    __syncthreads();
    const uint32_t excl = sm.red32[1][tid >> 5] + x - small;
    sm.scan[tid] = excl;
    sm.u[tid] = u;
    sm.uval[tid] = uval;
    sm.beg[tid] = beg;
    sm.deg[tid] = deg;
    if (tid == BS - 1) sm.scan[BS] = excl + small;
    if (big_path) {
        uint32_t k = atomicAdd(&sm.nbig, 1u);
        sm.big[k] = tid;
    }
    __syncthreads();
    // small: edge-parallel over the concatenated short lists (load-balanced gather)
    const uint32_t S = sm.scan[BS];
    for (uint32_t k = tid; k < S; k += BS) {
        uint32_t lo = 0, hi = BS;  // find owner: scan[owner] <= k < scan[owner+1]
        while (hi - lo > 1) {
            uint32_t mid = (lo + hi) >> 1;
            if (sm.scan[mid] <= k) lo = mid; else hi = mid;
        }
        ops.edge(sm.u[lo], sm.uval[lo], sm.beg[lo] + (k - sm.scan[lo]));
    }
    // mid: warp-cooperative over this warp's own mid elements
    {
        unsigned m = __ballot_sync(0xffffffffu, is_mid);
        while (m) {
            const int j = __ffs(m) - 1;
            m &= m - 1;
            uint32_t uj = __shfl_sync(0xffffffffu, u, j);
            uint32_t vj = __shfl_sync(0xffffffffu, uval, j);
            uint32_t dj = __shfl_sync(0xffffffffu, deg, j);
            Off bj = (Off)__shfl_sync(0xffffffffu, (unsigned long long)beg, j);
            ops.edges_coop(uj, vj, bj, dj, lane, 32);
        }
    }
    // big: CTA-cooperative
    const uint32_t nb = sm.nbig;
    for (uint32_t i = 0; i < nb; ++i) {
        const uint32_t t = sm.big[i];
        const uint32_t ub = sm.u[t], vb = sm.uval[t];
        const Off bb = sm.beg[t];
        const uint32_t db = sm.deg[t];
        ops.edges_coop(ub, vb, bb, db, tid, BS);
    }
    __syncthreads();
}

// drain the hub-chunk tasks of this iteration (hybrid mapping)
template <int ALG, int ORD, typename Off>
__device__ __forceinline__ void drain_hubs(Ops<ALG, ORD, Off> &ops, TileSmem<Off> &sm, uint32_t slot,
                                           uint32_t tag) {
    const TravArgs<Off> &a = ops.a;
    Ctl *ctl = a.ctl;
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        atomicAdd(&ctl->stage_done[slot], 1u);
    }
    for (;;) {
        if (threadIdx.x == 0) {
            uint32_t t = atomicAdd(&ctl->hub_head[slot], 1u);
            uint32_t status = 0;  // 0 = done, 1 = ready
            for (;;) {
                uint32_t tail = ld_acquire(&ctl->hub_tail[slot]);
                if (t < tail) {
                    if (t >= a.hub_cap) { status = 0; break; }
                    while (ld_acquire(a.hub + 4ull * t + 3) != tag) __nanosleep(32);
                    status = 1;
                    break;
                }
                if (ld_acquire(&ctl->stage_done[slot]) == a.nblocks) {
                    if (t < ld_acquire(&ctl->hub_tail[slot])) continue;
                    status = 0;
                    break;
                }
                __nanosleep(64);
            }
            sm.task = t;
            sm.status = status;
        }
        __syncthreads();
        const uint32_t t = sm.task, st = sm.status;
        __syncthreads();
        if (!st) break;
        const uint32_t *tk = a.hub + 4ull * t;
        const uint32_t u = tk[0], uval = tk[1], k = tk[2];
        const Off b0 = a.rp[u], e0 = a.rp[u + 1];
        const Off b = b0 + (Off)k * HUB_CHUNK;
        const Off e = (e0 - b > (Off)HUB_CHUNK) ? b + HUB_CHUNK : e0;
        ops.edges_coop(u, uval, b, (uint32_t)(e - b), threadIdx.x, BS);
    }
}

// ordered SSSP: bitmap -> queue compaction of the pending set, O(V/32) (the "converted in O(V/32)"
// working-set switch; Merrill's prefix-scan alternative to per-element atomics, 22.s24)
__device__ __forceinline__ void compact_bitmap(const uint32_t *bm, uint32_t nwords, uint32_t *q, unsigned *qlen,
                                               uint32_t gwarp, uint32_t nwarps) {
    const unsigned lane = lane_id();
    for (uint32_t w0 = gwarp * 32; w0 < nwords; w0 += nwarps * 32) {
        uint32_t wi = w0 + lane;
        uint32_t word = wi < nwords ? bm[wi] : 0u;
        uint32_t c = __popc(word), x = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= (unsigned)o) x += y;
        }
        uint32_t total = __shfl_sync(0xffffffffu, x, 31);
        if (total == 0) continue;
        uint32_t base = 0;
        if (lane == 31) base = atomicAdd(qlen, total);
        base = __shfl_sync(0xffffffffu, base, 31);
        uint32_t pos = base + x - c;
        while (word) {
            int b = __ffs(word) - 1;
            word &= word - 1;
            q[pos++] = wi * 32 + b;
        }
    }
}

// ------------------------------------------------------------------------------------------------
// The persistent kernel
// ------------------------------------------------------------------------------------------------
template <int ALG, int ORD, typename Off>
__global__ void __launch_bounds__(BS, MIN_BLOCKS) traverse_kernel(const TravArgs<Off> a) {
    __shared__ TileSmem<Off> sm;
    Ctl *ctl = a.ctl;
    const uint32_t gtid = blockIdx.x * BS + threadIdx.x, gthreads = a.nblocks * BS;
    const uint32_t src = a.src;
    constexpr bool ROT = !(ALG == ALG_SSSP && ORD == ORD_O);

    // ---------------- phase 0: init (Fig. 4 lines 3-4; Fig. 8 lines 1-3) ----------------
    if (ALG == ALG_BFS) {
        for (uint32_t v = gtid; v < a.V; v += gthreads) {
            a.level[v] = (v == src) ? 0u : INF;
            if (a.parent) a.parent[v] = (v == src) ? src : INF;
        }
    } else {
        for (uint32_t v = gtid; v < a.V; v += gthreads)
            a.P[v] = (v == src) ? (unsigned long long)src : INF64;   // dist 0, parent src
    }
    const uint32_t sbit = 1u << (src & 31), sword = src >> 5;
    for (uint32_t wi = gtid; wi < a.nwords; wi += gthreads) {
        a.bm[0][wi] = (wi == sword) ? sbit : 0u;
        if (ROT) {
            a.bm[1][wi] = 0u;
            a.bm[2][wi] = 0u;
        }
        if (ALG == ALG_BFS && ORD == ORD_O) a.vis[wi] = (wi == sword) ? sbit : 0u;
    }
    if (gtid == 0) {
        a.q[0][0] = src;
        for (int s = 0; s < 3; ++s) {
            ctl->q_len[s] = (s == 0) ? 1u : 0u;
            ctl->next_min[s] = (s == 0) ? 0u : INF;
            ctl->tile_ctr[s] = 0;
            ctl->hub_tail[s] = 0;
            ctl->hub_head[s] = 0;
            ctl->stage_done[s] = 0;
            ctl->it_edges[s] = 0;
            ctl->it_verts[s] = 0;
        }
        ctl->pend_count = 1;
        ctl->overflow = 0;
        ctl->iterations = 0;
        ctl->aborted = 0;
        ctl->vexp = 0;
        ctl->eexp = 0;
    }
    grid_barrier(ctl, a.nblocks);

    uint32_t prev_ws = WS_QU;   // representation used in the previous iteration
    uint8_t prev_var = 0;
    uint32_t n_prev = 0;
    uint32_t it = 0;
    for (;; ++it) {
        const uint32_t slot = it % 3;
        const uint32_t n = ROT ? ld_relaxed(&ctl->q_len[slot]) : ld_relaxed(&ctl->pend_count);
        if (n == 0 || it >= a.max_iters) break;
        // decision maker, re-evaluated every sample_every iterations (inspector sampling, 26.s7-9)
        const uint8_t var = (it % a.pol.sample_every == 0 || prev_var == 0) ? select_variant(a.pol, n, 0) : prev_var;
        const uint32_t map = var >> 2, ws = var & 3;
        const uint32_t tag = a.epoch * 0x9E3779B1u + it + 1;

        if (blockIdx.x == 0 && threadIdx.x == 0) {
            if (it > 0) {
                const uint32_t ps = (it + 2) % 3;   // slot of iteration it-1
                unsigned long long e = ctl->it_edges[ps], v = ctl->it_verts[ps];
                ctl->eexp += e;
                ctl->vexp += v;
                if (it - 1 < a.trace_cap && a.trace_edges) a.trace_edges[it - 1] = e;
            }
            if (it < a.trace_cap && a.trace_ws) {
                a.trace_ws[it] = n;
                a.trace_var[it] = var;
            }
            const uint32_t rs = (it + 2) % 3;       // reset slot(it+2) (last used by iteration it-1)
            ctl->q_len[rs] = 0;
            ctl->next_min[rs] = INF;
            ctl->tile_ctr[rs] = 0;
            ctl->hub_tail[rs] = 0;
            ctl->hub_head[rs] = 0;
            ctl->stage_done[rs] = 0;
            ctl->it_edges[rs] = 0;
            ctl->it_verts[rs] = 0;
        }

        uint64_t hi = 0;
        bool append = true;
        if (!ROT) {
            const uint32_t lo = ld_relaxed(&ctl->next_min[slot]);
            hi = (uint64_t)lo + a.pol.delta;
            append = (ws == WS_QU);
            if (ws == WS_QU && prev_ws != WS_QU) {
                // the pending list is stale: rebuild it from the pending bitmap
                compact_bitmap(a.bm[0], a.nwords, a.q[slot], &ctl->q_len[slot], gtid >> 5, gthreads >> 5);
                grid_barrier(ctl, a.nblocks);
            }
        } else {
            // clear the bitmap that iteration it+1 will write: bm[(it+2)%3] (read in iteration it-1)
            uint32_t *bz = a.bm[(it + 2) % 3];
            if (it > 0) {
                if ((unsigned long long)n_prev * 32ull < a.nwords) {
                    const uint32_t *qp = a.q[(it + 2) % 3];
                    for (uint32_t i = gtid; i < n_prev; i += gthreads) bz[qp[i] >> 5] = 0u;
                } else {
                    for (uint32_t wi = gtid; wi < a.nwords; wi += gthreads) bz[wi] = 0u;
                }
            }
        }

        Ops<ALG, ORD, Off> ops(a, it, hi, append);
        const uint32_t *bmc = ROT ? a.bm[slot] : a.bm[0];
        const uint32_t *qc = a.q[slot];
        const uint32_t qn = ROT ? n : ld_relaxed(&ctl->q_len[slot]);
        const uint32_t ntiles = (ws == WS_BM) ? (a.V + BS - 1) / BS : (qn + BS - 1) / BS;
        const bool hubs = (map == MAP_H) && a.has_hubs;

        // dynamic tile scheduler: first tile static, then one atomic per tile
        uint32_t t = blockIdx.x;
        while (t < ntiles) {
            bool valid;
            uint32_t u;
            if (ws == WS_BM) {
                u = t * BS + threadIdx.x;
                valid = u < a.V && ((bmc[u >> 5] >> (u & 31)) & 1u);
            } else {
                uint32_t i = t * BS + threadIdx.x;
                valid = i < qn;
                u = valid ? qc[i] : 0u;
            }
            process_tile(ops, sm, map, valid, u, a.pol.cta_group, hubs, slot, tag);
            __syncthreads();
            if (threadIdx.x == 0) sm.tile = a.nblocks + atomicAdd(&ctl->tile_ctr[slot], 1u);
            __syncthreads();
            t = sm.tile;
        }
        if (hubs) drain_hubs(ops, sm, slot, tag);
        block_reduce_flush(ops, sm, ctl, slot);
        grid_barrier(ctl, a.nblocks);
        prev_ws = ws;
        prev_var = var;
        n_prev = n;
    }

    // ---------------- termination ----------------
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        if (it > 0) {
            const uint32_t ps = (it + 2) % 3;
            unsigned long long e = ctl->it_edges[ps], v = ctl->it_verts[ps];
            ctl->eexp += e;
            ctl->vexp += v;
            if (it - 1 < a.trace_cap && a.trace_edges) a.trace_edges[it - 1] = e;
        }
        ctl->iterations = it;
        if (it >= a.max_iters) ctl->aborted = 1;
    }
    if (ALG == ALG_SSSP) {  // unpack (dist, parent) into the caller's arrays
        for (uint32_t v = gtid; v < a.V; v += gthreads) {
            unsigned long long pv = a.P[v];
            a.dist_out[v] = (uint32_t)(pv >> 32);
            if (a.parent_out) a.parent_out[v] = (pv == INF64) ? INF : (uint32_t)pv;
        }
    }
}

}  // namespace ag
