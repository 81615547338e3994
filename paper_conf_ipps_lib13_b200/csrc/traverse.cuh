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
//           CC (NEXT-4)    : atomicMin(label[v], label[u]), "if (m.label > n.label)": Fig. 4 l.8'
//                            with level -> label and no +1; WS_0 = every vertex (R23)
//     a5  the next working set is written as the update vector = next-frontier bitmap (atomicOr,
//         20.s39-40) AND as a queue by warp-aggregated atomic append (22.s18), so either
//         representation is ready for the next iteration without an extra pass.
//
// Mappings (axis ii), all over "tiles" of BS working-set elements (BS queue entries, or BS
// consecutive vertex ids of the bitmap — thread per node id as in Fig. 9 line 1/2):
//   T  thread per element, the thread visits all neighbours                  (Fig. 9 line 4)
//   W  warp per element, lanes visit neighbours (block mapping at 32 threads, 24.s15)
//   B  group of `cta_group` threads per element (26.s28), threads visit neighbours (Fig. 9 l.4')
//   H  load-balanced: the tile's adjacency lists are concatenated (CTA scan of degrees) and
//      every thread takes EB edges per step; degree >= HUB_DEG is split into HUB_CHUNK-edge
//      tasks drained by all CTAs (18.s43-44 "intermediate solutions", not built in the paper).
#pragma once

#include "common.cuh"

namespace ag {

#ifdef AG_PROF
// diagnostic build only: per (iteration, CTA) timestamps — iteration start, tile loop done, hub drain
// done — read back with ag_debug_prof() (tools/prof_iters.py)
constexpr int PROF_IT = 64, PROF_CTA = 2048;
__device__ unsigned long long g_prof[PROF_IT][PROF_CTA][6];   // [3]: adjacency entries gated by the CTA's tiles,
                                                               // [4]: hub tasks it expanded, [5]: when its first task arrived
#define AG_PROF_MARK(it, k) \
    if (threadIdx.x == 0 && (it) < PROF_IT && blockIdx.x < PROF_CTA) g_prof[it][blockIdx.x][k] = globaltimer_ns()
#else
#define AG_PROF_MARK(it, k)
#endif

template <typename Off>
struct TravArgs {
    const Off *rp;
    const uint32_t *col;
    const uint2 *cw;            // SSSP: interleaved (col, w)
    uint32_t V;
    uint32_t nwords;
    uint32_t *level;            // BFS level array / CC label array (V), in device-layout ids
    uint32_t *parent;           // BFS parent array (V) or nullptr, in device-layout ids
    const uint32_t *perm;       // degree layout: new id -> caller id (nullptr = identity layout)
    const uint32_t *inv;        //                caller id -> new id
    uint32_t *out_level;        // BFS outputs in caller ids (written by the final pass if relabelled)
    uint32_t *out_parent;
    unsigned long long *P;      // SSSP packed state (V): (dist << 32) | parent, decided by 64-bit atomicMin
    uint32_t *vis;              // BFS ordered: visited bitmap
    uint32_t *bm[3];            // rotating frontier bitmaps (SSSP ordered: bm[0] = pending bitmap)
    uint32_t *q[3];             // rotating queues (capacity V)
    unsigned long long *hub;    // hybrid hub-chunk task ring (one 64-bit word per task, 0 = empty)
    uint32_t hub_cap;
    Ctl *ctl;
    uint32_t *dist_out;         // SSSP outputs (V) — may alias nothing
    uint32_t *parent_out;
    uint32_t *trace_ws;
    unsigned long long *trace_edges;
    uint8_t *trace_var;
    unsigned long long *trace_ns;
    uint32_t trace_cap;
    DevPolicy pol;
    uint32_t src;
    uint32_t nblocks;
    uint32_t max_iters;
    uint32_t has_hubs;
    const uint2 *ulist;         // listed working set (multi-GPU SSSP): entry i = (u, dist of u); the value
                                // travels with the entry, hub tasks carry the entry index (nullptr: off)
};

#ifndef AG_HTILE
#define AG_HTILE BS   // hybrid mapping: queue entries per tile at most (the tile's pieces still span the CTA)
#endif
#ifndef AG_BLIND
#define AG_BLIND 1
#endif
// per-warp staging capacity: one batch appends at most 32 x (edges per thread per batch), plus < 32 left over
// (sized per algorithm: the smaller SSSP buffer lets the L1/shared carveout leave more L1 to the status
// gathers, see launch_traverse)
template <int ALG>
constexpr int wq_cap() {
    return 32 * ((ALG == ALG_SSSP) ? (AG_EB_SSSP > 2 * AG_QB_SSSP ? AG_EB_SSSP : 2 * AG_QB_SSSP)
                                   : (AG_EB_BFS > 4 * AG_QB ? AG_EB_BFS : 4 * AG_QB)) + 32;
}

template <typename Off, int WQ_CAP>
struct __align__(16) TileSmem {
    Off beg[BS];
    uint32_t u[BS];
    uint32_t uval[BS];
    uint32_t deg[BS];
    uint32_t scan[BS + 1];
    uint32_t woff[2][WARPS_PER_CTA];
    uint32_t wq[WARPS_PER_CTA][WQ_CAP];   // per-warp staged queue appends (hybrid mapping)
    unsigned long long red64[2][WARPS_PER_CTA];
    uint32_t red32[2][WARPS_PER_CTA];
    int redi[WARPS_PER_CTA];
    uint32_t redrx[WARPS_PER_CTA];
    uint32_t redany[WARPS_PER_CTA];
    uint32_t tnext[2];
    uint32_t bcast;
    unsigned long long htask[2];   // hub-drain task slots (task word, 0 = drained)
};

// ------------------------------------------------------------------------------------------------
// Per-iteration operations of one algorithm (gate = which WS elements are expanded; visit = the
// per-edge update).  Per-thread counters are reduced once per CTA at the end of the iteration.
// ------------------------------------------------------------------------------------------------
// DO (SSSP, tuned kernels, no parents requested): the per-vertex state is the u32 distance alone (32-bit
// atomicMin, 4-byte status gathers: half the L2/L1 footprint of the packed (dist, parent) word); the packed
// 64-bit word is kept whenever parents are requested, so the parent stays consistent with its distance.
template <int ALG, int ORD, typename Off, bool DO = false>
struct Ops {
    static_assert(!DO || ALG == ALG_SSSP, "distance-only state is an SSSP specialisation");
    static constexpr int EB = (ALG == ALG_SSSP) ? AG_EB_SSSP : AG_EB_BFS;
    const TravArgs<Off> &a;
    uint32_t it;
    uint64_t hi;            // SSSP ordered: exclusive bound lo + delta of the current bucket
    uint64_t hub_hi = ~0ull;  // SSSP: deferral bound for high-degree vertices
    uint32_t *bm_next;      // next-frontier bitmap (SSSP ordered: the pending bitmap)
    uint32_t *q_next;
    unsigned *qlen_next;
    bool append_next;
    bool fenced;            // ordered SSSP with delta > 1: a bucket vertex can improve while claimed
    uint64_t pol_stream;    // L2 evict-first policy for the CSR streams
    uint64_t pol_keep;      // L2 evict-last policy for the status arrays
    uint32_t *wbuf;         // this warp's staging buffer in shared memory (hybrid mapping)
    uint32_t wfill;         // its fill level (warp-uniform)
    unsigned long long ne, nv;
    uint32_t reexp = 0;     // SSSP with an adaptive order: re-expansions (measured redundancy)
    uint32_t vmin;
    int dpend;
    bool ovf;
    bool freeo = false;     // free output: next working set = raw bitmap by fire-and-forget reductions
    bool any = false;       //   ... and this thread set at least one bit of it
    uint32_t nact;          // CTAs taking part in this iteration (default: the whole grid)
    bool bm_upd = true;     // BFS: write the update-vector bitmap (tuned queue-only kernels never read it)
    uint32_t hdeg = HUB_DEG, hchunk = HUB_CHUNK;   // hub-task degree threshold and chunk (per iteration)

    __device__ Ops(const TravArgs<Off> &a_, uint32_t it_, uint64_t hi_, bool append_)
        : a(a_), it(it_), hi(hi_), append_next(append_), fenced(ALG == ALG_SSSP && ORD == ORD_O && (a_.pol.delta > 1 || a_.pol.adapt)),
          pol_stream(policy_evict_first()), pol_keep(policy_evict_last()), wbuf(nullptr), wfill(0), ne(0), nv(0),
          vmin(INF), dpend(0), ovf(false), nact(a_.nblocks) {
        const uint32_t sn = (it_ + 1) % 3;
        bm_next = (ALG == ALG_SSSP && ORD == ORD_O) ? a_.bm[0] : a_.bm[sn];
        q_next = a_.q[sn];
        qlen_next = &a_.ctl->q_len[sn];
    }

    // SSSP state accessors: distance of u (relaxed / status read), and the relaxation itself (returns the
    // previous distance; the packed form also records the parent u in the same atomic)
    __device__ __forceinline__ uint32_t *D() const { return reinterpret_cast<uint32_t *>(a.P); }
    __device__ __forceinline__ uint32_t dist_now(uint32_t u) const {
        if constexpr (DO) return ld_relaxed(D() + u);
        else return (uint32_t)(ld_relaxed64(&a.P[u]) >> 32);
    }
    __device__ __forceinline__ uint32_t relax(uint32_t v, uint32_t nd, uint32_t u) const {
        if constexpr (DO) return atomicMin(D() + v, nd);
        else return (uint32_t)(atomicMin(&a.P[v], ((unsigned long long)nd << 32) | u) >> 32);
    }
    __device__ __forceinline__ void relax_red(uint32_t v, uint32_t nd, uint32_t u) const {
        if constexpr (DO) red_min32(D() + v, nd);
        else red_min64(&a.P[v], ((unsigned long long)nd << 32) | u);
    }

    // Is working-set element u expanded in this iteration?  Fills its adjacency range and value.
    __device__ __forceinline__ bool gate(uint32_t u, Off &beg, uint32_t &deg, uint32_t &uval) {
        bool ex = true;
        // the adjacency range is loaded first, in parallel with the value that decides (SSSP): nearly
        // every working-set element is expanded, and the two loads no longer wait for each other
        const Off rb = a.rp[u], re = a.rp[u + 1];
        if constexpr (ALG == ALG_BFS) {
            uval = it;  // the frontier of iteration it is exactly level it (level-synchronous, 26.s33)
        } else if constexpr (ALG == ALG_CC) {
            uval = ld_relaxed(&a.level[u]);   // the current label (never above the one that queued u)
            // shortcut (pointer jumping): the label of u's label also reaches u, so u can take it before
            // it is expanded — on a high-diameter graph the reach of a label doubles per iteration
            // instead of growing by one hop (R23; results unchanged: same fixed point)
            const uint32_t l2 = ld_relaxed(&a.level[a.inv ? a.inv[uval] : uval]);
            if (l2 < uval) {
                red_min32(&a.level[u], l2);
                uval = l2;
            }
        } else if (a.ulist) {
            // listed entry: uval (the sender's distance of u) was set by the caller; every entry expands
        } else {
            uint32_t t = dist_now(u);
            uval = t;
            if constexpr (ORD == ORD_O) {
                if ((uint64_t)t < hi) {  // in the current bucket: claim (settle) it
                    const uint32_t m = 1u << (u & 31);
                    uint32_t old = atomicAnd(&a.bm[0][u >> 5], ~m);
                    ex = (old & m) != 0;
                    if (ex) {
                        dpend -= 1;
                        if (fenced) {
                            // an improvement that found the pending bit still set (so did not re-add u)
                            // is visible after this fence: expand with the current value (the improver
                            // fences between its atomicMin and its atomicOr on the pending bit)
                            __threadfence();
                            uval = dist_now(u);
                        }
                    }
                } else {  // pending survivor: stays in the working set, feeds findmin (22.s11)
                    ex = false;
                    vmin = min(vmin, t);
                }
                if (append_next) warp_append(q_next, qlen_next, !ex && (uint64_t)t >= hi, u);
            } else if ((uint64_t)t >= hi || ((uint64_t)t >= hub_hi && (uint32_t)(re - rb) >= HUBW_DEG)) {
                // unordered SSSP with a deferral window: a far vertex stays in the working set
                // (re-added to the next frontier unless an improvement already did) and feeds the
                // minimum that places the next window
                ex = false;
                vmin = min(vmin, t);
                const uint32_t m = 1u << (u & 31);
                if (freeo) {
                    red_or(bm_next + (u >> 5), m);
                    any = true;
                } else {
                    const bool fresh = !(atomicOr(bm_next + (u >> 5), m) & m);
                    warp_append(q_next, qlen_next, fresh, u);
                }
            }
        }
        if (ex) {
            beg = rb;
            deg = (uint32_t)(re - rb);
            nv += 1;
            ne += deg;
            if (ALG == ALG_SSSP && a.pol.adapt && !a.ulist) {   // first expansion of u in this query?
                const uint32_t m = 1u << (u & 31);
                if (atomicOr(&a.vis[u >> 5], m) & m) reexp += 1;
            }
        } else {
            deg = 0;
        }
        return ex;
    }

    // The (u, uval) of a hub task key: the vertex itself, or the listed entry index
    __device__ __forceinline__ void task_vertex(uint32_t key, uint32_t &u, uint32_t &uval) const {
        if (a.ulist) {
            const uint2 e = a.ulist[key];
            u = e.x;
            uval = e.y;
        } else {
            u = key;
            uval = (ALG == ALG_BFS) ? it
                 : (ALG == ALG_CC)  ? ld_relaxed(&a.level[u])
                                    : dist_now(u);
        }
    }

    // Status word of v, read before deciding to update.  Plain (L1-cacheable) load: a stale value is
    // always safe because levels/distances only decrease and visited bits are only set — a stale
    // read can only cause an extra atomic, never a missed update.
    using St = uint32_t;
    __device__ __forceinline__ St status(uint32_t v) const {
        if constexpr (ALG == ALG_SSSP && DO) return ld_keep(D() + v, pol_keep);
        else if constexpr (ALG == ALG_SSSP) return (uint32_t)(ld_keep(a.P + v, pol_keep) >> 32);
        else if constexpr (ALG == ALG_CC) return ld_keep(a.level + v, pol_keep);   // label[v]
        else return ld_keep(a.vis + (v >> 5), pol_keep);   // BFS: visited bit (level-synchronous: set <=> level <= current+1)
    }

    // The updates of NB edges with their atomics phased: (1) candidates from the status words,
    // (2) every claiming atomic of the batch issued back to back, (3) results resolved.  A thread with
    // several discoveries then waits for one atomic round trip, not several in a row.  Same semantics
    // as NB calls of update(); returns bit j set if v[j] newly entered the next working set.
    template <int NB, bool CONV = false>
    __device__ __forceinline__ uint32_t update_batch(const uint32_t (&u)[NB], const uint32_t (&uv)[NB],
                                                     const uint32_t (&v)[NB], const uint32_t (&wt)[NB],
                                                     const St (&st)[NB], const bool (&ok)[NB]) {
        // (1) candidates from the (possibly stale) status words; CONV (all 32 lanes converged): a warp
        // with no candidate at all skips the atomic and resolution code (the common case on big levels)
        uint32_t cm = 0;   // bit j: an atomic is issued for edge j
        uint32_t nd[NB];   // SSSP: candidate distance (<= MAX_FINITE whenever bit j of cm is set)
#pragma unroll
        for (int j = 0; j < NB; ++j) {
            if constexpr (ALG == ALG_BFS) {
                nd[j] = 0;
                if (ok[j] && !((st[j] >> (v[j] & 31)) & 1u)) cm |= 1u << j;   // m.level == INF / > level
            } else if constexpr (ALG == ALG_CC) {
                nd[j] = uv[j];
                if (ok[j] && st[j] > uv[j]) cm |= 1u << j;                      // m.label > n.label
            } else {
                const uint64_t d = (uint64_t)uv[j] + wt[j];                     // d = n.distance + w (l.6)
                nd[j] = (uint32_t)d;
                if (ok[j]) {
                    if (d > MAX_FINITE) ovf = true;
                    else if (st[j] > nd[j]) cm |= 1u << j;                      // d < m.distance      (l.7)
                }
            }
        }
        if (CONV && !__any_sync(0xffffffffu, cm != 0)) return 0u;

        if (freeo) {
            // free output: every candidate marks v in the next bitmap with a reduction that returns
            // nothing (the update vector, 22.s13-14); BFS levels are assigned when the next iteration
            // compacts the bitmap, SSSP lowers the packed (dist, parent) word with red.min
#pragma unroll
            for (int j = 0; j < NB; ++j) {
                if ((cm >> j) & 1u) {
                    if constexpr (ALG == ALG_SSSP) {
                        relax_red(v[j], nd[j], u[j]);                           // m.distance = d (l.8)
                        vmin = min(vmin, (uint32_t)nd[j]);
                    } else if constexpr (ALG == ALG_CC) {
                        red_min32(&a.level[v[j]], uv[j]);                       // m.label = n.label
                    }
                    red_or(bm_next + (v[j] >> 5), 1u << (v[j] & 31));           // ws.add(m)       (l.9)
                }
            }
            any |= cm != 0;
            return 0u;
        }
        uint32_t nwm = 0;
        if constexpr (ALG == ALG_CC) {
            uint32_t r[NB];
#pragma unroll
            for (int j = 0; j < NB; ++j) r[j] = ((cm >> j) & 1u) ? atomicMin(&a.level[v[j]], uv[j]) : 0u;
            uint32_t ob[NB];
#pragma unroll
            for (int j = 0; j < NB; ++j) {
                ob[j] = 0u;
                if (((cm >> j) & 1u) && r[j] > uv[j]) ob[j] = atomicOr(bm_next + (v[j] >> 5), 1u << (v[j] & 31));
            }
#pragma unroll
            for (int j = 0; j < NB; ++j)   // lowered AND first to set the bit: ws.add(m), deduped
                if (((cm >> j) & 1u) && r[j] > uv[j] && !(ob[j] & (1u << (v[j] & 31)))) nwm |= 1u << j;
        } else if constexpr (ALG == ALG_BFS) {
            // (2) every claiming atomic of the batch issued back to back, (3) results resolved
            uint32_t r[NB];
#pragma unroll
            for (int j = 0; j < NB; ++j) {
                const uint32_t m = 1u << (v[j] & 31);
                r[j] = 0u;
                if ((cm >> j) & 1u) {
                    if constexpr (ORD == ORD_O) r[j] = atomicOr(a.vis + (v[j] >> 5), m);  // claim
                    else r[j] = atomicMin(&a.level[v[j]], uv[j] + 1);
                }
            }
#pragma unroll
            for (int j = 0; j < NB; ++j) {
                const uint32_t m = 1u << (v[j] & 31);
                const uint32_t nl = uv[j] + 1;
                const bool won = ((cm >> j) & 1u) && ((ORD == ORD_O) ? !(r[j] & m) : (r[j] > nl));
                if (won) {
                    if constexpr (ORD == ORD_O) {
                        a.level[v[j]] = nl;                            // m.level = level    (l.9)
                        if (bm_upd) red_or(a.bm[(it + 1) % 3] + (v[j] >> 5), m);   // update vector (l.10)
                    } else {
                        red_or(a.vis + (v[j] >> 5), m);
                        if (bm_upd) red_or(bm_next + (v[j] >> 5), m);
                    }
                    if (a.parent) a.parent[v[j]] = u[j];
                    nwm |= 1u << j;
                }
            }
        } else {
            uint32_t r[NB];   // previous distance of v[j]
#pragma unroll
            for (int j = 0; j < NB; ++j) {
                r[j] = 0u;
                if ((cm >> j) & 1u) r[j] = relax(v[j], nd[j], u[j]);
            }
            uint32_t ob[NB];
            uint32_t im = 0;   // bit j: we lowered m.distance
#pragma unroll
            for (int j = 0; j < NB; ++j) {
                ob[j] = 0u;
                if (((cm >> j) & 1u) && r[j] > nd[j]) {                  // m.distance = d      (l.8)
                    if (fenced) __threadfence();
                    im |= 1u << j;
                    ob[j] = atomicOr(bm_next + (v[j] >> 5), 1u << (v[j] & 31));
                    vmin = min(vmin, (uint32_t)nd[j]);
                }
            }
#pragma unroll
            for (int j = 0; j < NB; ++j) {
                const bool nw = ((im >> j) & 1u) && !(ob[j] & (1u << (v[j] & 31)));  // ws.add(m) (l.9)
                if (nw) {
                    if constexpr (ORD == ORD_O) dpend += 1;
                    if (ORD == ORD_U || append_next) nwm |= 1u << j;
                }
            }
        }
        return nwm;
    }

    // NB independent edges: all CSR loads first, then all status loads, then the updates, so NB
    // memory requests per phase are in flight per thread (the per-edge chain col -> status -> atomic
    // is latency-bound otherwise).  New working-set elements are appended either warp-aggregated to
    // the global queue, or (STAGED: all 32 lanes converged) staged in this warp's shared-memory
    // buffer, flushed to the global queue 32 entries at a time with one atomic per flush.
    template <int NB, bool STAGED = false>
    __device__ __forceinline__ void batch(const uint32_t (&u)[NB], const uint32_t (&uv)[NB], const Off (&e)[NB],
                                          const bool (&ok)[NB]) {
        uint32_t v[NB], wt[NB];
#pragma unroll
        for (int j = 0; j < NB; ++j) {
            if constexpr (ALG == ALG_SSSP) {
                const uint2 c = ok[j] ? ld_stream2(a.cw + e[j], pol_stream) : make_uint2(0u, 1u);
                v[j] = c.x;
                wt[j] = c.y;
            } else {
                v[j] = ok[j] ? ld_stream(a.col + e[j], pol_stream) : 0u;
                wt[j] = 1u;
            }
        }
        batch_vals<NB, STAGED>(u, uv, v, wt, ok);
    }

    // The status + update half of a batch, for neighbour ids already in registers.
    template <int NB, bool STAGED>
    __device__ __forceinline__ void batch_vals(const uint32_t (&u)[NB], const uint32_t (&uv)[NB], const uint32_t (&v)[NB],
                                               const uint32_t (&wt)[NB], const bool (&ok)[NB]) {
        St st[NB];
#pragma unroll
        for (int j = 0; j < NB; ++j) {
            // free-output BFS: no status gather — every target is marked with one fire-and-forget red.or
            // and the next iteration's compaction drops the visited ones (one L2 operation per edge with
            // no round trip, instead of a gather plus a red.or per unvisited target)
            if (AG_BLIND && ALG == ALG_BFS && freeo) st[j] = (St)0;
            else st[j] = ok[j] ? status(v[j]) : (St)0;
        }
        if constexpr (STAGED) {
            const uint32_t nwm = update_batch<NB, true>(u, uv, v, wt, st, ok);  // bit j: v[j] entered the next WS
            if (__any_sync(0xffffffffu, nwm != 0)) {   // rare on the big levels: skip the ballots otherwise
#pragma unroll
                for (int j = 0; j < NB; ++j) {
                    const bool nw = (nwm >> j) & 1u;
                    const unsigned m = __ballot_sync(0xffffffffu, nw);
                    if (nw) wbuf[wfill + __popc(m & ((1u << lane_id()) - 1u))] = v[j];
                    wfill += __popc(m);
                }
                __syncwarp();
                if (wfill >= 32) warp_flush(false);
            }
        } else {
            const uint32_t nwm = update_batch<NB>(u, uv, v, wt, st, ok);
#pragma unroll
            for (int j = 0; j < NB; ++j) warp_append(q_next, qlen_next, (nwm >> j) & 1u, v[j]);
        }
    }

    // QB aligned 16-byte pieces per thread: piece q holds CSR entries [q*QE, q*QE + QE) (one 128-bit
    // load), of which those in [lo, hi) (one adjacency list) are expanded.  All loads of the QB pieces
    // are issued first, then all status loads, then the updates (warp-converged; staged appends).
    static constexpr uint32_t QE = (ALG == ALG_SSSP) ? 2u : 4u;
    static constexpr int QB = (ALG == ALG_SSSP) ? AG_QB_SSSP : AG_QB;
    template <int NQ>
    __device__ __forceinline__ void pieces(const uint32_t (&pu)[NQ], const uint32_t (&pv)[NQ], const Off (&pq)[NQ],
                                           const Off (&plo)[NQ], const Off (&phi)[NQ], const bool (&pok)[NQ]) {
        constexpr int N = NQ * (int)QE;
        uint32_t uu[N], vv[N], v[N], wt[N];
        bool ok[N];
#pragma unroll
        for (int j = 0; j < NQ; ++j) {
            uint4 c = pok[j] ? ld_stream4(reinterpret_cast<const uint4 *>(
                                              (ALG == ALG_SSSP) ? (const void *)(a.cw + pq[j] * QE)
                                                                : (const void *)(a.col + pq[j] * QE)),
                                          pol_stream)
                             : make_uint4(0u, 0u, 0u, 0u);
            const Off e0 = pq[j] * QE;
            if constexpr (ALG == ALG_SSSP) {
                v[2 * j] = c.x; wt[2 * j] = c.y; v[2 * j + 1] = c.z; wt[2 * j + 1] = c.w;
            } else {
                v[4 * j] = c.x; v[4 * j + 1] = c.y; v[4 * j + 2] = c.z; v[4 * j + 3] = c.w;
#pragma unroll
                for (int k = 0; k < 4; ++k) wt[4 * j + k] = 1u;
            }
#pragma unroll
            for (int k = 0; k < (int)QE; ++k) {
                ok[j * QE + k] = pok[j] && e0 + k >= plo[j] && e0 + k < phi[j];
                uu[j * QE + k] = pu[j];
                vv[j * QE + k] = pv[j];
            }
        }
        batch_vals<N, true>(uu, vv, v, wt, ok);
    }

    // Copy this warp's staged entries (all, or whole groups of 32) to the global queue.
    __device__ __forceinline__ void warp_flush(bool all) {
        const unsigned lane = lane_id();
        const uint32_t n = all ? wfill : (wfill & ~31u);
        if (n == 0) return;
        uint32_t base = 0;
        if (lane == 0) base = atomicAdd(qlen_next, n);
        base = __shfl_sync(0xffffffffu, base, 0);
        for (uint32_t i = lane; i < n; i += 32) q_next[base + i] = wbuf[i];
        const uint32_t rem = wfill - n;  // < 32
        uint32_t t = (lane < rem) ? wbuf[n + lane] : 0u;
        __syncwarp();
        if (lane < rem) wbuf[lane] = t;
        __syncwarp();
        wfill = rem;
    }

    // thread-mapped neighbour loop (Fig. 9 line 4: "current thread visits all neighbors")
    __device__ __forceinline__ void edges_thread(uint32_t u, uint32_t uval, Off beg, uint32_t deg) {
        for (uint32_t k = 0; k < deg; k += EB) {
            uint32_t uu[EB], vv[EB];
            Off e[EB];
            bool ok[EB];
#pragma unroll
            for (int j = 0; j < EB; ++j) {
                uu[j] = u; vv[j] = uval; e[j] = beg + k + j; ok[j] = k + j < deg;
            }
            batch<EB>(uu, vv, e, ok);
        }
    }

    // cooperative neighbour loop: `lane` of `width` threads (Fig. 9 line 4': "each thread in block
    // visits a neighbor")
    __device__ __forceinline__ void edges_coop(uint32_t u, uint32_t uval, Off beg, uint32_t deg, uint32_t lane,
                                               uint32_t width) {
        for (uint32_t k = lane; k < deg; k += EB * width) {
            uint32_t uu[EB], vv[EB];
            Off e[EB];
            bool ok[EB];
#pragma unroll
            for (int j = 0; j < EB; ++j) {
                uu[j] = u; vv[j] = uval; e[j] = beg + k + j * width; ok[j] = k + j * width < deg;
            }
            batch<EB>(uu, vv, e, ok);
        }
    }
};

// ------------------------------------------------------------------------------------------------
template <int ALG, int ORD, typename Off, bool DO, typename SmT>
__device__ __forceinline__ void block_reduce_flush(Ops<ALG, ORD, Off, DO> &ops, SmT &sm, Ctl *ctl,
                                                   uint32_t slot) {
    const unsigned lane = lane_id(), wid = threadIdx.x >> 5;
    unsigned long long ne = warp_sum(ops.ne), nv = warp_sum(ops.nv);
    uint32_t vmin = warp_min(ops.vmin);
    int dp = warp_sum(ops.dpend);
    const uint32_t rx = warp_sum(ops.reexp);
    unsigned ovf = __any_sync(0xffffffffu, ops.ovf);
    unsigned anyw = __any_sync(0xffffffffu, ops.any);
    if (lane == 0) {
        sm.redany[wid] = anyw;
        sm.red64[0][wid] = ne;
        sm.red64[1][wid] = nv;
        sm.red32[0][wid] = vmin;
        sm.red32[1][wid] = ovf;
        sm.redi[wid] = dp;
        sm.redrx[wid] = rx;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long se = 0, sv = 0;
        uint32_t mn = INF, ov = 0, an = 0;
        int sd = 0;
        uint32_t srx = 0;
        for (int i = 0; i < WARPS_PER_CTA; ++i) {
            srx += sm.redrx[i];
            an |= sm.redany[i];
            se += sm.red64[0][i];
            sv += sm.red64[1][i];
            mn = min(mn, sm.red32[0][i]);
            ov |= sm.red32[1][i];
            sd += sm.redi[i];
        }
        if (se) {
            atomicAdd(&ctl->eexp, se);
            atomicAdd(&ctl->it_edges[slot], se);   // m_F of this working set (selector input, trace)
        }
        if (sv) {
            atomicAdd(&ctl->vexp, sv);
            atomicAdd(&ctl->it_nv[slot], sv);
        }
        if (srx) atomicAdd(&ctl->it_reexp[slot], srx);
        if (ALG == ALG_SSSP) {
            if (mn != INF) atomicMin(&ctl->next_min[(slot + 1) % 3], mn);
            if (ORD == ORD_O && sd) atomicAdd(&ctl->pend_count, (unsigned)sd);
        }
        if (ov) ctl->overflow = 1;
        if (an) ctl->free_any[(slot + 1) % 3] = 1u;
    }
    // (the following grid barrier begins with __syncthreads)
}

// ------------------------------------------------------------------------------------------------
// One tile: thread tid holds working-set element (valid, u).  Applies the mapping.
// ------------------------------------------------------------------------------------------------
template <bool TUNED, int ALG, int ORD, typename Off, bool DO, typename SmT>
__device__ __forceinline__ void process_tile(Ops<ALG, ORD, Off, DO> &ops, SmT &sm, uint32_t map,
                                             bool valid, uint32_t u, uint32_t group, bool hubs, uint32_t slot,
                                             uint32_t uval_in = 0, uint32_t key = 0xFFFFFFFFu) {
    const TravArgs<Off> &a = ops.a;
    Off beg = 0;
    uint32_t deg = 0, uval = uval_in;
    if (key == 0xFFFFFFFFu) key = u;   // hub-task key: the vertex, or its listed entry index
    bool ex = valid && ops.gate(u, beg, deg, uval);
    if (!ex) deg = 0;
    const uint32_t tid = threadIdx.x, lane = lane_id();

    if (map == MAP_T) {
        if (ex) ops.edges_thread(u, uval, beg, deg);
        return;
    }
    if (!TUNED && (map == MAP_W || (map == MAP_B && group == 32))) {
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
    if (!TUNED && map == MAP_B) {
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
    // ---- MAP_H: load-balanced gather over the tile's concatenated adjacency lists; vertices of
    // degree >= HUB_DEG are split into HUB_CHUNK-edge tasks drained by all CTAs.
    const bool is_hub = hubs && deg >= ops.hdeg;
    if (is_hub) {
        const uint32_t nch = (deg + ops.hchunk - 1) / ops.hchunk;
        uint32_t base = atomicAdd(&a.ctl->hub_tail[slot], nch);
        // hub_cap >= E/chunk + E/degree + 16 (smallest in use) covers any frontier (each vertex is at most once
        // per iteration in it); the guard only protects memory.
        // a task is ONE self-contained 64-bit word (u << 32 | chunk << 1 | 1), published with a single
        // relaxed store: the consumer needs no acquire (which would invalidate its L1) and clears the
        // slot after reading it, so a nonzero word is always a task of the current iteration
        for (uint32_t k = 0; k < nch; ++k) {
            uint32_t idx = base + k;
            if (idx < a.hub_cap) st_relaxed64(a.hub + idx, ((unsigned long long)key << 32) | ((unsigned long long)k << 1) | 1ull);
            else a.ctl->aborted = 2;
        }
    }
    // every (non-hub) adjacency list is cut into aligned 16-byte pieces (QE entries each: 4 col ids for
    // BFS, 2 (col, w) pairs for SSSP); a CTA scan of the piece counts gives each thread QB pieces per
    // step: one owner search + one 128-bit load per piece, coalesced across the warp
    constexpr uint32_t QE = Ops<ALG, ORD, Off>::QE;
    const uint32_t d = is_hub ? 0u : deg;
    const uint32_t np = d ? (uint32_t)((beg + d + QE - 1) / QE - beg / QE) : 0u;
    // (the __syncthreads_or that opened this tile guarantees nobody still reads the previous tile)
    sm.u[tid] = u;
    sm.uval[tid] = uval;
    sm.beg[tid] = beg;
    sm.deg[tid] = d;
    uint32_t x = np;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint32_t xo = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= (unsigned)o) x += xo;
    }
    if (lane == 31) sm.red32[0][tid >> 5] = x;
    __syncthreads();
    uint32_t woff = 0;   // every thread sums the preceding warps' totals (broadcast reads)
    for (uint32_t w = 0; w < (tid >> 5); ++w) woff += sm.red32[0][w];
    const uint32_t excl = woff + x - np;
    sm.scan[tid] = excl;
    if (tid == BS - 1) sm.scan[BS] = excl + np;
    __syncthreads();
    const uint32_t NP = sm.scan[BS];
    constexpr int QB = Ops<ALG, ORD, Off>::QB;
    for (uint32_t base = 0; base < NP; base += QB * BS) {
        uint32_t pu[QB], pv[QB];
        Off pq[QB], plo[QB], phi[QB];
        bool pok[QB];
#pragma unroll
        for (int j = 0; j < QB; ++j) {
            const uint32_t p = base + j * BS + tid;
            pok[j] = p < NP;
            uint32_t lo = 0, hi = BS;   // owner: the largest i with scan[i] <= p
#pragma unroll
            for (int step = 0; step < LOG_BS; ++step) {
                const uint32_t mid = (lo + hi) >> 1;
                if (sm.scan[mid] <= p) lo = mid; else hi = mid;
            }
            pu[j] = sm.u[lo];
            pv[j] = sm.uval[lo];
            const Off bo = sm.beg[lo];
            plo[j] = bo;
            phi[j] = bo + sm.deg[lo];
            pq[j] = bo / QE + (p - sm.scan[lo]);   // aligned piece index
        }
        ops.template pieces<QB>(pu, pv, pq, plo, phi, pok);
    }
    // no trailing barrier: the next tile's __syncthreads_or orders the reuse of the tile arrays
}

// Wait for hub task t of this iteration: its word, or 0 once the producers are all done and t is
// past the final tail (thread 0 only).
template <typename Off>
__device__ __forceinline__ unsigned long long hub_wait(const TravArgs<Off> &a, uint32_t t, uint32_t slot, uint32_t nact) {
    Ctl *ctl = a.ctl;
    if (t >= a.hub_cap) return 0ull;   // overflow (flagged by the producer)
    for (;;) {
        const unsigned long long w = ld_relaxed64(a.hub + t);
        if (w) return w;
        if (t < ld_relaxed(&ctl->hub_tail[slot])) {   // reserved, not yet written
            __nanosleep(32);
            continue;
        }
        if (ld_relaxed(&ctl->stage_done[slot]) == nact) {
            (void)ld_acquire(&ctl->stage_done[slot]);   // every producer's tail reservation is visible
            if (t < ld_relaxed(&ctl->hub_tail[slot])) continue;
            return 0ull;
        }
        __nanosleep(64);
    }
}

// drain the hub-chunk tasks of this iteration (hybrid mapping).  Thread 0 claims the next task when the
// current one starts and loads its word while the CTA expands the current one, so in steady state the
// claim and fetch latency hides behind the expansion; tasks reach the CTA through two shared-memory slots.
template <int ALG, int ORD, typename Off, bool DO, typename SmT>
__device__ __forceinline__ void drain_hubs(Ops<ALG, ORD, Off, DO> &ops, SmT &sm, uint32_t slot) {
    const TravArgs<Off> &a = ops.a;
    Ctl *ctl = a.ctl;
    __syncthreads();
    // ONE task claimed ahead of the one being expanded (two ahead left up to two claimed-but-unstarted tasks
    // per CTA when the ring ran dry, a tail of up to two tasks: C2 BFS -2.6%, SSSP -2.4% with one, A/B 11)
    uint32_t c1 = 0;                  // claimed index of the next task
    unsigned long long pre = 0ull;    // its word, fetched while the current task is expanded
    if (threadIdx.x == 0) {
        __threadfence();
        atomicAdd(&ctl->stage_done[slot], 1u);
        const uint32_t c0 = atomicAdd(&ctl->hub_head[slot], 1u);
        const unsigned long long w = hub_wait(a, c0, slot, ops.nact);
        if (w) {
            a.hub[c0] = 0ull;
            c1 = atomicAdd(&ctl->hub_head[slot], 1u);
        }
        sm.htask[0] = w;
#ifdef AG_PROF
        if (ops.it < PROF_IT && blockIdx.x < PROF_CTA) {
            g_prof[ops.it][blockIdx.x][4] = 0;
            g_prof[ops.it][blockIdx.x][5] = w ? globaltimer_ns() : 0ull;
        }
#endif
    }
    __syncthreads();
    int par = 0;
    for (;;) {
        const unsigned long long w = sm.htask[par];
        if (!w) break;
        const uint32_t k = (uint32_t)(w & 0xFFFFFFFFull) >> 1;
        uint32_t u, uval;
        ops.task_vertex((uint32_t)(w >> 32), u, uval);
        const Off b0 = a.rp[u], e0 = a.rp[u + 1];
        const Off b = b0 + (Off)k * ops.hchunk;
        const Off e = (e0 - b > (Off)ops.hchunk) ? b + ops.hchunk : e0;
        constexpr uint32_t QE = Ops<ALG, ORD, Off>::QE;
        constexpr int QB = Ops<ALG, ORD, Off>::QB;
        const Off q0 = b / QE, q1 = (e + QE - 1) / QE;
        // the next task was claimed before this one started; its word is fetched now, behind the expansion
        if (threadIdx.x == 0) pre = c1 < a.hub_cap ? ld_relaxed64(a.hub + c1) : 0ull;
        for (Off qb = q0; qb < q1; qb += (Off)QB * BS) {
            uint32_t pu[QB], pv[QB];
            Off pq[QB], plo[QB], phi[QB];
            bool pok[QB];
#pragma unroll
            for (int j = 0; j < QB; ++j) {
                pq[j] = qb + (Off)(j * BS + threadIdx.x);
                pok[j] = pq[j] < q1;
                pu[j] = u;
                pv[j] = uval;
                plo[j] = b;
                phi[j] = e;
            }
            ops.template pieces<QB>(pu, pv, pq, plo, phi, pok);
        }
#ifdef AG_PROF
        if (threadIdx.x == 0 && ops.it < PROF_IT && blockIdx.x < PROF_CTA) g_prof[ops.it][blockIdx.x][4] += 1;
#endif
        if (threadIdx.x == 0) {
            const unsigned long long wn = pre ? pre : hub_wait(a, c1, slot, ops.nact);
            if (wn) {
                a.hub[c1] = 0ull;
                c1 = atomicAdd(&ctl->hub_head[slot], 1u);
            }
            sm.htask[par ^ 1] = wn;
        }
        __syncthreads();
        par ^= 1;
    }
}


// Warp-cooperative, in-order emission of the set bits of the warp's 32 consecutive words (word w0 + lane,
// popcount c, inclusive warp count x, warp total tot) as vertex ids out[0 .. tot): output i goes to lane
// i % 32, which finds the owning word (binary search over the lanes' inclusive counts, by shuffles) and
// its bit (n-th set bit), so the warp's stores are consecutive instead of one lane writing its word's run
// (32 scattered sectors per store instruction).  f(v) is called for every emitted vertex.
template <typename F>
__device__ __forceinline__ void warp_emit_f(uint32_t *out, uint32_t x, uint32_t c, uint32_t word, uint32_t w0,
                                            uint32_t tot, F f) {
    const uint32_t lane = lane_id();
    for (uint32_t i0 = 0; i0 < tot; i0 += 32) {
        const uint32_t i = i0 + lane;
        uint32_t o = 0;   // first lane whose inclusive count exceeds i
#pragma unroll
        for (uint32_t step = 16; step >= 1; step >>= 1) {
            const uint32_t xs = __shfl_sync(0xffffffffu, x, o + step - 1);
            if (xs <= i) o += step;
        }
        o = o > 31u ? 31u : o;
        const uint32_t ow = __shfl_sync(0xffffffffu, word, o);
        const uint32_t oe = __shfl_sync(0xffffffffu, x - c, o);
        if (i < tot) {
            const uint32_t v = (w0 + o) * 32u + __fns(ow, 0u, (int)(i - oe) + 1);
            out[i] = v;
            f(v);
        }
    }
}
__device__ __forceinline__ void warp_emit(uint32_t *out, uint32_t x, uint32_t c, uint32_t word, uint32_t w0, uint32_t tot) {
    warp_emit_f(out, x, c, word, w0, tot, [](uint32_t) {});
}

// Free-output successor -> queue: O(V/32) compaction of the raw next bitmap (the "converted in
// O(V/32)" working-set switch; prefix scan instead of per-element atomics, 22.s24).  Each thread
// takes one word per step, one atomic per CTA step.  BFS keeps only the unvisited bits, marks them
// visited and assigns their level (the bitmap held candidates, not claims); SSSP keeps every bit.
// Every word is cleared for reuse.
template <int ALG, typename Off, typename SmT>
__device__ __forceinline__ void compact_raw(const TravArgs<Off> &a, SmT &sm, uint32_t *bm, uint32_t lvl,
                                            uint32_t *q, unsigned *qlen, uint32_t nact, uint32_t vid) {
    const uint32_t lane = lane_id(), wid = threadIdx.x >> 5;
    for (uint32_t w0 = vid * BS; w0 < a.nwords; w0 += nact * BS) {
        const uint32_t wi = w0 + threadIdx.x;
        uint32_t word = wi < a.nwords ? bm[wi] : 0u;
        if (word) {
            bm[wi] = 0u;
            if constexpr (ALG == ALG_BFS) {
                const uint32_t vw = a.vis[wi];
                word &= ~vw;
                if (word) a.vis[wi] = vw | word;
            }
        }
        const uint32_t c = __popc(word);
        uint32_t x = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= (unsigned)o) x += y;
        }
        if (lane == 31) sm.red32[0][wid] = x;
        __syncthreads();
        if (threadIdx.x == 0) {
            uint32_t tot = 0;
            for (int i = 0; i < WARPS_PER_CTA; ++i) {
                const uint32_t t = sm.red32[0][i];
                sm.red32[1][i] = tot;
                tot += t;
            }
            sm.bcast = tot ? atomicAdd(qlen, tot) : 0u;
        }
        __syncthreads();
        const uint32_t wbase = sm.bcast + sm.red32[1][wid], wtot = __shfl_sync(0xffffffffu, x, 31);
        warp_emit_f(q + wbase, x, c, word, w0 + (wid << 5), wtot, [&](uint32_t v) {
            if constexpr (ALG == ALG_BFS) a.level[v] = lvl;   // m.level = level (Fig. 4 l.9)
        });
        __syncthreads();   // red32 / bcast reuse
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
        warp_emit(q + base, x, c, word, w0, total);
    }
}

// ------------------------------------------------------------------------------------------------
// The persistent kernel
// ------------------------------------------------------------------------------------------------
// TUNED = the adaptive B200 policy only (thread / hybrid mappings over the queue): the paper's
// static variants are compiled out, which frees registers for occupancy.
template <int ALG, int ORD, typename Off, bool TUNED, bool DO = false>
__global__ void __launch_bounds__(BS, ALG == ALG_SSSP ? (TUNED ? AG_MINB_SSSP_T : AG_MINB_SSSP)
                                                      : (TUNED ? AG_MINB_BFS_T : AG_MINB_BFS))
    traverse_kernel(const TravArgs<Off> a) {
    __shared__ TileSmem<Off, wq_cap<ALG>()> sm;

    Ctl *ctl = a.ctl;
    const uint32_t gtid = blockIdx.x * BS + threadIdx.x, gthreads = a.nblocks * BS;
    const uint32_t src = a.inv ? a.inv[a.src] : a.src;
    constexpr bool ROT = !(ALG == ALG_SSSP && ORD == ORD_O);

    // ---------------- phase 0: init (Fig. 4 lines 3-4; Fig. 8 lines 1-3) ----------------
    if (ALG == ALG_BFS) {
        for (uint32_t v = gtid; v < a.V; v += gthreads) {
            a.level[v] = (v == src) ? 0u : INF;
            if (a.parent) a.parent[v] = (v == src) ? src : INF;
        }
    } else if (ALG == ALG_CC) {   // label = own (caller) id; WS_0 = every vertex, as queue and as bitmap
        for (uint32_t v = gtid; v < a.V; v += gthreads) {
            a.level[v] = a.perm ? a.perm[v] : v;
            a.q[0][v] = v;
        }
    } else if (DO) {
        uint32_t *D = reinterpret_cast<uint32_t *>(a.P);
        for (uint32_t v = gtid; v < a.V; v += gthreads) D[v] = (v == src) ? 0u : INF;
    } else {
        for (uint32_t v = gtid; v < a.V; v += gthreads)
            a.P[v] = (v == src) ? (unsigned long long)src : INF64;   // dist 0, parent src
    }
    const uint32_t sbit = 1u << (src & 31), sword = src >> 5;
    for (uint32_t wi = gtid; wi < a.nwords; wi += gthreads) {
        a.bm[0][wi] = (ALG == ALG_CC) ? ((wi + 1 < a.nwords || (a.V & 31) == 0) ? ~0u : (1u << (a.V & 31)) - 1u)
                                      : ((wi == sword) ? sbit : 0u);
        if (ROT) {
            a.bm[1][wi] = 0u;
            a.bm[2][wi] = 0u;
        }
        if (ALG == ALG_BFS) a.vis[wi] = (wi == sword) ? sbit : 0u;
        if (ALG == ALG_SSSP && a.pol.adapt) a.vis[wi] = 0u;   // "expanded before" bits (redundancy measure)
    }
    if (gtid == 0) {
        if (ALG != ALG_CC) a.q[0][0] = src;
        for (int s = 0; s < 3; ++s) {
            ctl->q_len[s] = (s == 0) ? (ALG == ALG_CC ? a.V : 1u) : 0u;
            ctl->next_min[s] = (s == 0) ? 0u : INF;
            ctl->tile_ctr[s] = 0;
            ctl->hub_tail[s] = 0;
            ctl->hub_head[s] = 0;
            ctl->stage_done[s] = 0;
            ctl->it_edges[s] = 0;
            ctl->it_nv[s] = 0;
            ctl->it_reexp[s] = 0;
            ctl->free_any[s] = 0;
        }
        ctl->pend_count = 1;
        ctl->overflow = 0;
        ctl->iterations = 0;
        ctl->aborted = 0;
        ctl->vexp = 0;
        ctl->eexp = 0;
    }
    // small-frontier mode: wake events seen so far (read before the barrier: no wake can precede it),
    // and the virtual CTA id: one leader per SM first, so a small iteration runs on every SM
    uint32_t wgen = ld_relaxed(&ctl->wake_gen);
    if (threadIdx.x == 0) {
        // launch parity from the device-side launch counter (advanced at the end of every launch,
        // after this read: every CTA reads it before its first grid-barrier arrival)
        const uint32_t lpar = ld_relaxed(&ctl->launch_seq) & 1u;
        uint32_t smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        const uint32_t per_sm = a.pol.small_ctas ? (a.nblocks + a.pol.small_ctas - 1) / a.pol.small_ctas : 1u;
        const bool leader = atomicAdd(&ctl->sm_rank[smid & 255u], 1u) % per_sm == 0u;
        sm.red32[1][0] = leader;
        sm.red32[1][1] = leader ? atomicAdd(&ctl->lead_cnt[lpar], 1u) : atomicAdd(&ctl->other_cnt[lpar], 1u);
        sm.red32[1][2] = lpar;
        if (blockIdx.x == 0) {
            ctl->lead_cnt[lpar ^ 1u] = 0u;   // for the next launch (stream-ordered after this one)
            ctl->other_cnt[lpar ^ 1u] = 0u;
        }
    }
    grid_barrier(ctl, a.nblocks);
    const uint32_t nlead = ld_relaxed(&ctl->lead_cnt[sm.red32[1][2]]);
    const uint32_t vid = sm.red32[1][0] ? sm.red32[1][1] : nlead + sm.red32[1][1];   // permutation of [0, nblocks)
    const uint32_t vgtid = vid * BS + threadIdx.x;
    __syncthreads();   // (red32 reuse)
    uint32_t n = (ALG == ALG_CC) ? a.V : 1u;   // |WS_0| = |{src}| (CC: every vertex)
    uint32_t nact = a.nblocks;   // CTAs taking part in the current iteration: vid < nact
    const bool small_ok = TUNED && (a.has_hubs ? a.pol.t_small_hub > 0 : a.pol.t_small > 0) && nlead > 0 &&
                          nlead < a.nblocks;

    // BFS whose every iteration uses the queue (tuned kernels, or the tuned decisions of unordered BFS in the
    // general kernel): the update-vector bitmap is never read, so it is neither written nor cleared
    // (C2 BFS 0.543 -> 0.533 ms, profiles/r02_ab/ab_summary.txt 5v)
    const bool bfs_qonly = ALG == ALG_BFS && (TUNED || (a.pol.kind == AG_POLICY_TUNED && !a.pol.ordered &&
                                                         a.pol.force_ws != WS_BM));
    uint32_t prev_ws = WS_QU;   // representation used in the previous iteration
    uint8_t prev_var = 0;
    uint32_t n_prev = 0;
    // SSSP order axis (NEXT-3): the unordered deferral window / the ordered bucket width; adapted per
    // iteration from the measured redundancy when the policy asks for it (identical on every CTA: the
    // inputs are global counters, and a parked CTA receives the current value when woken)
    uint32_t win = ROT ? a.pol.window : a.pol.delta;
    // (unordered: never below the start value — narrower windows measured slower on C2/C3/C4)
    const uint32_t win_min = ROT ? (win ? win : 1u) : 1u;
    uint32_t it = 0;
    bool in_raw = false;   // this iteration's working set is the raw bitmap of a free-output iteration
    for (;; ++it) {
        if (TUNED && in_raw) {
            compact_raw<ALG>(a, sm, a.bm[it % 3], it, a.q[it % 3], &ctl->q_len[it % 3], nact, vid);
            grid_barrier(ctl, nact, vid == 0);
            n = ld_relaxed(&ctl->q_len[it % 3]);
        }
        if (n == 0 || it >= a.max_iters) break;
        if (small_ok) {
            // small-frontier mode: below t_small only CTAs [0, small_ctas) run the iteration (the grid
            // barrier then has small_ctas arrivals); the others park until CTA 0 wakes them with the
            // iteration to resume at.  Every CTA takes the same decision (same n).
            // (graphs with hub tasks: only in the falling tail, where the hubs have long been expanded)
            const bool small = a.has_hubs ? (n < a.pol.t_small_hub && it > 0 && n < n_prev) : n < a.pol.t_small;
            const uint32_t want = small ? nlead : a.nblocks;
            if (want > nact) {          // grow: wake the parked CTAs into this iteration
                if (vid == 0 && threadIdx.x == 0) {
                    ctl->wake_it = it;
                    ctl->wake_n = n;
                    ctl->wake_nprev = n_prev;
                    ctl->wake_win = win;
                    __threadfence();
                    st_release(&ctl->wake_gen, wgen + 1u);
                }
                wgen += 1u;
                nact = want;
            } else if (want < nact) {   // shrink
                nact = want;
                if (vid >= nact) {
                    if (threadIdx.x == 0) {
                        while (ld_relaxed(&ctl->wake_gen) == wgen) __nanosleep(1000);
                        (void)ld_acquire(&ctl->wake_gen);
                        sm.red32[1][0] = ld_relaxed(&ctl->wake_it);
                        sm.red32[1][1] = ld_relaxed(&ctl->wake_n);
                        sm.red32[1][2] = ld_relaxed(&ctl->wake_nprev);
                        sm.red32[1][3] = ld_relaxed(&ctl->wake_win);
                    }
                    __syncthreads();
                    wgen += 1u;
                    it = sm.red32[1][0];
                    n = sm.red32[1][1];
                    n_prev = sm.red32[1][2];
                    win = sm.red32[1][3];
                    __syncthreads();
                    nact = a.nblocks;
                    prev_var = 0;
                    if (n == 0) break;      // the small group finished: join the final pass
                }
            }
        }
        const uint32_t slot = it % 3;
        const uint32_t gact = nact * BS;   // threads taking part (grid-strided loops of this iteration)
        AG_PROF_MARK(it, 0);
        // decision maker, re-evaluated every sample_every iterations (inspector sampling, 26.s7-9)
        // m_F estimate for the selector: |WS| x the previous frontier's average out-degree (the graph's
        // average at it = 0) — the inspector's working-set statistic (26.s4-7)
        // (every CTA reads the same global counter: the decision must be grid-uniform)
        const uint64_t mf_prev = it ? ld_relaxed64(&ctl->it_edges[(it + 2) % 3]) : 0ull;
        const uint64_t mf = n_prev ? (uint64_t)n * mf_prev / n_prev : (uint64_t)n * ((a.pol.E + a.V - 1) / a.V);
        const uint8_t var = (it % a.pol.sample_every == 0 || prev_var == 0) ? select_variant(a.pol, n, mf) : prev_var;
        const uint32_t map = TUNED ? ((var >> 2) == MAP_T ? (uint32_t)MAP_T : (uint32_t)MAP_H) : (var >> 2);
        // tuned kernels: the queue, except the ordered-SSSP pending set, whose bitmap tier the selector
        // picks once the set is dense (select_variant)
        const uint32_t ws = (TUNED && ROT) ? (uint32_t)WS_QU : (var & 3u);
        if (vid == 0 && threadIdx.x == 0) {
            if (it < a.trace_cap && a.trace_ws) {
                a.trace_ws[it] = n;
                a.trace_var[it] = var;
                a.trace_ns[it] = globaltimer_ns();
                if (it > 0) a.trace_edges[it - 1] = ld_relaxed64(&ctl->it_edges[(it + 2) % 3]);
            }
            const uint32_t rs = (it + 2) % 3;   // reset slot(it+2): last used by iteration it-1,
            ctl->q_len[rs] = 0;                 // next written in iteration it+1
            ctl->next_min[rs] = INF;
            ctl->tile_ctr[rs] = 0;
            ctl->hub_tail[rs] = 0;
            ctl->hub_head[rs] = 0;
            ctl->stage_done[rs] = 0;
            ctl->it_edges[(it + 1) % 3] = 0;   // (slot it%3 is still read after this iteration's barrier)
            ctl->it_nv[(it + 1) % 3] = 0;
            ctl->it_reexp[(it + 1) % 3] = 0;
            ctl->free_any[rs] = 0;
        }

        uint64_t hi = ~0ull;
        bool append = true;
        uint32_t qn = n;
        if (ALG == ALG_SSSP && a.pol.adapt && it > 0) {
            // redundancy of the previous iteration: re-expanded / expanded.  Much waste -> a narrower
            // window (more ordered, fewer redundant relaxations); little waste -> a wider one (more
            // parallel work per iteration, fewer iterations).  Results are unchanged either way.
            const unsigned long long nvp = ld_relaxed64(&ctl->it_nv[(it + 2) % 3]);
            const uint32_t rxp = ld_relaxed(&ctl->it_reexp[(it + 2) % 3]);
            if ((unsigned long long)rxp * 4ull > nvp) win = win > win_min ? win >> 1 : win_min;
            else if ((unsigned long long)rxp * 16ull < nvp && win < a.pol.win_max) win <<= 1;
        }
        if (ALG == ALG_SSSP && ROT && win) {
            const uint32_t lo = ld_relaxed(&ctl->next_min[slot]);
            hi = (uint64_t)lo + win;
        }
        if (!ROT) {
            const uint32_t lo = ld_relaxed(&ctl->next_min[slot]);
            hi = (uint64_t)lo + win;
            append = (ws == WS_QU);
            if (ws == WS_QU) {
                if (prev_ws != WS_QU) {
                    // the pending list is stale: rebuild it from the pending bitmap
                    compact_bitmap(a.bm[0], a.nwords, a.q[slot], &ctl->q_len[slot], vgtid >> 5, gact >> 5);
                    grid_barrier(ctl, nact, vid == 0);
                    qn = ld_relaxed(&ctl->q_len[slot]);
                } else {
                    qn = ld_relaxed(&ctl->q_len[slot]);
                }
            }
        } else if (!TUNED && !bfs_qonly) {
            // clear the bitmap that iteration it+1 will write: bm[(it+2)%3] (read in iteration it-1).
            // (tuned kernels instead clear each frontier word when its vertex is read from the queue)
            uint32_t *bz = a.bm[(it + 2) % 3];
            if (it > 0) {
                if ((unsigned long long)n_prev * 32ull < a.nwords) {
                    const uint32_t *qp = a.q[(it + 2) % 3];
                    for (uint32_t i = vgtid; i < n_prev; i += gact) bz[qp[i] >> 5] = 0u;
                } else {
                    for (uint32_t wi = vgtid; wi < a.nwords; wi += gact) bz[wi] = 0u;
                }
            }
        }

        Ops<ALG, ORD, Off, DO> ops(a, it, hi, append);
        ops.wbuf = sm.wq[threadIdx.x >> 5];
        ops.nact = nact;
        ops.bm_upd = !bfs_qonly;
        if (TUNED && (uint64_t)qn < (uint64_t)a.pol.smallchunk_per_cta * nact) {   // few tasks per CTA: finer tasks
            ops.hdeg = HUB_CHUNK_SMALL < HUB_DEG ? HUB_CHUNK_SMALL : HUB_DEG;
            ops.hchunk = HUB_CHUNK_SMALL;
        }
        // free output (tuned, unordered, big working sets; BFS only without parents: a claim decides them)
        ops.freeo = TUNED && ROT && (ALG != ALG_BFS ? (uint64_t)qn >= a.pol.t_free_sssp
                                                    : ((uint64_t)qn >= a.pol.t_free && a.parent == nullptr));
        if (ALG == ALG_SSSP && ROT && a.pol.hub_window)
            ops.hub_hi = (uint64_t)ld_relaxed(&ctl->next_min[slot]) + a.pol.hub_window;
        const uint32_t *bmc = ROT ? a.bm[slot] : a.bm[0];
        const uint32_t *qc = a.q[slot];
        // queue tiles: BS entries for thread mapping (element per thread); for the cooperative
        // mappings a short queue is spread over all CTAs (>= 2 tiles per CTA)
        uint32_t tile_n = BS;
        if (ws == WS_QU && map != MAP_T) {
            uint32_t want = (qn + 2 * nact - 1) / (2 * nact);
            const uint32_t cap = (map == MAP_H) ? (uint32_t)AG_HTILE : (uint32_t)BS;
            tile_n = want < 1u ? 1u : (want > cap ? cap : want);
        }
        // entry slot of this thread: spread across warps for the warp mapping
        const uint32_t s_idx = (map == MAP_W || (map == MAP_B && a.pol.cta_group == 32))
                                   ? (lane_id() * WARPS_PER_CTA + (threadIdx.x >> 5)) : threadIdx.x;
        const uint32_t ntiles = (ws == WS_BM) ? (a.V + BS - 1) / BS : (qn + tile_n - 1) / tile_n;
        const bool hubs = (map == MAP_H) && a.has_hubs;

        {
            // dynamic tile scheduler: first tile static, then one atomic per tile, fetched one tile ahead
            // (double-buffered in smem; the __syncthreads_or below orders the write before the read)
            uint32_t t = vid;
            int par = 0;
            while (t < ntiles) {
                // (no dynamic tiles when every tile is a static first tile: no atomic on the critical path)
                if (threadIdx.x == 0) sm.tnext[par] = ntiles > nact ? nact + atomicAdd(&ctl->tile_ctr[slot], 1u) : ntiles;
                bool valid;
                uint32_t u;
                if (ws == WS_BM) {
                    u = t * BS + threadIdx.x;
                    valid = u < a.V && ((bmc[u >> 5] >> (u & 31)) & 1u);
                } else {
                    uint32_t i = t * tile_n + s_idx;
                    valid = s_idx < tile_n && i < qn;
                    u = valid ? qc[i] : 0u;
                    // tuned, rotating bitmaps: every set bit of this iteration's bitmap is a queued vertex and
                    // nothing reads the bitmap any more, so its words are cleared here for reuse in it+3
                    if (TUNED && ROT && ALG != ALG_BFS && valid) a.bm[slot][u >> 5] = 0u;
                }
                if (__syncthreads_or(valid))  // skip empty tiles (sparse bitmap): uniform branch
                    process_tile<TUNED>(ops, sm, map, valid, u, a.pol.cta_group, hubs, slot);
                t = sm.tnext[par];
                par ^= 1;
            }
        }
        AG_PROF_MARK(it, 1);
#ifdef AG_PROF
        {
            const unsigned long long x = warp_sum(ops.ne);
            __syncthreads();
            if (lane_id() == 0) sm.red64[0][threadIdx.x >> 5] = x;
            __syncthreads();
            if (threadIdx.x == 0 && it < PROF_IT && blockIdx.x < PROF_CTA) {
                unsigned long long t = 0;
                for (int w = 0; w < WARPS_PER_CTA; ++w) t += sm.red64[0][w];
                g_prof[it][blockIdx.x][3] = t;
            }
            __syncthreads();
        }
#endif
        if (hubs) drain_hubs(ops, sm, slot);   // (begins with __syncthreads)
        AG_PROF_MARK(it, 2);
        ops.warp_flush(true);
        block_reduce_flush(ops, sm, ctl, slot);
        grid_barrier(ctl, nact, vid == 0);
        if (ops.freeo) {
            n = ld_relaxed(&ctl->free_any[(it + 1) % 3]) ? 1u : 0u;   // exact size after the compaction
            in_raw = true;
        } else {
            n = ROT ? ld_relaxed(&ctl->q_len[(it + 1) % 3]) : ld_relaxed(&ctl->pend_count);
            in_raw = false;
        }
        prev_ws = ws;
        prev_var = var;
        n_prev = qn;
    }

    // ---------------- termination ----------------
    if (nact < a.nblocks && vid == 0 && threadIdx.x == 0) {   // wake the parked CTAs for the final pass
        ctl->wake_it = it;
        ctl->wake_n = 0u;
        ctl->wake_nprev = 0u;
        __threadfence();
        st_release(&ctl->wake_gen, wgen + 1u);
    }
    if (vid == 0 && threadIdx.x == 0) {
        ctl->iterations = it;
        if (it > 0 && it - 1 < a.trace_cap && a.trace_edges) a.trace_edges[it - 1] = ld_relaxed64(&ctl->it_edges[(it + 2) % 3]);
        if (it >= a.max_iters) ctl->aborted = 1;
        if (it <= a.trace_cap && a.trace_ns) a.trace_ns[it] = globaltimer_ns();
        const uint32_t ab = ld_relaxed(&ctl->aborted);
        if (ab) atomicMax(&ctl->sticky, ab << 8);
        ctl->launch_seq += 1u;   // every CTA read it before the first grid barrier
    }
    // final pass: results into the caller's arrays in caller ids.  The state is final here (every CTA passed
    // the barrier that ended the last iteration, or was parked without writing), so no further barrier is
    // needed.  (The exact overflow test is a separate kernel, api.cu overflow_check_kernel.)
    if (ALG == ALG_SSSP && DO) {  // distances into the caller's array (caller ids)
        // (a gather per output: measured 1-3% faster than coalesced reads with scattered stores, A/B 10)
        const uint32_t *D = reinterpret_cast<const uint32_t *>(a.P);
        for (uint32_t v = gtid; v < a.V; v += gthreads) a.dist_out[v] = D[a.inv ? a.inv[v] : v];
    } else if (ALG == ALG_SSSP) {  // unpack (dist, parent) into the caller's arrays (caller ids)
        for (uint32_t v = gtid; v < a.V; v += gthreads) {
            const unsigned long long pv = a.P[a.inv ? a.inv[v] : v];
            a.dist_out[v] = (uint32_t)(pv >> 32);
            if (a.parent_out) {
                uint32_t pp = (uint32_t)pv;
                a.parent_out[v] = (pv == INF64) ? INF : (a.perm ? a.perm[pp] : pp);
            }
        }
    } else if (a.inv) {     // BFS / CC in the degree layout: gather back to caller ids
        for (uint32_t v = gtid; v < a.V; v += gthreads) {
            const uint32_t i = a.inv[v];
            a.out_level[v] = a.level[i];
            if (a.out_parent) {
                uint32_t pp = a.parent[i];
                a.out_parent[v] = pp == INF ? INF : a.perm[pp];
            }
        }
    }
}

}  // namespace ag
