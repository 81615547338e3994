// dist.cu — multi-GPU BFS: 1-D destination partition, per-level frontier-bitmap all-gather.
//
// Not in the paper (one C2070, PAPER.md:26.s15); required by BASELINE.json north_star / SURVEY.md §8(e).
//  * Rank p owns vertices [p*S, min(V,(p+1)*S)), S = ceil(V/P) rounded up to 1024 (whole 128-B bitmap
//    slices).  It stores every CSR entry whose DESTINATION it owns, indexed by source over all V, so
//    expanding any frontier vertex touches only owned level/visited entries: no remote writes, no
//    cross-GPU atomics (NCCL has no bitwise-OR reduction; destination ownership needs none).
//  * Per level: the identical global frontier bitmap (V/8 B) is compacted to a local queue
//    (O(V/32) warp scan), expanded over the local CSR with the load-balanced hybrid mapping
//    (a4), the owned next-frontier slice is published with ncclAllGather(slice -> global bitmap)
//    over NVLink, and termination is a popcount of the gathered bitmap on every rank (no extra
//    collective).
//  * Transport: NCCL (one process per GPU), or a "local group" of P virtual ranks inside one
//    process on one GPU whose all-gather is a device copy — used by the tests to check the
//    partitioning / ownership logic at any P on a single device.
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <cstdlib>
#include <cstring>
#include <mutex>
#include <vector>

#include <cub/device/device_scan.cuh>

#include "agraph.h"
#include "common.cuh"
#include "graph.h"
#include "traverse.cuh"

// Minimal NCCL ABI declarations (nccl.h 2.x): the library dlopens libnccl.so.2 at run time.
typedef struct ncclComm *ncclComm_t;
typedef struct { char internal[128]; } ncclUniqueId;
typedef enum { ncclSuccess = 0 } ncclResult_t;
typedef enum { ncclUint8 = 1, ncclUint32 = 3 } ncclDataType_t;

namespace {

// ---- NCCL loaded at run time (the library itself must load without NCCL)
struct NcclApi {
    bool ok = false;
    ncclResult_t (*GetUniqueId)(ncclUniqueId *) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*AllGather)(const void *, void *, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    const char *(*GetErrorString)(ncclResult_t) = nullptr;
};
NcclApi g_nccl;
std::mutex g_nccl_mu;

bool load_nccl() {
    std::lock_guard<std::mutex> lk(g_nccl_mu);
    if (g_nccl.ok) return true;
    void *h = nullptr;
    if (const char *p = getenv("AG_NCCL_LIB")) h = dlopen(p, RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return false;
    g_nccl.GetUniqueId = (decltype(g_nccl.GetUniqueId))dlsym(h, "ncclGetUniqueId");
    g_nccl.CommInitRank = (decltype(g_nccl.CommInitRank))dlsym(h, "ncclCommInitRank");
    g_nccl.CommDestroy = (decltype(g_nccl.CommDestroy))dlsym(h, "ncclCommDestroy");
    g_nccl.AllGather = (decltype(g_nccl.AllGather))dlsym(h, "ncclAllGather");
    g_nccl.GetErrorString = (decltype(g_nccl.GetErrorString))dlsym(h, "ncclGetErrorString");
    g_nccl.ok = g_nccl.GetUniqueId && g_nccl.CommInitRank && g_nccl.CommDestroy && g_nccl.AllGather;
    return g_nccl.ok;
}

ag_status nccl_status(ncclResult_t r, const char *what) {
    if (r == ncclSuccess) return AG_OK;
    return ag::set_error(AG_ERR_NCCL, "%s: %s", what, g_nccl.GetErrorString ? g_nccl.GetErrorString(r) : "nccl error");
}

}  // namespace

struct ag_local_group;

struct ag_comm_s {
    int rank = 0, world = 1, device = 0;
    int live_parts = 0;                // graphs partitioned over this comm and not yet freed
    ncclComm_t nccl = nullptr;
    ag_local_group *group = nullptr;   // virtual mode
};

struct ag_local_group {
    int world = 0;
    int refs = 0;                      // live comms of the group
    std::vector<ag_graph_s *> parts;   // registered local graphs, index = rank
};

struct ag_dist_part {
    ag_comm_s *comm = nullptr;
    int world = 1;                     // copy of comm->world (the release path must not need the comm)
    uint32_t own_b = 0, own_e = 0;     // owned vertex range
    uint32_t S = 0;                    // slice size (bits), multiple of 1024
    uint32_t gwords = 0;               // words of the padded global bitmap (world * S / 32)
    uint32_t *d_front = nullptr;       // global frontier bitmap (gathered)
    uint32_t *d_next = nullptr;        // next-frontier bitmap (only owned words written)
    unsigned long long *d_cnt = nullptr;
    unsigned long long *h_cnt = nullptr;  // pinned
    unsigned *d_done = nullptr;        // BFS device-side termination: [0] frontier empty, [1] block arrivals,
                                       // [2] levels after the first, [3] |WS| of the next level
    unsigned *h_done = nullptr;        // pinned copy, read once per batch of enqueued levels
    uint32_t *d_trace = nullptr;       // per-level frontier sizes (stats)
    uint32_t trace_cap = 0;
    // SSSP exchange buffers (allocated on the first ag_dist_sssp)
    uint2 *d_send = nullptr;           // S entries: (owned improved vertex, its distance)
    uint2 *d_list = nullptr;           // world * S entries: the gathered global frontier
    unsigned *d_counts = nullptr;      // world x CW words per rank: (sent, carried, min pending dist, 0), gathered
    unsigned *h_counts = nullptr;      // pinned copy
    uint32_t *d_carry[2] = {nullptr, nullptr};   // owned pending vertices held back (hub window), double-buffered
    uint32_t *d_indeg = nullptr;       // in-degree of every owned vertex (all its in-edges live on this rank)
};
constexpr int CW = 4;                  // words per rank in the SSSP count exchange

namespace ag {

void dist_graph_release(ag_graph_s *g) {
    if (!g->dist) return;
    ag_dist_part *d = g->dist;
    dev_free(d->d_front, (size_t)d->gwords * 4 + 128, g->device);
    dev_free(d->d_next, (size_t)d->gwords * 4 + 128, g->device);
    dev_free(d->d_cnt, 64, g->device);
    if (d->h_cnt) cudaFreeHost(d->h_cnt);
    dev_free(d->d_done, 64, g->device);
    if (d->h_done) cudaFreeHost(d->h_done);
    dev_free(d->d_trace, (size_t)d->trace_cap * 4 + 64, g->device);
    const int W = d->world;
    if (d->comm) d->comm->live_parts -= 1;
    dev_free(d->d_send, (size_t)d->S * 8 + 128, g->device);
    dev_free(d->d_list, (size_t)W * d->S * 8 + 128, g->device);
    dev_free(d->d_counts, (size_t)W * CW * 4 + 128, g->device);
    if (d->h_counts) cudaFreeHost(d->h_counts);
    dev_free(d->d_carry[0], (size_t)d->S * 4 + 128, g->device);
    dev_free(d->d_carry[1], (size_t)d->S * 4 + 128, g->device);
    dev_free(d->d_indeg, (size_t)d->S * 4 + 128, g->device);
    delete d;
    g->dist = nullptr;
}

}  // namespace ag

using namespace ag;

// ------------------------------------------------------------------------------------------------
// kernels
// ------------------------------------------------------------------------------------------------
// count the owned entries of each row
// ---- partition extraction from a streamed global CSR (ag_dist_graph_load_csr): the global col_idx /
// weights arrive in chunks; each pass handles the CSR entries [e0, e1) of one chunk, whose rows are
// [ra, rb] (owner row of entry k: the largest u in [ra, rb] with rp[u] <= k).
__device__ __forceinline__ uint32_t chunk_owner(const uint64_t *rp, uint32_t ra, uint32_t rb, uint64_t k) {
    uint32_t lo = ra, hi = rb + 1;   // rp[lo] <= k < rp[hi]
    while (hi - lo > 1) {
        const uint32_t mid = lo + (hi - lo) / 2;
        if (rp[mid] <= k) lo = mid; else hi = mid;
    }
    return lo;
}

__global__ void dist_validate_rows_kernel(const uint64_t *rp, uint32_t V, uint64_t E, unsigned *bad) {
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < V; u += gridDim.x * blockDim.x)
        if (rp[u + 1] < rp[u]) *bad = 1u;
    if (blockIdx.x == 0 && threadIdx.x == 0 && (rp[0] != 0 || rp[V] != E)) *bad = 1u;
}

// pass 1: validate the chunk's entries (col < V, weight in [1, 2^31)) and count the owned ones per row
__global__ void dist_chunk_count_kernel(const uint64_t *rp, uint32_t V, const uint32_t *colc, const uint32_t *wc,
                                        uint64_t e0, uint64_t e1, uint32_t ra, uint32_t rb, uint32_t b, uint32_t e,
                                        unsigned long long *cnt, unsigned *bad) {
    unsigned bd = 0;
    for (uint64_t k = e0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < e1; k += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t c = colc[k - e0];
        if (c >= V) bd |= 2u;
        if (wc) {
            const uint32_t x = wc[k - e0];
            if (x == 0 || x >= 0x80000000u) bd |= 4u;
        }
        if (c >= b && c < e) atomicAdd(&cnt[chunk_owner(rp, ra, rb, k)], 1ull);
    }
    if (bd) atomicOr(bad, bd);
}

// pass 2: scatter the chunk's owned entries to their rows (order inside a row is not kept: rows need
// not be sorted, include/agraph.h)
__global__ void dist_chunk_scatter_kernel(const uint64_t *rp, const uint32_t *colc, const uint32_t *wc, uint64_t e0,
                                          uint64_t e1, uint32_t ra, uint32_t rb, uint32_t b, uint32_t e,
                                          unsigned long long *cursor, uint32_t *ncol, uint32_t *nw) {
    for (uint64_t k = e0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < e1; k += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t c = colc[k - e0];
        if (c >= b && c < e) {
            const unsigned long long pos = atomicAdd(&cursor[chunk_owner(rp, ra, rb, k)], 1ull);
            ncol[pos] = c;
            if (wc) nw[pos] = wc[k - e0];
        }
    }
}

__global__ void dist_init_kernel(uint32_t *level, uint32_t *parent, uint32_t *vis, uint32_t *front, uint32_t *next,
                                 uint32_t V, uint32_t gwords, uint32_t src) {
    const uint32_t gt = blockIdx.x * blockDim.x + threadIdx.x, gs = gridDim.x * blockDim.x;
    for (uint32_t v = gt; v < V; v += gs) {
        level[v] = v == src ? 0u : INF;
        if (parent) parent[v] = v == src ? src : INF;
    }
    for (uint32_t wi = gt; wi < gwords; wi += gs) {
        const uint32_t bit = (wi == (src >> 5)) ? (1u << (src & 31)) : 0u;
        vis[wi] = bit;
        front[wi] = bit;
        next[wi] = 0u;
    }
}

__global__ void owned_check_kernel(const uint32_t *col, uint64_t E, uint32_t b, uint32_t e, unsigned *bad) {
    for (uint64_t k = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < E; k += (uint64_t)gridDim.x * blockDim.x)
        if (col[k] < b || col[k] >= e) *bad = 1;
}

// After the exchange of a level: clear this rank's owned next slice, count the gathered frontier (every
// rank holds the same bitmap, so every rank takes the same decision), record |WS| of the next level
// and set done[0] when it is empty.  The last block to finish decides.
__global__ void dist_level_finish_kernel(const uint32_t *front, uint32_t gwords, uint32_t *next_owned, uint32_t owned_words,
                                         unsigned long long *cnt, unsigned *done, uint32_t *trace, uint32_t trace_cap) {
    __shared__ unsigned long long part[32];
    unsigned long long c = 0;
    for (uint32_t wi = blockIdx.x * blockDim.x + threadIdx.x; wi < gwords; wi += gridDim.x * blockDim.x) c += __popc(front[wi]);
    for (uint32_t wi = blockIdx.x * blockDim.x + threadIdx.x; wi < owned_words; wi += gridDim.x * blockDim.x) next_owned[wi] = 0u;
    c = warp_sum(c);
    if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = c;
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long t = 0;
        for (uint32_t i = 0; i < blockDim.x / 32; ++i) t += part[i];
        if (t) atomicAdd(cnt, t);
        __threadfence();
        if (atomicAdd(done + 1, 1u) == gridDim.x - 1) {
            __threadfence();
            const unsigned long long tot = *(volatile unsigned long long *)cnt;
            if (!*(volatile unsigned *)done) {
                done[3] = (unsigned)(tot > 0xFFFFFFFFull ? 0xFFFFFFFFull : tot);
                if (tot == 0) {
                    done[0] = 1u;
                } else {
                    done[2] += 1u;
                    if (trace && done[2] < trace_cap) trace[done[2]] = done[3];
                }
            }
            *cnt = 0ull;
            done[1] = 0u;
        }
    }
}

// One BFS level on one rank.  The decision maker (Fig. 11 / the tuned rule) runs on the gathered
// frontier's size (done[3], identical on every rank): for the queue working set the global frontier
// bitmap is compacted into a local queue (O(V/32)), for the bitmap working set the tiles are the
// bitmap's vertex ids directly (Fig. 9 line 1/2); either way the working set is expanded over the local
// (destination-owned) CSR with the selected mapping, and discovered owned vertices get their level and
// their bit in the next-frontier bitmap.  Device-side termination: a level launched after the frontier
// became empty (done[0], raised by the previous finish kernel) returns at once, so the host enqueues
// several levels without reading the frontier size.
template <typename Off>
__global__ void __launch_bounds__(BS, AG_MINB_BFS) dist_level_kernel(const TravArgs<Off> a, uint32_t L,
                                                                     const uint32_t *front, const unsigned *done) {
    if (*(volatile const unsigned *)done) return;
    __shared__ TileSmem<Off, wq_cap<ALG_BFS>()> sm;
    Ctl *ctl = a.ctl;
    const uint32_t slot = 0;
    const uint32_t gtid = blockIdx.x * BS + threadIdx.x, gthreads = a.nblocks * BS;
    const uint32_t n = *(volatile const unsigned *)(done + 3);
    const uint8_t var = select_variant(a.pol, n, 0);
    const uint32_t map = var >> 2, ws = var & 3u;
    uint32_t qn = 0, tile_n = BS, ntiles;
    if (ws == WS_QU) {
        compact_bitmap(front, a.nwords, a.q[0], &ctl->q_len[0], gtid >> 5, gthreads >> 5);
        grid_barrier(ctl, a.nblocks);
        qn = ld_relaxed(&ctl->q_len[0]);
        if (map != MAP_T) {
            tile_n = (qn + 2 * a.nblocks - 1) / (2 * a.nblocks);
            tile_n = tile_n < 1u ? 1u : (tile_n > (uint32_t)BS ? (uint32_t)BS : tile_n);
        }
        ntiles = (qn + tile_n - 1) / tile_n;
    } else {
        ntiles = (a.V + BS - 1) / BS;
    }
    Ops<ALG_BFS, ORD_O, Off> ops(a, L, 0, true);
    ops.wbuf = sm.wq[threadIdx.x >> 5];
    const bool hubs = (map == MAP_H) && a.has_hubs;
    const uint32_t s_idx = (map == MAP_W || (map == MAP_B && a.pol.cta_group == 32))
                               ? (lane_id() * WARPS_PER_CTA + (threadIdx.x >> 5)) : threadIdx.x;
    uint32_t t = blockIdx.x;
    int par = 0;
    while (t < ntiles) {
        if (threadIdx.x == 0) sm.tnext[par] = ntiles > a.nblocks ? a.nblocks + atomicAdd(&ctl->tile_ctr[slot], 1u) : ntiles;
        bool valid;
        uint32_t u;
        if (ws == WS_BM) {
            u = t * BS + threadIdx.x;
            valid = u < a.V && ((front[u >> 5] >> (u & 31)) & 1u);
        } else {
            const uint32_t i = t * tile_n + s_idx;
            valid = s_idx < tile_n && i < qn;
            u = valid ? a.q[0][i] : 0u;
        }
        if (__syncthreads_or(valid)) process_tile<false>(ops, sm, map, valid, u, a.pol.cta_group, hubs, slot);
        t = sm.tnext[par];
        par ^= 1;
    }
    if (hubs) drain_hubs(ops, sm, slot);
    ops.warp_flush(true);
    block_reduce_flush(ops, sm, ctl, slot);
}

// ---- multi-GPU SSSP on the same destination partition --------------------
// One unordered round (Fig. 5 unordered, 18.s30: every working-set node relaxes its out-edges) on one
// rank: the gathered global frontier is a LIST of (u, dist u) entries — the value travels with the
// entry because only u's owner holds P[u] — expanded over the local CSR (edges u -> v with v owned)
// with the hybrid mapping; an improved owned v gets its bit in the next bitmap (dedup) and is
// appended to the local next queue.  Padding entries have u = INF.
template <typename Off>
__global__ void __launch_bounds__(BS, AG_MINB_SSSP) dist_sssp_kernel(const TravArgs<Off> a, const uint2 *list,
                                                                     uint32_t n) {
    __shared__ TileSmem<Off, wq_cap<ALG_SSSP>()> sm;
    Ctl *ctl = a.ctl;
    const uint32_t slot = 0;
    Ops<ALG_SSSP, ORD_U, Off> ops(a, 0, ~0ull, true);   // it 0: next bitmap bm[1], next queue q[1]
    ops.wbuf = sm.wq[threadIdx.x >> 5];
    uint32_t tile_n = (n + 2 * a.nblocks - 1) / (2 * a.nblocks);
    tile_n = tile_n < 1u ? 1u : (tile_n > (uint32_t)BS ? (uint32_t)BS : tile_n);
    const uint32_t ntiles = (n + tile_n - 1) / tile_n;
    uint32_t t = blockIdx.x;
    int par = 0;
    while (t < ntiles) {
        if (threadIdx.x == 0) sm.tnext[par] = a.nblocks + atomicAdd(&ctl->tile_ctr[slot], 1u);
        const uint32_t i = t * tile_n + threadIdx.x;
        uint2 e = make_uint2(INF, INF);
        if (threadIdx.x < tile_n && i < n) e = list[i];
        const bool valid = e.x != INF;
        if (__syncthreads_or(valid))
            process_tile<true>(ops, sm, MAP_H, valid, valid ? e.x : 0u, 32u, a.has_hubs != 0, slot, e.y, i);
        t = sm.tnext[par];
        par ^= 1;
    }
    if (a.has_hubs) drain_hubs(ops, sm, slot);
    ops.warp_flush(true);
    block_reduce_flush(ops, sm, ctl, slot);
}

// The rank's contribution to the next global frontier, decided by the OWNER (so every rank expands the
// same list): its pending vertices are the ones held back last round (cin) and the ones improved in this
// round (q, deduplicated by the pending bitmap).  A pending vertex is sent as (v, dist v) — its latest
// distance — unless it is a hub (in-degree >= HUBW_DEG: re-expanding it re-scans its whole list on every
// rank) whose distance is at least `hi` = (global minimum pending distance of the last exchange) +
// hub window; those stay pending (cout, bit kept set).  Sent vertices leave the pending bitmap.
// cnt[0] = sent, cnt[1] = carried, cnt[2] = minimum pending distance (all zeroed / INF by the caller).
// The hub window only reorders work: the global minimum pending vertex is always sent next round.
__global__ void dist_sssp_collect_kernel(const uint32_t *cin, uint32_t ncin, const uint32_t *q, const unsigned *qlen,
                                         const unsigned long long *P, const uint32_t *indeg, uint32_t own_b,
                                         unsigned long long hi, uint32_t *pend_bm, uint2 *send, uint32_t *cout,
                                         unsigned *cnt) {
    const uint32_t nq = *qlen, tot = ncin + nq;
    uint32_t lmin = INF;
    const uint32_t gs = gridDim.x * blockDim.x;
    for (uint32_t i0 = blockIdx.x * blockDim.x; i0 < tot; i0 += gs) {   // warp-uniform trip count
        const uint32_t i = i0 + threadIdx.x;
        bool ok = i < tot, snd = false;
        uint32_t v = 0, dv = INF;
        if (ok) {
            v = i < ncin ? cin[i] : q[i - ncin];
            dv = (uint32_t)(P[v] >> 32);
            lmin = min(lmin, dv);
            snd = indeg[v - own_b] < HUBW_DEG || (unsigned long long)dv < hi;
        }
        const unsigned ms = __ballot_sync(0xffffffffu, ok && snd), mc = __ballot_sync(0xffffffffu, ok && !snd);
        const unsigned lane = threadIdx.x & 31u, below = (1u << lane) - 1u;
        uint32_t bs = 0, bc = 0;
        if (lane == 0) {
            if (ms) bs = atomicAdd(&cnt[0], (unsigned)__popc(ms));
            if (mc) bc = atomicAdd(&cnt[1], (unsigned)__popc(mc));
        }
        bs = __shfl_sync(0xffffffffu, bs, 0);
        bc = __shfl_sync(0xffffffffu, bc, 0);
        if (ok && snd) {
            send[bs + __popc(ms & below)] = make_uint2(v, dv);
            atomicAnd(&pend_bm[v >> 5], ~(1u << (v & 31)));
        } else if (ok) {
            cout[bc + __popc(mc & below)] = v;
        }
    }
    lmin = warp_min(lmin);
    if ((threadIdx.x & 31u) == 0 && lmin != INF) atomicMin(&cnt[2], lmin);
}

// in-degree of the owned vertices: every CSR entry of this rank has an owned destination
__global__ void dist_indeg_kernel(const uint32_t *col, unsigned long long E, uint32_t own_b, uint32_t *indeg) {
    for (unsigned long long e = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; e < E;
         e += (unsigned long long)gridDim.x * blockDim.x)
        atomicAdd(&indeg[col[e] - own_b], 1u);
}

__global__ void dist_sssp_init_kernel(unsigned long long *P, uint32_t *next_bm, uint32_t V, uint32_t gwords,
                                      uint32_t src, uint32_t own_b, uint32_t own_e) {
    const uint32_t gt = blockIdx.x * blockDim.x + threadIdx.x, gs = gridDim.x * blockDim.x;
    for (uint32_t v = gt; v < V; v += gs)
        P[v] = (v == src && src >= own_b && src < own_e) ? (unsigned long long)src : INF64;   // dist 0, parent src
    for (uint32_t wi = gt; wi < gwords; wi += gs) next_bm[wi] = 0u;
}

// owned slice -> caller arrays: dist, parent (INF for unreached)
__global__ void dist_sssp_out_kernel(const unsigned long long *P, uint32_t b, uint32_t e, uint32_t *dist,
                                     uint32_t *parent) {
    for (uint32_t v = b + blockIdx.x * blockDim.x + threadIdx.x; v < e; v += gridDim.x * blockDim.x) {
        const unsigned long long pv = P[v];
        dist[v - b] = (uint32_t)(pv >> 32);
        if (parent) parent[v - b] = pv == INF64 ? INF : (uint32_t)pv;
    }
}

// ------------------------------------------------------------------------------------------------
// host side
// ------------------------------------------------------------------------------------------------
namespace {

ag_status part_alloc(ag_graph_s *g, ag_comm_s *c) {
    ag_dist_part *d = new ag_dist_part();
    d->comm = c;
    d->world = c->world;
    c->live_parts += 1;
    ag_dist_owned_range(g->V, c->rank, c->world, &d->own_b, &d->own_e);
    uint64_t S = ((uint64_t)g->V + c->world - 1) / c->world;
    S = (S + 1023) & ~1023ull;
    d->S = (uint32_t)S;
    d->gwords = (uint32_t)(S * c->world / 32);
    g->dist = d;
    ag_status s;
    if ((s = dev_alloc((void **)&d->d_front, (size_t)d->gwords * 4 + 128, g->device)) != AG_OK) return s;
    if ((s = dev_alloc((void **)&d->d_next, (size_t)d->gwords * 4 + 128, g->device)) != AG_OK) return s;
    if ((s = dev_alloc((void **)&d->d_cnt, 64, g->device)) != AG_OK) return s;
    if (cudaMallocHost(&d->h_cnt, 64) != cudaSuccess) return set_error(AG_ERR_OOM, "pinned alloc");
    if ((s = dev_alloc((void **)&d->d_done, 64, g->device)) != AG_OK) return s;
    if (cudaMallocHost(&d->h_done, 64) != cudaSuccess) return set_error(AG_ERR_OOM, "pinned alloc");
    return AG_OK;
}

// scratch the level kernel needs (same layout as the single-GPU handle; bitmaps sized to gwords)
ag_status dist_scratch(ag_graph_s *g) {
    ag_status s;
    const size_t V = g->V, gw = g->dist->gwords;
    if (!g->d_ctl) {
        if ((s = dev_alloc(&g->d_ctl, sizeof(Ctl), g->device)) != AG_OK) return s;
        cudaMemset(g->d_ctl, 0, sizeof(Ctl));
        g->ctl_init = true;
    }
    if (!g->d_q[0] && (s = dev_alloc((void **)&g->d_q[0], V * 4 + 128, g->device)) != AG_OK) return s;
    if (!g->d_q[1] && (s = dev_alloc((void **)&g->d_q[1], V * 4 + 128, g->device)) != AG_OK) return s;
    if (!g->d_vis && (s = dev_alloc((void **)&g->d_vis, gw * 4 + 128, g->device)) != AG_OK) return s;
    if (!g->d_hub) {
        if ((s = dev_alloc((void **)&g->d_hub, (size_t)g->hub_cap * 8, g->device)) != AG_OK) return s;
        cudaMemset(g->d_hub, 0, (size_t)g->hub_cap * 8);
    }
    if (!g->d_level && (s = dev_alloc((void **)&g->d_level, V * 4 + 128, g->device)) != AG_OK) return s;
    if (!g->d_acc && (s = dev_alloc(&g->d_acc, 64, g->device)) != AG_OK) return s;
    return AG_OK;
}

struct LevelCfg {
    int nblocks = 0;
};

template <typename Off>
ag_status launch_level(ag_graph_s *g, uint32_t L, uint32_t *parent_local, const ag_policy &pol, cudaStream_t st) {
    ag_dist_part *d = g->dist;
    TravArgs<Off> a;
    memset(&a, 0, sizeof a);
    a.pol = resolve_policy(pol, *g);
    a.rp = (const Off *)g->d_rp;
    a.col = g->d_col;
    a.V = g->V;
    a.nwords = d->gwords;
    a.level = g->d_level;
    a.parent = parent_local;
    a.vis = g->d_vis;
    a.bm[0] = a.bm[1] = a.bm[2] = d->d_next;
    a.q[0] = g->d_q[0];
    a.q[1] = a.q[2] = g->d_q[1];   // appends of the expansion (not consumed: the bitmap is exchanged)
    a.hub = g->d_hub;
    a.hub_cap = g->hub_cap;
    a.ctl = (Ctl *)g->d_ctl;
    a.has_hubs = g->info.max_deg >= HUB_DEG;
    auto fn = dist_level_kernel<Off>;
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, BS, 0);
    if (occ < 1) return set_error(AG_ERR_CUDA, "dist kernel does not fit");
    a.nblocks = (uint32_t)(occ * g->num_sms);
    // reset the per-level counters of slot 0/1 (q_len, tile/hub scheduler)
    cudaMemsetAsync((char *)g->d_ctl + offsetof(Ctl, q_len), 0, offsetof(Ctl, it_edges) - offsetof(Ctl, q_len), st);
    const unsigned *done = d->d_done;
    void *args[] = {(void *)&a, (void *)&L, (void *)&d->d_front, (void *)&done};
    cudaError_t e = cudaLaunchCooperativeKernel((const void *)fn, dim3(a.nblocks), dim3(BS), args, 0, st);
    note_launch(1);
    return cuda_status(e, "dist level");
}

// SSSP scratch: packed state P (V), exchange buffers
ag_status dist_sssp_scratch(ag_graph_s *g) {
    ag_status s;
    ag_dist_part *d = g->dist;
    const int W = d->comm->world;
    if (!g->d_P && (s = dev_alloc((void **)&g->d_P, (size_t)g->V * 8 + 128, g->device)) != AG_OK) return s;
    if (!d->d_send && (s = dev_alloc((void **)&d->d_send, (size_t)d->S * 8 + 128, g->device)) != AG_OK) return s;
    if (!d->d_list && (s = dev_alloc((void **)&d->d_list, (size_t)W * d->S * 8 + 128, g->device)) != AG_OK) return s;
    if (!d->d_counts && (s = dev_alloc((void **)&d->d_counts, (size_t)W * CW * 4 + 128, g->device)) != AG_OK) return s;
    if (!d->h_counts && cudaMallocHost(&d->h_counts, (size_t)W * CW * 4 + 64) != cudaSuccess)
        return set_error(AG_ERR_OOM, "pinned alloc");
    for (int k = 0; k < 2; ++k)
        if (!d->d_carry[k] && (s = dev_alloc((void **)&d->d_carry[k], (size_t)d->S * 4 + 128, g->device)) != AG_OK) return s;
    if (!d->d_indeg) {
        if ((s = dev_alloc((void **)&d->d_indeg, (size_t)d->S * 4 + 128, g->device)) != AG_OK) return s;
        cudaMemset(d->d_indeg, 0, (size_t)d->S * 4 + 128);
        if (g->E) dist_indeg_kernel<<<g->num_sms * 8, 256>>>(g->d_col, g->E, d->own_b, d->d_indeg);
        note_launch(1);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) return cuda_status(e, "in-degrees");
    }
    return AG_OK;
}

template <typename Off>
ag_status launch_sssp_round(ag_graph_s *g, const uint2 *list, uint32_t n, uint32_t ncin, int cpar,
                            unsigned long long hi, cudaStream_t st) {
    ag_dist_part *d = g->dist;
    TravArgs<Off> a;
    memset(&a, 0, sizeof a);
    a.rp = (const Off *)g->d_rp;
    a.cw = g->d_cw;
    a.V = g->V;
    a.nwords = d->gwords;
    a.P = g->d_P;
    a.bm[0] = a.bm[1] = a.bm[2] = d->d_next;
    a.q[0] = a.q[2] = g->d_q[0];
    a.q[1] = g->d_q[1];
    a.hub = g->d_hub;
    a.hub_cap = g->hub_cap;
    a.ctl = (Ctl *)g->d_ctl;
    a.has_hubs = g->info.max_deg >= HUB_DEG;
    a.ulist = list;
    auto fn = dist_sssp_kernel<Off>;
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, BS, 0);
    if (occ < 1) return set_error(AG_ERR_CUDA, "dist sssp kernel does not fit");
    a.nblocks = (uint32_t)(occ * g->num_sms);
    cudaMemsetAsync((char *)g->d_ctl + offsetof(Ctl, q_len), 0, offsetof(Ctl, it_edges) - offsetof(Ctl, q_len), st);
    void *args[] = {(void *)&a, (void *)&list, (void *)&n};
    cudaError_t e = cudaLaunchCooperativeKernel((const void *)fn, dim3(a.nblocks), dim3(BS), args, 0, st);
    note_launch(1);
    if (e != cudaSuccess) return cuda_status(e, "dist sssp round");
    unsigned *cnt = d->d_counts + (size_t)d->comm->rank * CW;
    cudaMemsetAsync(cnt, 0, 8, st);
    cudaMemsetAsync(cnt + 2, 0xFF, 4, st);
    dist_sssp_collect_kernel<<<g->num_sms * 2, 256, 0, st>>>(d->d_carry[cpar], ncin, g->d_q[1], &((Ctl *)g->d_ctl)->q_len[1],
                                                             g->d_P, d->d_indeg, d->own_b, hi, d->d_next, d->d_send,
                                                             d->d_carry[cpar ^ 1], cnt);
    note_launch(1);
    return cuda_status(cudaGetLastError(), "dist sssp collect");
}

ag_status run_sssp_round(ag_graph_s *g, const uint2 *list, uint32_t n, uint32_t ncin, int cpar, unsigned long long hi,
                         cudaStream_t st) {
    return g->offs32 ? launch_sssp_round<uint32_t>(g, list, n, ncin, cpar, hi, st)
                     : launch_sssp_round<unsigned long long>(g, list, n, ncin, cpar, hi, st);
}

ag_status run_level(ag_graph_s *g, uint32_t L, uint32_t *parent_local, const ag_policy &pol, cudaStream_t st) {
    return g->offs32 ? launch_level<uint32_t>(g, L, parent_local, pol, st)
                     : launch_level<unsigned long long>(g, L, parent_local, pol, st);
}

}  // namespace

// ------------------------------------------------------------------------------------------------
// C ABI
// ------------------------------------------------------------------------------------------------
extern "C" {

ag_status ag_dist_owned_range(uint32_t V, int rank, int world, uint32_t *begin, uint32_t *end) {
    if (!begin || !end || world < 1 || rank < 0 || rank >= world)
        return ag::set_error(AG_ERR_INVALID_ARG, "bad rank/world");
    uint64_t S = ((uint64_t)V + world - 1) / world;
    S = (S + 1023) & ~1023ull;  // whole, 128-B aligned bitmap slices
    uint64_t b = S * (uint64_t)rank, e = b + S;
    if (b > V) b = V;
    if (e > V) e = V;
    *begin = (uint32_t)b;
    *end = (uint32_t)e;
    return AG_OK;
}

ag_status ag_dist_unique_id(void *out128) {
    if (!out128) return set_error(AG_ERR_INVALID_ARG, "NULL");
    if (!load_nccl()) return set_error(AG_ERR_NCCL, "cannot load libnccl.so.2 (set AG_NCCL_LIB)");
    ncclUniqueId id;
    ag_status s = nccl_status(g_nccl.GetUniqueId(&id), "ncclGetUniqueId");
    if (s == AG_OK) memcpy(out128, &id, sizeof id);
    return s;
}

ag_status ag_dist_init(int rank, int world, const void *id128, int device, ag_comm *out) {
    if (!out || !id128 || world < 1 || rank < 0 || rank >= world) return set_error(AG_ERR_INVALID_ARG, "bad args");
    ag_status s = check_device(device, nullptr);
    if (s != AG_OK) return s;
    if (!load_nccl()) return set_error(AG_ERR_NCCL, "cannot load libnccl.so.2 (set AG_NCCL_LIB)");
    cudaSetDevice(device);
    ncclUniqueId id;
    memcpy(&id, id128, sizeof id);
    ag_comm_s *c = new ag_comm_s();
    c->rank = rank;
    c->world = world;
    c->device = device;
    s = nccl_status(g_nccl.CommInitRank(&c->nccl, world, id, rank), "ncclCommInitRank");
    if (s != AG_OK) {
        delete c;
        return s;
    }
    *out = c;
    return AG_OK;
}

ag_status ag_dist_init_local(int world, int device, ag_comm *comms_out) {
    if (!comms_out || world < 1) return set_error(AG_ERR_INVALID_ARG, "bad args");
    ag_status s = check_device(device, nullptr);
    if (s != AG_OK) return s;
    ag_local_group *grp = new ag_local_group();
    grp->world = world;
    grp->refs = world;
    grp->parts.assign(world, nullptr);
    for (int r = 0; r < world; ++r) {
        ag_comm_s *c = new ag_comm_s();
        c->rank = r;
        c->world = world;
        c->device = device;
        c->group = grp;
        comms_out[r] = c;
    }
    return AG_OK;
}

ag_status ag_dist_free(ag_comm c) {
    if (!c) return set_error(AG_ERR_INVALID_ARG, "NULL");
    if (c->live_parts > 0)
        return set_error(AG_ERR_INVALID_ARG, "ag_dist_free: %d graph(s) partitioned over this comm are still live; "
                         "ag_graph_free them first", c->live_parts);
    if (c->nccl && g_nccl.ok) g_nccl.CommDestroy(c->nccl);
    if (c->group) {
        c->group->parts[c->rank] = nullptr;
        if (--c->group->refs == 0) delete c->group;
    }
    delete c;
    return AG_OK;
}

ag_status ag_dist_graph_load_csr(ag_comm c, uint32_t V, uint64_t E, const uint64_t *row_ptr, const uint32_t *col_idx,
                                 const uint32_t *weights, ag_graph *out_local) {
    if (!c || !out_local || !row_ptr || (!col_idx && E)) return set_error(AG_ERR_INVALID_ARG, "NULL argument");
    *out_local = nullptr;
    if (V == 0 || V >= 0xFFFFFFFFu) return set_error(AG_ERR_BAD_CSR, "V must be in [1, 2^32-1)");
    if (V >= 0x80000000u) return set_error(AG_ERR_UNSUPPORTED, "ag_dist_graph_load_csr needs V < 2^31 (31-bit scan)");
    const int dev = c->device;
    int sms = 0;
    ag_status s = check_device(dev, &sms);
    if (s != AG_OK) return s;
    cudaSetDevice(dev);
    uint32_t b, e;
    ag_dist_owned_range(V, c->rank, c->world, &b, &e);
    // The global CSR is never held on the device: the row offsets are copied once, col_idx / weights
    // stream through two chunk buffers twice — pass 1 validates and counts the owned entries per row,
    // pass 2 scatters them — so device memory holds the row offsets, the chunk buffers and the owned
    // part only (C5 / 8 ranks: ~3.5 GB instead of the ~34 GB of a staged global graph).
    const uint64_t CH = 1ull << 24;
    const size_t rpb = (size_t)(V + 1) * 8;
    uint64_t *rp64 = nullptr, *rph = nullptr;
    unsigned long long *cnt = nullptr, *nrp = nullptr;
    uint32_t *colc = nullptr, *wc = nullptr, *ncol = nullptr, *nw = nullptr;
    unsigned *bad = nullptr;
    void *tmp = nullptr;
    size_t tb = 0;
    uint64_t El = 0;
    auto cleanup = [&]() {
        dev_free(rp64, rpb, dev);
        dev_free(cnt, rpb, dev);
        dev_free(nrp, rpb, dev);
        dev_free(colc, CH * 4, dev);
        dev_free(wc, CH * 4, dev);
        dev_free(ncol, El * 4 + 128, dev);
        dev_free(nw, El * 4 + 128, dev);
        dev_free(bad, 16, dev);
        dev_free(tmp, tb, dev);
        free(rph);
    };
    auto fail = [&](ag_status st) { cleanup(); return st; };
    if ((s = dev_alloc((void **)&rp64, rpb, dev)) != AG_OK) return fail(s);
    if ((s = dev_alloc((void **)&cnt, rpb, dev)) != AG_OK) return fail(s);
    if ((s = dev_alloc((void **)&nrp, rpb, dev)) != AG_OK) return fail(s);
    if ((s = dev_alloc((void **)&bad, 16, dev)) != AG_OK) return fail(s);
    if (E && (s = dev_alloc((void **)&colc, CH * 4, dev)) != AG_OK) return fail(s);
    if (E && weights && (s = dev_alloc((void **)&wc, CH * 4, dev)) != AG_OK) return fail(s);
    rph = (uint64_t *)malloc(rpb);   // chunk -> row ranges are found on the host
    if (!rph) return fail(set_error(AG_ERR_OOM, "host row_ptr copy"));
    cudaError_t ce = cudaMemcpy(rph, row_ptr, rpb, cudaMemcpyDefault);
    if (ce == cudaSuccess) ce = cudaMemcpy(rp64, rph, rpb, cudaMemcpyHostToDevice);
    if (ce == cudaSuccess) ce = cudaMemset(bad, 0, 16);
    if (ce == cudaSuccess) ce = cudaMemset(cnt, 0, rpb);
    if (ce != cudaSuccess) return fail(cuda_status(ce, "dist partition"));
    dist_validate_rows_kernel<<<sms * 4, 256>>>(rp64, V, E, bad);
    note_launch(1);
    unsigned hbad = 0;
    ce = cudaMemcpy(&hbad, bad, 4, cudaMemcpyDeviceToHost);
    if (ce != cudaSuccess) return fail(cuda_status(ce, "dist partition"));
    if (hbad) return fail(set_error(AG_ERR_BAD_CSR, "invalid CSR (row offsets)"));
    auto rows_of = [&](uint64_t e0, uint64_t e1, uint32_t &ra, uint32_t &rb) {   // rows touching [e0, e1)
        uint32_t lo = 0, hi = V;   // ra: first u with rp[u+1] > e0
        while (lo < hi) {
            const uint32_t mid = lo + (hi - lo) / 2;
            if (rph[mid + 1] > e0) hi = mid; else lo = mid + 1;
        }
        ra = lo;
        lo = ra;
        hi = V;   // rb: last u with rp[u] < e1
        while (lo < hi) {
            const uint32_t mid = lo + (hi - lo + 1) / 2;
            if (rph[mid] < e1) lo = mid; else hi = mid - 1;
        }
        rb = lo;
    };
    for (int pass = 0; pass < 2; ++pass) {
        if (pass == 1) {   // owned-entry offsets, then the owned part's arrays
            cub::DeviceScan::ExclusiveSum(nullptr, tb, cnt, nrp, (int)V + 1);
            if ((s = dev_alloc(&tmp, tb, dev)) != AG_OK) return fail(s);
            cub::DeviceScan::ExclusiveSum(tmp, tb, cnt, nrp, (int)V + 1);
            ce = cudaMemcpy(&El, nrp + V, 8, cudaMemcpyDeviceToHost);
            if (ce != cudaSuccess) return fail(cuda_status(ce, "dist partition"));
            if ((s = dev_alloc((void **)&ncol, El * 4 + 128, dev)) != AG_OK) return fail(s);
            if (weights && (s = dev_alloc((void **)&nw, El * 4 + 128, dev)) != AG_OK) return fail(s);
            ce = cudaMemcpy(cnt, nrp, rpb, cudaMemcpyDeviceToDevice);   // cnt = per-row write cursor
            if (ce != cudaSuccess) return fail(cuda_status(ce, "dist partition"));
        }
        for (uint64_t e0 = 0; e0 < E; e0 += CH) {
            const uint64_t e1 = (E - e0 > CH) ? e0 + CH : E;
            uint32_t ra, rb;
            rows_of(e0, e1, ra, rb);
            ce = cudaMemcpy(colc, col_idx + e0, (e1 - e0) * 4, cudaMemcpyDefault);
            if (ce == cudaSuccess && weights) ce = cudaMemcpy(wc, weights + e0, (e1 - e0) * 4, cudaMemcpyDefault);
            if (ce != cudaSuccess) return fail(cuda_status(ce, "dist partition copy"));
            if (pass == 0)
                dist_chunk_count_kernel<<<sms * 8, 256>>>(rp64, V, colc, weights ? wc : nullptr, e0, e1, ra, rb, b, e, cnt, bad);
            else
                dist_chunk_scatter_kernel<<<sms * 8, 256>>>(rp64, colc, weights ? wc : nullptr, e0, e1, ra, rb, b, e, cnt, ncol, nw);
            note_launch(1);
        }
        if (pass == 0) {
            ce = cudaMemcpy(&hbad, bad, 4, cudaMemcpyDeviceToHost);
            if (ce != cudaSuccess) return fail(cuda_status(ce, "dist partition"));
            if (hbad)
                return fail(set_error(AG_ERR_BAD_CSR, "invalid CSR (%s%s)", hbad & 2 ? "col>=V " : "",
                                      hbad & 4 ? "weight not in [1,2^31) " : ""));
        }
    }
    ce = cudaDeviceSynchronize();
    if (ce != cudaSuccess) return fail(cuda_status(ce, "dist partition"));
    // the local part is an ordinary graph handle (rows over all V, owned destinations only)
    ag_graph gl = nullptr;
    s = ag_graph_load_csr_ex(V, El, (const uint64_t *)nrp, ncol, nw, dev, AG_LAYOUT_IDENTITY, &gl);
    cleanup();
    if (s != AG_OK) return s;
    if ((s = part_alloc(gl, c)) != AG_OK) { ag_graph_free(gl); return s; }
    if (c->group) c->group->parts[c->rank] = gl;
    *out_local = gl;
    return AG_OK;
}

ag_status ag_dist_graph_load_local(ag_comm c, uint32_t V, uint64_t E_local, const uint64_t *row_ptr,
                                   const uint32_t *col_idx, const uint32_t *weights, ag_graph *out_local) {
    if (!c || !out_local) return set_error(AG_ERR_INVALID_ARG, "NULL argument");
    *out_local = nullptr;
    ag_graph gl = nullptr;
    ag_status s = ag_graph_load_csr_ex(V, E_local, row_ptr, col_idx, weights, c->device, AG_LAYOUT_IDENTITY, &gl);
    if (s != AG_OK) return s;
    uint32_t b, e;
    ag_dist_owned_range(V, c->rank, c->world, &b, &e);
    unsigned *bad = nullptr;
    if ((s = dev_alloc((void **)&bad, 16, c->device)) != AG_OK) { ag_graph_free(gl); return s; }
    cudaMemset(bad, 0, 4);
    if (E_local) owned_check_kernel<<<gl->num_sms * 4, 256>>>(gl->d_col, E_local, b, e, bad);
    note_launch(1);
    unsigned h = 0;
    cudaMemcpy(&h, bad, 4, cudaMemcpyDeviceToHost);
    dev_free(bad, 16, c->device);
    if (h) { ag_graph_free(gl); return set_error(AG_ERR_BAD_CSR, "local CSR has a destination outside [%u, %u)", b, e); }
    if ((s = part_alloc(gl, c)) != AG_OK) { ag_graph_free(gl); return s; }
    if (c->group) c->group->parts[c->rank] = gl;
    *out_local = gl;
    return AG_OK;
}

}  // extern "C"

namespace {

// Lock-step driver over the participating ranks of THIS process (1 rank for NCCL, all for a group).
// Device-side termination: per level the host ENQUEUES [level kernel, exchange, finish kernel] without
// looking at the frontier; the finish kernel counts the gathered frontier on the device and raises
// d_done when it is empty, after which the level kernels of later enqueued levels return at once.  The
// host reads d_done once per BATCH of levels (4, doubling up to 64), not once per level.
ag_status dist_bfs_driver(std::vector<ag_graph_s *> &parts, uint32_t src, uint32_t **levels_owned,
                          uint32_t **parents_owned, const ag_policy *pin, ag_run_stats *stats, cudaStream_t st) {
    const int P = (int)parts.size();
    ag_status s;
    ag_policy pol;
    if (pin) {
        pol = *pin;
    } else if ((s = ag_policy_default(&pol, parts[0]->device)) != AG_OK) {
        return s;
    }
    if ((s = check_policy(&pol)) != AG_OK) return s;
    const uint32_t tcap = stats && stats->trace_ws ? stats->trace_cap : 0;
    for (auto *g : parts) {
        cudaSetDevice(g->device);
        if ((s = dist_scratch(g)) != AG_OK) return s;
        if (parents_owned && !g->d_lpar && (s = dev_alloc((void **)&g->d_lpar, (size_t)g->V * 4 + 128, g->device)) != AG_OK)
            return s;
        ag_dist_part *d = g->dist;
        if (tcap > d->trace_cap) {
            dev_free(d->d_trace, (size_t)d->trace_cap * 4 + 64, g->device);
            d->d_trace = nullptr;
            d->trace_cap = 0;
            if ((s = dev_alloc((void **)&d->d_trace, (size_t)tcap * 4 + 64, g->device)) != AG_OK) return s;
            d->trace_cap = tcap;
        }
    }
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    if (stats) {
        cudaEventCreate(&e0);
        cudaEventCreate(&e1);
        cudaEventRecord(e0, st);
    }
    const uint32_t V = parts[0]->V;
    static const uint32_t one = 1u;
    for (auto *g : parts) {
        ag_dist_part *d = g->dist;
        dist_init_kernel<<<g->num_sms * 4, 256, 0, st>>>(g->d_level, parents_owned ? g->d_lpar : nullptr, g->d_vis,
                                                        d->d_front, d->d_next, V, d->gwords, src);
        cudaMemsetAsync(g->d_ctl, 0, offsetof(Ctl, q_len), st);   // no-op for the barrier word (self-resetting)
        cudaMemsetAsync((char *)g->d_ctl + offsetof(Ctl, vexp), 0, 16, st);
        cudaMemsetAsync(d->d_done, 0, 12, st);
        cudaMemcpyAsync(d->d_done + 3, &one, 4, cudaMemcpyHostToDevice, st);   // |WS_0| = |{src}|
        cudaMemsetAsync(d->d_cnt, 0, 8, st);
        if (tcap) cudaMemcpyAsync(d->d_trace, &one, 4, cudaMemcpyHostToDevice, st);
        note_launch(1);
    }
    uint32_t L = 0, batch = 4;
    bool fin = false;
    while (!fin) {
        for (uint32_t k = 0; k < batch; ++k, ++L) {
            for (auto *g : parts)
                if ((s = run_level(g, L, parents_owned ? g->d_lpar : nullptr, pol, st)) != AG_OK) return s;
            // exchange: every rank contributes its owned slice of the next bitmap
            if (P == 1 && parts[0]->dist->comm->nccl) {
                ag_graph_s *g = parts[0];
                ag_dist_part *d = g->dist;
                ncclResult_t r = g_nccl.AllGather(d->d_next + (size_t)d->comm->rank * (d->S / 32), d->d_front, d->S / 8,
                                                  ncclUint8, d->comm->nccl, st);
                if ((s = nccl_status(r, "ncclAllGather")) != AG_OK) return s;
            } else {
                for (auto *gd : parts) {
                    for (auto *gs : parts) {
                        ag_dist_part *dd = gd->dist, *ds = gs->dist;
                        const size_t off = (size_t)ds->comm->rank * (ds->S / 32);
                        cudaMemcpyAsync(dd->d_front + off, ds->d_next + off, ds->S / 8, cudaMemcpyDeviceToDevice, st);
                    }
                }
            }
            // every rank: clear its owned next slice, count the gathered frontier, decide termination
            for (auto *g : parts) {
                ag_dist_part *d = g->dist;
                dist_level_finish_kernel<<<g->num_sms, 256, 0, st>>>(d->d_front, d->gwords,
                                                                   d->d_next + (size_t)d->comm->rank * (d->S / 32), d->S / 32,
                                                                   d->d_cnt, d->d_done, tcap ? d->d_trace : nullptr, tcap);
                note_launch(1);
            }
        }
        ag_dist_part *d0 = parts[0]->dist;
        cudaMemcpyAsync(d0->h_done, d0->d_done, 16, cudaMemcpyDeviceToHost, st);
        cudaError_t ce = cudaStreamSynchronize(st);
        if (ce != cudaSuccess) return cuda_status(ce, "dist level");
        fin = d0->h_done[0] != 0;
        if (!fin && L > V + 1) return set_error(AG_ERR_CUDA, "dist bfs did not terminate");
        batch = batch < 64 ? 2 * batch : 64;
    }
    const uint32_t levels = parts[0]->dist->h_done[2] + 1;   // nonempty frontiers, {src} included
    // outputs: owned slices of level / parent
    for (int r = 0; r < P; ++r) {
        ag_graph_s *g = parts[r];
        ag_dist_part *d = g->dist;
        const size_t n = d->own_e - d->own_b;
        if (levels_owned && levels_owned[r] && n)
            cudaMemcpyAsync(levels_owned[r], g->d_level + d->own_b, n * 4, cudaMemcpyDefault, st);
        if (parents_owned && parents_owned[r] && n)
            cudaMemcpyAsync(parents_owned[r], g->d_lpar + d->own_b, n * 4, cudaMemcpyDefault, st);
    }
    if (stats) cudaEventRecord(e1, st);
    cudaError_t ce = cudaStreamSynchronize(st);
    if (ce != cudaSuccess) return cuda_status(ce, "dist bfs");
    if (stats) {
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        cudaEventDestroy(e0);
        cudaEventDestroy(e1);
        stats->iterations = levels;
        stats->device_ms = ms;
        unsigned long long vx = 0, ex = 0;
        for (auto *g : parts) {
            Ctl c;
            cudaMemcpy(&c, g->d_ctl, sizeof c, cudaMemcpyDeviceToHost);
            vx += c.vexp;
            ex += c.eexp;
        }
        stats->vertices_expanded = vx;  // summed over the ranks of this process
        stats->edges_inspected = ex;
        const uint32_t n = levels < tcap ? levels : tcap;
        stats->trace_len = n;
        if (n) cudaMemcpy(stats->trace_ws, parts[0]->dist->d_trace, (size_t)n * 4, cudaMemcpyDeviceToHost);
    }
    return AG_OK;
}

// Lock-step unordered SSSP over the participating ranks of THIS process.  Per round: every rank
// expands the same gathered list, collects its improved owned vertices, the per-rank counts are
// all-gathered (termination: all zero), then the (v, dist) lists padded to the largest count.
ag_status dist_sssp_driver(std::vector<ag_graph_s *> &parts, uint32_t src, uint32_t **dist_owned,
                           uint32_t **parents_owned, ag_run_stats *stats, cudaStream_t st,
                           uint32_t hub_window) {
    const int P = (int)parts.size();
    ag_status s;
    for (auto *g : parts) {
        cudaSetDevice(g->device);
        if (!g->d_cw) return set_error(AG_ERR_NO_WEIGHTS, "SSSP on an unweighted distributed graph");
        if ((s = dist_scratch(g)) != AG_OK) return s;
        if ((s = dist_sssp_scratch(g)) != AG_OK) return s;
    }
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    if (stats) {
        cudaEventCreate(&e0);
        cudaEventCreate(&e1);
        cudaEventRecord(e0, st);
    }
    const uint32_t V = parts[0]->V;
    const int world = parts[0]->dist->comm->world;
    const bool nccl = P == 1 && parts[0]->dist->comm->nccl;
    const uint2 first = make_uint2(src, 0u);
    for (auto *g : parts) {
        ag_dist_part *d = g->dist;
        dist_sssp_init_kernel<<<g->num_sms * 4, 256, 0, st>>>(g->d_P, d->d_next, V, d->gwords, src, d->own_b, d->own_e);
        cudaMemsetAsync(g->d_ctl, 0, offsetof(Ctl, q_len), st);
        cudaMemsetAsync((char *)g->d_ctl + offsetof(Ctl, vexp), 0, 16, st);
        cudaMemsetAsync((char *)g->d_ctl + offsetof(Ctl, overflow), 0, 4, st);
        cudaMemcpyAsync(d->d_list, &first, sizeof first, cudaMemcpyHostToDevice, st);
        note_launch(1);
    }
    uint32_t n = 1, R = 0;   // entries of the gathered list (with padding), rounds
    uint64_t front = 1;      // real entries
    const uint32_t tcap = stats ? stats->trace_cap : 0;
    // owner-side hub window: hi = (global minimum pending distance) + hub_window; 0 = off (send all)
    unsigned long long hi = hub_window ? (unsigned long long)hub_window : ~0ull;
    int cpar = 0;                               // carry buffer read this round
    std::vector<uint32_t> ncin(P, 0u);          // carried (held-back) entries per local part
    for (;; ++R) {
        if (stats && R < tcap && stats->trace_ws) stats->trace_ws[R] = (uint32_t)front;
        for (int r = 0; r < P; ++r)
            if ((s = run_sssp_round(parts[r], parts[r]->dist->d_list, n, ncin[r], cpar, hi, st)) != AG_OK) return s;
        // counts: every rank's (sent, carried, min pending) to every rank
        if (nccl) {
            ag_dist_part *d = parts[0]->dist;
            ncclResult_t r = g_nccl.AllGather(d->d_counts + (size_t)d->comm->rank * CW, d->d_counts, CW, ncclUint32,
                                              d->comm->nccl, st);
            if ((s = nccl_status(r, "ncclAllGather(counts)")) != AG_OK) return s;
        } else {
            for (auto *gd : parts)
                for (auto *gs : parts)
                    if (gd != gs)
                        cudaMemcpyAsync(gd->dist->d_counts + (size_t)gs->dist->comm->rank * CW,
                                        gs->dist->d_counts + (size_t)gs->dist->comm->rank * CW, CW * 4,
                                        cudaMemcpyDeviceToDevice, st);
        }
        ag_dist_part *d0 = parts[0]->dist;
        cudaMemcpyAsync(d0->h_counts, d0->d_counts, (size_t)world * CW * 4, cudaMemcpyDeviceToHost, st);
        cudaError_t ce = cudaStreamSynchronize(st);
        if (ce != cudaSuccess) return cuda_status(ce, "dist sssp round");
        uint32_t maxc = 0, lo = INF;
        uint64_t carried = 0;
        front = 0;
        for (int r = 0; r < world; ++r) {
            const unsigned *c = d0->h_counts + (size_t)r * CW;
            maxc = c[0] > maxc ? c[0] : maxc;
            front += c[0];
            carried += c[1];
            lo = c[2] < lo ? c[2] : lo;
        }
        for (int r = 0; r < P; ++r) ncin[r] = d0->h_counts[(size_t)parts[r]->dist->comm->rank * CW + 1];
        cpar ^= 1;
        if (hub_window) hi = lo == INF ? ~0ull : (unsigned long long)lo + hub_window;
        if ((front == 0 && carried == 0) || R > 4u * V + 64u) break;
        n = (uint32_t)world * maxc;
        if (maxc == 0) continue;   // everything pending is held back: next round sends the window's minimum
        // pad every send list to maxc with (INF, INF), then gather rank-ordered into the global list
        for (auto *g : parts) {
            ag_dist_part *d = g->dist;
            const uint32_t c = d0->h_counts[(size_t)d->comm->rank * CW];
            if (c < maxc) cudaMemsetAsync(d->d_send + c, 0xFF, (size_t)(maxc - c) * 8, st);
        }
        if (nccl) {
            ag_dist_part *d = parts[0]->dist;
            ncclResult_t r = g_nccl.AllGather(d->d_send, d->d_list, (size_t)maxc * 8, ncclUint8, d->comm->nccl, st);
            if ((s = nccl_status(r, "ncclAllGather(frontier)")) != AG_OK) return s;
        } else {
            for (auto *gd : parts)
                for (auto *gs : parts)
                    cudaMemcpyAsync(gd->dist->d_list + (size_t)gs->dist->comm->rank * maxc, gs->dist->d_send,
                                    (size_t)maxc * 8, cudaMemcpyDeviceToDevice, st);
        }
    }
    for (int r = 0; r < P; ++r) {
        ag_graph_s *g = parts[r];
        ag_dist_part *d = g->dist;
        if (d->own_e > d->own_b && dist_owned && dist_owned[r]) {
            // device outputs directly; host outputs through the queue buffer q[0] as staging
            uint32_t *dd = dist_owned[r], *pp = parents_owned ? parents_owned[r] : nullptr;
            const bool dh = !is_device_ptr(dd), ph = pp && !is_device_ptr(pp);
            const size_t cnt = d->own_e - d->own_b;
            uint32_t *sd = dh ? g->d_q[0] : dd, *sp = ph ? g->d_q[1] : pp;   // staging: V entries each
            dist_sssp_out_kernel<<<g->num_sms * 2, 256, 0, st>>>(g->d_P, d->own_b, d->own_e, sd, sp);
            note_launch(1);
            if (dh) cudaMemcpyAsync(dd, sd, cnt * 4, cudaMemcpyDeviceToHost, st);
            if (ph) cudaMemcpyAsync(pp, sp, cnt * 4, cudaMemcpyDeviceToHost, st);
        }
    }
    if (stats) cudaEventRecord(e1, st);
    cudaError_t ce = cudaStreamSynchronize(st);
    if (ce != cudaSuccess) return cuda_status(ce, "dist sssp");
    unsigned long long vx = 0, ex = 0;
    bool ovf = false;
    for (auto *g : parts) {
        Ctl c;
        cudaMemcpy(&c, g->d_ctl, sizeof c, cudaMemcpyDeviceToHost);
        vx += c.vexp;
        ex += c.eexp;
        ovf |= c.overflow != 0;
        if (c.aborted) return set_error(AG_ERR_CUDA, "dist sssp aborted (code %u)", c.aborted);
    }
    if (stats) {
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        cudaEventDestroy(e0);
        cudaEventDestroy(e1);
        stats->iterations = R + 1;
        stats->device_ms = ms;
        stats->vertices_expanded = vx;
        stats->edges_inspected = ex;
        stats->trace_len = (R + 1) < tcap ? (R + 1) : tcap;
    }
    // a relaxation past 0xFFFFFFFE was dropped somewhere: reported conservatively (the distributed path
    // has no exact re-check like the single-GPU one; the outputs are still written)
    if (ovf) return set_error(AG_ERR_OVERFLOW, "a distance exceeds 0xFFFFFFFE");
    return AG_OK;
}

}  // namespace

extern "C" {

ag_status ag_dist_bfs(ag_graph local, uint32_t src, uint32_t *levels_owned, uint32_t *parents_owned,
                      const ag_policy *policy, ag_run_stats *stats, void *stream) {
    if (!local || !local->dist) return set_error(AG_ERR_INVALID_ARG, "not a distributed graph");
    if (src >= local->V) return set_error(AG_ERR_SRC_RANGE, "src %u >= V %u", src, local->V);
    if (stats && stats->struct_size != sizeof(ag_run_stats)) return set_error(AG_ERR_INVALID_ARG, "stats size");
    if (local->dist->comm->group) return set_error(AG_ERR_INVALID_ARG, "virtual-group graph: use ag_dist_bfs_group");
    std::vector<ag_graph_s *> parts{local};
    uint32_t *lv[1] = {levels_owned};
    uint32_t *pa[1] = {parents_owned};
    cudaSetDevice(local->device);
    return dist_bfs_driver(parts, src, lv, parents_owned ? pa : nullptr, policy, stats, (cudaStream_t)stream);
}

ag_status ag_dist_bfs_group(ag_graph *locals, int world, uint32_t src, uint32_t **levels_owned,
                            uint32_t **parents_owned, ag_run_stats *stats, void *stream) {
    if (!locals || world < 1) return set_error(AG_ERR_INVALID_ARG, "bad args");
    std::vector<ag_graph_s *> parts;
    for (int r = 0; r < world; ++r) {
        if (!locals[r] || !locals[r]->dist || !locals[r]->dist->comm->group || locals[r]->dist->comm->rank != r)
            return set_error(AG_ERR_INVALID_ARG, "locals[%d] is not rank %d of a virtual group", r, r);
        parts.push_back(locals[r]);
    }
    if (src >= parts[0]->V) return set_error(AG_ERR_SRC_RANGE, "src out of range");
    if (stats && stats->struct_size != sizeof(ag_run_stats)) return set_error(AG_ERR_INVALID_ARG, "stats size");
    cudaSetDevice(parts[0]->device);
    return dist_bfs_driver(parts, src, levels_owned, parents_owned, nullptr, stats, (cudaStream_t)stream);
}

ag_status ag_dist_sssp(ag_graph local, uint32_t src, uint32_t *dist_owned, uint32_t *parents_owned,
                       const ag_policy *policy, ag_run_stats *stats, void *stream) {
    if (!local || !local->dist) return set_error(AG_ERR_INVALID_ARG, "not a distributed graph");
    if (!dist_owned) return set_error(AG_ERR_INVALID_ARG, "dist_owned is NULL");
    if (src >= local->V) return set_error(AG_ERR_SRC_RANGE, "src %u >= V %u", src, local->V);
    if (stats && stats->struct_size != sizeof(ag_run_stats)) return set_error(AG_ERR_INVALID_ARG, "stats size");
    if (local->dist->comm->group) return set_error(AG_ERR_INVALID_ARG, "virtual-group graph: use ag_dist_sssp_group");
    std::vector<ag_graph_s *> parts{local};
    uint32_t *dv[1] = {dist_owned};
    uint32_t *pa[1] = {parents_owned};
    cudaSetDevice(local->device);
    // owner-side hub window: policy->sssp_hub_window, AUTO = max(1, max weight / 50)
    uint32_t hw = local->info.max_weight / 50u > 1u ? local->info.max_weight / 50u : 1u;
    if (policy && policy->struct_size == sizeof(ag_policy) && policy->sssp_hub_window != AG_WINDOW_AUTO)
        hw = policy->sssp_hub_window;
    return dist_sssp_driver(parts, src, dv, parents_owned ? pa : nullptr, stats, (cudaStream_t)stream, hw);
}

ag_status ag_dist_sssp_group(ag_graph *locals, int world, uint32_t src, uint32_t **dist_owned,
                             uint32_t **parents_owned, ag_run_stats *stats, void *stream) {
    if (!locals || world < 1 || !dist_owned) return set_error(AG_ERR_INVALID_ARG, "bad args");
    std::vector<ag_graph_s *> parts;
    for (int r = 0; r < world; ++r) {
        if (!locals[r] || !locals[r]->dist || !locals[r]->dist->comm->group || locals[r]->dist->comm->rank != r)
            return set_error(AG_ERR_INVALID_ARG, "locals[%d] is not rank %d of a virtual group", r, r);
        parts.push_back(locals[r]);
    }
    if (src >= parts[0]->V) return set_error(AG_ERR_SRC_RANGE, "src out of range");
    if (stats && stats->struct_size != sizeof(ag_run_stats)) return set_error(AG_ERR_INVALID_ARG, "stats size");
    cudaSetDevice(parts[0]->device);
    const uint32_t mw = parts[0]->info.max_weight;
    return dist_sssp_driver(parts, src, dist_owned, parents_owned, stats, (cudaStream_t)stream, mw / 50u > 1u ? mw / 50u : 1u);
}

}  // extern "C"
