// common.cuh — shared device/host definitions of libagraph (B200, sm_100a).
//
// Control block, device policy + the decision maker (Fig. 11, PAPER.md:24.s34-42), PTX helpers
// and the software grid barrier of the device-resident traversal loop (the paper splits every
// iteration into two kernel launches only because "CUDA does not offer primitives for global
// synchronization inside kernels", 20.s42; sm_100 has co-resident cooperative grids).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <cstddef>
#include <type_traits>

#include "agraph.h"

namespace ag {

#ifndef AG_BS
#define AG_BS 256
#endif
constexpr int BS = AG_BS;           // threads per CTA of the persistent traversal kernel
constexpr int WARPS_PER_CTA = BS / 32;
constexpr int LOG_BS = (BS == 1024) ? 10 : (BS == 512) ? 9 : (BS == 256) ? 8 : (BS == 128) ? 7 : -1;
static_assert(LOG_BS > 0, "BS must be 128, 256, 512 or 1024");
// Occupancy / batch depth per algorithm (measured on B200; profiles/r01_occupancy_ab.txt):
// BFS/CC 5 CTAs/SM with 4-edge pieces, SSSP (8-byte states, more atomics) 5 CTAs/SM with 2-edge pieces.
#ifndef AG_MINB_BFS
#define AG_MINB_BFS 5
#endif
#ifndef AG_MINB_SSSP
#define AG_MINB_SSSP 5   // re-tuned after the carveout / staging changes: C2 -3.8%, C4 -12.5%, C3 -3% vs 6 (12 B of spills instead of 152)
#endif
#ifndef AG_MINB_BFS_T
#define AG_MINB_BFS_T AG_MINB_BFS
#endif
#ifndef AG_MINB_SSSP_T
#define AG_MINB_SSSP_T AG_MINB_SSSP
#endif
#ifndef AG_EB_BFS
#define AG_EB_BFS 4
#endif
#ifndef AG_EB_SSSP
#define AG_EB_SSSP 2
#endif
constexpr uint32_t INF = 0xFFFFFFFFu;
constexpr unsigned long long INF64 = 0xFFFFFFFFFFFFFFFFull;
constexpr uint32_t MAX_FINITE = 0xFFFFFFFEu;

enum { ALG_BFS = 0, ALG_SSSP = 1, ALG_CC = 2 };   // CC: min-label components (NEXT-4, R23)
enum { ORD_U = 0, ORD_O = 1 };
enum { MAP_T = 1, MAP_W = 2, MAP_B = 3, MAP_H = 4 };
enum { WS_BM = 1, WS_QU = 2 };

// Hybrid mapping (beyond the paper, 18.s43-44): vertices with out-degree >= HUB_DEG are split into
// HUB_CHUNK-edge tasks drained by all CTAs.
#ifndef AG_HUBCHUNK
#define AG_HUBCHUNK 4096
#endif
#ifndef AG_QB
#define AG_QB 2           // hybrid mapping: aligned 16-byte pieces per thread per step (BFS)
#endif
#ifndef AG_QB_SSSP
#define AG_QB_SSSP 2      //                                                  (SSSP)
#endif
#ifndef AG_LONG_MIN
#define AG_LONG_MIN 512   // hybrid mapping: lists this long go to aligned warp windows
#endif
#ifndef AG_HUBDEG
#define AG_HUBDEG 2048
#endif
constexpr uint32_t HUB_DEG = AG_HUBDEG;
constexpr uint32_t HUBW_DEG = 64;   // SSSP hub-window degree threshold (measured on C1/C2/C4)
constexpr uint32_t HUB_CHUNK = AG_HUBCHUNK;
// Small working sets (|WS| < SMALLCHUNK_PER_CTA x CTAs: few hub tasks per CTA, the iteration ends with the
// slowest task) split lists of >= HUB_CHUNK_SMALL entries into HUB_CHUNK_SMALL-entry tasks instead.
#ifndef AG_HUBCHUNK_SMALL
#define AG_HUBCHUNK_SMALL 1024
#endif
#ifndef AG_SMALLCHUNK_PER_CTA
#define AG_SMALLCHUNK_PER_CTA 32
#endif
constexpr uint32_t HUB_CHUNK_SMALL = AG_HUBCHUNK_SMALL;
constexpr uint32_t SMALLCHUNK_PER_CTA = AG_SMALLCHUNK_PER_CTA;
// small-frontier mode on graphs with hub tasks: only in the falling tail, below this |WS|
#ifndef AG_T_SMALL_HUB
#define AG_T_SMALL_HUB 4096
#endif
// unordered BFS on degree-layout graphs runs the general specialisation with the tuned decisions
#ifndef AG_BFS_ROUTE
#define AG_BFS_ROUTE 1
#endif
// Edges processed per thread per batch: loads of all EB edges are issued before any dependent use.
constexpr int EB_MAX = (AG_EB_BFS > AG_EB_SSSP) ? AG_EB_BFS : AG_EB_SSSP;

// ---------------------------------------------------------------------------------------------
// Device-side control block.  Per-iteration counters rotate over 3 slots (slot = it % 3): slot(it)
// describes the working set processed in iteration it, slot(it+1) accumulates the next one, and
// slot(it+2) is reset at the start of iteration it (its last reader finished at the barrier).
// ---------------------------------------------------------------------------------------------
constexpr int NGRP = 32;            // barrier arrival groups (hierarchical arrival)
#ifndef AG_CTL_SPREAD
#define AG_CTL_SPREAD 1
#endif
#if AG_CTL_SPREAD
#define AG_CTL_LINE alignas(128)
#else
#define AG_CTL_LINE
#endif

struct alignas(128) Ctl {
    unsigned long long bar_word;      // (generation << 32) | payload, released by the last arriver
    unsigned int pad0[30];
    unsigned int bar_count;           // groups arrived
    unsigned int pad1[31];
    unsigned int grp_count[NGRP * 32];  // CTAs arrived per group (one 128-B line each)
    // The counters every CTA hits with atomics or polls each iteration, one 128-B line each: an L2 slice
    // serialises the operations on one line, and with the counters packed into two lines the queue appends,
    // tile claims, hub claims, the drain's polls and the per-CTA reductions all queued behind each other
    // (C2 BFS -3.5%, SSSP -6.6%, profiles/r02_ab/ab_summary.txt item 5p)
    AG_CTL_LINE unsigned int q_len[3];       // queue append cursor == |WS| for BFS and unordered SSSP
    AG_CTL_LINE unsigned int next_min[3];    // ordered SSSP: min tentative distance of pending vertices
    AG_CTL_LINE unsigned int tile_ctr[3];    // dynamic tile scheduler
    AG_CTL_LINE unsigned int hub_tail[3];    // hybrid mapping: produced hub-chunk tasks
    AG_CTL_LINE unsigned int hub_head[3];    //                 consumed hub-chunk tasks
    AG_CTL_LINE unsigned int stage_done[3];  //                 CTAs done producing
    AG_CTL_LINE unsigned long long it_edges[3];   // edges inspected in iteration (m_F: selector input, trace)
    AG_CTL_LINE unsigned long long it_nv[3];      // working-set elements expanded in iteration
    AG_CTL_LINE unsigned int it_reexp[3];         // SSSP: expansions of a vertex already expanded earlier in the query
    AG_CTL_LINE unsigned int free_any[3];         // free-output iteration wrote at least one next-bitmap bit
    AG_CTL_LINE unsigned int pend_count;          // ordered SSSP: |pending|
    AG_CTL_LINE unsigned int overflow;            // a relaxation exceeded MAX_FINITE
    unsigned int iterations;
    unsigned int aborted;             // iteration cap hit (never expected)
    AG_CTL_LINE unsigned long long vexp;   // totals (adjacent: cleared together; ONE declarator per alignas,
    unsigned long long eexp;               // which would otherwise align each of them)
    // small-frontier mode (tuned kernels): CTAs >= small_ctas park while |WS| < t_small and are woken
    // with the iteration to resume at (wake_n = 0: terminate).  Own 128-B line: the parked CTAs poll
    // it, and must not slow the atomics on the per-iteration counters above.
    alignas(128) unsigned int wake_gen;   // wake events so far (monotone across launches)
    unsigned int wake_it, wake_n, wake_nprev;
    unsigned int wake_win;            //   ... and the current adaptive window / bucket width
    unsigned int pad2[27];
    // virtual CTA numbering (small-frontier mode): one "leader" CTA per SM gets vid [0, leaders), the
    // others [leaders, nblocks); counters double-buffered by launch parity (the other half is zeroed)
    unsigned int sm_rank[256];        // CTAs that have arrived on SM s (mod CTAs per SM = rank on s)
    unsigned int lead_cnt[2], other_cnt[2];
    // launches completed on this control block: its parity selects the (lead_cnt, other_cnt) pair of
    // the next launch, which zeroes the other pair for the one after.  Advanced by the kernel itself
    // (never by the host), so a call that fails before or at launch cannot desynchronise it.
    unsigned int launch_seq;
    // deferred status, sticky across launches until ag_graph_check() clears it: bit 0 = a finite
    // distance exceeds MAX_FINITE (exact, checked in-kernel), bits 8.. = max abort code seen
    unsigned int sticky;
};
// layout invariants: the distributed path clears the totals as one 16-byte range; with AG_CTL_SPREAD every
// hot per-iteration counter sits on its own 128-B line (an alignas on a multi-declarator member would align
// each declarator, which once split vexp / eexp apart)
static_assert(offsetof(Ctl, eexp) == offsetof(Ctl, vexp) + 8, "vexp, eexp must be adjacent");
#if AG_CTL_SPREAD
static_assert(offsetof(Ctl, q_len) / 128 != offsetof(Ctl, tile_ctr) / 128 &&
                  offsetof(Ctl, tile_ctr) / 128 != offsetof(Ctl, hub_tail) / 128 &&
                  offsetof(Ctl, hub_tail) / 128 != offsetof(Ctl, hub_head) / 128 &&
                  offsetof(Ctl, hub_head) / 128 != offsetof(Ctl, stage_done) / 128 &&
                  offsetof(Ctl, stage_done) / 128 != offsetof(Ctl, it_edges) / 128,
              "per-iteration control counters on separate lines");
#endif

// Policy as seen by the device (plain integers; filled from ag_policy on the host).
struct DevPolicy {
    uint32_t kind;        // AG_POLICY_PAPER / AG_POLICY_TUNED
    uint32_t force_map;   // 0 = auto
    uint32_t force_ws;    // 0 = auto
    uint32_t t1;
    uint64_t t2;
    uint64_t t3;          // absolute (already scaled by V)
    uint32_t sample_every;
    uint32_t delta;
    uint32_t cta_group;   // resolved block-mapping group size (multiple of 32, <= BS)
    uint32_t window;      // unordered SSSP deferral window (0 = off)
    uint32_t hub_window;  // unordered SSSP deferral window for vertices of degree >= HUBW_DEG (0 = off)
    uint32_t V;
    uint64_t E;
    uint32_t max_deg;     // inspector: maximum out-degree (tuned policy)
    uint32_t t2_tuned;    // tuned policy: thread mapping below this |WS| on low-degree graphs
    uint64_t t_free;      // tuned policy: free (raw-bitmap) output from this |WS| on (~0 = never), BFS
    uint64_t t_free_sssp; //   ... SSSP (never on skewed graphs: red.min on hot targets loses, tools/gpu_free_ab.sh)
    uint32_t small_ctas;  // tuned kernels: CTAs that run an iteration whose |WS| < t_small (the rest park)
    uint32_t t_small;     //   0 = off
    uint32_t t_small_hub; //   graphs with hub tasks: only in the shrinking tail (|WS| below this and falling)
    uint32_t smallchunk_per_cta;  // tuned kernels: |WS| < this x CTAs -> HUB_CHUNK_SMALL-entry hub tasks
    uint32_t ordered;     // ordered SSSP: |WS| is the pending set (its representation is selected)
    uint32_t adapt;       // SSSP order axis adapted per iteration (NEXT-3): the unordered deferral window
                          // (sssp_window = AG_WINDOW_ADAPTIVE) or the ordered bucket width (delta = 0)
    uint32_t win_max;     //   upper bound of the adapted window / width
};

// The decision maker.  PAPER: Fig. 11 with readings R12/R13:
//   ws < T2 -> B_QU; else workset = ws >= T3 ? BM : QU; mapping = E >= T1*V ? B : T.
// TUNED (B200, calibrated with tools/sweep.py / tools/calibrate.py on C2/C3/C4), from
//   |WS| and m_F (the working set's out-degree sum; the kernel passes |WS| x the previous frontier's
//   average degree, the paper's inspector statistic, 26.s4-7):
//   * working set: the queue (appends are warp-staged, the bitmap scan costs O(V/32) per iteration),
//     except the ordered-SSSP pending set once it holds >= V/32 vertices: a bucket then re-reads most
//     of it, and one O(V/32) scan of the pending bitmap beats re-reading (and re-appending) the list;
//   * mapping: THREAD for small working sets of low out-degree (m_F <= 6 |WS|) on graphs without
//     straggler lists (max degree <= 64), else HYBRID (load-balanced pieces + hub tasks).
__host__ __device__ inline uint8_t select_variant(const DevPolicy &p, uint64_t ws, uint64_t ws_edges) {
    uint32_t map, wsr;
    if (p.kind == AG_POLICY_PAPER) {
        if (ws < p.t2) {
            map = MAP_B;
            wsr = WS_QU;
        } else {
            wsr = ws >= p.t3 ? WS_BM : WS_QU;
            map = (p.E >= (uint64_t)p.t1 * p.V) ? MAP_B : MAP_T;
        }
    } else {
        wsr = (p.ordered && ws >= ((uint64_t)p.V + 31) / 32) ? WS_BM : WS_QU;
        const bool low_deg = ws_edges <= 6ull * ws;   // grid-like (avg 2-4); ER's 8 already prefers H (r02 sweep)
        map = (p.max_deg <= 64 && low_deg && ws < p.t2_tuned) ? MAP_T : MAP_H;
    }
    if (p.force_map) map = p.force_map;
    if (p.force_ws) wsr = p.force_ws;
    return (uint8_t)(map * 4 + wsr);
}

#ifdef __CUDACC__
// ---------------------------------------------------------------------------------------------
// PTX helpers
// ---------------------------------------------------------------------------------------------
__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(unsigned *p, unsigned v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned ld_relaxed(const unsigned *p) {
    unsigned v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed64(unsigned long long *p, unsigned long long v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_relaxed64(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
// L2 eviction policies: the CSR arrays stream through once per traversal (evict first, no L1
// allocation) while the per-vertex status arrays (visited bitmap, levels, packed distances) should
// stay resident in the 126 MB L2 (evict last).
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
// streaming read of a CSR array: read once per traversal, keep it out of L1, evict first from L2
__device__ __forceinline__ uint32_t ld_stream(const uint32_t *p, uint64_t pol) {
    uint32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ uint2 ld_stream2(const uint2 *p, uint64_t pol) {
    uint2 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.u32 {%0, %1}, [%2], %3;"
                 : "=r"(v.x), "=r"(v.y) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ uint4 ld_stream4(const uint4 *p, uint64_t pol) {
    uint4 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0, %1, %2, %3}, [%4], %5;"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p), "l"(pol));
    return v;
}
// status read: L1-cacheable, evict last from L2
__device__ __forceinline__ uint32_t ld_keep(const uint32_t *p, uint64_t pol) {
    uint32_t v;
    asm volatile("ld.global.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ unsigned long long ld_keep(const unsigned long long *p, uint64_t pol) {
    unsigned long long v;
    asm volatile("ld.global.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ void red_or(uint32_t *p, uint32_t v) {
    asm volatile("red.relaxed.gpu.global.or.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void red_min32(uint32_t *p, uint32_t v) {
    asm volatile("red.relaxed.gpu.global.min.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void red_min64(unsigned long long *p, unsigned long long v) {
    asm volatile("red.relaxed.gpu.global.min.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ unsigned lane_id() { return threadIdx.x & 31u; }

__device__ __forceinline__ unsigned long long globaltimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// Software grid barrier for a co-resident (cooperative) grid, one atomic per CTA on a single word:
// CTA 0 adds 0x80000000 - (nblocks - 1), every other CTA adds 1, so the top bit flips exactly when
// the last CTA arrives; everyone spins on that bit (measured on B200: ~1.6 us at 592 CTAs, faster
// than a two-level tree with a separate release word).  Self-resetting across launches.
// `first`: exactly one participating CTA passes true (default: CTA 0).
__device__ __forceinline__ void grid_barrier(Ctl *ctl, unsigned nblocks, bool first) {
    __syncthreads();
    if (threadIdx.x == 0) {
        const unsigned inc = first ? (0x80000000u - (nblocks - 1)) : 1u;
        __threadfence();
        const unsigned old = atomicAdd(&ctl->bar_count, inc);
        while (((old ^ ld_relaxed(&ctl->bar_count)) & 0x80000000u) == 0) {
        }
        __threadfence();
    }
    __syncthreads();
}
__device__ __forceinline__ void grid_barrier(Ctl *ctl, unsigned nblocks) { grid_barrier(ctl, nblocks, blockIdx.x == 0); }

// Warp-aggregated append of v (where flag) to a queue: one atomic per warp-step ("each thread uses an
// atomic operation only to get a unique insertion index", 22.s18, aggregated per warp).
__device__ __forceinline__ void warp_append(uint32_t *q, unsigned *qlen, bool flag, uint32_t v) {
    unsigned act = __activemask();
    unsigned m = __ballot_sync(act, flag);
    if (m == 0) return;
    unsigned lane = lane_id();
    int leader = __ffs(m) - 1;
    unsigned base = 0;
    if ((int)lane == leader) base = atomicAdd(qlen, (unsigned)__popc(m));
    base = __shfl_sync(act, base, leader);
    if (flag) q[base + __popc(m & ((1u << lane) - 1u))] = v;
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}
__device__ __forceinline__ unsigned warp_min(unsigned v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = min(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}
#endif  // __CUDACC__

}  // namespace ag
