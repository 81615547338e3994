// common.cuh — shared device/host definitions of libagraph (B200, sm_100a).
//
// Control block, device policy + the decision maker (Fig. 11, PAPER.md:24.s34-42), PTX helpers
// and the software grid barrier of the device-resident traversal loop (the paper splits every
// iteration into two kernel launches only because "CUDA does not offer primitives for global
// synchronization inside kernels", 20.s42; sm_100 has co-resident cooperative grids).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "agraph.h"

namespace ag {

constexpr int BS = 256;             // threads per CTA of the persistent traversal kernel
constexpr int WARPS_PER_CTA = BS / 32;
constexpr int MIN_BLOCKS = 4;       // __launch_bounds__ min CTAs/SM (=> <= 64 regs/thread)
constexpr uint32_t INF = 0xFFFFFFFFu;
constexpr unsigned long long INF64 = 0xFFFFFFFFFFFFFFFFull;
constexpr uint32_t MAX_FINITE = 0xFFFFFFFEu;

enum { ALG_BFS = 0, ALG_SSSP = 1 };
enum { ORD_U = 0, ORD_O = 1 };
enum { MAP_T = 1, MAP_W = 2, MAP_B = 3, MAP_H = 4 };
enum { WS_BM = 1, WS_QU = 2 };

// Hybrid mapping (beyond the paper, 18.s43-44): vertices with out-degree >= HUB_DEG are split into
// HUB_CHUNK-edge tasks drained by all CTAs.
constexpr uint32_t HUB_DEG = 4096;
constexpr uint32_t HUB_CHUNK = 2048;

// ---------------------------------------------------------------------------------------------
// Device-side control block.  Per-iteration counters rotate over 3 slots (slot = it % 3): slot(it)
// describes the working set processed in iteration it, slot(it+1) accumulates the next one, and
// slot(it+2) is reset at the start of iteration it (its last reader finished at the barrier).
// ---------------------------------------------------------------------------------------------
struct alignas(128) Ctl {
    unsigned int bar_count;
    unsigned int pad0[31];
    unsigned int bar_gen;
    unsigned int pad1[31];
    unsigned int q_len[3];            // queue append cursor == |WS| for BFS and unordered SSSP
    unsigned int next_min[3];         // ordered SSSP: min tentative distance of pending vertices
    unsigned int tile_ctr[3];         // dynamic tile scheduler
    unsigned int hub_tail[3];         // hybrid mapping: produced hub-chunk tasks
    unsigned int hub_head[3];         //                 consumed hub-chunk tasks
    unsigned int stage_done[3];       //                 CTAs done producing
    unsigned long long it_edges[3];   // edges inspected in iteration
    unsigned long long it_verts[3];   // vertices expanded in iteration
    unsigned int pend_count;          // ordered SSSP: |pending|
    unsigned int overflow;            // a relaxation exceeded MAX_FINITE
    unsigned int iterations;
    unsigned int aborted;             // iteration cap hit (never expected)
    unsigned long long vexp, eexp;    // totals
};

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
    uint32_t V;
    uint64_t E;
};

// The decision maker.  PAPER: Fig. 11 with readings R12/R13:
//   ws < T2 -> B_QU; else workset = ws >= T3 ? BM : QU; mapping = E >= T1*V ? B : T.
// TUNED (B200): workset by the same T3 rule; mapping HYBRID (per-vertex degree
//   classes + hub splitting) unless the graph is near-regular and low-degree, where THREAD wins.
__host__ __device__ inline uint8_t select_variant(const DevPolicy &p, uint64_t ws, uint64_t ws_edges) {
    uint32_t map, wsr;
    (void)ws_edges;
    if (p.kind == AG_POLICY_PAPER) {
        if (ws < p.t2) {
            map = MAP_B;
            wsr = WS_QU;
        } else {
            wsr = ws >= p.t3 ? WS_BM : WS_QU;
            map = (p.E >= (uint64_t)p.t1 * p.V) ? MAP_B : MAP_T;
        }
    } else {
        wsr = ws >= p.t3 ? WS_BM : WS_QU;
        map = MAP_H;
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
__device__ __forceinline__ unsigned long long ld_relaxed64(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
// streaming read of a CSR array: read once per traversal, keep it out of L1
__device__ __forceinline__ uint32_t ld_stream(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ uint32_t ld_ro(const uint32_t *p) { return __ldg(p); }
__device__ __forceinline__ unsigned long long ld_ro(const unsigned long long *p) { return __ldg(p); }
__device__ __forceinline__ void red_or(uint32_t *p, uint32_t v) {
    asm volatile("red.relaxed.gpu.global.or.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ unsigned lane_id() { return threadIdx.x & 31u; }

// Software grid barrier for a co-resident (cooperative) grid.  Sense via a generation counter;
// the last arriver resets the count, so the barrier needs no per-launch reset.
__device__ __forceinline__ void grid_barrier(Ctl *ctl, unsigned nblocks) {
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned gen = ld_acquire(&ctl->bar_gen);
        __threadfence();
        unsigned arrived = atomicAdd(&ctl->bar_count, 1u);
        if (arrived == nblocks - 1) {
            ctl->bar_count = 0;
            __threadfence();
            st_release(&ctl->bar_gen, gen + 1);
        } else {
            while (ld_acquire(&ctl->bar_gen) == gen) __nanosleep(20);
        }
        __threadfence();
    }
    __syncthreads();
}

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
