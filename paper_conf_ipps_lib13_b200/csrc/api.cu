// api.cu — the C ABI of libagraph (include/agraph.h): graph store + inspector (a1), policy and
// decision maker (a3), and the launch of the device-resident traversal (a2, a4-a7).
#include <cuda_runtime.h>

#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <unordered_map>
#include <vector>

#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include "agraph.h"
#include "common.cuh"
#include "graph.h"
#include "traverse.cuh"

using namespace ag;

// ------------------------------------------------------------------------------------------------
// errors, allocator, launch accounting
// ------------------------------------------------------------------------------------------------
static thread_local std::string g_last_error;
static std::atomic<unsigned long long> g_launches{0};

namespace ag {
void note_launch(unsigned n) { g_launches += n; }

ag_status set_error(ag_status s, const char *fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_last_error = buf;
    return s;
}

ag_status cuda_status(cudaError_t e, const char *what) {
    if (e == cudaSuccess) return AG_OK;
    cudaGetLastError();
    if (e == cudaErrorMemoryAllocation) return set_error(AG_ERR_OOM, "%s: %s", what, cudaGetErrorString(e));
    if (e == cudaErrorNoDevice || e == cudaErrorInsufficientDriver)
        return set_error(AG_ERR_NO_DEVICE, "%s: %s", what, cudaGetErrorString(e));
    return set_error(AG_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
}

static void *(*g_alloc)(size_t, int, void *, void *) = nullptr;
static void (*g_free)(void *, size_t, int, void *, void *) = nullptr;
static void *g_alloc_ctx = nullptr;

// Every hook allocation remembers the free function that owns it, so a buffer is always returned to the
// allocator it came from — also when the hook is changed or removed between allocation and free (a
// graph loaded with cudaMalloc and freed while the PyTorch hook is active, or the reverse).
struct HookRec {
    void (*free_)(void *, size_t, int, void *, void *);
    void *ctx;
};
static std::unordered_map<void *, HookRec> g_hook_ptrs;
static std::mutex g_hook_mu;

ag_status dev_alloc(void **p, size_t bytes, int device) {
    *p = nullptr;
    if (bytes == 0) bytes = 16;
    bytes = (bytes + 255) & ~size_t(255);
    if (g_alloc) {
        *p = g_alloc(bytes, device, nullptr, g_alloc_ctx);
        if (!*p) return set_error(AG_ERR_OOM, "allocator hook returned NULL for %zu bytes", bytes);
        std::lock_guard<std::mutex> lk(g_hook_mu);
        g_hook_ptrs[*p] = HookRec{g_free, g_alloc_ctx};
        return AG_OK;
    }
    return cuda_status(cudaMalloc(p, bytes), "cudaMalloc");
}

void dev_free(void *p, size_t bytes, int device) {
    if (!p) return;
    bytes = (bytes == 0 ? 16 : (bytes + 255) & ~size_t(255));
    HookRec r{nullptr, nullptr};
    {
        std::lock_guard<std::mutex> lk(g_hook_mu);
        auto it = g_hook_ptrs.find(p);
        if (it != g_hook_ptrs.end()) {
            r = it->second;
            g_hook_ptrs.erase(it);
        }
    }
    if (r.free_) r.free_(p, bytes, device, nullptr, r.ctx);
    else cudaFree(p);
}

bool is_device_ptr(const void *p) {
    if (!p) return false;
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

// per-device attributes, queried once (cudaGetDeviceProperties is slow: milliseconds per call)
struct DevAttrs {
    bool valid = false;
    int major = 0, minor = 0, sms = 0, persist_max = 0, window_max = 0;
};
static DevAttrs g_dev[64];
static std::mutex g_dev_mu;

const DevAttrs *device_attrs(int device) {
    if (device < 0 || device >= 64) return nullptr;
    std::lock_guard<std::mutex> lk(g_dev_mu);
    DevAttrs &d = g_dev[device];
    if (!d.valid) {
        if (cudaDeviceGetAttribute(&d.major, cudaDevAttrComputeCapabilityMajor, device) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        cudaDeviceGetAttribute(&d.minor, cudaDevAttrComputeCapabilityMinor, device);
        cudaDeviceGetAttribute(&d.sms, cudaDevAttrMultiProcessorCount, device);
        cudaDeviceGetAttribute(&d.persist_max, cudaDevAttrMaxPersistingL2CacheSize, device);
        cudaDeviceGetAttribute(&d.window_max, cudaDevAttrMaxAccessPolicyWindowSize, device);
        cudaGetLastError();
        d.valid = true;
    }
    return &d;
}

ag_status check_device(int device, int *num_sms) {
    int n = 0;
    cudaError_t e = cudaGetDeviceCount(&n);
    if (e != cudaSuccess || n == 0) {
        cudaGetLastError();
        return set_error(AG_ERR_NO_DEVICE, "no CUDA device available");
    }
    if (device < 0 || device >= n) return set_error(AG_ERR_INVALID_ARG, "device %d out of range [0,%d)", device, n);
    const DevAttrs *d = device_attrs(device);
    if (!d) return set_error(AG_ERR_CUDA, "cannot query device %d", device);
    if (d->major != 10 || d->minor != 0)
        return set_error(AG_ERR_NO_DEVICE, "device %d is sm_%d%d; libagraph is built for sm_100a only", device,
                         d->major, d->minor);
    if (num_sms) *num_sms = d->sms;
    return AG_OK;
}
}  // namespace ag

// ------------------------------------------------------------------------------------------------
// graph load kernels: validation + inspector statistics (a1)
// ------------------------------------------------------------------------------------------------
struct LoadStats {
    unsigned int bad;            // bit 0 rp[0], 1 monotone, 2 rp[V], 3 col range, 4 weight range
    unsigned int min_deg, max_deg, isolated;
    unsigned int max_w;
};

__global__ void validate_rows_kernel(const uint64_t *rp, uint32_t V, uint64_t E, LoadStats *st) {
    uint32_t lmin = 0xFFFFFFFFu, lmax = 0, liso = 0, bad = 0;
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < V; u += gridDim.x * blockDim.x) {
        uint64_t b = rp[u], e = rp[u + 1];
        if (e < b) { bad |= 2; continue; }
        uint64_t d = e - b;
        uint32_t dd = d > 0xFFFFFFFFull ? 0xFFFFFFFFu : (uint32_t)d;
        lmin = min(lmin, dd);
        lmax = max(lmax, dd);
        liso += (d == 0);
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        if (rp[0] != 0) bad |= 1;
        if (rp[V] != E) bad |= 4;
    }
    lmin = warp_min(lmin);
    for (int o = 16; o > 0; o >>= 1) lmax = max(lmax, __shfl_xor_sync(0xffffffffu, lmax, o));
    liso = warp_sum(liso);
    bad |= __reduce_or_sync(0xffffffffu, bad);
    if ((threadIdx.x & 31) == 0) {
        atomicMin(&st->min_deg, lmin);
        atomicMax(&st->max_deg, lmax);
        if (liso) atomicAdd(&st->isolated, liso);
        if (bad) atomicOr(&st->bad, bad);
    }
}

__global__ void validate_edges_kernel(const uint32_t *col, const uint32_t *w, uint64_t E, uint32_t V, LoadStats *st) {
    unsigned bad = 0, mw = 0;
    for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < E; e += (uint64_t)gridDim.x * blockDim.x) {
        if (col[e] >= V) bad |= 8;
        if (w) {
            uint32_t x = w[e];
            if (x == 0 || x >= 0x80000000u) bad |= 16;
            mw = max(mw, x);
        }
    }
    bad = __reduce_or_sync(0xffffffffu, bad);
    mw = __reduce_max_sync(0xffffffffu, mw);
    if ((threadIdx.x & 31) == 0) {
        if (bad) atomicOr(&st->bad, bad);
        if (mw) atomicMax(&st->max_w, mw);
    }
}

// Degree layout, one chunk of the pipelined load: the CSR entries of old rows [ra, rb) (all arrived) go to
// their relabelled positions nrp[inv[u]] + (e - rp[u]) with the neighbour mapped through inv (an
// out-of-range id is flagged, never dereferenced); weights are validated and interleaved into cw.
// Edge-parallel (one owner binary search per entry) so hub rows do not serialise on one warp.
__global__ void relabel_edges_kernel(const uint64_t *rp, const uint32_t *col, const uint32_t *w, const uint32_t *inv,
                                     const uint64_t *nrp, uint32_t V, uint32_t ra, uint32_t rb, uint32_t *ncol, uint2 *cw,
                                     LoadStats *st) {
    const uint64_t e0 = rp[ra], e1 = rp[rb];
    unsigned bad = 0, mw = 0;
    for (uint64_t e = e0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < e1; e += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t lo = ra, hi = rb;   // rp[lo] <= e < rp[hi]: the owner is the largest u with rp[u] <= e
        while (hi - lo > 1) {
            const uint32_t mid = lo + (hi - lo) / 2;
            if (rp[mid] <= e) lo = mid; else hi = mid;
        }
        const uint32_t c = col[e];
        uint32_t nc = 0;
        if (c < V) nc = inv[c]; else bad |= 8;
        const uint64_t ne = nrp[inv[lo]] + (e - rp[lo]);
        ncol[ne] = nc;
        if (w) {
            const uint32_t x = w[e];
            if (x == 0 || x >= 0x80000000u) bad |= 16;
            mw = max(mw, x);
            cw[ne] = make_uint2(nc, x);
        }
    }
    bad = __reduce_or_sync(0xffffffffu, bad);
    mw = __reduce_max_sync(0xffffffffu, mw);
    if ((threadIdx.x & 31) == 0) {
        if (bad) atomicOr(&st->bad, bad);
        if (mw) atomicMax(&st->max_w, mw);
    }
}

__global__ void interleave_kernel(const uint32_t *col, const uint32_t *w, uint2 *cw, uint64_t E) {
    for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < E; e += (uint64_t)gridDim.x * blockDim.x)
        cw[e] = make_uint2(col[e], w[e]);
}

__global__ void narrow_offsets_kernel(const uint64_t *rp, uint32_t *rp32, uint32_t n) {
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
        rp32[i] = (uint32_t)rp[i];
}

// V_r and E_r of a result array (stats only; not in the timed path)
template <typename Off>
__global__ void reached_kernel(const uint32_t *out, const Off *rp, const uint32_t *inv, uint32_t V,
                               unsigned long long *acc) {
    unsigned long long a = 0, b = 0;
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < V; v += gridDim.x * blockDim.x)
        if (out[v] != INF) {
            const uint32_t i = inv ? inv[v] : v;
            a += 1;
            b += (unsigned long long)(rp[i + 1] - rp[i]);
        }
    a = warp_sum(a);
    b = warp_sum(b);
    if ((threadIdx.x & 31) == 0 && (a | b)) { atomicAdd(&acc[0], a); atomicAdd(&acc[1], b); }
}

// Exact overflow test after an SSSP traversal (enqueued behind it; returns at once unless a relaxation
// exceeded MAX_FINITE): a reachable vertex left at INF behind a finite one.  Packed state in device ids.
template <typename Off>
__global__ void overflow_check_kernel(const Ctl *ctl, const unsigned long long *P, bool packed, const Off *rp, const uint2 *cw,
                                      uint32_t V, unsigned *sticky) {
    if (!*(volatile const unsigned *)&ctl->overflow) return;
    // packed: (dist << 32) | parent words; else the distance-only u32 state (no parents requested)
    auto dist = [&](uint32_t x) { return packed ? (uint32_t)(P[x] >> 32) : reinterpret_cast<const uint32_t *>(P)[x]; };
    bool bad = false;
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < V && !bad; u += gridDim.x * blockDim.x) {
        if (dist(u) == INF) continue;
        for (Off e = rp[u]; e < rp[u + 1]; ++e)
            if (dist(cw[e].x) == INF) { bad = true; break; }
    }
    if (bad) atomicOr(sticky, 1u);
}

// ------------------------------------------------------------------------------------------------
// graph handle helpers
// ------------------------------------------------------------------------------------------------
namespace ag {

static ag_status ensure_scratch(ag_graph_s *g, bool sssp) {
    const size_t V = g->V, nw = g->nwords;
    ag_status s;
#define ALLOC(ptr, bytes)                                                          \
    if (!(ptr)) {                                                                  \
        if ((s = dev_alloc((void **)&(ptr), (bytes), g->device)) != AG_OK) return s; \
        g->scratch_bytes += (bytes);                                               \
    }
    ALLOC(g->d_ctl, sizeof(Ctl));
    if (!g->ctl_init) {
        cudaMemset(g->d_ctl, 0, sizeof(Ctl));
        g->ctl_init = true;
    }
    for (int i = 0; i < 3; ++i) { ALLOC(g->d_bm[i], nw * 4 + 128); }
    for (int i = 0; i < 3; ++i) { ALLOC(g->d_q[i], V * 4 + 128); }
    ALLOC(g->d_vis, nw * 4 + 128);
    if (!g->d_hub) {   // hub-task ring: every slot 0 (= empty) between iterations
        ALLOC(g->d_hub, (size_t)g->hub_cap * 8);
        cudaMemset(g->d_hub, 0, (size_t)g->hub_cap * 8);
    }
    ALLOC(g->d_acc, 64);
    if (sssp) { ALLOC(g->d_P, V * 8 + 128); }
#undef ALLOC
    return AG_OK;
}

static ag_status ensure_buf(ag_graph_s *g, uint32_t **p, size_t *have, size_t bytes) {
    if (*have >= bytes && *p) return AG_OK;
    if (*p) dev_free(*p, *have, g->device);
    *p = nullptr;
    *have = 0;
    ag_status s = dev_alloc((void **)p, bytes, g->device);
    if (s == AG_OK) *have = bytes;
    return s;
}

DevPolicy resolve_policy(const ag_policy &p, const ag_graph_s &g) {
    DevPolicy d;
    memset(&d, 0, sizeof d);
    d.kind = p.kind;
    d.force_map = p.mapping;
    d.force_ws = p.workset;
    d.t1 = p.t1_avg_degree;
    d.t2 = p.t2_ws;
    d.t3 = ((uint64_t)g.V * p.t3_ppm + 999999ull) / 1000000ull;
    d.sample_every = p.sample_every ? p.sample_every : 1;
    d.delta = p.delta ? p.delta : 1;   // 0 = adaptive, starting at 1 (below)
    uint32_t grp = p.cta_group;
    if (grp == 0) {  // multiple of 32 closest to the average out-degree, ties up (26.s28, R16)
        uint64_t k = g.V ? (2 * g.E + 32ull * g.V) / (64ull * g.V) : 1;
        grp = (uint32_t)(32 * (k < 1 ? 1 : k));
    }
    grp = grp < 32 ? 32 : grp;
    grp = grp > (uint32_t)BS ? (uint32_t)BS : grp;
    grp &= ~31u;
    d.cta_group = grp;
    if (p.sssp_window == AG_WINDOW_AUTO || p.sssp_window == AG_WINDOW_ADAPTIVE) {
        // tuned: Bellman-Ford re-expansion is distance-ordering waste on long-path graphs (grid: 152x,
        // ER: 4.3x) but not on power-law graphs (R-MAT: no gain) -- measured with tools/sweep.py
        const uint64_t avg = g.V ? (g.E + g.V - 1) / g.V : 1;
        const bool skewed = g.info.layout == AG_LAYOUT_DEGREE;
        uint64_t w = 8ull * g.info.max_weight / (avg ? avg : 1);
        if (w < 1) w = 1;
        if (w > 0x7FFFFFFFull) w = 0x7FFFFFFFull;
        d.window = (p.kind == AG_POLICY_TUNED && !skewed && g.info.max_weight) ? (uint32_t)w : 0u;
        if (p.sssp_window == AG_WINDOW_ADAPTIVE) d.window = (uint32_t)w;   // the start of the adapted window
    } else {
        d.window = p.sssp_window;
    }
    if (p.sssp_hub_window == AG_WINDOW_AUTO) {
        // tuned: expand high-degree vertices only near the frontier minimum (R-MAT s22: edges
        // inspected 2.75 E_r -> 1.15 E_r, 2.7 -> 1.9 ms; tools/sweep.py)
        d.hub_window = (p.kind == AG_POLICY_TUNED && g.info.max_weight)
                           ? (g.info.max_weight / 50 > 1 ? g.info.max_weight / 50 : 1u) : 0u;
    } else {
        d.hub_window = p.sssp_hub_window;
    }
    d.V = g.V;
    d.E = g.E;
    d.max_deg = g.info.max_deg;
    d.t2_tuned = 65536;
    d.t_free = (p.kind == AG_POLICY_TUNED && p.free_ppm) ? ((uint64_t)g.V * p.free_ppm + 999999ull) / 1000000ull : ~0ull;
    if (d.t_free == 0) d.t_free = 1;
    const uint64_t t_free_any = d.t_free;
    // BFS: free output only on non-skewed graphs too (measured over 32 sources, profiles/r01_free_output_ab.txt:
    // R-MAT s22 median 0.571 ms without vs 1.19 ms with — during a free-output level the visited bitmap is
    // not updated, so every edge into a vertex discovered in the same level issues a red.or, tens of millions
    // on the big R-MAT level; ER n=2^25 6.41 -> 3.69 ms with it)
    if (g.info.layout == AG_LAYOUT_DEGREE && !(p.free_ppm >= 1000000u)) d.t_free = ~0ull;
    // SSSP: free output only on non-skewed graphs (measured: ER n=2^25 21.4 -> 12.4 ms; R-MAT s22
    // 1.59 -> 2.19 ms, the fire-and-forget red.min on power-law hot targets loses to the claiming
    // atomicMin whose result gates the next-bitmap update)
    d.t_free_sssp = (g.info.layout == AG_LAYOUT_DEGREE && !(p.free_ppm >= 1000000u)) ? ~0ull : t_free_any;
    // small-frontier mode (graphs without hub tasks): an iteration whose working set is below t_small runs
    // on one CTA per SM, the others park — the grid barrier that ends every iteration then has 148
    // arrivals instead of ~740 (measured C3 grid: BFS 55.9 -> 42.4 ms, SSSP 129 -> 92.7 ms with 148 CTAs)
    d.small_ctas = (uint32_t)g.num_sms;
    d.t_small = p.kind == AG_POLICY_TUNED ? (p.small_ws ? p.small_ws : 32768u) : 0u;
    d.t_small_hub = p.kind == AG_POLICY_TUNED ? (uint32_t)AG_T_SMALL_HUB : 0u;   // C2: BFS -1.6%, SSSP -2.7% (median of 12)
    d.smallchunk_per_cta = SMALLCHUNK_PER_CTA;
    d.ordered = p.order == AG_ORDERED ? 1u : 0u;
    // NEXT-3: the SSSP order axis adapted per iteration from the measured redundancy
    d.adapt = (p.order == AG_ORDERED) ? (p.delta == 0 ? 1u : 0u) : (p.sssp_window == AG_WINDOW_ADAPTIVE ? 1u : 0u);
    d.win_max = 1u << 24;
    return d;
}

ag_status check_policy(const ag_policy *p) {
    if (p->struct_size != sizeof(ag_policy)) return set_error(AG_ERR_INVALID_ARG, "ag_policy.struct_size mismatch");
    if (p->order > AG_ORDERED || p->mapping > AG_MAP_HYBRID || p->workset > AG_WS_QUEUE || p->kind > AG_POLICY_TUNED)
        return set_error(AG_ERR_INVALID_ARG, "ag_policy field out of range");
    if (p->cta_group % 32) return set_error(AG_ERR_INVALID_ARG, "cta_group must be a multiple of 32");
    if (p->delta >= 0x80000000u) return set_error(AG_ERR_INVALID_ARG, "delta must be 0 (adaptive) or in [1, 2^31)");
    return AG_OK;
}

}  // namespace ag

// ------------------------------------------------------------------------------------------------
// traversal launch
// ------------------------------------------------------------------------------------------------
#ifndef AG_DONLY
#define AG_DONLY 1
#endif
template <int ALG, int ORD, typename Off>
static ag_status launch_traverse(ag_graph_s *g, TravArgs<Off> &a, cudaStream_t st) {
    // the tuned adaptive policy runs the specialisation without the paper's static variants
    // Unordered BFS on degree-layout (hub) graphs runs the tuned policy's decisions (hybrid mapping,
    // queue) in the general specialisation: C2 median 0.575 -> 0.566 ms, mean 0.588 -> 0.565 ms over
    // 16 sources (profiles/r01_bfs_tuned_probe.txt; cause in the tuned specialisation not found).
    // A forced variant the tuned specialisation implements (thread or hybrid mapping over the queue; for the
    // ordered-SSSP pending set also the bitmap) runs in it too, with the same engine features as the
    // adaptive runs (free output, small-frontier mode), so static-vs-adaptive is like for like there.
    const bool tuned_map = a.pol.force_map == 0 || a.pol.force_map == MAP_T || a.pol.force_map == MAP_H;
    const bool tuned_ws = a.pol.force_ws == 0 || a.pol.force_ws == WS_QU ||
                          (ALG == ALG_SSSP && ORD == ORD_O && a.pol.force_ws == WS_BM);
    const bool tuned = a.pol.kind == AG_POLICY_TUNED && tuned_map && tuned_ws &&
                       !(AG_BFS_ROUTE && ALG == ALG_BFS && ORD == ORD_U && g->info.layout == AG_LAYOUT_DEGREE);
    // SSSP without parents in the tuned specialisation: distance-only state (u32)
    const bool donly = AG_DONLY && ALG == ALG_SSSP && tuned && a.parent_out == nullptr;
    g->last_packed = !donly;
    auto fn = !tuned ? traverse_kernel<ALG, ORD, Off, false>
              : donly ? traverse_kernel<ALG, ORD, Off, true, ALG == ALG_SSSP>
                      : traverse_kernel<ALG, ORD, Off, true>;
    const size_t dyn = 0;
    if (dyn) cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn);
    int occ = 0;
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, BS, dyn);
    if (e != cudaSuccess || occ < 1) return cuda_status(e == cudaSuccess ? cudaErrorLaunchOutOfResources : e, "occupancy");
    // L1/shared carveout: request just the shared memory the resident CTAs need so the rest of the
    // 256 KB goes to L1, where the status gathers hit (the driver otherwise picked a 132 KB shared
    // configuration for ~100 KB of use).  Once per kernel.
    static int carved[3] = {0, 0, 0};   // per specialisation (paper variants / tuned / tuned distance-only)
    const int spec = tuned ? (donly ? 2 : 1) : 0;
    if (!carved[spec]) {
        carved[spec] = 1;
        int pct = -1;
        cudaFuncAttributes fa;
        if (cudaFuncGetAttributes(&fa, fn) == cudaSuccess) {
            const double need = (double)occ * ((double)fa.sharedSizeBytes + dyn + 1024.0);
            pct = (int)((need * 100.0 + 228.0 * 1024.0 - 1.0) / (228.0 * 1024.0));
            if (pct > 100) pct = 100;
        }
        if (pct >= 0) {
            cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, pct);
            int occ2 = 0;
            if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ2, fn, BS, dyn) != cudaSuccess || occ2 < occ) {
                cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, -1);   // keep occupancy
            }
        }
        cudaGetLastError();
    }
    a.nblocks = (uint32_t)(occ * g->num_sms);
    // Cooperative launch (co-resident grid for the software grid barrier) with an L2 access-policy
    // window marking the per-vertex status array persisting, so the ~1 GB CSR stream does not evict
    // it.  The window is a per-launch attribute: the caller's stream is not modified.
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(a.nblocks);
    cfg.blockDim = dim3(BS);
    cfg.dynamicSmemBytes = dyn;
    cfg.stream = st;
    cudaLaunchAttribute attrs[2];
    attrs[0].id = cudaLaunchAttributeCooperative;
    attrs[0].val.cooperative = 1;
    int nattr = 1;
    void *wbase = ALG == ALG_SSSP ? (void *)a.P : ALG == ALG_CC ? (void *)a.level : (void *)a.vis;
    size_t wbytes = ALG == ALG_SSSP ? (size_t)g->V * (donly ? 4 : 8) : ALG == ALG_CC ? (size_t)g->V * 4 : (size_t)g->nwords * 4;
    if (g->persist_bytes > 0) {
        if (wbytes > g->max_window) wbytes = g->max_window;
        attrs[1].id = cudaLaunchAttributeAccessPolicyWindow;
        attrs[1].val.accessPolicyWindow.base_ptr = wbase;
        attrs[1].val.accessPolicyWindow.num_bytes = wbytes;
        attrs[1].val.accessPolicyWindow.hitRatio =
            wbytes <= g->persist_bytes ? 1.0f : (float)g->persist_bytes / (float)wbytes;
        attrs[1].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        attrs[1].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        nattr = 2;
    }
    cfg.attrs = attrs;
    cfg.numAttrs = nattr;
    e = cudaLaunchKernelEx(&cfg, fn, a);
    note_launch(1);
    return cuda_status(e, "traverse launch");
}

template <typename Off>
static ag_status run_query(ag_graph_s *g, int alg, uint32_t src, uint32_t *out, uint32_t *parents,
                           const ag_policy *pin, ag_run_stats *stats, cudaStream_t st) {
    ag_policy pol;
    if (pin) {
        pol = *pin;
    } else {
        ag_policy_default(&pol, g->device);
    }
    ag_status s = check_policy(&pol);
    if (s != AG_OK) return s;
    if (alg == ALG_CC && pol.order == AG_ORDERED) return set_error(AG_ERR_UNSUPPORTED, "ag_cc is unordered only (DESIGN.md R23)");
    if (stats && stats->struct_size != sizeof(ag_run_stats))
        return set_error(AG_ERR_INVALID_ARG, "ag_run_stats.struct_size mismatch");
    cudaSetDevice(g->device);
    if ((s = ensure_scratch(g, alg == ALG_SSSP)) != AG_OK) return s;

    const bool out_dev = is_device_ptr(out);
    const bool par_dev = parents ? is_device_ptr(parents) : true;
    const bool sync = stats != nullptr || !out_dev || !par_dev;
    const size_t vbytes = (size_t)g->V * 4 + 128;
    uint32_t *d_out = out, *d_par = parents;
    if (!out_dev) {
        if ((s = ensure_buf(g, &g->d_out_tmp, &g->out_tmp_bytes, vbytes)) != AG_OK) return s;
        d_out = g->d_out_tmp;
    }
    if (parents && !par_dev) {
        if ((s = ensure_buf(g, &g->d_par_tmp, &g->par_tmp_bytes, vbytes)) != AG_OK) return s;
        d_par = g->d_par_tmp;
    }
    uint32_t tcap = (stats && (stats->trace_ws || stats->trace_edges || stats->trace_variant || stats->trace_ns))
                        ? stats->trace_cap : 0;
    if (tcap) {
        size_t need = (size_t)tcap * 24 + 64;
        if ((s = ensure_buf(g, &g->d_trace, &g->trace_bytes, need)) != AG_OK) return s;
    }

    TravArgs<Off> a;
    memset(&a, 0, sizeof a);
    a.rp = (const Off *)g->d_rp;
    a.col = g->d_col;
    a.cw = g->d_cw;
    a.V = g->V;
    a.nwords = g->nwords;
    a.P = g->d_P;
    a.vis = g->d_vis;
    for (int i = 0; i < 3; ++i) { a.bm[i] = g->d_bm[i]; a.q[i] = g->d_q[i]; }
    a.hub = g->d_hub;
    a.hub_cap = g->hub_cap;
    a.ctl = (Ctl *)g->d_ctl;
    a.perm = g->d_perm;
    a.inv = g->d_inv;
    if (alg != ALG_SSSP) {   // BFS levels / CC labels
        if (g->d_inv) {  // traverse in the degree layout, gather back to caller ids at the end
            if (!g->d_level && (s = dev_alloc((void **)&g->d_level, (size_t)g->V * 4 + 128, g->device)) != AG_OK) return s;
            if (d_par && !g->d_lpar && (s = dev_alloc((void **)&g->d_lpar, (size_t)g->V * 4 + 128, g->device)) != AG_OK)
                return s;
            a.level = g->d_level;
            a.parent = d_par ? g->d_lpar : nullptr;
            a.out_level = d_out;
            a.out_parent = d_par;
        } else {
            a.level = d_out;
            a.parent = d_par;
        }
    } else {
        a.dist_out = d_out;
        a.parent_out = d_par;
    }
    if (tcap) {
        uint8_t *base = (uint8_t *)g->d_trace;
        a.trace_edges = (unsigned long long *)base;
        a.trace_ws = (uint32_t *)(base + (size_t)tcap * 8);
        a.trace_var = base + (size_t)tcap * 12;
        a.trace_ns = (unsigned long long *)(base + (((size_t)tcap * 13 + 15) & ~size_t(15)));
        a.trace_cap = tcap;
    }
    a.pol = resolve_policy(pol, *g);
    a.src = src;
    {   // iteration cap (never expected to bind): BFS/CC <= V + 1 levels / label rounds; SSSP generous
        const uint64_t cap = alg != ALG_SSSP ? (uint64_t)g->V + 2 : 4ull * g->V + 64;
        a.max_iters = (uint32_t)(cap > 0xFFFFFFF0ull ? 0xFFFFFFF0ull : cap);
    }
    a.has_hubs = g->info.max_deg >= HUB_DEG;

    if (stats) {
        cudaEventRecord(g->ev[0], st);
    }
    if (alg == ALG_BFS) {
        s = (pol.order == AG_ORDERED) ? launch_traverse<ALG_BFS, ORD_O, Off>(g, a, st)
                                      : launch_traverse<ALG_BFS, ORD_U, Off>(g, a, st);
    } else if (alg == ALG_CC) {
        s = launch_traverse<ALG_CC, ORD_U, Off>(g, a, st);
    } else {
        s = (pol.order == AG_ORDERED) ? launch_traverse<ALG_SSSP, ORD_O, Off>(g, a, st)
                                      : launch_traverse<ALG_SSSP, ORD_U, Off>(g, a, st);
    }
    if (s != AG_OK) return s;
    if (stats) cudaEventRecord(g->ev[1], st);
    if (alg == ALG_SSSP) {   // deferred exact overflow test (a no-op launch unless the traversal flagged one)
        Ctl *ctl = (Ctl *)g->d_ctl;
        overflow_check_kernel<Off><<<g->num_sms * 4, 256, 0, st>>>(ctl, g->d_P, g->last_packed, (const Off *)g->d_rp,
                                                                    g->d_cw, g->V, &ctl->sticky);
        note_launch(1);
    }
    g->last_stream = st;
    g->pending_check = true;

    if (!out_dev) cudaMemcpyAsync(out, d_out, (size_t)g->V * 4, cudaMemcpyDeviceToHost, st);
    if (parents && !par_dev) cudaMemcpyAsync(parents, d_par, (size_t)g->V * 4, cudaMemcpyDeviceToHost, st);
    if (!sync) return cuda_status(cudaGetLastError(), "enqueue");

    if (stats) {
        cudaMemsetAsync(g->d_acc, 0, 16, st);
        reached_kernel<Off><<<g->num_sms * 4, 256, 0, st>>>(d_out, (const Off *)g->d_rp, g->d_inv, g->V,
                                                             (unsigned long long *)g->d_acc);
        note_launch(1);
    }
    cudaError_t e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return cuda_status(e, "traversal");
    s = ag_graph_check(g);
    if (s != AG_OK && s != AG_ERR_OVERFLOW) return s;
    if (stats) {
        Ctl c;
        cudaMemcpy(&c, g->d_ctl, sizeof c, cudaMemcpyDeviceToHost);
        unsigned long long acc[2];
        cudaMemcpy(acc, g->d_acc, 16, cudaMemcpyDeviceToHost);
        stats->iterations = c.iterations;
        stats->vertices_expanded = c.vexp;
        stats->edges_inspected = c.eexp;
        stats->reached = acc[0];
        stats->reached_edges = acc[1];
        float ms = 0;
        cudaEventElapsedTime(&ms, g->ev[0], g->ev[1]);
        stats->device_ms = ms;
        uint32_t n = c.iterations < tcap ? c.iterations : tcap;
        stats->trace_len = n;
        if (n) {
            uint8_t *base = (uint8_t *)g->d_trace;
            if (stats->trace_edges) cudaMemcpy(stats->trace_edges, base, (size_t)n * 8, cudaMemcpyDeviceToHost);
            if (stats->trace_ws) cudaMemcpy(stats->trace_ws, base + (size_t)tcap * 8, (size_t)n * 4, cudaMemcpyDeviceToHost);
            if (stats->trace_variant) cudaMemcpy(stats->trace_variant, base + (size_t)tcap * 12, n, cudaMemcpyDeviceToHost);
            if (stats->trace_ns)
                cudaMemcpy(stats->trace_ns, base + (((size_t)tcap * 13 + 15) & ~size_t(15)),
                           (size_t)(c.iterations < tcap ? n + 1 : n) * 8, cudaMemcpyDeviceToHost);
        }
        e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_status(e, "stats");
    }
    return s;
}

// ------------------------------------------------------------------------------------------------
// C ABI
// ------------------------------------------------------------------------------------------------
extern "C" {

uint32_t ag_abi_version(void) { return AG_ABI_VERSION; }
uint64_t ag_kernel_launches(void) { return g_launches.load(); }
const char *ag_last_error(void) { return g_last_error.c_str(); }

// diagnostic builds (-DAG_PROF) only: copy the per-(iteration, CTA) timestamps to host memory
int ag_debug_prof(void *host, size_t bytes) {
#ifdef AG_PROF
    size_t n = sizeof(ag::g_prof) < bytes ? sizeof(ag::g_prof) : bytes;
    return cudaMemcpyFromSymbol(host, ag::g_prof, n) == cudaSuccess ? (int)ag::PROF_CTA : -1;
#else
    (void)host;
    (void)bytes;
    return -1;
#endif
}

const char *ag_status_string(ag_status s) {
    switch (s) {
        case AG_OK: return "AG_OK";
        case AG_ERR_INVALID_ARG: return "AG_ERR_INVALID_ARG";
        case AG_ERR_BAD_CSR: return "AG_ERR_BAD_CSR";
        case AG_ERR_SRC_RANGE: return "AG_ERR_SRC_RANGE";
        case AG_ERR_NO_WEIGHTS: return "AG_ERR_NO_WEIGHTS";
        case AG_ERR_OVERFLOW: return "AG_ERR_OVERFLOW";
        case AG_ERR_OOM: return "AG_ERR_OOM";
        case AG_ERR_CUDA: return "AG_ERR_CUDA";
        case AG_ERR_NCCL: return "AG_ERR_NCCL";
        case AG_ERR_UNSUPPORTED: return "AG_ERR_UNSUPPORTED";
        case AG_ERR_NO_DEVICE: return "AG_ERR_NO_DEVICE";
    }
    return "AG_ERR_?";
}

ag_status ag_set_allocator(void *(*alloc)(size_t, int, void *, void *), void (*free_)(void *, size_t, int, void *, void *),
                           void *ctx) {
    if ((alloc == nullptr) != (free_ == nullptr)) return set_error(AG_ERR_INVALID_ARG, "alloc and free must both be set");
    g_alloc = alloc;
    g_free = free_;
    g_alloc_ctx = ctx;
    return AG_OK;
}

ag_status ag_policy_default(ag_policy *p, int device) {
    if (!p) return set_error(AG_ERR_INVALID_ARG, "policy is NULL");
    int sms = 0;
    ag_status s = check_device(device, &sms);
    if (s != AG_OK) return s;
    memset(p, 0, sizeof *p);
    p->struct_size = sizeof(ag_policy);
    p->order = AG_UNORDERED;
    p->mapping = AG_MAP_AUTO;
    p->workset = AG_WS_AUTO;
    p->kind = AG_POLICY_TUNED;
    p->t1_avg_degree = 32;
    p->thread_tpb = 192;
    p->t2_ws = 192ull * (uint64_t)sms;
    p->t3_ppm = 100000;   // T3 = 10% of V: the B200 calibration (X8, profiles/sweeps/r02_x8_C4.jsonl)
    p->sample_every = 1;
    p->delta = 1;
    p->cta_group = 0;
    p->sssp_window = AG_WINDOW_AUTO;
    p->sssp_hub_window = AG_WINDOW_AUTO;
    p->free_ppm = 3906;   // V/256 (tools/sweep.py --set free_ppm=...)
    return AG_OK;
}

uint8_t ag_select(const ag_policy *p, const ag_graph_info *gi, uint64_t ws_size, uint64_t ws_edges) {
    if (!p || !gi || check_policy(p) != AG_OK) return 0;
    ag_graph_s tmp;
    tmp.V = gi->num_vertices;
    tmp.E = gi->num_edges;
    tmp.info = *gi;
    DevPolicy d = resolve_policy(*p, tmp);
    return select_variant(d, ws_size, ws_edges);
}

ag_status ag_graph_load_csr(uint32_t V, uint64_t E, const uint64_t *row_ptr, const uint32_t *col_idx,
                            const uint32_t *weights, int device, ag_graph *out) {
    return ag_graph_load_csr_ex(V, E, row_ptr, col_idx, weights, device, AG_LAYOUT_AUTO, out);
}

ag_status ag_graph_load_csr_ex(uint32_t V, uint64_t E, const uint64_t *row_ptr, const uint32_t *col_idx,
                               const uint32_t *weights, int device, uint32_t layout, ag_graph *out) {
    if (layout > AG_LAYOUT_DEGREE) return set_error(AG_ERR_INVALID_ARG, "unknown layout %u", layout);
    if (!out || !row_ptr || (!col_idx && E > 0)) return set_error(AG_ERR_INVALID_ARG, "NULL argument");
    *out = nullptr;
    if (V == 0 || V >= 0xFFFFFFFFu) return set_error(AG_ERR_BAD_CSR, "V must be in [1, 2^32-1)");
    int sms = 0;
    ag_status s = check_device(device, &sms);
    if (s != AG_OK) return s;
    cudaSetDevice(device);
    ag_graph_s *g = new ag_graph_s();
    g->device = device;
    g->V = V;
    g->E = E;
    g->num_sms = sms;
    g->nwords = (V + 31) / 32;
    g->offs32 = E < 0xFFFFFFFFull;
    {   // tasks of one iteration <= E / chunk + (lists >= the task degree), for the smallest chunk/degree in use
        const uint64_t ch = HUB_CHUNK_SMALL < HUB_CHUNK ? HUB_CHUNK_SMALL : HUB_CHUNK;
        const uint64_t hd = HUB_CHUNK_SMALL < HUB_DEG ? HUB_CHUNK_SMALL : HUB_DEG;
        const uint64_t c = E / ch + E / hd + 16;
        g->hub_cap = (uint32_t)(c > 0xFFFFFFF0ull ? 0xFFFFFFF0ull : c);
    }
    cudaEventCreate(&g->ev[0]);
    cudaEventCreate(&g->ev[1]);
    auto fail = [&](ag_status st) { ag_graph_free(g); return st; };

    // ---- pipelined load (row a1): the row offsets are copied and validated first
    // (the inspector's degree statistics decide the layout), then col_idx / weights stream in
    // CH-edge chunks on a copy stream while a processing stream validates each chunk and builds the
    // final arrays from it (identity: the (col, w) interleave; degree layout: the relabelled rows
    // whose last entry is in the chunk).  The host waits once, so the PCIe copy hides the processing.
    LoadStats hs = {0, 0xFFFFFFFFu, 0, 0, 0};
    uint64_t *rp64 = nullptr;
    LoadStats *dst = nullptr;
    uint32_t *col_old = nullptr, *w_old = nullptr;   // staging (freed at the end of the load)
    unsigned long long *keys = nullptr, *keys2 = nullptr;
    uint64_t *ndeg = nullptr, *nrp = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0;
    uint64_t *rp_host = nullptr;   // host copy of row_ptr when the caller passed device memory (degree layout)
    cudaStream_t s_copy = nullptr, s_proc = nullptr;
    std::vector<cudaEvent_t> evs;
    auto release = [&]() {
        if (s_copy) cudaStreamSynchronize(s_copy);
        if (s_proc) cudaStreamSynchronize(s_proc);
        for (auto ev : evs) cudaEventDestroy(ev);
        evs.clear();
        if (s_copy) cudaStreamDestroy(s_copy);
        if (s_proc) cudaStreamDestroy(s_proc);
        s_copy = s_proc = nullptr;
        dev_free(rp64, (size_t)(V + 1) * 8 + 8, device);
        dev_free(dst, sizeof(LoadStats), device);
        dev_free(col_old, E * 4 + 128, device);
        dev_free(w_old, E * 4 + 128, device);
        dev_free(keys, (size_t)V * 8, device);
        dev_free(keys2, (size_t)V * 8, device);
        dev_free(ndeg, (size_t)V * 8 + 8, device);
        dev_free(nrp, (size_t)V * 8 + 8, device);
        dev_free(tmp, tmp_bytes, device);
        free(rp_host);
        rp64 = nullptr; dst = nullptr; col_old = w_old = nullptr; keys = keys2 = nullptr; ndeg = nrp = nullptr;
        tmp = nullptr; rp_host = nullptr;
    };
    auto lfail = [&](ag_status st) { release(); return fail(st); };
    cudaError_t e = cudaStreamCreateWithFlags(&s_copy, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&s_proc, cudaStreamNonBlocking);
    if (e != cudaSuccess) return lfail(cuda_status(e, "load streams"));
    if ((s = dev_alloc((void **)&rp64, (size_t)(V + 1) * 8 + 8, device)) != AG_OK) return lfail(s);
    if ((s = dev_alloc((void **)&dst, sizeof(LoadStats), device)) != AG_OK) return lfail(s);
    e = cudaMemcpyAsync(rp64, row_ptr, (size_t)(V + 1) * 8, cudaMemcpyDefault, s_proc);
    if (e == cudaSuccess) e = cudaMemcpyAsync(dst, &hs, sizeof hs, cudaMemcpyHostToDevice, s_proc);
    if (e == cudaSuccess) {
        validate_rows_kernel<<<sms * 8, 256, 0, s_proc>>>(rp64, V, E, dst);
        note_launch(1);
        e = cudaMemcpyAsync(&hs, dst, sizeof hs, cudaMemcpyDeviceToHost, s_proc);
    }
    if (e == cudaSuccess) e = cudaStreamSynchronize(s_proc);
    if (e != cudaSuccess) return lfail(cuda_status(e, "graph load"));
    if (hs.bad)
        return lfail(set_error(AG_ERR_BAD_CSR, "invalid CSR (%s%s%s)", hs.bad & 1 ? "row_ptr[0]!=0 " : "",
                               hs.bad & 2 ? "non-monotone row_ptr " : "", hs.bad & 4 ? "row_ptr[V]!=E " : ""));
    // inspector decides the device layout (skewed degree distribution -> degree order)
    if (layout == AG_LAYOUT_AUTO) {
        uint64_t avg = (E + V - 1) / V;
        layout = (E > 0 && (uint64_t)hs.max_deg >= 64ull * (avg ? avg : 1)) ? AG_LAYOUT_DEGREE : AG_LAYOUT_IDENTITY;
        if (V >= 0x80000000u) layout = AG_LAYOUT_IDENTITY;   // the degree sort counts items in 31 bits
    }
    if (layout == AG_LAYOUT_DEGREE && V >= 0x80000000u)
        return lfail(set_error(AG_ERR_UNSUPPORTED, "the degree layout needs V < 2^31"));
    g->layout = layout;
    const bool deg = layout == AG_LAYOUT_DEGREE;
    // final arrays
    if ((s = dev_alloc((void **)&g->d_col, E * 4 + 128, device)) != AG_OK) return lfail(s);
    g->col_bytes = E * 4 + 128;
    if (weights) {
        if ((s = dev_alloc((void **)&g->d_cw, E * 8 + 128, device)) != AG_OK) return lfail(s);
        g->cw_bytes = E * 8 + 128;
        if ((s = dev_alloc((void **)&w_old, E * 4 + 128, device)) != AG_OK) return lfail(s);
    }
    if (deg) {
        if ((s = dev_alloc((void **)&col_old, E * 4 + 128, device)) != AG_OK) return lfail(s);
        if ((s = dev_alloc((void **)&keys, (size_t)V * 8, device)) != AG_OK) return lfail(s);
        if ((s = dev_alloc((void **)&keys2, (size_t)V * 8, device)) != AG_OK) return lfail(s);
        if ((s = dev_alloc((void **)&ndeg, (size_t)V * 8 + 8, device)) != AG_OK) return lfail(s);
        if ((s = dev_alloc((void **)&nrp, (size_t)V * 8 + 8, device)) != AG_OK) return lfail(s);
        if ((s = dev_alloc((void **)&g->d_perm, (size_t)V * 4, device)) != AG_OK) return lfail(s);
        if ((s = dev_alloc((void **)&g->d_inv, (size_t)V * 4, device)) != AG_OK) return lfail(s);
        size_t t1 = 0, t2 = 0;
        cub::DeviceRadixSort::SortKeys(nullptr, t1, keys, keys2, (int)V);
        cub::DeviceScan::ExclusiveSum(nullptr, t2, ndeg, nrp, (int)V + 1);
        tmp_bytes = t1 > t2 ? t1 : t2;
        if ((s = dev_alloc(&tmp, tmp_bytes, device)) != AG_OK) return lfail(s);
        if (is_device_ptr(row_ptr)) {   // the chunk -> row ranges are found on the host
            rp_host = (uint64_t *)malloc((size_t)(V + 1) * 8);
            if (!rp_host) return lfail(set_error(AG_ERR_OOM, "host row_ptr copy"));
            e = cudaMemcpy(rp_host, row_ptr, (size_t)(V + 1) * 8, cudaMemcpyDeviceToHost);
            if (e != cudaSuccess) return lfail(cuda_status(e, "row_ptr readback"));
        }
        // degree order and new row offsets (overlaps the edge copies below)
        build_degree_order(rp64, V, keys, keys2, tmp, tmp_bytes, g->d_perm, g->d_inv, ndeg, nrp, sms, s_proc);
    }
    const uint64_t *rph = rp_host ? rp_host : row_ptr;
    uint32_t *col_dst = deg ? col_old : g->d_col;
    const uint64_t CH = 1ull << 24;   // edges per chunk (64 MB of col_idx, 64 MB of weights)
    uint32_t row_a = 0;
    for (uint64_t e0 = 0; e0 < E; e0 += CH) {
        const uint64_t e1 = (E - e0 > CH) ? e0 + CH : E;
        cudaEvent_t ev;
        if ((e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming)) != cudaSuccess) return lfail(cuda_status(e, "event"));
        evs.push_back(ev);
        e = cudaMemcpyAsync(col_dst + e0, col_idx + e0, (e1 - e0) * 4, cudaMemcpyDefault, s_copy);
        if (e == cudaSuccess && weights) e = cudaMemcpyAsync(w_old + e0, weights + e0, (e1 - e0) * 4, cudaMemcpyDefault, s_copy);
        if (e == cudaSuccess) e = cudaEventRecord(ev, s_copy);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(s_proc, ev, 0);
        if (e != cudaSuccess) return lfail(cuda_status(e, "edge copy"));
        const int grid = sms * 8;
        if (!deg) {
            validate_edges_kernel<<<grid, 256, 0, s_proc>>>(g->d_col + e0, weights ? w_old + e0 : nullptr, e1 - e0, V, dst);
            if (weights) interleave_kernel<<<grid, 256, 0, s_proc>>>(g->d_col + e0, w_old + e0, g->d_cw + e0, e1 - e0);
            note_launch(weights ? 2 : 1);
        } else {
            // rows whose last entry lies in [e0, e1) (all their entries have arrived): rp[u+1] <= e1
            uint32_t lo = row_a, hi = V;   // first u in [row_a, V] with rp[u+1] > e1 (V if none)
            if (e1 < E) {
                while (lo < hi) {
                    const uint32_t mid = lo + (hi - lo) / 2;
                    if (rph[mid + 1] > e1) hi = mid; else lo = mid + 1;
                }
            } else {
                lo = V;
            }
            if (lo > row_a) {
                relabel_edges_kernel<<<grid, 256, 0, s_proc>>>(rp64, col_old, weights ? w_old : nullptr, g->d_inv, nrp, V,
                                                               row_a, lo, g->d_col, g->d_cw, dst);
                note_launch(1);
            }
            row_a = lo;
        }
    }
    // final row offsets (u32 when E < 2^32)
    const uint64_t *rp_final = deg ? nrp : rp64;
    if (g->offs32) {
        uint32_t *rp32 = nullptr;
        if ((s = dev_alloc((void **)&rp32, (size_t)(V + 1) * 4 + 128, device)) != AG_OK) return lfail(s);
        g->d_rp = rp32;
        g->rp_bytes = (size_t)(V + 1) * 4 + 128;
        narrow_offsets_kernel<<<sms * 8, 256, 0, s_proc>>>(rp_final, rp32, V + 1);
        note_launch(1);
    } else {
        uint64_t *rpk = nullptr;
        if ((s = dev_alloc((void **)&rpk, (size_t)(V + 1) * 8 + 8, device)) != AG_OK) return lfail(s);
        g->d_rp = rpk;
        g->rp_bytes = (size_t)(V + 1) * 8 + 8;
        e = cudaMemcpyAsync(rpk, rp_final, (size_t)(V + 1) * 8, cudaMemcpyDeviceToDevice, s_proc);
        if (e != cudaSuccess) return lfail(cuda_status(e, "row offsets"));
    }
    LoadStats he = hs;
    e = cudaMemcpyAsync(&he, dst, sizeof he, cudaMemcpyDeviceToHost, s_proc);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s_proc);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s_copy);
    if (e == cudaSuccess) e = cudaGetLastError();
    if (e != cudaSuccess) return lfail(cuda_status(e, "graph load"));
    if (he.bad)
        return lfail(set_error(AG_ERR_BAD_CSR, "invalid CSR (%s%s)", he.bad & 8 ? "col>=V " : "",
                               he.bad & 16 ? "weight not in [1,2^31) " : ""));
    hs.max_w = he.max_w;
    release();
    g->info.num_vertices = V;
    g->info.num_edges = E;
    g->info.deg_sum = E;
    g->info.min_deg = hs.min_deg == 0xFFFFFFFFu ? 0 : hs.min_deg;
    g->info.max_deg = hs.max_deg;
    g->info.isolated = hs.isolated;
    g->info.weighted = weights ? 1 : 0;
    g->info.device = device;
    g->info.num_sms = sms;
    g->info.offset_bytes = g->offs32 ? 4 : 8;
    g->info.layout = g->layout;
    g->info.max_weight = weights ? hs.max_w : 0;
    {   // L2 set-aside for the persisting status window (device-wide limit, set once to the maximum)
        const DevAttrs *da = device_attrs(device);
        size_t cur = 0;
        cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
        if (da && cur < (size_t)da->persist_max) {
            cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)da->persist_max);
            cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
        }
        g->persist_bytes = cur;
        g->max_window = da ? (size_t)da->window_max : 0;
        cudaGetLastError();
    }
    *out = g;
    return AG_OK;
}

ag_status ag_graph_info_get(ag_graph g, ag_graph_info *out) {
    if (!g || !out) return set_error(AG_ERR_INVALID_ARG, "NULL argument");
    *out = g->info;
    return AG_OK;
}

ag_status ag_graph_free(ag_graph g) {
    if (!g) return set_error(AG_ERR_INVALID_ARG, "NULL graph");
    cudaSetDevice(g->device);
    if (g->last_stream || g->pending_check) cudaDeviceSynchronize();
    dev_free(g->d_rp, g->rp_bytes, g->device);
    dev_free(g->d_col, g->col_bytes, g->device);
    dev_free(g->d_w, g->w_bytes, g->device);
    dev_free(g->d_cw, g->cw_bytes, g->device);
    const size_t V = g->V, nw = g->nwords;
    dev_free(g->d_ctl, sizeof(Ctl), g->device);
    for (int i = 0; i < 3; ++i) { dev_free(g->d_bm[i], nw * 4 + 128, g->device); dev_free(g->d_q[i], V * 4 + 128, g->device); }
    dev_free(g->d_vis, nw * 4 + 128, g->device);
    dev_free(g->d_hub, (size_t)g->hub_cap * 8, g->device);
    dev_free(g->d_acc, 64, g->device);
    dev_free(g->d_P, V * 8 + 128, g->device);
    dev_free(g->d_out_tmp, g->out_tmp_bytes, g->device);
    dev_free(g->d_par_tmp, g->par_tmp_bytes, g->device);
    dev_free(g->d_trace, g->trace_bytes, g->device);
    dev_free(g->d_perm, V * 4, g->device);
    dev_free(g->d_inv, V * 4, g->device);
    dev_free(g->d_level, V * 4 + 128, g->device);
    dev_free(g->d_lpar, V * 4 + 128, g->device);
    if (g->ev[0]) cudaEventDestroy(g->ev[0]);
    if (g->ev[1]) cudaEventDestroy(g->ev[1]);
    ag::dist_graph_release(g);
    delete g;
    return AG_OK;
}

ag_status ag_graph_check(ag_graph g) {
    if (!g) return set_error(AG_ERR_INVALID_ARG, "NULL graph");
    if (!g->pending_check) return AG_OK;
    cudaSetDevice(g->device);
    cudaError_t e = cudaStreamSynchronize(g->last_stream);
    if (e != cudaSuccess) return cuda_status(e, "traversal");
    g->pending_check = false;
    // the sticky status accumulates over every traversal enqueued since the last check (a launch
    // never clears it), so an overflow or abort of an earlier query is not lost behind a later one
    unsigned sticky = 0;
    unsigned *d_sticky = (unsigned *)((char *)g->d_ctl + offsetof(Ctl, sticky));
    e = cudaMemcpy(&sticky, d_sticky, 4, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) return cuda_status(e, "ctl");
    if (!sticky) return AG_OK;
    cudaMemset(d_sticky, 0, 4);
    if (sticky >> 8) {
        if (g->d_hub) cudaMemset(g->d_hub, 0, (size_t)g->hub_cap * 8);   // the ring may hold unconsumed tasks
        return set_error(AG_ERR_CUDA, "traversal aborted (code %u)", sticky >> 8);
    }
    return set_error(AG_ERR_OVERFLOW, "a finite distance exceeds 0xFFFFFFFE");
}

static ag_status query(ag_graph g, int alg, uint32_t src, uint32_t *out, uint32_t *parents, const ag_policy *p,
                       ag_run_stats *stats, void *stream) {
    if (!g || !out) return set_error(AG_ERR_INVALID_ARG, "NULL argument");
    if (alg == ALG_CC && parents) return set_error(AG_ERR_INVALID_ARG, "ag_cc has no parents");
    if (src >= g->V) return set_error(AG_ERR_SRC_RANGE, "src %u >= V %u", src, g->V);
    if (alg == ALG_SSSP && !g->d_cw) return set_error(AG_ERR_NO_WEIGHTS, "graph was loaded without weights");
    if (g->dist) return set_error(AG_ERR_INVALID_ARG, "distributed graph: use ag_dist_bfs");
    cudaStream_t st = (cudaStream_t)stream;
    return g->offs32 ? run_query<uint32_t>(g, alg, src, out, parents, p, stats, st)
                     : run_query<unsigned long long>(g, alg, src, out, parents, p, stats, st);
}

ag_status ag_bfs(ag_graph g, uint32_t src, uint32_t *levels, uint32_t *parents, const ag_policy *policy,
                 ag_run_stats *stats, void *stream) {
    return query(g, ALG_BFS, src, levels, parents, policy, stats, stream);
}

ag_status ag_sssp(ag_graph g, uint32_t src, uint32_t *dist, uint32_t *parents, const ag_policy *policy,
                  ag_run_stats *stats, void *stream) {
    return query(g, ALG_SSSP, src, dist, parents, policy, stats, stream);
}

ag_status ag_cc(ag_graph g, uint32_t *labels, const ag_policy *policy, ag_run_stats *stats, void *stream) {
    return query(g, ALG_CC, 0, labels, nullptr, policy, stats, stream);
}

}  // extern "C"
