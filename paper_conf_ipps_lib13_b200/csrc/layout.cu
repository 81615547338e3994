// layout.cu — degree-ordered device vertex layout (part of the CSR store, row a1; load time, untimed).
//
// New id i holds old vertex perm[i], sorted by descending out-degree (ties by old id); inv = perm^-1.
// The CSR is rewritten in the new ids: row i = old row perm[i] with every neighbour mapped through
// inv.  Power-law graphs (R-MAT, the SNS/CiteSeer-like datasets of PAPER.md:14.s8-10) send most
// edges to a few high-degree vertices; after relabelling their visited bits / states sit in a
// small prefix that stays in L1/L2, which turns most per-edge status checks into cache hits.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include "common.cuh"
#include "graph.h"

namespace ag {

__global__ void degree_keys_kernel(const uint64_t *rp, uint32_t V, unsigned long long *keys) {
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < V; v += gridDim.x * blockDim.x) {
        uint64_t d = rp[v + 1] - rp[v];
        uint32_t dd = d > 0xFFFFFFFEull ? 0xFFFFFFFEu : (uint32_t)d;
        keys[v] = ((unsigned long long)(0xFFFFFFFFu - dd) << 32) | v;  // ascending = degree descending
    }
}

__global__ void perm_kernel(const unsigned long long *keys, uint32_t V, const uint64_t *rp, uint32_t *perm,
                            uint32_t *inv, uint64_t *ndeg) {
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < V; i += gridDim.x * blockDim.x) {
        uint32_t old = (uint32_t)keys[i];
        perm[i] = old;
        inv[old] = i;
        ndeg[i] = rp[old + 1] - rp[old];
    }
}

// one warp per new row: copy the old row with neighbours mapped through inv
__global__ void relabel_rows_kernel(const uint64_t *rp, const uint32_t *col, const uint32_t *w, const uint32_t *perm,
                                    const uint32_t *inv, const uint64_t *nrp, uint32_t V, uint32_t *ncol,
                                    uint32_t *nw) {
    const uint32_t lane = threadIdx.x & 31, warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t i = warp; i < V; i += nwarps) {
        const uint32_t old = perm[i];
        const uint64_t b = rp[old], d = rp[old + 1] - b, nb = nrp[i];
        for (uint64_t k = lane; k < d; k += 32) {
            ncol[nb + k] = inv[col[b + k]];
            if (w) nw[nb + k] = w[b + k];
        }
    }
}

// Rewrites g->d_col / g->d_w in place (new buffers) and returns the new u64 row offsets in *nrp_out.
ag_status build_degree_layout(ag_graph_s *g, const uint64_t *rp64, uint64_t **nrp_out) {
    const uint32_t V = g->V;
    const uint64_t E = g->E;
    const int dev = g->device, grid = g->num_sms * 8;
    ag_status s;
    unsigned long long *keys = nullptr, *keys2 = nullptr;
    uint64_t *ndeg = nullptr, *nrp = nullptr;
    uint32_t *ncol = nullptr, *nw = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0, t2 = 0;
    auto cleanup = [&]() {
        dev_free(keys, (size_t)V * 8, dev);
        dev_free(keys2, (size_t)V * 8, dev);
        dev_free(ndeg, (size_t)V * 8 + 8, dev);
        dev_free(tmp, tmp_bytes, dev);
    };
    if ((s = dev_alloc((void **)&keys, (size_t)V * 8, dev)) != AG_OK) return s;
    if ((s = dev_alloc((void **)&keys2, (size_t)V * 8, dev)) != AG_OK) { cleanup(); return s; }
    if ((s = dev_alloc((void **)&ndeg, (size_t)V * 8 + 8, dev)) != AG_OK) { cleanup(); return s; }
    if ((s = dev_alloc((void **)&g->d_perm, (size_t)V * 4, dev)) != AG_OK) { cleanup(); return s; }
    if ((s = dev_alloc((void **)&g->d_inv, (size_t)V * 4, dev)) != AG_OK) { cleanup(); return s; }
    if ((s = dev_alloc((void **)&nrp, (size_t)V * 8 + 8, dev)) != AG_OK) { cleanup(); return s; }
    cub::DeviceRadixSort::SortKeys(nullptr, tmp_bytes, keys, keys2, (int)V);
    cub::DeviceScan::ExclusiveSum(nullptr, t2, ndeg, nrp, (int)V + 1);
    tmp_bytes = tmp_bytes > t2 ? tmp_bytes : t2;
    if ((s = dev_alloc(&tmp, tmp_bytes, dev)) != AG_OK) { dev_free(nrp, (size_t)V * 8 + 8, dev); cleanup(); return s; }
    degree_keys_kernel<<<grid, 256>>>(rp64, V, keys);
    cub::DeviceRadixSort::SortKeys(tmp, tmp_bytes, keys, keys2, (int)V);
    perm_kernel<<<grid, 256>>>(keys2, V, rp64, g->d_perm, g->d_inv, ndeg);
    cudaMemset(ndeg + V, 0, 8);
    cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, ndeg, nrp, (int)V + 1);
    note_launch(6);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { dev_free(nrp, (size_t)V * 8 + 8, dev); cleanup(); return cuda_status(e, "layout sort"); }
    if ((s = dev_alloc((void **)&ncol, E * 4 + 128, dev)) != AG_OK) { dev_free(nrp, (size_t)V * 8 + 8, dev); cleanup(); return s; }
    if (g->d_w && (s = dev_alloc((void **)&nw, E * 4 + 128, dev)) != AG_OK) {
        dev_free(ncol, E * 4 + 128, dev);
        dev_free(nrp, (size_t)V * 8 + 8, dev);
        cleanup();
        return s;
    }
    relabel_rows_kernel<<<grid, 256>>>(rp64, g->d_col, g->d_w, g->d_perm, g->d_inv, nrp, V, ncol, nw);
    note_launch(1);
    e = cudaDeviceSynchronize();
    cleanup();
    if (e != cudaSuccess) {
        dev_free(ncol, E * 4 + 128, dev);
        dev_free(nw, E * 4 + 128, dev);
        dev_free(nrp, (size_t)V * 8 + 8, dev);
        return cuda_status(e, "relabel");
    }
    dev_free(g->d_col, g->col_bytes, dev);
    g->d_col = ncol;
    g->col_bytes = E * 4 + 128;
    if (g->d_w) {
        dev_free(g->d_w, g->w_bytes, dev);
        g->d_w = nw;
        g->w_bytes = E * 4 + 128;
    }
    *nrp_out = nrp;
    return AG_OK;
}

}  // namespace ag
