// layout.cu — degree-ordered device vertex layout (part of the CSR store, row a1; load time, untimed).
// (the relabelled CSR itself is written chunk by chunk during the pipelined load, api.cu)
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

// Degree order and the new row offsets, enqueued on `st` (no host synchronisation): keys = (~deg, id),
// radix-sorted -> perm (new -> old), inv (old -> new), nrp = exclusive scan of the new degrees.
// tmp must hold tmp_bytes >= the CUB temporary storage of both the sort (V keys) and the scan (V+1).
void build_degree_order(const uint64_t *rp64, uint32_t V, unsigned long long *keys, unsigned long long *keys2, void *tmp,
                        size_t tmp_bytes, uint32_t *perm, uint32_t *inv, uint64_t *ndeg, uint64_t *nrp, int sms,
                        cudaStream_t st) {
    const int grid = sms * 8;
    degree_keys_kernel<<<grid, 256, 0, st>>>(rp64, V, keys);
    cub::DeviceRadixSort::SortKeys(tmp, tmp_bytes, keys, keys2, (int)V, 0, 64, st);
    perm_kernel<<<grid, 256, 0, st>>>(keys2, V, rp64, perm, inv, ndeg);
    cudaMemsetAsync(ndeg + V, 0, 8, st);
    cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, ndeg, nrp, (int)V + 1, st);
    note_launch(6);
}

}  // namespace ag
