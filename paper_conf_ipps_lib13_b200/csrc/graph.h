// graph.h — the library-owned graph handle (device CSR + per-handle traversal scratch).
//
// HBM layout: row offsets u32 when E < 2^32 (else u64), col_idx u32, weights u32,
// all cudaMalloc'd (256-B aligned).  Scratch: 3 frontier bitmaps (V/8 B each), 3 queues (4V B
// each), visited bitmap (V/8 B), packed SSSP state (8V B), hub-chunk task ring, control block.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "agraph.h"

struct ag_dist_part;  // multi-GPU partition data (dist.cu)

struct ag_graph_s {
    int device = 0;
    uint32_t V = 0;
    uint64_t E = 0;
    uint32_t nwords = 0;
    int num_sms = 0;
    bool offs32 = true;
    ag_graph_info info{};
    // CSR
    void *d_rp = nullptr;
    size_t rp_bytes = 0;
    uint32_t *d_col = nullptr;
    size_t col_bytes = 0;
    uint32_t *d_w = nullptr;       // weights (load time only; freed once interleaved)
    size_t w_bytes = 0;
    uint2 *d_cw = nullptr;         // interleaved (col, w) pairs for SSSP: one 8-B load per edge
    size_t cw_bytes = 0;
    // degree layout (layout.cu): new id i = old vertex d_perm[i]; d_inv = inverse
    uint32_t layout = AG_LAYOUT_IDENTITY;
    uint32_t *d_perm = nullptr;
    uint32_t *d_inv = nullptr;
    uint32_t *d_level = nullptr;   // BFS level / parent arrays in the relabelled space
    uint32_t *d_lpar = nullptr;
    // scratch
    void *d_ctl = nullptr;
    bool ctl_init = false;
    uint32_t *d_bm[3] = {nullptr, nullptr, nullptr};
    uint32_t *d_q[3] = {nullptr, nullptr, nullptr};
    uint32_t *d_vis = nullptr;
    unsigned long long *d_hub = nullptr;   // hub-task ring (self-contained 64-bit task words)
    uint32_t hub_cap = 0;
    unsigned long long *d_P = nullptr;
    void *d_acc = nullptr;
    uint32_t *d_out_tmp = nullptr;
    size_t out_tmp_bytes = 0;
    uint32_t *d_par_tmp = nullptr;
    size_t par_tmp_bytes = 0;
    uint32_t *d_trace = nullptr;
    size_t trace_bytes = 0;
    size_t scratch_bytes = 0;
    size_t persist_bytes = 0;      // L2 persisting set-aside available
    size_t max_window = 0;         // cudaDeviceProp::accessPolicyMaxWindowSize
    cudaEvent_t ev[2] = {nullptr, nullptr};
    // deferred status: stream of the last enqueued traversal (the status itself is Ctl::sticky)
    cudaStream_t last_stream = nullptr;
    bool pending_check = false;
    bool last_packed = true;       // the last SSSP kept the packed (dist, parent) state (false: distance-only u32)
    // multi-GPU
    ag_dist_part *dist = nullptr;
};

namespace ag {
ag_status set_error(ag_status s, const char *fmt, ...);
ag_status cuda_status(cudaError_t e, const char *what);
ag_status dev_alloc(void **p, size_t bytes, int device);
void dev_free(void *p, size_t bytes, int device);
bool is_device_ptr(const void *p);
ag_status check_device(int device, int *num_sms);
void note_launch(unsigned n);
void dist_graph_release(ag_graph_s *g);
struct DevPolicy;
DevPolicy resolve_policy(const ag_policy &p, const ag_graph_s &g);
ag_status check_policy(const ag_policy *p);
void build_degree_order(const uint64_t *rp64, uint32_t V, unsigned long long *keys, unsigned long long *keys2, void *tmp,
                        size_t tmp_bytes, uint32_t *perm, uint32_t *inv, uint64_t *ndeg, uint64_t *nrp, int sms,
                        cudaStream_t st);
}  // namespace ag
