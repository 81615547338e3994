// dist.cu — multi-GPU 1-D destination partition.  Placeholder entry points until the
// NCCL path lands; every call reports AG_ERR_UNSUPPORTED.
#include "agraph.h"
#include "graph.h"

namespace ag {
void dist_graph_release(ag_graph_s *) {}
}  // namespace ag

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

ag_status ag_dist_unique_id(void *) { return ag::set_error(AG_ERR_UNSUPPORTED, "multi-GPU path not built yet"); }
ag_status ag_dist_init(int, int, const void *, int, ag_comm *) {
    return ag::set_error(AG_ERR_UNSUPPORTED, "multi-GPU path not built yet");
}
ag_status ag_dist_free(ag_comm) { return ag::set_error(AG_ERR_UNSUPPORTED, "multi-GPU path not built yet"); }
ag_status ag_dist_graph_load_csr(ag_comm, uint32_t, uint64_t, const uint64_t *, const uint32_t *, const uint32_t *,
                                 ag_graph *) {
    return ag::set_error(AG_ERR_UNSUPPORTED, "multi-GPU path not built yet");
}
ag_status ag_dist_bfs(ag_graph, uint32_t, uint32_t *, uint32_t *, const ag_policy *, ag_run_stats *, void *) {
    return ag::set_error(AG_ERR_UNSUPPORTED, "multi-GPU path not built yet");
}

}  // extern "C"
