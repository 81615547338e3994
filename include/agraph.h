/*
 * agraph.h — C ABI of the B200 adaptive BFS/SSSP frontier engine (libagraph.so).
 *
 * The paper's Graph API: "an abstract graph data type ... primitives to define and instantiate
 * graphs, as well as functions to run the SSSP and BFS algorithms on them" (PAPER.md:22.s36-37,
 * 12.s3), with the decision maker's policy exposed (Fig. 11, 24.s34-42).  extern "C", plain
 * pointers and sizes, no C++ types, no exceptions across the ABI.  Every compute step runs in
 * this library's own CUDA kernels (sm_100a); there is no CPU fallback.
 *
 * Conventions
 *  - Vertex ids are uint32 in [0, V); V < 2^32 - 1 because AG_INF is reserved (reading R1).
 *  - CSR (PAPER.md:20.s16-29, Fig. 7): the out-edges of u are col_idx[row_ptr[u] .. row_ptr[u+1]),
 *    row_ptr has V+1 entries, row_ptr[0] = 0, row_ptr[V] = E.  Rows need not be sorted;
 *    multi-edges and self-loops are accepted (reading R6).  Traversal follows out-edges (R5).
 *  - Weights (SSSP, 20.s32): uint32 in [1, 2^31) (reading R8).
 *  - Outputs: level / dist / parent arrays of V uint32, AG_INF for unreached vertices;
 *    parent[src] = src.  level = minimum number of edges on a path src -> v (14.s19 with Fig. 4,
 *    reading R2); dist = minimum total weight (14.s20, Fig. 5, reading R3).
 *  - Pointers: every array argument may be HOST or DEVICE memory (detected with
 *    cudaPointerGetAttributes).  Inputs are borrowed for the duration of the call and copied.
 *  - Errors: functions return ag_status and never abort; ag_last_error() gives thread-local detail.
 *  - Threading: a graph handle carries its own device scratch, so concurrent queries on the SAME
 *    handle are not allowed; separate handles are independent.
 */
#ifndef AGRAPH_H
#define AGRAPH_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define AG_ABI_VERSION 1u
#define AG_INF 0xFFFFFFFFu
#define AG_WINDOW_AUTO 0xFFFFFFFFu
#define AG_WINDOW_ADAPTIVE 0xFFFFFFFEu   /* sssp_window: adapted per iteration (NEXT-3) */

typedef struct ag_graph_s *ag_graph; /* opaque, library-owned device CSR + scratch */
typedef struct ag_comm_s *ag_comm;   /* opaque multi-GPU communicator (one per process/GPU) */

typedef enum {
    AG_OK = 0,
    AG_ERR_INVALID_ARG = 1,  /* NULL handle/array, bad policy field, struct_size mismatch */
    AG_ERR_BAD_CSR = 2,      /* row_ptr[0]!=0, non-monotone, row_ptr[V]!=E, col>=V, weight 0 or >=2^31, V>=2^32-1 */
    AG_ERR_SRC_RANGE = 3,    /* src >= V */
    AG_ERR_NO_WEIGHTS = 4,   /* ag_sssp on a graph loaded without weights */
    AG_ERR_OVERFLOW = 5,     /* some finite distance exceeds 0xFFFFFFFE (reading R8) */
    AG_ERR_OOM = 6,          /* device allocation failed */
    AG_ERR_CUDA = 7,         /* any other CUDA runtime error */
    AG_ERR_NCCL = 8,         /* NCCL failure or NCCL not loadable (multi-GPU only) */
    AG_ERR_UNSUPPORTED = 9,  /* variant/feature not available for this request */
    AG_ERR_NO_DEVICE = 10    /* no CUDA device / device is not sm_100 */
} ag_status;

/* Axis (ii): mapping of a working-set element to the GPU (PAPER.md:18.s13-45, Fig. 9).
 * THREAD = one thread per element (fine-grained); CTA = one thread-block group per element
 * (coarse-grained; group size per reading R16); WARP = the paper's block mapping at its minimum
 * block size of 32 (24.s15) / Hong's virtual warp (12.s19-20); HYBRID = per-element choice by
 * out-degree (thread / warp / CTA / split across CTAs) — the "intermediate solutions" of
 * 18.s43-44 that the paper names but does not build (beyond the paper; tuned policy). */
typedef enum { AG_MAP_AUTO = 0, AG_MAP_THREAD = 1, AG_MAP_WARP = 2, AG_MAP_CTA = 3, AG_MAP_HYBRID = 4 } ag_mapping;
/* Axis (iii): working-set representation (PAPER.md:20.s1-12, Fig. 6). */
typedef enum { AG_WS_AUTO = 0, AG_WS_BITMAP = 1, AG_WS_QUEUE = 2 } ag_workset;
/* Axis (i): ordered vs unordered algorithm (PAPER.md:16.s38-46, Fig. 4, Fig. 5). */
typedef enum { AG_UNORDERED = 0, AG_ORDERED = 1 } ag_order;
/* Decision-maker rule: PAPER = Fig. 11 with T1/T2/T3 (24.s34-42); TUNED = B200-calibrated rule
 * using the same inputs plus the frontier edge count. */
typedef enum { AG_POLICY_PAPER = 0, AG_POLICY_TUNED = 1 } ag_policy_kind;

/* A variant id packs (mapping, workset): id = mapping * 4 + workset, e.g. T_BM = 5, T_QU = 6,
 * W_BM = 9, W_QU = 10, B_BM = 13, B_QU = 14, H_BM = 17, H_QU = 18. */
#define AG_VARIANT(mapping, workset) ((uint8_t)((mapping) * 4 + (workset)))
#define AG_VARIANT_MAPPING(id) ((ag_mapping)((id) >> 2))
#define AG_VARIANT_WORKSET(id) ((ag_workset)((id) & 3))

typedef struct {
    uint32_t struct_size;    /* caller sets sizeof(ag_policy) (ABI versioning) */
    uint32_t order;          /* ag_order */
    uint32_t mapping;        /* ag_mapping; AUTO = the selector decides each iteration */
    uint32_t workset;        /* ag_workset; AUTO = the selector decides each iteration */
    uint32_t kind;           /* ag_policy_kind */
    uint32_t t1_avg_degree;  /* T1, default 32 = warp size (PAPER.md:28.s21-22) */
    uint64_t t2_ws;          /* T2, default thread_tpb x #SMs (28.s24-27; reading R17) */
    uint32_t t3_ppm;         /* T3 = ceil(t3_ppm * V / 1e6) (Fig. 13 sweeps 1-13% of V; reading R14) */
    uint32_t sample_every;   /* inspector sampling interval (26.s7-9; reading R15), >= 1 */
    uint32_t delta;          /* ordered-SSSP bucket width; 1 = the paper's Dijkstra batches (28.s8, R9);
                                0 = adaptive (NEXT-3): starts at 1 and is halved / doubled every iteration
                                from the measured re-expansion ratio (> 1/4: halve, < 1/16: double) */
    uint32_t thread_tpb;     /* thread-mapping block size used for T2, paper 192 (26.s27) */
    uint32_t cta_group;      /* block-mapping group size (multiple of 32); 0 = auto (26.s28, R16) */
    uint32_t sssp_window;    /* unordered SSSP: expand only frontier vertices with dist < min + window
                                (others stay in the working set); 0 = off (plain Bellman-Ford rounds);
                                AG_WINDOW_AUTO = tuned: off on skewed graphs, else 8 x max_weight / avg degree;
                                AG_WINDOW_ADAPTIVE = NEXT-3: start at that value, then halve / double it every
                                iteration from the measured re-expansion ratio (the order axis at run time) */
    uint32_t sssp_hub_window;/* unordered SSSP: vertices with out-degree >= 64 are expanded only when within
                                this distance of the frontier minimum (re-expanding a hub re-scans its whole
                                list); 0 = off; AG_WINDOW_AUTO = tuned: max(1, max_weight / 50) */
    uint32_t free_ppm;       /* tuned policy, unordered: an iteration whose working set has >= free_ppm * V / 1e6
                                elements writes its successor as a raw bitmap with fire-and-forget reductions (no
                                claiming atomics, no queue appends; BFS without parents only) and the next
                                iteration converts it to a queue in O(V/32) (the paper's update-vector bitmap,
                                22.s13-14).  Used only on graphs without the degree layout (non-skewed; measured
                                2x slower on R-MAT) unless free_ppm = 1000000 (every iteration, also on
                                skewed graphs: a diagnostic / test setting) — except unordered BFS on a degree-layout
                                graph, which the tuned policy runs in the general kernel specialisation (hybrid
                                queue, no free output: measured faster there).  BFS and ag_cc use
                                t_free from this field, ag_sssp the same threshold.
                                0 = never; ag_policy_default: 3906 (V/256) */
    uint32_t small_ws;       /* tuned policy, graphs without hub lists: an iteration whose working set has fewer than
                                small_ws elements runs on one CTA per SM while the others park (cheaper grid barrier;
                                DESIGN.md §5); 0 = AUTO (32768); 0xFFFFFFFF = always; 1 = never.  Results unchanged. */
} ag_policy;

typedef struct {
    uint32_t num_vertices;
    uint32_t min_deg, max_deg;   /* out-degree statistics (graph inspector, 22.s41) */
    uint64_t num_edges;          /* CSR entries E */
    uint64_t deg_sum;            /* = num_edges */
    uint32_t isolated;           /* vertices with out-degree 0 */
    uint32_t weighted;           /* 1 if loaded with weights */
    int32_t device;              /* CUDA device ordinal */
    uint32_t num_sms;            /* SM count of that device */
    uint32_t offset_bytes;       /* 4 if row offsets are stored as u32 (E < 2^32), else 8 */
    uint32_t layout;             /* ag_layout actually used (IDENTITY or DEGREE) */
    uint32_t max_weight;         /* largest edge weight (0 if unweighted) */
    uint32_t reserved2;
} ag_graph_info;

/* Device vertex layout.  DEGREE relabels vertices by descending out-degree at load
 * time so that the status words of high-degree vertices — the targets of most edges in a power-law
 * graph — are packed into a small, cache-resident prefix of the visited bitmap / state arrays.
 * Results are always returned in the caller's vertex ids.  AUTO picks DEGREE when the inspector
 * sees a skewed degree distribution (max_deg >= 64 x ceil(E/V)), else IDENTITY. DEGREE needs V < 2^31 (AG_ERR_UNSUPPORTED; AUTO then picks IDENTITY). */
typedef enum { AG_LAYOUT_AUTO = 0, AG_LAYOUT_IDENTITY = 1, AG_LAYOUT_DEGREE = 2 } ag_layout;

typedef struct {
    uint32_t struct_size;        /* caller sets sizeof(ag_run_stats) */
    uint32_t iterations;         /* traversal iterations (levels / relaxation rounds / buckets) */
    uint64_t vertices_expanded;  /* working-set elements whose neighbourhood was visited */
    uint64_t edges_inspected;    /* out-edges visited (sum of degrees of expanded elements) */
    uint64_t reached;            /* V_r: vertices with a finite result */
    uint64_t reached_edges;      /* E_r: CSR entries whose source is reached */
    float device_ms;             /* device time of the traversal (init -> termination) */
    uint32_t trace_cap;          /* in: capacity of the caller-owned trace arrays below */
    uint32_t trace_len;          /* out: entries written (min(iterations, trace_cap)) */
    uint32_t reserved;
    uint32_t *trace_ws;          /* per iteration |WS| (host, nullable) */
    uint64_t *trace_edges;       /* per iteration edges inspected (host, nullable) */
    uint8_t *trace_variant;      /* per iteration variant id AG_VARIANT(m, w) (host, nullable) */
    uint64_t *trace_ns;          /* per iteration device timestamp (ns, %globaltimer) at the start
                                    of the iteration; entry [iterations] = end (host, nullable,
                                    capacity trace_cap + 1) */
} ag_run_stats;

/* ---------------------------------------------------------------------------------------------
 * Policy and selector
 * ------------------------------------------------------------------------------------------- */

/* Fill *p with defaults for `device`: order UNORDERED, mapping/workset AUTO, kind TUNED,
 * T1 = 32, thread_tpb = 192, T2 = 192 x #SMs, t3_ppm = 100000 (10% of V, calibrated on B200: X8), delta = 1, sample_every = 1,
 * sssp_window = AG_WINDOW_AUTO.
 * Errors: AG_ERR_INVALID_ARG (p NULL), AG_ERR_NO_DEVICE. */
ag_status ag_policy_default(ag_policy *p, int device);

/* The decision maker (Fig. 11, 24.s34-42; readings R12, R13): returns AG_VARIANT(mapping, workset)
 * for a working set of ws_size elements whose out-degrees sum to ws_edges, on graph `gi`.
 * A forced mapping/workset in *p overrides the corresponding axis.  Pure function; the traversal
 * kernels evaluate the same rule on the device every iteration.  Returns 0 on invalid input. */
uint8_t ag_select(const ag_policy *p, const ag_graph_info *gi, uint64_t ws_size, uint64_t ws_edges);

/* ---------------------------------------------------------------------------------------------
 * Graphs (CSR store + graph inspector, 20.s16-33, 22.s40-41)
 * ------------------------------------------------------------------------------------------- */

/* Validate the CSR (AG_ERR_BAD_CSR list above), copy it into library-owned device memory on
 * `device`, and compute the inspector statistics.  row_ptr: V+1 uint64; col_idx: E uint32;
 * weights: E uint32 or NULL (BFS only).  Host or device pointers.  Untimed, once per graph.
 * *out receives the handle (owned by the library until ag_graph_free). */
ag_status ag_graph_load_csr(uint32_t V, uint64_t E, const uint64_t *row_ptr, const uint32_t *col_idx,
                            const uint32_t *weights, int device, ag_graph *out);
/* As ag_graph_load_csr with an explicit device layout (ag_layout). */
ag_status ag_graph_load_csr_ex(uint32_t V, uint64_t E, const uint64_t *row_ptr, const uint32_t *col_idx,
                               const uint32_t *weights, int device, uint32_t layout, ag_graph *out);
ag_status ag_graph_info_get(ag_graph g, ag_graph_info *out);
ag_status ag_graph_free(ag_graph g);

/* ---------------------------------------------------------------------------------------------
 * Traversals.  `stream` is a cudaStream_t (NULL = legacy default stream).
 * Synchronisation: if stats != NULL or any output pointer is host memory, the call synchronises
 * `stream` before returning (stats and host outputs are then valid).  Otherwise the traversal is
 * only ENQUEUED (outputs valid once the stream reaches that point) and deferred errors
 * (AG_ERR_OVERFLOW) are reported by the next ag_graph_check().
 * policy NULL = ag_policy_default() (adaptive).
 * ------------------------------------------------------------------------------------------- */

/* BFS levels from src (Fig. 4).  levels: V uint32 (required); parents: V uint32 or NULL.
 * Ordered (16.s43: each node processed exactly once, visited-claim) or unordered (16.s44:
 * level lowered by atomicMin, proceeds level by level on the GPU, 26.s33).
 * Errors: AG_ERR_INVALID_ARG, AG_ERR_SRC_RANGE, AG_ERR_OOM, AG_ERR_CUDA. */
ag_status ag_bfs(ag_graph g, uint32_t src, uint32_t *levels, uint32_t *parents, const ag_policy *policy,
                 ag_run_stats *stats, void *stream);

/* SSSP distances from src (Fig. 5).  dist: V uint32 (required); parents: V uint32 or NULL.
 * Unordered = Bellman-Ford-style label correcting (18.s3, 18.s5); ordered = bucketed with width
 * policy->delta (delta = 1: all pending nodes at the current minimum distance per iteration, the
 * paper's GPU Dijkstra, 28.s8; findmin by parallel reduction, 22.s11).
 * parents = NULL (distances only, as Fig. 5 computes them) lets the tuned kernels keep a 4-byte distance per
 * vertex instead of the packed 8-byte (distance, parent) word that keeps a parent consistent with its
 * distance: same distances, fewer bytes per status read and per atomic.
 * Errors: as ag_bfs plus AG_ERR_NO_WEIGHTS, AG_ERR_OVERFLOW. */
ag_status ag_sssp(ag_graph g, uint32_t src, uint32_t *dist, uint32_t *parents, const ag_policy *policy,
                  ag_run_stats *stats, void *stream);

/* Min-label connected components ("other graph algorithms that exhibit
 * similar computational patterns", PAPER.md:10.s9; connected components, 12.s13; R23):
 * labels[v] = min{ u : u reaches v along out-edges } (u = v included) in caller ids, i.e. on a
 * symmetric graph the smallest vertex id of v's connected component.  Same working-set engine as
 * ag_bfs: WS_0 = every vertex with label = own id; each iteration expands the WS with
 * atomicMin(label[m], label[n]) and a vertex whose label dropped enters the next WS (Fig. 4 l.8'
 * with level -> label, no +1), until the WS is empty.  labels: V uint32 (required), host or device.
 * policy: order must be AG_UNORDERED (AG_ERR_UNSUPPORTED otherwise); mapping / workset / selector
 * as for ag_bfs.  stats: iterations = label-propagation rounds; reached = V.  Synchronisation as
 * for ag_bfs.  Errors: AG_ERR_INVALID_ARG, AG_ERR_UNSUPPORTED, AG_ERR_OOM, AG_ERR_CUDA. */
ag_status ag_cc(ag_graph g, uint32_t *labels, const ag_policy *policy, ag_run_stats *stats, void *stream);

/* Wait for the graph's last enqueued traversal and return the deferred status accumulated over
 * EVERY traversal enqueued on this handle since the previous check (sticky on the device: a later
 * launch never clears an earlier query's overflow or abort): AG_ERR_CUDA if any aborted, else
 * AG_ERR_OVERFLOW if any SSSP left a reachable vertex beyond 0xFFFFFFFE (exact test, run inside the
 * traversal kernel only when a relaxation exceeded that bound), else AG_OK.  Clears the status. */
ag_status ag_graph_check(ag_graph g);

/* ---------------------------------------------------------------------------------------------
 * Multi-GPU, one process per GPU (not in the paper; BASELINE.json north_star).
 * 1-D partition by destination vertex: rank p owns vertices [p*S, min(V,(p+1)*S)), S a multiple
 * of 1024; it stores every edge whose destination it owns, indexed by source over all V.  Per BFS
 * level the owned next-frontier bitmap slices are exchanged with ncclAllGather over NVLink.
 * ------------------------------------------------------------------------------------------- */

/* Write a fresh 128-byte ncclUniqueId into out128 (call on rank 0, broadcast to the others). */
ag_status ag_dist_unique_id(void *out128);
/* Create the communicator for (rank, world) on `device`. */
ag_status ag_dist_init(int rank, int world, const void *nccl_unique_id128, int device, ag_comm *out);
/* Free a communicator.  AG_ERR_INVALID_ARG while graphs partitioned over it are still live
 * (ag_graph_free them first). */
ag_status ag_dist_free(ag_comm c);
/* Owned vertex range of `rank` for a V-vertex graph partitioned over `world` ranks. */
ag_status ag_dist_owned_range(uint32_t V, int rank, int world, uint32_t *begin, uint32_t *end);
/* Every rank passes the SAME global CSR (host or device); each keeps its destination-owned part.  The
 * global col_idx / weights are streamed through the device in 16M-entry chunks twice (count, then
 * scatter), so a rank never holds the global graph, only its row offsets (8 (V+1) B) and its own part.
 * Rows of the part keep their entries but not their order.  V < 2^31 (AG_ERR_UNSUPPORTED otherwise). */
ag_status ag_dist_graph_load_csr(ag_comm c, uint32_t V, uint64_t E, const uint64_t *row_ptr,
                                 const uint32_t *col_idx, const uint32_t *weights, ag_graph *out_local);
/* As above but every rank passes only ITS part: CSR rows over all V whose entries all have their
 * destination in the rank's owned range (AG_ERR_BAD_CSR otherwise).  Lets each process build its
 * part without holding the whole graph (R-MAT scale 26 = 8.6 GB of col_idx). */
ag_status ag_dist_graph_load_local(ag_comm c, uint32_t V, uint64_t E_local, const uint64_t *row_ptr,
                                   const uint32_t *col_idx, const uint32_t *weights, ag_graph *out_local);
/* Virtual group for tests on ONE GPU: creates `world` comms (ranks 0..world-1) in this process on
 * `device`; their all-gather is a device copy.  Load each rank's part with ag_dist_graph_load_csr
 * and run them in lock step with ag_dist_bfs_group.  comms_out: array of `world` handles. */
ag_status ag_dist_init_local(int world, int device, ag_comm *comms_out);
/* Lock-step BFS over all ranks of a virtual group (locals[r] = rank r's part); levels_owned[r] /
 * parents_owned[r] (nullable) receive rank r's owned slices. */
ag_status ag_dist_bfs_group(ag_graph *locals, int world, uint32_t src, uint32_t **levels_owned,
                            uint32_t **parents_owned, ag_run_stats *stats, void *stream);
/* Distributed BFS (unordered = ordered level-synchronous here).  levels_owned / parents_owned:
 * (end - begin) uint32 for this rank's owned range.  Collective: all ranks call with the same src. */
ag_status ag_dist_bfs(ag_graph local, uint32_t src, uint32_t *levels_owned, uint32_t *parents_owned,
                      const ag_policy *policy, ag_run_stats *stats, void *stream);
/* Distributed SSSP (the algorithm is Fig. 5 unordered, PAPER.md:18.s30:
 * every working-set node relaxes its out-edges until no distance improves).  Same destination
 * partition; per round every rank expands the gathered global list of (vertex, distance) entries —
 * the distance travels with the entry since only a vertex's owner holds it — over its local edges,
 * then the improved owned vertices are exchanged: ncclAllGather of the per-rank counts (termination
 * when all are 0) and of the (v, dist) lists padded to the largest count.  The local part must
 * carry weights (AG_ERR_NO_WEIGHTS).  dist_owned (required) / parents_owned (nullable): (end - begin)
 * uint32 for the owned range, host or device memory, caller-owned; AG_INF for unreached vertices.
 * AG_ERR_OVERFLOW is reported conservatively if any relaxation exceeded 0xFFFFFFFE.  Collective. */
ag_status ag_dist_sssp(ag_graph local, uint32_t src, uint32_t *dist_owned, uint32_t *parents_owned,
                       const ag_policy *policy, ag_run_stats *stats, void *stream);
/* Lock-step distributed SSSP over all ranks of a virtual group (test transport, see above). */
ag_status ag_dist_sssp_group(ag_graph *locals, int world, uint32_t src, uint32_t **dist_owned,
                             uint32_t **parents_owned, ag_run_stats *stats, void *stream);

/* ---------------------------------------------------------------------------------------------
 * Misc
 * ------------------------------------------------------------------------------------------- */
/* Optional device allocator hook (e.g. the PyTorch caching allocator).  alloc returns device
 * memory of `bytes` on `device` or NULL; free_ releases it.  NULL/NULL restores cudaMalloc. */
ag_status ag_set_allocator(void *(*alloc)(size_t bytes, int device, void *stream, void *ctx),
                           void (*free_)(void *ptr, size_t bytes, int device, void *stream, void *ctx), void *ctx);
const char *ag_status_string(ag_status s);
const char *ag_last_error(void);
uint32_t ag_abi_version(void);
/* Number of kernel launches this process has issued through the library (for bench accounting). */
uint64_t ag_kernel_launches(void);

#ifdef __cplusplus
}
#endif
#endif /* AGRAPH_H */
