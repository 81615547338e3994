/*
 * aggen — seeded synthetic graph generators (input recipe only).
 *
 * This module produces the INPUTS that both the oracle (oracle/) and the CUDA
 * path (paper_conf_ipps_lib13_b200/) consume.  It holds none of the method's
 * arithmetic: no traversal, no levels, no distances, no selector.  It only
 * builds CSR graphs (SURVEY.md §8(d) "Synthetic inputs"):
 *
 *   - R-MAT / Kronecker (Graph500 A,B,C,D = .57,.19,.19,.05), random vertex
 *     relabelling by a keyed bijection on [0, 2^scale)      (configs C1, C2, C5)
 *   - 2-D 4-neighbour grid, row-major ids, optional bond percolation (C3, C3')
 *   - Erdos-Renyi G(n, m) with uniform endpoints                          (C4)
 *   - symmetric integer weights w(u,v) = 1 + splitmix64(seed ^ pack(min,max)) % wmax
 *     (reading R7; PAPER.md:20.s32 only says SSSP needs a weight array)
 *
 * Every random draw is a counter-based SplitMix64 of (seed, index), so the
 * result is independent of the thread count.  Undirected tuples are stored
 * both ways (symmetrised), self-loops dropped, duplicates merged, rows sorted
 * ascending (readings R5, R6).
 *
 * Build: gcc -O3 -fopenmp -shared -fPIC aggen.c -o libaggen.so
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <omp.h>

typedef struct {
    uint32_t V;
    uint64_t E;
    uint64_t *row_ptr; /* V+1 */
    uint32_t *col;     /* E   */
} aggen_csr;

static inline uint64_t splitmix64(uint64_t x) {
    uint64_t z = x + 0x9e3779b97f4a7c15ULL;
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
}

/* ------------------------------------------------------------------ */
/* tuple sources: tuple index -> (u, v) or "skip"                      */
/* ------------------------------------------------------------------ */
enum { GEN_RMAT = 1, GEN_ER = 2, GEN_GRID = 3 };

typedef struct {
    int kind;
    uint64_t seed;
    /* rmat */
    uint32_t scale;
    uint64_t tA, tAB, tABC; /* thresholds in 2^64 units */
    int permute;
    uint64_t pa1, pc1, pa2, pc2; /* permutation keys */
    /* er */
    uint32_t n;
    /* grid */
    uint32_t W, H;
    uint64_t keep_thr; /* keep edge iff hash < keep_thr (2^64 units); 0 => keep all */
    int keep_all;
} gen_t;

/* keyed bijection on [0, 2^s): two rounds of (odd-multiply + add) and xorshift */
static inline uint32_t perm_s(const gen_t *g, uint64_t x) {
    uint32_t s = g->scale;
    uint64_t mask = (s == 64) ? ~0ULL : ((1ULL << s) - 1);
    uint32_t k = s / 2 + 1;
    x = (x * g->pa1 + g->pc1) & mask;
    x ^= x >> k;
    x = (x * g->pa2 + g->pc2) & mask;
    x ^= x >> k;
    x = (x * g->pa1 + g->pc2) & mask;
    return (uint32_t)x;
}

static inline uint32_t bounded(uint64_t h, uint32_t n) {
    return (uint32_t)(((h >> 32) * (uint64_t)n) >> 32);
}

/* returns 0 if the tuple is skipped */
static inline int gen_tuple(const gen_t *g, uint64_t i, uint32_t *pu, uint32_t *pv) {
    if (g->kind == GEN_RMAT) {
        uint64_t state = splitmix64(g->seed ^ (i * 0xd1b54a32d192ed03ULL));
        uint64_t u = 0, v = 0;
        for (uint32_t l = 0; l < g->scale; ++l) {
            state += 0x9e3779b97f4a7c15ULL;
            uint64_t z = splitmix64(state);
            uint64_t ub, vb;
            if (z < g->tA) { ub = 0; vb = 0; }
            else if (z < g->tAB) { ub = 0; vb = 1; }
            else if (z < g->tABC) { ub = 1; vb = 0; }
            else { ub = 1; vb = 1; }
            u = (u << 1) | ub;
            v = (v << 1) | vb;
        }
        if (g->permute) { u = perm_s(g, u); v = perm_s(g, v); }
        *pu = (uint32_t)u; *pv = (uint32_t)v;
        return 1;
    } else if (g->kind == GEN_ER) {
        uint64_t h1 = splitmix64(g->seed ^ splitmix64(2 * i));
        uint64_t h2 = splitmix64(g->seed ^ splitmix64(2 * i + 1));
        *pu = bounded(h1, g->n);
        *pv = bounded(h2, g->n);
        return 1;
    } else { /* GRID */
        uint64_t W = g->W, H = g->H;
        uint64_t nh = H * (W - 1);
        uint64_t a, b;
        if (i < nh) {
            uint64_t y = i / (W - 1), x = i % (W - 1);
            a = y * W + x; b = a + 1;
        } else {
            uint64_t j = i - nh;
            uint64_t y = j / W, x = j % W;
            a = y * W + x; b = a + W;
        }
        if (!g->keep_all) {
            uint64_t h = splitmix64(g->seed ^ ((a << 32) | b));
            if (h >= g->keep_thr) return 0;
        }
        *pu = (uint32_t)a; *pv = (uint32_t)b;
        return 1;
    }
}

/* ------------------------------------------------------------------ */
/* row sort + dedup                                                    */
/* ------------------------------------------------------------------ */
static void sort_u32(uint32_t *a, uint64_t n, uint32_t *tmp) {
    if (n <= 48) {
        for (uint64_t i = 1; i < n; ++i) {
            uint32_t x = a[i];
            uint64_t j = i;
            while (j > 0 && a[j - 1] > x) { a[j] = a[j - 1]; --j; }
            a[j] = x;
        }
        return;
    }
    /* LSD radix, 2 passes x 16 bits */
    uint64_t *cnt = (uint64_t *)calloc(65536, sizeof(uint64_t));
    for (int pass = 0; pass < 2; ++pass) {
        int sh = pass * 16;
        memset(cnt, 0, 65536 * sizeof(uint64_t));
        uint32_t *src = pass == 0 ? a : tmp;
        uint32_t *dst = pass == 0 ? tmp : a;
        for (uint64_t i = 0; i < n; ++i) cnt[(src[i] >> sh) & 0xFFFF]++;
        uint64_t s = 0;
        for (int k = 0; k < 65536; ++k) { uint64_t c = cnt[k]; cnt[k] = s; s += c; }
        for (uint64_t i = 0; i < n; ++i) dst[cnt[(src[i] >> sh) & 0xFFFF]++] = src[i];
    }
    free(cnt);
}

/* keep only CSR entries whose destination is in [own_b, own_e) (multi-GPU 1-D partition);
 * own_b = 0, own_e = V keeps everything */
static uint32_t g_own_b = 0, g_own_e = 0xFFFFFFFFu;
static inline int owned(uint32_t v) { return v >= g_own_b && v < g_own_e; }

static int build_csr(const gen_t *g, uint32_t V, uint64_t M, aggen_csr *out) {
    uint64_t *deg = (uint64_t *)calloc((size_t)V + 1, sizeof(uint64_t));
    if (!deg) return -1;
    /* pass 1: degrees of the symmetrised tuple multiset (self loops dropped) */
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)M; ++i) {
        uint32_t u, v;
        if (!gen_tuple(g, (uint64_t)i, &u, &v) || u == v) continue;
        if (owned(v)) __atomic_fetch_add(&deg[u], 1, __ATOMIC_RELAXED);
        if (owned(u)) __atomic_fetch_add(&deg[v], 1, __ATOMIC_RELAXED);
    }
    uint64_t *off = (uint64_t *)malloc(((size_t)V + 1) * sizeof(uint64_t));
    if (!off) { free(deg); return -1; }
    uint64_t s = 0;
    for (uint32_t u = 0; u < V; ++u) { off[u] = s; s += deg[u]; }
    off[V] = s;
    uint64_t Eraw = s;
    uint32_t *col = (uint32_t *)malloc((Eraw ? Eraw : 1) * sizeof(uint32_t));
    if (!col) { free(deg); free(off); return -1; }
    /* pass 2: scatter (deg reused as cursor) */
    memcpy(deg, off, (size_t)V * sizeof(uint64_t));
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)M; ++i) {
        uint32_t u, v;
        if (!gen_tuple(g, (uint64_t)i, &u, &v) || u == v) continue;
        if (owned(v)) col[__atomic_fetch_add(&deg[u], 1, __ATOMIC_RELAXED)] = v;
        if (owned(u)) col[__atomic_fetch_add(&deg[v], 1, __ATOMIC_RELAXED)] = u;
    }
    /* sort + dedup each row; deg[u] := unique count */
#pragma omp parallel
    {
        uint64_t cap = 0;
        uint32_t *tmp = NULL;
#pragma omp for schedule(dynamic, 1024)
        for (int64_t u = 0; u < (int64_t)V; ++u) {
            uint64_t b = off[u], n = off[u + 1] - b;
            if (n > 48 && n > cap) { free(tmp); cap = n; tmp = (uint32_t *)malloc(cap * sizeof(uint32_t)); }
            sort_u32(col + b, n, tmp);
            uint64_t k = 0;
            for (uint64_t i = 0; i < n; ++i)
                if (k == 0 || col[b + k - 1] != col[b + i]) col[b + k++] = col[b + i];
            deg[u] = k;
        }
        free(tmp);
    }
    /* compact in place, ascending (destination never overtakes source) */
    uint64_t *rp = (uint64_t *)malloc(((size_t)V + 1) * sizeof(uint64_t));
    if (!rp) { free(deg); free(off); free(col); return -1; }
    s = 0;
    for (uint32_t u = 0; u < V; ++u) {
        rp[u] = s;
        if (s != off[u] && deg[u]) memmove(col + s, col + off[u], deg[u] * sizeof(uint32_t));
        s += deg[u];
    }
    rp[V] = s;
    free(deg);
    free(off);
    uint32_t *c2 = (uint32_t *)realloc(col, (s ? s : 1) * sizeof(uint32_t));
    if (c2) col = c2;
    out->V = V;
    out->E = s;
    out->row_ptr = rp;
    out->col = col;
    return 0;
}

/* ------------------------------------------------------------------ */
/* public entry points                                                 */
/* ------------------------------------------------------------------ */
int aggen_rmat(uint32_t scale, uint32_t edgefactor, uint64_t seed, uint32_t a_ppm, uint32_t b_ppm,
               uint32_t c_ppm, int permute, aggen_csr *out) {
    if (scale < 1 || scale > 31 || a_ppm + b_ppm + c_ppm > 1000000) return -2;
    gen_t g;
    memset(&g, 0, sizeof g);
    g.kind = GEN_RMAT;
    g.seed = splitmix64(seed);
    g.scale = scale;
    const long double two64 = 18446744073709551616.0L;
    g.tA = (uint64_t)(two64 * (long double)a_ppm / 1e6L);
    g.tAB = (uint64_t)(two64 * (long double)(a_ppm + b_ppm) / 1e6L);
    g.tABC = (uint64_t)(two64 * (long double)(a_ppm + b_ppm + c_ppm) / 1e6L);
    g.permute = permute;
    g.pa1 = splitmix64(seed ^ 0x1111) | 1ULL;
    g.pc1 = splitmix64(seed ^ 0x2222);
    g.pa2 = splitmix64(seed ^ 0x3333) | 1ULL;
    g.pc2 = splitmix64(seed ^ 0x4444);
    uint32_t V = 1u << scale;
    uint64_t M = (uint64_t)edgefactor << scale;
    return build_csr(&g, V, M, out);
}

int aggen_er(uint32_t n, uint64_t m, uint64_t seed, aggen_csr *out) {
    if (n < 1) return -2;
    gen_t g;
    memset(&g, 0, sizeof g);
    g.kind = GEN_ER;
    g.seed = splitmix64(seed);
    g.n = n;
    return build_csr(&g, n, m, out);
}

int aggen_grid(uint32_t W, uint32_t H, uint32_t keep_ppm, uint64_t seed, aggen_csr *out) {
    if (W < 1 || H < 1 || (uint64_t)W * H >= 0xFFFFFFFFULL) return -2;
    gen_t g;
    memset(&g, 0, sizeof g);
    g.kind = GEN_GRID;
    g.seed = splitmix64(seed);
    g.W = W;
    g.H = H;
    g.keep_all = keep_ppm >= 1000000;
    const long double two64 = 18446744073709551616.0L;
    g.keep_thr = (uint64_t)(two64 * (long double)keep_ppm / 1e6L);
    uint64_t M = (uint64_t)H * (W - 1) + (uint64_t)(H - 1) * W;
    return build_csr(&g, W * H, M, out);
}

/* symmetric weights in [1, wmax]; wmax == 0 => constant weight `seed` (closed-form tests) */
void aggen_weights(uint32_t V, const uint64_t *row_ptr, const uint32_t *col, uint64_t seed, uint32_t wmax,
                   uint32_t *w) {
    uint64_t k = splitmix64(seed);
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t u = 0; u < (int64_t)V; ++u) {
        for (uint64_t e = row_ptr[u]; e < row_ptr[u + 1]; ++e) {
            uint64_t v = col[e];
            uint64_t lo = (uint64_t)u < v ? (uint64_t)u : v, hi = (uint64_t)u < v ? v : (uint64_t)u;
            w[e] = wmax == 0 ? (uint32_t)seed : 1u + (uint32_t)(splitmix64(k ^ ((lo << 32) | hi)) % wmax);
        }
    }
}

/* seeded list of `count` source vertices with out-degree >= 1 */
int aggen_sources(uint32_t V, const uint64_t *row_ptr, uint64_t seed, uint32_t count, uint32_t *out) {
    uint64_t k = splitmix64(seed);
    uint32_t got = 0;
    for (uint64_t t = 0; got < count && t < 64ULL * V + 1024; ++t) {
        uint32_t v = bounded(splitmix64(k ^ splitmix64(t)), V);
        if (row_ptr[v + 1] > row_ptr[v]) out[got++] = v;
    }
    return (int)got;
}

void aggen_free(aggen_csr *g) {
    free(g->row_ptr);
    free(g->col);
    g->row_ptr = NULL;
    g->col = NULL;
}

int aggen_num_threads(void) { return omp_get_max_threads(); }

/* restrict subsequent generators to destinations in [b, e) (call with 0, 0xFFFFFFFF to reset) */
void aggen_set_owned(uint32_t b, uint32_t e) {
    g_own_b = b;
    g_own_e = e;
}
