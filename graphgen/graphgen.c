/*
 * graphgen.c — seeded synthetic CSR generator (INPUT ONLY).
 *
 * This module is shared by the CUDA path's tests/bench and by the oracle's
 * tests. It holds none of the method's arithmetic (no frontier, no placer,
 * no BFS/SSSP/CC/PR): it only produces the graphs the paper's workloads are
 * shaped like (SURVEY.md §8(d) "Generators"; Table 3, P:973-980,
 * "RMAT-rand" P:980; SSSP weight field P:993-995).
 *
 * Recipe (restated in DESIGN.md §"Input recipe"):
 *   * RMAT(scale, tuples, a,b,c,d = 0.57,0.19,0.19,0.05), no noise. Tuple i,
 *     attempt j draws its quadrant bits from a counter-based hash
 *     mix64(key ^ ctr) so the graph is identical at any thread count.
 *   * Optional bijective seeded permutation of [0, 2^scale) ("RMAT-rand").
 *   * Endpoints >= n_limit are rejected and the tuple redrawn with the next
 *     attempt counter (friendster/uk shapes with exact n and tuple count).
 *   * Symmetrize, drop self-loops, sort each row, drop duplicates.
 *   * Weights (SSSP): w(u,v) = 1 + mix64(seed ^ (min<<32 | max)) % 64,
 *     symmetric and uniform in 1..64.
 *
 * Memory: two arc arrays (raw with duplicates, then the caller's compacted
 * buffer). Offsets are uint64, ids uint32.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <omp.h>

static inline uint64_t gg_mix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

/* bijection on [0, 2^bits): 3 rounds of (odd multiply, add, xorshift) mod 2^bits */
static inline uint64_t gg_perm(uint64_t x, int bits, uint64_t seed) {
    const uint64_t mask = (bits >= 64) ? ~0ull : ((1ull << bits) - 1);
    int sh = bits / 2 > 0 ? bits / 2 : 1;
    for (int r = 0; r < 3; ++r) {
        uint64_t k = gg_mix64(seed * 0x100000001B3ull + (uint64_t)r);
        x = (x * (k | 1ull)) & mask;
        x = (x + (k >> 17)) & mask;
        x ^= x >> sh;
    }
    return x;
}

typedef struct {
    int scale;
    uint64_t tuples;
    uint32_t n;          /* vertex count (<= 2^scale) */
    uint64_t seed;
    int permute;
    uint32_t th_a, th_ab, th_abc; /* 32-bit quadrant thresholds */
    /* built state */
    uint64_t* off;       /* n+1, after dedup */
    uint32_t* raw;       /* raw arcs, rows sorted + deduped in place (prefix of each raw row) */
    uint64_t* raw_off;   /* n+1, raw row starts */
    uint64_t m;          /* arcs after dedup */
} gg_graph;

/* draw one tuple (u,v) for counter i, attempt j */
static inline void gg_draw(const gg_graph* g, uint64_t i, uint64_t j, uint64_t* u, uint64_t* v) {
    uint64_t key = gg_mix64(g->seed ^ 0xA5A5A5A5DEADBEEFull) ^ (i * 0x9E3779B97F4A7C15ull) ^ (j << 58);
    uint64_t su = 0, sv = 0;
    uint64_t h = 0;
    for (int l = 0; l < g->scale; ++l) {
        uint32_t r;
        if ((l & 1) == 0) { h = gg_mix64(key + (uint64_t)(l >> 1)); r = (uint32_t)h; }
        else r = (uint32_t)(h >> 32);
        uint64_t bu, bv;
        if (r < g->th_a) { bu = 0; bv = 0; }
        else if (r < g->th_ab) { bu = 0; bv = 1; }
        else if (r < g->th_abc) { bu = 1; bv = 0; }
        else { bu = 1; bv = 1; }
        su = (su << 1) | bu;
        sv = (sv << 1) | bv;
    }
    if (g->permute) {
        su = gg_perm(su, g->scale, g->seed);
        sv = gg_perm(sv, g->scale, g->seed);
    }
    *u = su; *v = sv;
}

static inline int gg_tuple(const gg_graph* g, uint64_t i, uint32_t* u, uint32_t* v) {
    for (uint64_t j = 0;; ++j) {
        uint64_t a, b;
        gg_draw(g, i, j, &a, &b);
        if (a < g->n && b < g->n) { *u = (uint32_t)a; *v = (uint32_t)b; return a != b; }
    }
}

static int cmp_u32(const void* a, const void* b) {
    uint32_t x = *(const uint32_t*)a, y = *(const uint32_t*)b;
    return (x > y) - (x < y);
}

/* insertion sort for short rows, qsort for long */
static void sort_row(uint32_t* p, uint64_t len) {
    if (len < 32) {
        for (uint64_t i = 1; i < len; ++i) {
            uint32_t x = p[i]; uint64_t j = i;
            while (j > 0 && p[j - 1] > x) { p[j] = p[j - 1]; --j; }
            p[j] = x;
        }
    } else {
        qsort(p, len, sizeof(uint32_t), cmp_u32);
    }
}

void* gg_rmat_build(int scale, uint64_t tuples, uint32_t n_limit, uint64_t seed, int permute,
                    double a, double b, double c) {
    if (scale < 1 || scale > 32) return NULL;
    gg_graph* g = (gg_graph*)calloc(1, sizeof(gg_graph));
    g->scale = scale; g->tuples = tuples; g->seed = seed; g->permute = permute;
    uint64_t full = 1ull << scale;
    g->n = (n_limit == 0 || (uint64_t)n_limit > full) ? (uint32_t)(full > 0xFFFFFFFFull ? 0xFFFFFFFFull : full) : n_limit;
    g->th_a = (uint32_t)(a * 4294967296.0);
    g->th_ab = (uint32_t)((a + b) * 4294967296.0);
    g->th_abc = (uint32_t)((a + b + c) * 4294967296.0);
    const uint32_t n = g->n;
    /* pass 1: degree counts (both directions, self-loops dropped) */
    uint64_t* cnt = (uint64_t*)calloc((size_t)n + 1, sizeof(uint64_t));
    #pragma omp parallel for schedule(static, 1 << 16)
    for (int64_t i = 0; i < (int64_t)tuples; ++i) {
        uint32_t u, v;
        if (!gg_tuple(g, (uint64_t)i, &u, &v)) continue;
        __atomic_fetch_add(&cnt[u], 1, __ATOMIC_RELAXED);
        __atomic_fetch_add(&cnt[v], 1, __ATOMIC_RELAXED);
    }
    g->raw_off = (uint64_t*)malloc(((size_t)n + 1) * sizeof(uint64_t));
    uint64_t acc = 0;
    for (uint32_t v = 0; v < n; ++v) { g->raw_off[v] = acc; acc += cnt[v]; }
    g->raw_off[n] = acc;
    g->raw = (uint32_t*)malloc((acc ? acc : 1) * sizeof(uint32_t));
    /* cursor */
    #pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < (int64_t)n; ++v) cnt[v] = g->raw_off[v];
    /* pass 2: fill */
    #pragma omp parallel for schedule(static, 1 << 16)
    for (int64_t i = 0; i < (int64_t)tuples; ++i) {
        uint32_t u, v;
        if (!gg_tuple(g, (uint64_t)i, &u, &v)) continue;
        uint64_t pu = __atomic_fetch_add(&cnt[u], 1, __ATOMIC_RELAXED);
        uint64_t pv = __atomic_fetch_add(&cnt[v], 1, __ATOMIC_RELAXED);
        g->raw[pu] = v;
        g->raw[pv] = u;
    }
    /* pass 3: sort + dedup each row in place; cnt[v] = deduped degree */
    #pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t v = 0; v < (int64_t)n; ++v) {
        uint32_t* p = g->raw + g->raw_off[v];
        uint64_t len = g->raw_off[v + 1] - g->raw_off[v];
        sort_row(p, len);
        uint64_t k = 0;
        for (uint64_t x = 0; x < len; ++x)
            if (k == 0 || p[x] != p[k - 1]) p[k++] = p[x];
        cnt[v] = k;
    }
    g->off = (uint64_t*)malloc(((size_t)n + 1) * sizeof(uint64_t));
    acc = 0;
    for (uint32_t v = 0; v < n; ++v) { g->off[v] = acc; acc += cnt[v]; }
    g->off[n] = acc;
    g->m = acc;
    free(cnt);
    return g;
}

void gg_size(void* h, uint32_t* n, uint64_t* m) {
    gg_graph* g = (gg_graph*)h;
    *n = g->n; *m = g->m;
}

static inline uint32_t gg_weight(uint64_t seed, uint32_t u, uint32_t v) {
    uint64_t lo = u < v ? u : v, hi = u < v ? v : u;
    return 1u + (uint32_t)(gg_mix64(seed ^ ((lo << 32) | hi)) % 64ull);
}

/* export: off_out (n+1 uint64), nbr_out (m uint32, or 2m if pairs), wgt_out (m uint32, nullable).
 * pairs!=0: nbr_out receives interleaved (id, w) uint32 pairs. */
int gg_export(void* h, uint64_t* off_out, uint32_t* nbr_out, uint32_t* wgt_out, int pairs, uint64_t wseed) {
    gg_graph* g = (gg_graph*)h;
    const uint32_t n = g->n;
    memcpy(off_out, g->off, ((size_t)n + 1) * sizeof(uint64_t));
    #pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t v = 0; v < (int64_t)n; ++v) {
        const uint32_t* src = g->raw + g->raw_off[v];
        uint64_t o = g->off[v], len = g->off[v + 1] - g->off[v];
        if (pairs) {
            for (uint64_t x = 0; x < len; ++x) {
                nbr_out[2 * (o + x)] = src[x];
                nbr_out[2 * (o + x) + 1] = gg_weight(wseed, (uint32_t)v, src[x]);
            }
        } else {
            memcpy(nbr_out + o, src, len * sizeof(uint32_t));
            if (wgt_out)
                for (uint64_t x = 0; x < len; ++x) wgt_out[o + x] = gg_weight(wseed, (uint32_t)v, src[x]);
        }
    }
    return 0;
}

void gg_free(void* h) {
    gg_graph* g = (gg_graph*)h;
    if (!g) return;
    free(g->off); free(g->raw); free(g->raw_off); free(g);
}

/* Build CSR from an explicit edge list (tests, tiny graphs): symmetrize? flag. */
void* gg_from_edges(uint32_t n, uint64_t ne, const uint32_t* src, const uint32_t* dst, int symmetrize, int keep_dups) {
    gg_graph* g = (gg_graph*)calloc(1, sizeof(gg_graph));
    g->n = n;
    uint64_t* cnt = (uint64_t*)calloc((size_t)n + 1, sizeof(uint64_t));
    for (uint64_t i = 0; i < ne; ++i) {
        if (!keep_dups && src[i] == dst[i]) continue;
        cnt[src[i]]++;
        if (symmetrize && src[i] != dst[i]) cnt[dst[i]]++;
    }
    g->raw_off = (uint64_t*)malloc(((size_t)n + 1) * sizeof(uint64_t));
    uint64_t acc = 0;
    for (uint32_t v = 0; v < n; ++v) { g->raw_off[v] = acc; acc += cnt[v]; }
    g->raw_off[n] = acc;
    g->raw = (uint32_t*)malloc((acc ? acc : 1) * sizeof(uint32_t));
    for (uint32_t v = 0; v < n; ++v) cnt[v] = g->raw_off[v];
    for (uint64_t i = 0; i < ne; ++i) {
        if (!keep_dups && src[i] == dst[i]) continue;
        g->raw[cnt[src[i]]++] = dst[i];
        if (symmetrize && src[i] != dst[i]) g->raw[cnt[dst[i]]++] = src[i];
    }
    for (uint32_t v = 0; v < n; ++v) {
        uint32_t* p = g->raw + g->raw_off[v];
        uint64_t len = g->raw_off[v + 1] - g->raw_off[v];
        sort_row(p, len);
        uint64_t k = len;
        if (!keep_dups) {
            k = 0;
            for (uint64_t x = 0; x < len; ++x)
                if (k == 0 || p[x] != p[k - 1]) p[k++] = p[x];
        }
        cnt[v] = k;
    }
    g->off = (uint64_t*)malloc(((size_t)n + 1) * sizeof(uint64_t));
    acc = 0;
    for (uint32_t v = 0; v < n; ++v) { g->off[v] = acc; acc += cnt[v]; }
    g->off[n] = acc;
    g->m = acc;
    free(cnt);
    return g;
}

int gg_threads(void) { return omp_get_max_threads(); }
