/*
 * inputs/gen.c -- seeded synthetic digraph generators shared by the oracle
 * tests and the product benchmarks.  Holds NONE of DiGraph's arithmetic: it
 * only draws edges (R-MAT power-law digraphs, long-chain digraphs), integer
 * weights and per-vertex random parameters, and packs them as CSR.
 *
 * Every random number is a pure function of (seed, stream, index) through
 * splitmix64, so the output is identical for any OpenMP thread count.
 * Build: gcc -O3 -fopenmp -shared -fPIC gen.c -o libdginputs.so
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <omp.h>

static inline uint64_t mix64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}
static inline uint64_t h3(uint64_t seed, uint64_t a, uint64_t b) {
    return mix64(mix64(mix64(seed) ^ a) ^ (b * 0xD6E8FEB86659FD93ull));
}
static inline double u01(uint64_t h) { return (double)(h >> 11) * (1.0 / 9007199254740992.0); }

/* Random bijection on [0, n) (cycle-walking 4-round Feistel). */
static inline uint64_t feistel(uint64_t x, uint64_t n, uint64_t seed) {
    int bits = 2;
    while ((1ull << bits) < n) bits += 2;
    int half = bits / 2;
    uint64_t mask = (1ull << half) - 1;
    do {
        uint64_t l = x >> half, r = x & mask;
        for (int i = 0; i < 4; i++) {
            uint64_t nl = r;
            uint64_t nr = l ^ (h3(seed, r, (uint64_t)i) & mask);
            l = nl; r = nr;
        }
        x = (l << half) | r;
    } while (x >= n);
    return x;
}

/* vertex id scrambling: 0 stays 0 (the R-MAT hub the configs use as source),
 * ids 1..n-1 are permuted among themselves. */
uint64_t dgi_perm(uint64_t v, uint64_t n, uint64_t seed) {
    if (v == 0 || n <= 2) return v;
    return 1 + feistel(v - 1, n - 1, seed);
}

/* R-MAT (Chakrabarti et al.): edge k descends `scale` quadrant levels with
 * probabilities (a, b, c, 1-a-b-c).  Endpoints >= n are redrawn (attempt
 * counter in the hash) so exactly m edges on [0, n) come out. */
void dgi_rmat(int scale, int64_t m, int64_t n, double a, double b, double c,
              uint64_t seed, int permute, int32_t *src, int32_t *dst) {
    #pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < m; k++) {
        for (uint64_t attempt = 0;; attempt++) {
            uint64_t u = 0, v = 0;
            for (int l = 0; l < scale; l++) {
                double r = u01(h3(seed, (uint64_t)k, (attempt << 8) | (uint64_t)l));
                int q = r < a ? 0 : r < a + b ? 1 : r < a + b + c ? 2 : 3;
                u = (u << 1) | (uint64_t)(q >> 1);
                v = (v << 1) | (uint64_t)(q & 1);
            }
            if ((int64_t)u < n && (int64_t)v < n) {
                if (permute) { u = dgi_perm(u, (uint64_t)n, seed ^ 0x5bd1e995ull);
                               v = dgi_perm(v, (uint64_t)n, seed ^ 0x5bd1e995ull); }
                src[k] = (int32_t)u; dst[k] = (int32_t)v;
                break;
            }
        }
    }
}

/* Long-chain-heavy digraph: vertices laid out as chains of `chain_len`
 * (edge v -> v+1 inside a chain; chain heads are random-permuted), plus
 * `m_extra` cross edges u -> u + offset (geometric forward offset, so
 * dependencies are deep), a fraction `back_frac` of them reversed (cycles).
 * Output: m = (#chain edges) + m_extra edges. */
int64_t dgi_chains(int64_t n, int64_t chain_len, int64_t m_extra, double back_frac,
                   uint64_t seed, int32_t *src, int32_t *dst) {
    int64_t n_chains = (n + chain_len - 1) / chain_len;
    int64_t m_chain = n - n_chains;
    #pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < n; v++) {
        int64_t pos = v % chain_len;
        int64_t base = v - pos;
        if (pos + 1 < chain_len && v + 1 < n) {
            int64_t k = base - base / chain_len + pos;   /* edges before this chain + pos */
            src[k] = (int32_t)dgi_perm((uint64_t)v, (uint64_t)n, seed);
            dst[k] = (int32_t)dgi_perm((uint64_t)(v + 1), (uint64_t)n, seed);
        }
    }
    #pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < m_extra; k++) {
        uint64_t u = h3(seed, 1, (uint64_t)k) % (uint64_t)n;
        double r = u01(h3(seed, 2, (uint64_t)k));
        /* geometric offset with mean ~ 4 chain lengths */
        double mean = 4.0 * (double)chain_len;
        uint64_t off = 1 + (uint64_t)(-mean * __builtin_log(1.0 - r));
        uint64_t v = (u + off) % (uint64_t)n;
        int back = u01(h3(seed, 3, (uint64_t)k)) < back_frac;
        uint64_t a = back ? v : u, b2 = back ? u : v;
        src[m_chain + k] = (int32_t)dgi_perm(a, (uint64_t)n, seed);
        dst[m_chain + k] = (int32_t)dgi_perm(b2, (uint64_t)n, seed);
    }
    return m_chain + m_extra;
}

/* Uniform random digraph on n vertices (Erdos-Renyi G(n, m) with replacement). */
void dgi_uniform(int64_t n, int64_t m, uint64_t seed, int32_t *src, int32_t *dst) {
    #pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < m; k++) {
        src[k] = (int32_t)(h3(seed, 11, (uint64_t)k) % (uint64_t)n);
        dst[k] = (int32_t)(h3(seed, 12, (uint64_t)k) % (uint64_t)n);
    }
}

static int cmp_i32(const void *x, const void *y) {
    int32_t a = *(const int32_t *)x, b = *(const int32_t *)y;
    return (a > b) - (a < b);
}

/* Edge list -> CSR (rows sorted by destination).  dedupe: drop repeated
 * (u,v); drop_self: drop u->u.  keep_m > 0: if more edges survive, keep the
 * keep_m ones with the smallest hash(u,v) (deterministic thinning to an exact
 * edge count).  row_ptr has n+1 entries; col must hold m entries.
 * Returns the final edge count.  Every pass is parallel; the output does not
 * depend on the thread count (rows are sorted after an unordered fill, and the
 * thinning threshold is the exact keep_m-th smallest hash). */
static inline uint64_t thin_hash(uint64_t seed, int64_t v, int32_t x) {
    return h3(seed ^ 0x7f4a7c15ull, (uint64_t)v, (uint64_t)x);
}
static int cmp_u64(const void *x, const void *y) {
    uint64_t a = *(const uint64_t *)x, b = *(const uint64_t *)y;
    return (a > b) - (a < b);
}
int64_t dgi_build_csr(int64_t n, int64_t m, const int32_t *src, const int32_t *dst,
                      int dedupe, int drop_self, int64_t keep_m, uint64_t seed,
                      int64_t *row_ptr, int32_t *col) {
    int64_t *cnt = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
    #pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < m; k++)
        if (!(drop_self && src[k] == dst[k])) __atomic_fetch_add(&cnt[src[k] + 1], 1, __ATOMIC_RELAXED);
    for (int64_t v = 0; v < n; v++) cnt[v + 1] += cnt[v];
    int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
    memcpy(fill, cnt, sizeof(int64_t) * (size_t)n);
    #pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < m; k++)
        if (!(drop_self && src[k] == dst[k])) col[__atomic_fetch_add(&fill[src[k]], 1, __ATOMIC_RELAXED)] = dst[k];
    free(fill);
    /* sort (and dedupe) each row in place */
    int64_t *keep = (int64_t *)malloc(sizeof(int64_t) * ((size_t)n + 1));
    #pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t v = 0; v < n; v++) {
        int64_t b = cnt[v], e = cnt[v + 1];
        qsort(col + b, (size_t)(e - b), sizeof(int32_t), cmp_i32);
        int64_t w = b;
        for (int64_t i = b; i < e; i++)
            if (!dedupe || i == b || col[i] != col[i - 1]) col[w++] = col[i];
        keep[v] = w - b;
    }
    int64_t total = 0;
    #pragma omp parallel for reduction(+:total) schedule(static)
    for (int64_t v = 0; v < n; v++) total += keep[v];
    /* optional thinning: the exact keep_m-th smallest hash(u,v) by a two-pass
     * radix select (histogram of the top 16 bits, then the one bucket sorted) */
    uint64_t thresh = UINT64_MAX;
    if (keep_m > 0 && total > keep_m) {
        enum { NB = 1 << 16 };
        uint64_t *hist = (uint64_t *)calloc(NB, sizeof(uint64_t));
        #pragma omp parallel
        {
            uint64_t *h = (uint64_t *)calloc(NB, sizeof(uint64_t));
            #pragma omp for schedule(dynamic, 1024)
            for (int64_t v = 0; v < n; v++)
                for (int64_t i = 0; i < keep[v]; i++) h[thin_hash(seed, v, col[cnt[v] + i]) >> 48]++;
            #pragma omp critical
            for (int b2 = 0; b2 < NB; b2++) hist[b2] += h[b2];
            free(h);
        }
        int64_t kth = keep_m - 1, below = 0;
        int bucket = 0;
        while (below + (int64_t)hist[bucket] <= kth) below += (int64_t)hist[bucket++];
        int64_t nb = (int64_t)hist[bucket], pos = 0;
        uint64_t *cand = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(nb > 0 ? nb : 1));
        #pragma omp parallel for schedule(dynamic, 1024)
        for (int64_t v = 0; v < n; v++)
            for (int64_t i = 0; i < keep[v]; i++) {
                uint64_t x = thin_hash(seed, v, col[cnt[v] + i]);
                if ((int)(x >> 48) == bucket) cand[__atomic_fetch_add(&pos, 1, __ATOMIC_RELAXED)] = x;
            }
        qsort(cand, (size_t)nb, sizeof(uint64_t), cmp_u64);
        thresh = cand[kth - below];
        free(cand); free(hist);
    }
    /* compact rows: kept count per row, offsets, parallel copy into a
     * temporary (rows move left, so an in-place parallel copy could overwrite
     * a row not yet read), then back into col */
    int64_t *kc = (int64_t *)malloc(sizeof(int64_t) * ((size_t)n + 1));
    #pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t v = 0; v < n; v++) {
        int64_t c = keep[v];
        if (thresh != UINT64_MAX) {
            c = 0;
            for (int64_t i = 0; i < keep[v]; i++) c += thin_hash(seed, v, col[cnt[v] + i]) <= thresh;
        }
        kc[v] = c;
    }
    row_ptr[0] = 0;
    for (int64_t v = 0; v < n; v++) row_ptr[v + 1] = row_ptr[v] + kc[v];
    int32_t *tmp = (int32_t *)malloc(sizeof(int32_t) * (size_t)(row_ptr[n] > 0 ? row_ptr[n] : 1));
    #pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t v = 0; v < n; v++) {
        int64_t b = cnt[v], w = row_ptr[v];
        for (int64_t i = 0; i < keep[v]; i++) {
            int32_t x = col[b + i];
            if (thresh != UINT64_MAX && thin_hash(seed, v, x) > thresh) continue;
            tmp[w++] = x;
        }
    }
    memcpy(col, tmp, sizeof(int32_t) * (size_t)row_ptr[n]);
    free(tmp); free(kc);
    free(cnt); free(keep);
    return row_ptr[n];
}

/* Integer weight of edge (u,v): uniform in [lo, hi], a function of (u,v). */
void dgi_weights(int64_t n, const int64_t *row_ptr, const int32_t *col,
                 int32_t lo, int32_t hi, uint64_t seed, int32_t *w) {
    uint64_t span = (uint64_t)(hi - lo + 1);
    #pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t v = 0; v < n; v++)
        for (int64_t i = row_ptr[v]; i < row_ptr[v + 1]; i++)
            w[i] = lo + (int32_t)(h3(seed ^ 0x2545F491ull, (uint64_t)v, (uint64_t)col[i]) % span);
}

/* Per-vertex uniform doubles in [lo, hi) (random parameters the method is
 * given as inputs, e.g. Adsorption's p_inj / p_cont / injected values). */
void dgi_uniform_f64(int64_t n, uint64_t seed, uint64_t stream, double lo, double hi, double *out) {
    #pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < n; v++) out[v] = lo + (hi - lo) * u01(h3(seed, stream, (uint64_t)v));
}
