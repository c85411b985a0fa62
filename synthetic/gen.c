/*
 * synthetic/gen.c -- seeded synthetic CSR matrices and dense operands.
 *
 * Shared input generators: the ONLY code both the oracle side (tests) and the
 * CUDA side (tests, bench) use.  Holds none of the method's arithmetic (no
 * SpMM, no permutation, no feature): it only draws matrices shaped like the
 * paper's workloads (power-law graphs, banded FEM stencils, uniform random,
 * block-clustered; SURVEY.md §8(d) "Synthetic inputs").
 *
 * Every random number is a counter-based hash  rnd(seed, counter)  (splitmix64
 * finaliser), so a draw depends only on (seed, counter) and never on thread
 * count or scheduling.  Output CSR: rowidx int64[M+1], colidx int32[nnz] strictly
 * increasing per row, value float32[nnz].
 *
 * Memory protocol: a generator builds the CSR in malloc'd staging buffers and
 * returns an opaque pointer; synth_sizes() reports M, N, nnz so the caller can
 * allocate, and synth_take() copies the arrays out and frees the staging.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#ifdef _OPENMP
#include <omp.h>
#endif

typedef struct {
    int64_t M, N, nnz;
    int64_t *rowidx;
    int32_t *colidx;
    float *value;
} staged_csr;

static inline uint64_t mix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}
/* counter-based draw: independent streams per (seed, stream id) */
static inline uint64_t rnd(uint64_t seed, uint64_t stream, uint64_t ctr) {
    return mix64(mix64(seed * 0xD1B54A32D192ED03ULL + stream) ^ (ctr * 0x9E3779B97F4A7C15ULL));
}
static inline double u01(uint64_t r) { return (double)(r >> 11) * (1.0 / 9007199254740992.0); }
/* U[-1,1) on a 2^-23 grid: exactly representable in fp32 */
static inline float um11(uint64_t r) { return (float)((int64_t)(r >> 40) - (1LL << 23)) * (1.0f / 8388608.0f); }

enum { STREAM_RMAT = 1, STREAM_LOCAL = 2, STREAM_LABEL = 3, STREAM_VALUE = 4, STREAM_B = 5,
       STREAM_UNIF = 6, STREAM_BLK = 7, STREAM_SHUF = 8, STREAM_INTV = 9 };

static int cmp_i32(const void *a, const void *b) {
    int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    return (x > y) - (x < y);
}

/* sort + dedup each row of a (row, col) edge list, build CSR, draw values */
static staged_csr *edges_to_csr(int64_t M, int64_t N, int64_t E, const int32_t *er, const int32_t *ec,
                                uint64_t seed, int value_mode) {
    staged_csr *s = (staged_csr *)calloc(1, sizeof(staged_csr));
    s->M = M; s->N = N;
    int64_t *cnt = (int64_t *)calloc((size_t)M + 1, sizeof(int64_t));
    for (int64_t e = 0; e < E; ++e) cnt[er[e] + 1]++;
    for (int64_t i = 0; i < M; ++i) cnt[i + 1] += cnt[i];
    int32_t *tmp = (int32_t *)malloc((size_t)(E ? E : 1) * sizeof(int32_t));
    int64_t *cur = (int64_t *)malloc((size_t)(M ? M : 1) * sizeof(int64_t));
    memcpy(cur, cnt, (size_t)M * sizeof(int64_t));
    for (int64_t e = 0; e < E; ++e) tmp[cur[er[e]]++] = ec[e];
    free(cur);
    int64_t *ucnt = (int64_t *)calloc((size_t)M + 1, sizeof(int64_t));
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t i = 0; i < M; ++i) {
        int64_t a = cnt[i], b = cnt[i + 1];
        if (b - a > 1) qsort(tmp + a, (size_t)(b - a), sizeof(int32_t), cmp_i32);
        int64_t u = 0;
        for (int64_t j = a; j < b; ++j)
            if (j == a || tmp[j] != tmp[j - 1]) tmp[a + u++] = tmp[j];
        ucnt[i + 1] = u;
    }
    for (int64_t i = 0; i < M; ++i) ucnt[i + 1] += ucnt[i];
    s->nnz = ucnt[M];
    s->rowidx = ucnt;
    s->colidx = (int32_t *)malloc((size_t)(s->nnz ? s->nnz : 1) * sizeof(int32_t));
    s->value = (float *)malloc((size_t)(s->nnz ? s->nnz : 1) * sizeof(float));
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t i = 0; i < M; ++i)
        memcpy(s->colidx + ucnt[i], tmp + cnt[i], (size_t)(ucnt[i + 1] - ucnt[i]) * sizeof(int32_t));
    free(tmp);
    free(cnt);
    const int64_t nnz = s->nnz;
#pragma omp parallel for schedule(static)
    for (int64_t j = 0; j < nnz; ++j) {
        uint64_t r = rnd(seed, value_mode ? STREAM_INTV : STREAM_VALUE, (uint64_t)j);
        if (value_mode) {          /* integer-valued: {-2,-1,1,2} (exact fp32 products) */
            static const float tab[4] = {-2.f, -1.f, 1.f, 2.f};
            s->value[j] = tab[r >> 62];
        } else {
            s->value[j] = um11(r);
        }
    }
    return s;
}

/* a permutation of [0,n) from a counter-based Fisher-Yates */
static int32_t *random_perm(int64_t n, uint64_t seed, uint64_t stream) {
    int32_t *p = (int32_t *)malloc((size_t)(n ? n : 1) * sizeof(int32_t));
    for (int64_t i = 0; i < n; ++i) p[i] = (int32_t)i;
    for (int64_t i = n - 1; i > 0; --i) {
        uint64_t r = rnd(seed, stream, (uint64_t)i);
        int64_t j = (int64_t)(((unsigned __int128)r * (unsigned __int128)(i + 1)) >> 64);
        int32_t t = p[i]; p[i] = p[j]; p[j] = t;
    }
    return p;
}

/* ---------------------------------------------------------------------------------------
 * R-MAT (Graph500 a,b,c,d = .57,.19,.19,.05), 2^S rows/cols, E = 2^S * edge_factor draws.
 * variant 0 = natural labels, 1 = random-label (same permutation on rows and columns),
 * 2 = local: R-MAT rows; each edge's column lands w.p. p_local uniformly in the row's
 *     community window [floor(i/2^12)*2^12, +2^12), otherwise on an R-MAT column.
 * ------------------------------------------------------------------------------------- */
void *synth_rmat(int32_t S, double edge_factor, uint64_t seed, int32_t variant, double p_local,
                 int32_t value_mode) {
    const int64_t n = (int64_t)1 << S;
    const int64_t E = (int64_t)((double)n * edge_factor);
    int32_t *er = (int32_t *)malloc((size_t)(E ? E : 1) * sizeof(int32_t));
    int32_t *ec = (int32_t *)malloc((size_t)(E ? E : 1) * sizeof(int32_t));
    const double a = 0.57, b = 0.19, c = 0.19;
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < E; ++e) {
        int64_t r = 0, q = 0;
        for (int l = 0; l < S; ++l) {
            double u = u01(rnd(seed, STREAM_RMAT, (uint64_t)e * 64u + (uint64_t)l));
            int rb, cb;
            if (u < a) { rb = 0; cb = 0; }
            else if (u < a + b) { rb = 0; cb = 1; }
            else if (u < a + b + c) { rb = 1; cb = 0; }
            else { rb = 1; cb = 1; }
            r = (r << 1) | rb;
            q = (q << 1) | cb;
        }
        if (variant == 2) {
            uint64_t h = rnd(seed, STREAM_LOCAL, (uint64_t)e);
            if (u01(h) < p_local) {
                int64_t w = 12 < S ? 12 : S;
                int64_t base = (r >> w) << w;
                q = base + (int64_t)(rnd(seed, STREAM_LOCAL + 100, (uint64_t)e) & (((uint64_t)1 << w) - 1));
            }
        }
        er[e] = (int32_t)r;
        ec[e] = (int32_t)q;
    }
    if (variant == 1) {
        int32_t *pi = random_perm(n, seed, STREAM_LABEL);
#pragma omp parallel for schedule(static)
        for (int64_t e = 0; e < E; ++e) { er[e] = pi[er[e]]; ec[e] = pi[ec[e]]; }
        free(pi);
    }
    staged_csr *s = edges_to_csr(n, n, E, er, ec, seed, value_mode);
    free(er); free(ec);
    return s;
}

/* 3-D 27-point stencil on an n^3 grid, lexicographic order i = (x*n + y)*n + z */
void *synth_stencil27(int32_t n, uint64_t seed, int32_t value_mode) {
    const int64_t M = (int64_t)n * n * n;
    staged_csr *s = (staged_csr *)calloc(1, sizeof(staged_csr));
    s->M = M; s->N = M;
    s->rowidx = (int64_t *)calloc((size_t)M + 1, sizeof(int64_t));
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < M; ++i) {
        int64_t x = i / ((int64_t)n * n), y = (i / n) % n, z = i % n;
        int64_t cx = 1 + (x > 0) + (x < n - 1), cy = 1 + (y > 0) + (y < n - 1), cz = 1 + (z > 0) + (z < n - 1);
        s->rowidx[i + 1] = cx * cy * cz;
    }
    for (int64_t i = 0; i < M; ++i) s->rowidx[i + 1] += s->rowidx[i];
    s->nnz = s->rowidx[M];
    s->colidx = (int32_t *)malloc((size_t)(s->nnz ? s->nnz : 1) * sizeof(int32_t));
    s->value = (float *)malloc((size_t)(s->nnz ? s->nnz : 1) * sizeof(float));
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < M; ++i) {
        int64_t x = i / ((int64_t)n * n), y = (i / n) % n, z = i % n, k = s->rowidx[i];
        for (int dx = -1; dx <= 1; ++dx)
            for (int dy = -1; dy <= 1; ++dy)
                for (int dz = -1; dz <= 1; ++dz) {
                    int64_t X = x + dx, Y = y + dy, Z = z + dz;
                    if (X < 0 || Y < 0 || Z < 0 || X >= n || Y >= n || Z >= n) continue;
                    s->colidx[k++] = (int32_t)((X * n + Y) * n + Z);
                }
    }
    const int64_t nnz = s->nnz;
#pragma omp parallel for schedule(static)
    for (int64_t j = 0; j < nnz; ++j) {
        uint64_t r = rnd(seed, value_mode ? STREAM_INTV : STREAM_VALUE, (uint64_t)j);
        static const float tab[4] = {-2.f, -1.f, 1.f, 2.f};
        s->value[j] = value_mode ? tab[r >> 62] : um11(r);
    }
    return s;
}

/* d distinct uniform columns per row; d_mode 0 = fixed d, 1 = Poisson(d) per row (capped at N) */
void *synth_uniform(int64_t M, int64_t N, double d, int32_t d_mode, uint64_t seed, int32_t value_mode) {
    int64_t *deg = (int64_t *)malloc((size_t)(M ? M : 1) * sizeof(int64_t));
    int64_t E = 0;
    for (int64_t i = 0; i < M; ++i) {
        int64_t k;
        if (d_mode == 0) {
            k = (int64_t)d;
        } else {            /* Poisson by inversion on a counter draw */
            double u = u01(rnd(seed, STREAM_UNIF + 50, (uint64_t)i)), p = exp(-d), cdf = p;
            k = 0;
            while (u > cdf && k < 100000) { ++k; p *= d / (double)k; cdf += p; }
        }
        if (k > N) k = N;
        deg[i] = k;
        E += k;
    }
    int32_t *er = (int32_t *)malloc((size_t)(E ? E : 1) * sizeof(int32_t));
    int32_t *ec = (int32_t *)malloc((size_t)(E ? E : 1) * sizeof(int32_t));
    int64_t *off = (int64_t *)malloc((size_t)(M + 1) * sizeof(int64_t));
    off[0] = 0;
    for (int64_t i = 0; i < M; ++i) off[i + 1] = off[i] + deg[i];
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t i = 0; i < M; ++i) {
        /* Floyd's algorithm: deg[i] distinct values in [0,N) */
        int64_t k = deg[i], base = off[i], got = 0;
        for (int64_t t = N - k; t < N; ++t) {
            int64_t v = (int64_t)(((unsigned __int128)rnd(seed, STREAM_UNIF, (uint64_t)(base + got) * 2u) *
                                   (unsigned __int128)(t + 1)) >> 64);
            int dup = 0;
            for (int64_t q = 0; q < got; ++q)
                if (ec[base + q] == (int32_t)v) { dup = 1; break; }
            ec[base + got] = (int32_t)(dup ? t : v);
            er[base + got] = (int32_t)i;
            ++got;
        }
    }
    free(off); free(deg);
    staged_csr *s = edges_to_csr(M, N, E, er, ec, seed, value_mode);
    free(er); free(ec);
    return s;
}

/* Block-clustered: groups of g consecutive rows; each group draws c column blocks of bw columns,
 * each row draws d columns from its group's blocks; then a random row shuffle.
 * planted = 1: groups own disjoint block sets (block ids k*c .. k*c+c-1 before a random block
 * relabel) and every row hits every one of its group's blocks (d >= c). */
void *synth_blockcluster(int64_t M, int64_t N, int64_t g, int64_t c, int64_t d, int32_t bw, int32_t planted,
                         uint64_t seed, int32_t value_mode) {
    const int64_t nblk = (N + bw - 1) / bw;
    const int64_t G = (M + g - 1) / g;
    if (c > nblk) c = nblk;
    if (d > c * bw) d = c * bw;
    int32_t *blk = (int32_t *)malloc((size_t)(G * c ? G * c : 1) * sizeof(int32_t));
    int32_t *brel = planted ? random_perm(nblk, seed, STREAM_BLK + 10) : NULL;
    for (int64_t k = 0; k < G; ++k) {
        for (int64_t t = 0; t < c; ++t) {
            if (planted) {
                blk[k * c + t] = brel[(k * c + t) % nblk];
            } else {  /* distinct blocks per group by Floyd */
                int64_t tt = nblk - c + t;
                int64_t v = (int64_t)(((unsigned __int128)rnd(seed, STREAM_BLK, (uint64_t)(k * c + t)) *
                                       (unsigned __int128)(tt + 1)) >> 64);
                int dup = 0;
                for (int64_t q = 0; q < t; ++q)
                    if (blk[k * c + q] == (int32_t)v) { dup = 1; break; }
                blk[k * c + t] = (int32_t)(dup ? tt : v);
            }
        }
    }
    free(brel);
    const int64_t E = M * d;
    int32_t *er = (int32_t *)malloc((size_t)(E ? E : 1) * sizeof(int32_t));
    int32_t *ec = (int32_t *)malloc((size_t)(E ? E : 1) * sizeof(int32_t));
    int32_t *rowshuf = random_perm(M, seed, STREAM_SHUF);
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < M; ++i) {
        const int32_t *gb = blk + (i / g) * c;
        int64_t got = 0;
        int32_t *out = ec + i * d;
        if (planted) {  /* one column per block first, so every block is hit */
            for (int64_t t = 0; t < c && got < d; ++t) {
                int64_t lo = (int64_t)gb[t] * bw, hi = lo + bw < N ? lo + bw : N;
                int64_t col = lo + (int64_t)(rnd(seed, STREAM_BLK + 20, (uint64_t)(i * d + got)) % (uint64_t)(hi - lo));
                out[got++] = (int32_t)col;
            }
        }
        uint64_t ctr = 0;
        while (got < d) {
            uint64_t r = rnd(seed, STREAM_BLK + 30, (uint64_t)i * 1048576u + ctr++);
            int64_t t = (int64_t)(r % (uint64_t)c);
            int64_t lo = (int64_t)gb[t] * bw, hi = lo + bw < N ? lo + bw : N;
            int64_t col = lo + (int64_t)((r >> 32) % (uint64_t)(hi - lo));
            int dup = 0;
            for (int64_t q = 0; q < got; ++q)
                if (out[q] == (int32_t)col) { dup = 1; break; }
            if (!dup) out[got++] = (int32_t)col;
            if (ctr > (uint64_t)(64 * d + 1024)) break;  /* group blocks too narrow (N tail) */
        }
        for (int64_t q = 0; q < d; ++q) er[i * d + q] = q < got ? rowshuf[i] : -1;
        for (int64_t q = got; q < d; ++q) out[q] = 0;
    }
    free(rowshuf); free(blk);
    /* drop padding (-1) entries */
    int64_t E2 = 0;
    for (int64_t e = 0; e < E; ++e)
        if (er[e] >= 0) { er[E2] = er[e]; ec[E2] = ec[e]; ++E2; }
    staged_csr *s = edges_to_csr(M, N, E2, er, ec, seed, value_mode);
    free(er); free(ec);
    return s;
}

/* Arbitrary CSR from an explicit per-row degree list with uniform columns
 * (corpus helper for log-uniform nnz/row mixes). */
void *synth_from_degrees(int64_t M, int64_t N, const int64_t *deg_in, uint64_t seed, int32_t value_mode) {
    int64_t E = 0;
    for (int64_t i = 0; i < M; ++i) E += deg_in[i] < N ? deg_in[i] : N;
    int32_t *er = (int32_t *)malloc((size_t)(E ? E : 1) * sizeof(int32_t));
    int32_t *ec = (int32_t *)malloc((size_t)(E ? E : 1) * sizeof(int32_t));
    int64_t *off = (int64_t *)malloc((size_t)(M + 1) * sizeof(int64_t));
    off[0] = 0;
    for (int64_t i = 0; i < M; ++i) off[i + 1] = off[i] + (deg_in[i] < N ? deg_in[i] : N);
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t i = 0; i < M; ++i) {
        int64_t k = off[i + 1] - off[i], base = off[i], got = 0;
        for (int64_t t = N - k; t < N; ++t) {
            int64_t v = (int64_t)(((unsigned __int128)rnd(seed, STREAM_UNIF + 7, (uint64_t)(base + got)) *
                                   (unsigned __int128)(t + 1)) >> 64);
            int dup = 0;
            if (k <= 64) {
                for (int64_t q = 0; q < got; ++q)
                    if (ec[base + q] == (int32_t)v) { dup = 1; break; }
            }
            ec[base + got] = (int32_t)(dup ? t : v);
            er[base + got] = (int32_t)i;
            ++got;
        }
    }
    free(off);
    staged_csr *s = edges_to_csr(M, N, E, er, ec, seed, value_mode);
    free(er); free(ec);
    return s;
}

/* Banded random: row i draws min(d, band) distinct columns uniformly in [i-w, i+w] (clipped to [0,N)). */
void *synth_banded(int64_t M, int64_t N, int64_t d, int64_t w, uint64_t seed, int32_t value_mode) {
    int64_t *off = (int64_t *)malloc((size_t)(M + 1) * sizeof(int64_t));
    off[0] = 0;
    for (int64_t i = 0; i < M; ++i) {
        int64_t lo = i - w < 0 ? 0 : i - w, hi = i + w + 1 > N ? N : i + w + 1;
        int64_t band = hi > lo ? hi - lo : 0;
        off[i + 1] = off[i] + (d < band ? d : band);
    }
    const int64_t E = off[M];
    int32_t *er = (int32_t *)malloc((size_t)(E ? E : 1) * sizeof(int32_t));
    int32_t *ec = (int32_t *)malloc((size_t)(E ? E : 1) * sizeof(int32_t));
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t i = 0; i < M; ++i) {
        int64_t lo = i - w < 0 ? 0 : i - w, hi = i + w + 1 > N ? N : i + w + 1;
        int64_t band = hi - lo, k = off[i + 1] - off[i], base = off[i], got = 0;
        for (int64_t t = band - k; t < band; ++t) {   /* Floyd over [0, band) */
            int64_t v = (int64_t)(((unsigned __int128)rnd(seed, STREAM_UNIF + 11, (uint64_t)(base + got)) *
                                   (unsigned __int128)(t + 1)) >> 64);
            int dup = 0;
            for (int64_t q = 0; q < got; ++q)
                if (ec[base + q] == (int32_t)(lo + v)) { dup = 1; break; }
            ec[base + got] = (int32_t)(lo + (dup ? t : v));
            er[base + got] = (int32_t)i;
            ++got;
        }
    }
    free(off);
    staged_csr *s = edges_to_csr(M, N, E, er, ec, seed, value_mode);
    free(er); free(ec);
    return s;
}

void synth_sizes(const void *h, int64_t *M, int64_t *N, int64_t *nnz) {
    const staged_csr *s = (const staged_csr *)h;
    *M = s->M; *N = s->N; *nnz = s->nnz;
}

void synth_take(void *h, int64_t *rowidx, int32_t *colidx, float *value) {
    staged_csr *s = (staged_csr *)h;
    memcpy(rowidx, s->rowidx, (size_t)(s->M + 1) * sizeof(int64_t));
    memcpy(colidx, s->colidx, (size_t)s->nnz * sizeof(int32_t));
    memcpy(value, s->value, (size_t)s->nnz * sizeof(float));
    free(s->rowidx); free(s->colidx); free(s->value); free(s);
}

/* dense row-major [rows][K] operand, U[-1,1) on a 2^-23 grid (value_mode 0) or integers in [-8,8]
 * (value_mode 1); rows [row0, row0+rows) of the full operand so a block can be drawn alone */
void synth_dense(int64_t row0, int64_t rows, int64_t K, uint64_t seed, int32_t value_mode, float *out) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < rows; ++i)
        for (int64_t k = 0; k < K; ++k) {
            uint64_t r = rnd(seed, STREAM_B, (uint64_t)(row0 + i) * (uint64_t)K + (uint64_t)k);
            out[i * K + k] = value_mode ? (float)((int64_t)(r % 17u) - 8) : um11(r);
        }
}

int32_t synth_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
