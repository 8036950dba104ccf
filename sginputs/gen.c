/*
 * sginputs/gen.c — seeded synthetic input generators (ER, R-MAT, special matrices).
 *
 * This module is SHARED by the oracle tests and the CUDA path (input recipe).
 * It holds none of the method's arithmetic: it only builds canonical CSR inputs (sorted,
 * unique columns per row) and their values. Everything is a pure function of
 * (parameters, seed) through a counter-based SplitMix64 hash, so any process on any host
 * reproduces the same matrix bit-for-bit.
 *
 * Readings:
 *   Q4  h(seed, tag, j) = sm(seed ^ sm(tag ^ sm(j)))  with SplitMix64 finaliser sm.
 *   Q10 duplicates merged (sort + unique per row); values drawn per unique (i, j) after dedupe.
 *   Q11 value modes: real U[0.5,1.5) / integers {1,2,3,4} / all ones.
 *   Q12 R-MAT: per edge, `scale` quadrant draws against cumulative (a, a+b, a+b+c) in 2^64
 *       fixed point, MSB first; b sets the column bit, c the row bit, d both; seeded symmetric
 *       label permutation pi(v) = rank of h(seed, PERM, v); self-loops kept; directed.
 *   Q13 ER G(n, m): m = d*n edges, i = h(seed,ER_ROW,e) mod n, j = h(seed,ER_COL,e) mod p.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define TAG_VAL    0x56414c5545530001ULL
#define TAG_RMAT   0x524d415445444745ULL
#define TAG_PERM   0x5045524d55544531ULL
#define TAG_ER_ROW 0x45525f524f570001ULL
#define TAG_ER_COL 0x45525f434f4c0001ULL

static inline uint64_t sm64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}
static inline uint64_t h3(uint64_t seed, uint64_t tag, uint64_t j) {
    return sm64(seed ^ sm64(tag ^ sm64(j)));
}

uint64_t sginputs_hash(uint64_t seed, uint64_t tag, uint64_t j) { return h3(seed, tag, j); }

/* ER G(n, m) edge list (Q13). */
void sginputs_er_edges(int64_t n, int64_t p, int64_t m, uint64_t seed, int32_t* ei, int32_t* ej) {
    #pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < m; ++e) {
        ei[e] = (int32_t)(h3(seed, TAG_ER_ROW, (uint64_t)e) % (uint64_t)n);
        ej[e] = (int32_t)(h3(seed, TAG_ER_COL, (uint64_t)e) % (uint64_t)p);
    }
}

typedef struct { uint64_t key; int32_t v; int32_t pad; } keyed_t;
static int cmp_keyed(const void* a, const void* b) {
    const keyed_t* x = (const keyed_t*)a; const keyed_t* y = (const keyed_t*)b;
    if (x->key != y->key) return x->key < y->key ? -1 : 1;
    return x->v < y->v ? -1 : (x->v > y->v);
}

/* pi(v) = rank of h(seed, PERM, v) among all v (ties by v). perm must hold nv entries. */
void sginputs_rmat_perm(int64_t nv, uint64_t seed, int32_t* perm) {
    keyed_t* k = (keyed_t*)malloc(sizeof(keyed_t) * (size_t)nv);
    for (int64_t v = 0; v < nv; ++v) { k[v].key = h3(seed, TAG_PERM, (uint64_t)v); k[v].v = (int32_t)v; k[v].pad = 0; }
    qsort(k, (size_t)nv, sizeof(keyed_t), cmp_keyed);
    for (int64_t r = 0; r < nv; ++r) perm[k[r].v] = (int32_t)r;
    free(k);
}

/* R-MAT edge list (Q12). Probabilities given as 2^64 fixed-point cumulative thresholds
 * computed on the host by the caller (ta = a, tb = a+b, tc = a+b+c). */
void sginputs_rmat_edges(int scale, int64_t m, uint64_t ta, uint64_t tb, uint64_t tc,
                         uint64_t seed, int permute, int32_t* ei, int32_t* ej) {
    int64_t nv = (int64_t)1 << scale;
    int32_t* perm = NULL;
    if (permute) { perm = (int32_t*)malloc(sizeof(int32_t) * (size_t)nv); sginputs_rmat_perm(nv, seed, perm); }
    #pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < m; ++e) {
        uint32_t r = 0, c = 0;
        for (int l = 0; l < scale; ++l) {
            uint64_t x = h3(seed, TAG_RMAT, (uint64_t)e * (uint64_t)scale + (uint64_t)l);
            uint32_t bit = 1u << (scale - 1 - l);
            if (x < ta) { /* quadrant a */ }
            else if (x < tb) { c |= bit; }
            else if (x < tc) { r |= bit; }
            else { r |= bit; c |= bit; }
        }
        if (perm) { r = (uint32_t)perm[r]; c = (uint32_t)perm[c]; }
        ei[e] = (int32_t)r; ej[e] = (int32_t)c;
    }
    free(perm);
}

static int cmp_i32(const void* a, const void* b) {
    int32_t x = *(const int32_t*)a, y = *(const int32_t*)b; return (x > y) - (x < y);
}

/* Canonical CSR from an edge list: counting sort by row, then sort + unique per row.
 * row_ptr: n+1 entries; col_out: m entries (first nnz used). Returns nnz. */
int64_t sginputs_csr_from_edges(int64_t n, int64_t m, const int32_t* ei, const int32_t* ej,
                                int64_t* row_ptr, int32_t* col_out) {
    int64_t* cnt = (int64_t*)calloc((size_t)n + 1, sizeof(int64_t));
    for (int64_t e = 0; e < m; ++e) cnt[ei[e] + 1]++;
    for (int64_t i = 0; i < n; ++i) cnt[i + 1] += cnt[i];
    int64_t* pos = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n + 1));
    memcpy(pos, cnt, sizeof(int64_t) * (size_t)(n + 1));
    for (int64_t e = 0; e < m; ++e) col_out[pos[ei[e]]++] = ej[e];
    free(pos);
    int64_t* ucnt = (int64_t*)malloc(sizeof(int64_t) * (size_t)n);
    #pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t i = 0; i < n; ++i) {
        int32_t* s = col_out + cnt[i];
        int64_t len = cnt[i + 1] - cnt[i];
        if (len > 1) qsort(s, (size_t)len, sizeof(int32_t), cmp_i32);
        int64_t u = 0;
        for (int64_t q = 0; q < len; ++q) if (u == 0 || s[q] != s[u - 1]) s[u++] = s[q];
        ucnt[i] = u;
    }
    /* compact rows to the front (sequential, stable, in place since dst <= src) */
    int64_t off = 0;
    row_ptr[0] = 0;
    for (int64_t i = 0; i < n; ++i) {
        if (off != cnt[i]) memmove(col_out + off, col_out + cnt[i], sizeof(int32_t) * (size_t)ucnt[i]);
        off += ucnt[i];
        row_ptr[i + 1] = off;
    }
    free(ucnt); free(cnt);
    return off;
}

/* Values per unique (i, j) (Q11). mode 0: real U[0.5,1.5); 1: integer {1,2,3,4}; 2: all ones;
 * 3: signed integer {-2,-1,1,2} (exact cancellation to 0 happens: structural zeros, R9);
 * 4: {-1, 0, 1, 2} (explicitly STORED zeros in the inputs).
 * out is double (is_f32 == 0) or float (is_f32 == 1). */
void sginputs_values(int64_t n, int64_t p, const int64_t* row_ptr, const int32_t* col,
                     uint64_t seed, int mode, int is_f32, void* out) {
    #pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t i = 0; i < n; ++i) {
        for (int64_t q = row_ptr[i]; q < row_ptr[i + 1]; ++q) {
            double v;
            if (mode == 2) v = 1.0;
            else {
                uint64_t x = h3(seed, TAG_VAL, (uint64_t)i * (uint64_t)p + (uint64_t)col[q]);
                if (mode == 1) v = (double)(1 + (x & 3));
                else if (mode == 3) v = (double)((int)(x & 3) - 2 + ((x & 3) >= 2));
                else if (mode == 4) v = (double)((int)(x & 3) - 1);
                else v = 0.5 + (double)(x >> 11) * 0x1.0p-53;
            }
            if (is_f32) ((float*)out)[q] = (float)v; else ((double*)out)[q] = v;
        }
    }
}
