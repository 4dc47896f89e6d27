/* gen/gen.c — seeded synthetic-input generators shared by the oracle and the
 * CUDA path.  This file holds NO arithmetic of the method (no normalisation,
 * permutation, partitioning, SpMM, GEMM, loss or optimiser); it only draws
 * random numbers and assembles the input CSR / features / labels / weights
 * with the recipe of SURVEY.md §8(d) "Synthetic inputs" (restated in
 * DESIGN.md §3):
 *
 *  - Philox4x32-10 (Salmon et al., SC'11; the Random123 / cuRAND constants),
 *    key = (seed lo32, seed hi32), counter = (c0, c1, c2, c3).
 *  - U(seed, i) = (word i%4 of Philox(seed, (i/4 lo, i/4 hi, 0, 0)) >> 8) * 2^-24.
 *  - R-MAT, Graph500 (a,b,c,d) = (0.57,0.19,0.19,0.05), s = ceil(log2 n)
 *    levels; candidate k draws its level words from counter (k lo, k hi, w, 0),
 *    word j of call w = level 4w+j (level 0 = most significant bit).  Rejected
 *    if u>=n, v>=n or u==v; the first m/2 accepted candidates in k order emit
 *    (u,v) and (v,u).  Duplicates are kept (multiplicity).  CSR sorted by
 *    (row, col).
 *  - X[v][k] = 2 U(seed, v*d + k) - 1; y[v] = (k24 * C) >> 24;
 *    W_l[c][k] = a (2 U(seed, c*dout + k) - 1), a = sqrt(6/(din+dout)).
 *
 * Built as gen/libmggcn_gen.so (OpenMP for the R-MAT candidate stream; the
 * result is independent of the thread count because candidates are counter
 * based and concatenated in k order).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define PHILOX_M0 0xD2511F53u
#define PHILOX_M1 0xCD9E8D57u
#define PHILOX_W0 0x9E3779B9u
#define PHILOX_W1 0xBB67AE85u

static inline void philox_round(uint32_t c[4], const uint32_t k[2]) {
    uint64_t p0 = (uint64_t)PHILOX_M0 * c[0];
    uint64_t p1 = (uint64_t)PHILOX_M1 * c[2];
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    uint32_t o0 = hi1 ^ c[1] ^ k[0];
    uint32_t o2 = hi0 ^ c[3] ^ k[1];
    c[0] = o0; c[1] = lo1; c[2] = o2; c[3] = lo0;
}

/* Philox4x32 with R rounds (R = 10 everywhere in this repo). */
void gen_philox4x32(int rounds, const uint32_t ctr_in[4], const uint32_t key_in[2], uint32_t out[4]) {
    uint32_t c[4] = {ctr_in[0], ctr_in[1], ctr_in[2], ctr_in[3]};
    uint32_t k[2] = {key_in[0], key_in[1]};
    for (int r = 0; r < rounds; ++r) {
        if (r > 0) { k[0] += PHILOX_W0; k[1] += PHILOX_W1; }
        philox_round(c, k);
    }
    out[0] = c[0]; out[1] = c[1]; out[2] = c[2]; out[3] = c[3];
}

static inline void philox10(uint64_t seed, uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3, uint32_t out[4]) {
    uint32_t ctr[4] = {c0, c1, c2, c3};
    uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
    gen_philox4x32(10, ctr, key, out);
}

/* 24-bit integer behind U(seed, i). */
static inline uint32_t u24(uint64_t seed, uint64_t i) {
    uint64_t q = i >> 2;
    uint32_t w[4];
    philox10(seed, (uint32_t)q, (uint32_t)(q >> 32), 0, 0, w);
    return w[i & 3] >> 8;
}

/* U(seed, i) for i in [start, start+count), as doubles in [0,1). */
void gen_uniform(uint64_t seed, uint64_t start, int64_t count, double* out) {
#pragma omp parallel for schedule(static)
    for (int64_t t = 0; t < count; ++t) out[t] = (double)u24(seed, start + (uint64_t)t) * (1.0 / 16777216.0);
}

/* X (n x d, row stride ld >= d, padding columns set to 0): X[v][k] = 2U(seed, v*d+k) - 1. */
void gen_features(int64_t n, int64_t d, int64_t ld, uint64_t seed, float* X) {
#pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < n; ++v) {
        float* row = X + v * ld;
        for (int64_t k = 0; k < d; ++k) {
            double u = (double)u24(seed, (uint64_t)(v * d + k)) * (1.0 / 16777216.0);
            row[k] = (float)(2.0 * u - 1.0);   /* exact: 24-bit value */
        }
        for (int64_t k = d; k < ld; ++k) row[k] = 0.0f;
    }
}

/* Labels y[v] = (k24 * C) >> 24.  If unlabelled_per_mille > 0, vertex v is
 * unlabelled (y = -1) when u24(seed ^ 0x5bd1e995, v) * 1000 < per_mille * 2^24. */
void gen_labels(int64_t n, int32_t C, uint64_t seed, int32_t unlabelled_per_mille, int32_t* y) {
#pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < n; ++v) {
        uint32_t k = u24(seed, (uint64_t)v);
        int32_t lab = (int32_t)(((uint64_t)k * (uint64_t)C) >> 24);
        if (unlabelled_per_mille > 0) {
            uint32_t q = u24(seed ^ 0x5bd1e995ull, (uint64_t)v);
            if ((uint64_t)q * 1000ull < (uint64_t)unlabelled_per_mille * 16777216ull) lab = -1;
        }
        y[v] = lab;
    }
}

/* Glorot-uniform W (din x dout, row-major): a (2U(seed, c*dout+k) - 1). */
void gen_glorot(int64_t din, int64_t dout, uint64_t seed, float* W) {
    double a = sqrt(6.0 / (double)(din + dout));
    for (int64_t c = 0; c < din; ++c)
        for (int64_t k = 0; k < dout; ++k) {
            double u = (double)u24(seed, (uint64_t)(c * dout + k)) * (1.0 / 16777216.0);
            W[c * dout + k] = (float)(a * (2.0 * u - 1.0));
        }
}

/* ---------------------------------------------------------------- R-MAT */
#define RMAT_T1 2448131358u  /* floor(0.57 * 2^32) */
#define RMAT_T2 3264175144u  /* floor(0.76 * 2^32) */
#define RMAT_T3 4080218931u  /* floor(0.95 * 2^32) */

static int levels_for(int64_t n) {
    int s = 0;
    while (((int64_t)1 << s) < n) ++s;
    return s;
}

/* Candidate k -> (u, v).  Returns 1 if accepted. */
static inline int rmat_candidate(uint64_t seed, uint64_t k, int s, int64_t n, int32_t* pu, int32_t* pv) {
    uint64_t u = 0, v = 0;
    uint32_t w[4];
    for (int l = 0; l < s; ++l) {
        if ((l & 3) == 0) philox10(seed, (uint32_t)k, (uint32_t)(k >> 32), (uint32_t)(l >> 2), 0, w);
        uint32_t r = w[l & 3];
        uint64_t bu, bv;
        if (r < RMAT_T1)      { bu = 0; bv = 0; }
        else if (r < RMAT_T2) { bu = 0; bv = 1; }
        else if (r < RMAT_T3) { bu = 1; bv = 0; }
        else                  { bu = 1; bv = 1; }
        u = (u << 1) | bu;
        v = (v << 1) | bv;
    }
    if ((int64_t)u >= n || (int64_t)v >= n || u == v) return 0;
    *pu = (int32_t)u; *pv = (int32_t)v;
    return 1;
}

/* Generate the accepted pair stream: first `npairs` accepted (u,v) in k order.
 * Returns the number of candidates consumed, or -1 on allocation failure. */
int64_t gen_rmat_pairs(int64_t n, int64_t npairs, uint64_t seed, int32_t* U, int32_t* V) {
    int s = levels_for(n);
    int64_t have = 0;
    uint64_t k0 = 0;
    int nthr = 1;
#ifdef _OPENMP
    nthr = omp_get_max_threads();
#endif
    const int64_t chunk = 1 << 18;
    int32_t* bu = (int32_t*)malloc(sizeof(int32_t) * (size_t)chunk * nthr);
    int32_t* bv = (int32_t*)malloc(sizeof(int32_t) * (size_t)chunk * nthr);
    int64_t* cnt = (int64_t*)calloc((size_t)nthr, sizeof(int64_t));
    if (!bu || !bv || !cnt) { free(bu); free(bv); free(cnt); return -1; }
    while (have < npairs) {
#pragma omp parallel num_threads(nthr)
        {
            int t = 0;
#ifdef _OPENMP
            t = omp_get_thread_num();
#endif
            uint64_t kb = k0 + (uint64_t)t * (uint64_t)chunk;
            int64_t c = 0;
            for (int64_t q = 0; q < chunk; ++q) {
                int32_t u, v;
                if (rmat_candidate(seed, kb + (uint64_t)q, s, n, &u, &v)) {
                    bu[(size_t)t * chunk + c] = u; bv[(size_t)t * chunk + c] = v; ++c;
                }
            }
            cnt[t] = c;
        }
        for (int t = 0; t < nthr && have < npairs; ++t) {
            int64_t take = cnt[t];
            if (take > npairs - have) take = npairs - have;
            memcpy(U + have, bu + (size_t)t * chunk, sizeof(int32_t) * (size_t)take);
            memcpy(V + have, bv + (size_t)t * chunk, sizeof(int32_t) * (size_t)take);
            if (have + take == npairs) {
                /* consumed candidates: up to and including the last taken one */
                int64_t acc = 0; uint64_t kb = k0 + (uint64_t)t * (uint64_t)chunk;
                int32_t u, v;
                for (int64_t q = 0; q < chunk; ++q)
                    if (rmat_candidate(seed, kb + (uint64_t)q, s, n, &u, &v) && ++acc == take) { k0 = kb + (uint64_t)q + 1; break; }
                have += take;
                free(bu); free(bv); free(cnt);
                return (int64_t)k0;
            }
            have += take;
        }
        k0 += (uint64_t)chunk * (uint64_t)nthr;
    }
    free(bu); free(bv); free(cnt);
    return (int64_t)k0;
}

/* Symmetric R-MAT CSR with m (even) entries: rowptr[n+1], col[m], sorted by
 * (row, col); duplicates kept.  Returns candidates consumed or -1. */
int64_t gen_rmat_csr(int64_t n, int64_t m, uint64_t seed, int64_t* rowptr, int32_t* col) {
    if (n < 2 || m < 0 || (m & 1)) return -1;
    int64_t np = m / 2;
    int32_t* U = (int32_t*)malloc(sizeof(int32_t) * (size_t)(np ? np : 1));
    int32_t* V = (int32_t*)malloc(sizeof(int32_t) * (size_t)(np ? np : 1));
    int32_t* tmp_r = (int32_t*)malloc(sizeof(int32_t) * (size_t)(m ? m : 1));
    int32_t* tmp_c = (int32_t*)malloc(sizeof(int32_t) * (size_t)(m ? m : 1));
    int64_t* cnt = (int64_t*)calloc((size_t)n + 1, sizeof(int64_t));
    if (!U || !V || !tmp_r || !tmp_c || !cnt) { free(U); free(V); free(tmp_r); free(tmp_c); free(cnt); return -1; }
    int64_t used = gen_rmat_pairs(n, np, seed, U, V);
    if (used < 0) { free(U); free(V); free(tmp_r); free(tmp_c); free(cnt); return -1; }
    /* pass 1: counting sort of all 2*np entries by column (stable) */
    for (int64_t e = 0; e < np; ++e) { cnt[V[e] + 1]++; cnt[U[e] + 1]++; }
    for (int64_t i = 0; i < n; ++i) cnt[i + 1] += cnt[i];
    for (int64_t e = 0; e < np; ++e) {
        int64_t p = cnt[V[e]]++; tmp_r[p] = U[e]; tmp_c[p] = V[e];
        int64_t q = cnt[U[e]]++; tmp_r[q] = V[e]; tmp_c[q] = U[e];
    }
    free(U); free(V);
    /* pass 2: counting sort by row (stable) -> sorted by (row, col) */
    memset(rowptr, 0, sizeof(int64_t) * (size_t)(n + 1));
    for (int64_t e = 0; e < m; ++e) rowptr[tmp_r[e] + 1]++;
    for (int64_t i = 0; i < n; ++i) rowptr[i + 1] += rowptr[i];
    memcpy(cnt, rowptr, sizeof(int64_t) * (size_t)(n + 1));
    for (int64_t e = 0; e < m; ++e) col[cnt[tmp_r[e]]++] = tmp_c[e];
    free(tmp_r); free(tmp_c); free(cnt);
    return used;
}
