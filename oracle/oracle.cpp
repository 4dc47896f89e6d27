// oracle/oracle.cpp — TEST INFRASTRUCTURE ONLY.
//
// Plain, slow, single-threaded CPU reference of MG-GCN's full-batch GCN
// epoch (Balın, Sancak, Çatalyürek, ICPP '22; /root/reference/PAPER.md, cited
// as P:line).  Only tests/, __graft_entry__.smoke() and bench.py's
// cpu_baseline / --impl reference legs may load this library.  It shares no
// code with the CUDA path (paper_conf_icpp_balinsc22_b200/).
//
// Numeric core: every dot product / aggregation accumulates in fp64 in
// ascending index order and rounds once to the storage type T (float for the
// parity reference, double for the fp64 self-tests).  No blocking, fusion or
// reordering.  Built with -O2 -ffp-contract=off, no OpenMP, no BLAS.
//
// Parity pins for every function are listed in oracle/__init__.py and
// DESIGN.md §4 (tests/test_oracle_*.py).
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <vector>

namespace {

// SpMM over one CSR (Eq. 6 and Eq. 9):
//   out[r][k] = sum_{e in row r, ascending position} val[e] * B[col[e]][k]
// Forward uses the CSR of Â'^T (rows = destination v, entries = in-neighbours
// u); backward uses the CSR of Â' (rows = u, entries = out-neighbours v).
template <typename T>
void spmm(int64_t nrows, const int64_t* rowptr, const int64_t* col, const T* val,
          const T* B, int64_t ldb, int64_t width, T* out, int64_t ldo) {
    double* acc = new double[width > 0 ? width : 1];
    for (int64_t r = 0; r < nrows; ++r) {
        for (int64_t k = 0; k < width; ++k) acc[k] = 0.0;
        for (int64_t e = rowptr[r]; e < rowptr[r + 1]; ++e) {
            const double a = (double)val[e];
            const T* b = B + col[e] * ldb;
            for (int64_t k = 0; k < width; ++k) acc[k] += a * (double)b[k];
        }
        for (int64_t k = 0; k < width; ++k) out[r * ldo + k] = (T)acc[k];
    }
    delete[] acc;
}

// P-way simulation of the staged SpMM (Fig. 2-3): for the rows of
// one row block, stages j = 0..P-1 ascending, each tile's entries in
// ascending local column; the fp64 accumulator of every output element
// persists across stages, so the result is bit-identical to spmm() over the
// unpartitioned CSR (SURVEY.md §8(c) "P-way simulation mode").
template <typename T>
void spmm_tiles(int64_t nrows, int32_t P, const int64_t* const* rowptr, const int64_t* const* col,
                const T* const* val, const T* const* B, int64_t ldb, int64_t width, T* out, int64_t ldo) {
    double* acc = new double[width > 0 ? width : 1];
    for (int64_t r = 0; r < nrows; ++r) {
        for (int64_t k = 0; k < width; ++k) acc[k] = 0.0;
        for (int32_t j = 0; j < P; ++j)
            for (int64_t e = rowptr[j][r]; e < rowptr[j][r + 1]; ++e) {
                const double a = (double)val[j][e];
                const T* b = B[j] + col[j][e] * ldb;
                for (int64_t k = 0; k < width; ++k) acc[k] += a * (double)b[k];
            }
        for (int64_t k = 0; k < width; ++k) out[r * ldo + k] = (T)acc[k];
    }
    delete[] acc;
}

// Dense product (Eq. 5, Eq. 10-11):
//   C[m][n] = sum_{k ascending} opA[m][k] * opB[k][n]
// opA = A (M x K, lda) or A^T (A stored K x M); opB = B (K x N) or B^T (B stored N x K).
template <typename T>
void gemm(int64_t M, int64_t N, int64_t K, const T* A, int64_t lda, int transA,
          const T* B, int64_t ldb, int transB, T* C, int64_t ldc) {
    for (int64_t m = 0; m < M; ++m)
        for (int64_t n = 0; n < N; ++n) {
            double acc = 0.0;
            for (int64_t k = 0; k < K; ++k) {
                const double a = transA ? (double)A[k * lda + m] : (double)A[m * lda + k];
                const double b = transB ? (double)B[n * ldb + k] : (double)B[k * ldb + n];
                acc += a * b;
            }
            C[m * ldc + n] = (T)acc;
        }
}

// Softmax cross-entropy ("softmax cross-entropy loss [9]";
// readings C5): for labelled v (y >= 0):
//   lse_v = max_c z + log sum_c exp(z_c - max), loss_v = lse_v - z_{y_v}
//   G_v,c = (exp(z_c - lse_v) - [c == y_v]) / ntrain ;  G_v = 0 if unlabelled.
// *loss_sum = sum_v loss_v in ascending v (fp64); the mean is loss_sum/ntrain.
template <typename T>
void softmax_ce(int64_t n, int64_t C, const T* Z, int64_t ldz, const int32_t* y, int64_t ntrain,
                T* G, int64_t ldg, double* loss_sum) {
    double total = 0.0;
    for (int64_t v = 0; v < n; ++v) {
        const T* z = Z + v * ldz;
        T* g = G + v * ldg;
        if (y[v] < 0) {
            for (int64_t c = 0; c < C; ++c) g[c] = (T)0;
            continue;
        }
        double mx = (double)z[0];
        for (int64_t c = 1; c < C; ++c) if ((double)z[c] > mx) mx = (double)z[c];
        double s = 0.0;
        for (int64_t c = 0; c < C; ++c) s += std::exp((double)z[c] - mx);
        const double lse = mx + std::log(s);
        total += lse - (double)z[y[v]];
        for (int64_t c = 0; c < C; ++c) {
            double p = std::exp((double)z[c] - lse);
            if (c == y[v]) p -= 1.0;
            g[c] = (T)(p / (double)ntrain);
        }
    }
    *loss_sum = total;
}

// Adam ("We have implemented and used the Adam optimizer [23]";
// Kingma & Ba, Algorithm 1, reading C6: bias correction, eps outside sqrt).
//   m <- b1 m + (1-b1) g ; v <- b2 v + (1-b2) g^2
//   W <- W - lr * (m / (1-b1^t)) / (sqrt(v / (1-b2^t)) + eps)
template <typename T>
void adam(int64_t count, T* W, const T* g, T* m, T* v, int64_t t, double lr, double b1, double b2, double eps) {
    const double c1 = 1.0 - std::pow(b1, (double)t);
    const double c2 = 1.0 - std::pow(b2, (double)t);
    for (int64_t i = 0; i < count; ++i) {
        const double gi = (double)g[i];
        const double mi = b1 * (double)m[i] + (1.0 - b1) * gi;
        const double vi = b2 * (double)v[i] + (1.0 - b2) * gi * gi;
        m[i] = (T)mi;
        v[i] = (T)vi;
        W[i] = (T)((double)W[i] - lr * (mi / c1) / (std::sqrt(vi / c2) + eps));
    }
}

}  // namespace

extern "C" {

// Random vertex permutation (§5.2; RNG unspecified in the paper,
// reading C15): splitmix64 with state = seed; Fisher-Yates from k = n-1 down
// to 1 with j = floor(r * (k+1) / 2^64); perm[old] = new.  seed 0 = identity.
void orc_permutation(int64_t n, uint64_t seed, int64_t* perm) {
    for (int64_t i = 0; i < n; ++i) perm[i] = i;
    if (seed == 0) return;
    uint64_t state = seed;
    for (int64_t k = n - 1; k >= 1; --k) {
        state += 0x9E3779B97F4A7C15ull;
        uint64_t z = state;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        z = z ^ (z >> 31);
        const uint64_t j = (uint64_t)(((unsigned __int128)z * (unsigned __int128)(uint64_t)(k + 1)) >> 64);
        const int64_t tmp = perm[k];
        perm[k] = perm[j];
        perm[j] = tmp;
    }
}

// CSR from triplets (O4's ordering): entries sorted by (row, col) with ties
// kept in input order.  Plain bucket sort: count per row, scatter in input
// order (stable), then a stable sort of each row by column.  order[k] = input
// index of the k-th output entry; rowptr int64[n+1].
void orc_csr_order(int64_t n, int64_t nnz, const int64_t* rows, const int64_t* cols, int64_t* rowptr,
                   int64_t* order) {
    std::vector<int64_t> next(n + 1, 0);
    for (int64_t e = 0; e < nnz; ++e) next[rows[e] + 1] += 1;
    for (int64_t r = 0; r < n; ++r) next[r + 1] += next[r];
    for (int64_t r = 0; r <= n; ++r) rowptr[r] = next[r];
    for (int64_t e = 0; e < nnz; ++e) order[next[rows[e]]++] = e;
    std::vector<std::pair<int64_t, int64_t>> row;   // (col, input index): ties by input index = stable
    for (int64_t r = 0; r < n; ++r) {
        row.clear();
        for (int64_t k = rowptr[r]; k < rowptr[r + 1]; ++k) row.emplace_back(cols[order[k]], order[k]);
        std::sort(row.begin(), row.end());
        for (int64_t k = rowptr[r]; k < rowptr[r + 1]; ++k) order[k] = row[k - rowptr[r]].second;
    }
}

uint64_t orc_splitmix64_next(uint64_t* state) {
    *state += 0x9E3779B97F4A7C15ull;
    uint64_t z = *state;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

#define ORC_INSTANTIATE(SUF, T)                                                                          \
    void orc_spmm_##SUF(int64_t nrows, const int64_t* rowptr, const int64_t* col, const T* val,          \
                        const T* B, int64_t ldb, int64_t width, T* out, int64_t ldo) {                   \
        spmm<T>(nrows, rowptr, col, val, B, ldb, width, out, ldo);                                      \
    }                                                                                                    \
    void orc_spmm_tiles_##SUF(int64_t nrows, int32_t P, const int64_t* const* rowptr,                    \
                              const int64_t* const* col, const T* const* val, const T* const* B,         \
                              int64_t ldb, int64_t width, T* out, int64_t ldo) {                         \
        spmm_tiles<T>(nrows, P, rowptr, col, val, B, ldb, width, out, ldo);                             \
    }                                                                                                    \
    void orc_gemm_##SUF(int64_t M, int64_t N, int64_t K, const T* A, int64_t lda, int transA,           \
                        const T* B, int64_t ldb, int transB, T* C, int64_t ldc) {                        \
        gemm<T>(M, N, K, A, lda, transA, B, ldb, transB, C, ldc);                                       \
    }                                                                                                    \
    void orc_softmax_ce_##SUF(int64_t n, int64_t C, const T* Z, int64_t ldz, const int32_t* y,           \
                              int64_t ntrain, T* G, int64_t ldg, double* loss_sum) {                     \
        softmax_ce<T>(n, C, Z, ldz, y, ntrain, G, ldg, loss_sum);                                       \
    }                                                                                                    \
    void orc_adam_##SUF(int64_t count, T* W, const T* g, T* m, T* v, int64_t t, double lr, double b1,    \
                        double b2, double eps) {                                                         \
        adam<T>(count, W, g, m, v, t, lr, b1, b2, eps);                                                 \
    }

ORC_INSTANTIATE(f32, float)
ORC_INSTANTIATE(f64, double)

}  // extern "C"
