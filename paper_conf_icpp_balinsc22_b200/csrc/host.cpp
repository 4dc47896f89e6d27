// host.cpp — ingest (mggcn_load_csr), permutation and 1D partitioner
// (mggcn_partition) of the B200 MG-GCN library.  Pure host C++.
//
// Paper: /root/reference/PAPER.md (P:line).  Eq. 2 normalisation P:312-318;
// random permutation §5.2; partition vector Eq. 13 P:646-648;
// tiles Eq. 14-15; 1D row distribution with broadcast P:705-720.
#include <cmath>
#include <cstring>
#include <mutex>
#include <new>

#include "internal.h"

namespace mggcn {
static thread_local std::string g_last_error;
void set_error(const std::string& msg) { g_last_error = msg; }
}  // namespace mggcn

using mggcn::set_error;

extern "C" const char* mggcn_last_error(void) { return mggcn::g_last_error.c_str(); }
extern "C" int mggcn_version(void) { return 100; /* 0.1.0 */ }

#define FAIL(code, msg)        \
    do {                       \
        set_error(msg);        \
        return (code);         \
    } while (0)

// ------------------------------------------------------------------ ingest
extern "C" int mggcn_load_csr(int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                              const float* vals, mggcn_graph* out) {
    if (!out) FAIL(MGGCN_EINVAL, "load_csr: out is NULL");
    *out = nullptr;
    if (n <= 0 || n >= ((int64_t)1 << 31)) FAIL(MGGCN_EINVAL, "load_csr: n must be in [1, 2^31)");
    if (nnz < 0 || !rowptr || (nnz > 0 && !colidx)) FAIL(MGGCN_EINVAL, "load_csr: bad nnz / NULL arrays");
    if (rowptr[0] != 0) FAIL(MGGCN_EINVAL, "load_csr: rowptr[0] != 0");
    for (int64_t u = 0; u < n; ++u)
        if (rowptr[u + 1] < rowptr[u]) FAIL(MGGCN_EINVAL, "load_csr: rowptr not non-decreasing");
    if (rowptr[n] != nnz) FAIL(MGGCN_EINVAL, "load_csr: rowptr[n] != nnz");
    for (int64_t e = 0; e < nnz; ++e)
        if (colidx[e] < 0 || colidx[e] >= n) FAIL(MGGCN_EINVAL, "load_csr: colidx out of range");
    if (vals)
        for (int64_t e = 0; e < nnz; ++e)
            if (!std::isfinite(vals[e]) || !(vals[e] > 0.0f)) FAIL(MGGCN_EINVAL, "load_csr: vals must be finite and > 0");
    mggcn_graph_s* g = new (std::nothrow) mggcn_graph_s();
    if (!g) FAIL(MGGCN_ENOMEM, "load_csr: out of memory");
    try {
        g->n = n;
        g->nnz = nnz;
        g->rowptr.assign(rowptr, rowptr + n + 1);
        g->col.assign(colidx, colidx + nnz);
        if (vals) g->val.assign(vals, vals + nnz);
        // Eq. 2 denominator: weighted in-degree, fp64 sum in CSR order (reading C18)
        std::vector<double> d(n, 0.0);
        for (int64_t e = 0; e < nnz; ++e) d[colidx[e]] += vals ? (double)vals[e] : 1.0;
        g->deg.resize(n);
        for (int64_t v = 0; v < n; ++v) g->deg[v] = (float)d[v];
        // multiset pattern symmetry: sort entries by (row, col) and by (col, row), compare
        if (!vals) {
            std::vector<int64_t> cnt(n + 1, 0);
            std::vector<int32_t> byc_row(nnz), srt_col(nnz);  // LSD: by col, then by row
            for (int64_t e = 0; e < nnz; ++e) cnt[colidx[e] + 1]++;
            for (int64_t i = 0; i < n; ++i) cnt[i + 1] += cnt[i];
            std::vector<int32_t> byc_col(nnz);
            for (int64_t u = 0; u < n; ++u)
                for (int64_t e = rowptr[u]; e < rowptr[u + 1]; ++e) {
                    int64_t q = cnt[colidx[e]]++;
                    byc_row[q] = (int32_t)u;
                    byc_col[q] = colidx[e];
                }
            // byc_* are sorted by (col, row): that is A^T in (row', col') order.
            // A sorted by (row, col): stable counting sort of byc_* by row.
            std::vector<int64_t> rs(rowptr, rowptr + n + 1);
            for (int64_t q = 0; q < nnz; ++q) srt_col[rs[byc_row[q]]++] = byc_col[q];
            // compare: A (rows via rowptr, cols srt_col) vs A^T (rows = byc_col, cols = byc_row)
            bool sym = true;
            int64_t q = 0;
            for (int64_t u = 0; u < n && sym; ++u) {
                for (int64_t e = rowptr[u]; e < rowptr[u + 1]; ++e, ++q) {
                    if (byc_col[q] != u || byc_row[q] != srt_col[e]) { sym = false; break; }
                }
            }
            g->symmetric = sym && q == nnz;
        }
    } catch (const std::bad_alloc&) {
        delete g;
        FAIL(MGGCN_ENOMEM, "load_csr: out of memory");
    }
    *out = g;
    return MGGCN_OK;
}

extern "C" int mggcn_graph_info(mggcn_graph g, int64_t* n, int64_t* nnz, int32_t* symmetric, int32_t* unit,
                                float* deg) {
    if (!g) FAIL(MGGCN_EINVAL, "graph_info: NULL graph");
    if (n) *n = g->n;
    if (nnz) *nnz = g->nnz;
    if (symmetric) *symmetric = g->symmetric ? 1 : 0;
    if (unit) *unit = g->val.empty() ? 1 : 0;
    if (deg) std::memcpy(deg, g->deg.data(), sizeof(float) * (size_t)g->n);
    return MGGCN_OK;
}

extern "C" void mggcn_graph_free(mggcn_graph g) { delete g; }

// ------------------------------------------------------------ permutation
// §5.2: random vertex permutation for nnz balance; the paper
// does not name its RNG, reading C15: splitmix64 Fisher-Yates, perm[old]=new.
static void random_permutation(int64_t n, uint64_t seed, std::vector<int64_t>& perm) {
    perm.resize(n);
    for (int64_t i = 0; i < n; ++i) perm[i] = i;
    if (seed == 0) return;
    uint64_t s = seed;
    for (int64_t k = n - 1; k >= 1; --k) {
        s += 0x9E3779B97F4A7C15ull;
        uint64_t z = s;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        z ^= z >> 31;
        uint64_t j = (uint64_t)(((unsigned __int128)z * (unsigned __int128)(uint64_t)(k + 1)) >> 64);
        std::swap(perm[k], perm[j]);
    }
}

// ------------------------------------------------------------- partition
// Row block [lo, hi) of Â'^T (fwd) or Â' (bwd), sorted by (row, col, original
// position) with two stable counting sorts, then cut into P column tiles.
static int build_tiles(const mggcn_graph_s& g, mggcn_part_s& pt, bool fwd, std::vector<HostTile>& tiles) {
    const int64_t n = g.n, lo = pt.p[pt.rank], hi = pt.p[pt.rank + 1], nr = hi - lo;
    const bool keep_pos = !pt.pattern;
    const std::vector<int64_t>& perm = pt.perm;
    // pass 0: histogram of the sort key "col" (new id) over entries landing in the block
    std::vector<int64_t> cstart(n + 1, 0);
    int64_t total = 0;
    for (int64_t u = 0; u < n; ++u) {
        const int64_t pu = perm[u];
        for (int64_t e = g.rowptr[u]; e < g.rowptr[u + 1]; ++e) {
            const int64_t pv = perm[g.col[e]];
            const int64_t row = fwd ? pv : pu, c = fwd ? pu : pv;
            if (row >= lo && row < hi) { cstart[c + 1]++; ++total; }
        }
    }
    for (int64_t i = 0; i < n; ++i) cstart[i + 1] += cstart[i];
    std::vector<int32_t> t_row(total), t_col(total);
    std::vector<int64_t> t_pos(keep_pos ? total : 0);
    // pass 1: stable scatter by col, iterating entries in original CSR position order
    for (int64_t u = 0; u < n; ++u) {
        const int64_t pu = perm[u];
        for (int64_t e = g.rowptr[u]; e < g.rowptr[u + 1]; ++e) {
            const int64_t pv = perm[g.col[e]];
            const int64_t row = fwd ? pv : pu, c = fwd ? pu : pv;
            if (row >= lo && row < hi) {
                int64_t q = cstart[c]++;
                t_row[q] = (int32_t)(row - lo);
                t_col[q] = (int32_t)c;
                if (keep_pos) t_pos[q] = e;
            }
        }
    }
    // pass 2: stable scatter by row -> sorted by (row, col, position)
    std::vector<int64_t> rs(nr + 1, 0);
    for (int64_t q = 0; q < total; ++q) rs[t_row[q] + 1]++;
    for (int64_t r = 0; r < nr; ++r) rs[r + 1] += rs[r];
    std::vector<int64_t> rfill(rs.begin(), rs.end() - 1);
    std::vector<int32_t> s_col(total);
    std::vector<int64_t> s_pos(keep_pos ? total : 0);
    for (int64_t q = 0; q < total; ++q) {
        int64_t d = rfill[t_row[q]]++;
        s_col[d] = t_col[q];
        if (keep_pos) s_pos[d] = t_pos[q];
    }
    std::vector<int32_t>().swap(t_row);
    std::vector<int32_t>().swap(t_col);
    std::vector<int64_t>().swap(t_pos);
    // cut each row into P column tiles (cols ascending => contiguous per tile)
    const int P = pt.P;
    tiles.assign(P, HostTile());
    std::vector<int64_t> tnnz(P, 0);
    for (int j = 0; j < P; ++j) {
        tiles[j].nrows = nr;
        tiles[j].col0 = pt.p[j];
        tiles[j].ncols = pt.p[j + 1] - pt.p[j];
        tiles[j].rowptr.assign(nr + 1, 0);
    }
    for (int64_t r = 0; r < nr; ++r) {
        int j = 0;
        for (int64_t q = rs[r]; q < rs[r + 1]; ++q) {
            while (s_col[q] >= pt.p[j + 1]) ++j;
            tiles[j].rowptr[r + 1]++;
        }
    }
    for (int j = 0; j < P; ++j) {
        auto& rp = tiles[j].rowptr;
        int64_t acc = 0;
        for (int64_t r = 0; r < nr; ++r) {
            acc += rp[r + 1];
            if (acc >= ((int64_t)1 << 31)) {
                set_error("partition: a tile has >= 2^31 entries (use more parts)");
                return MGGCN_EUNSUPPORTED;
            }
            rp[r + 1] = (int32_t)acc;
        }
        tnnz[j] = acc;
        tiles[j].col.resize(acc);
        if (!pt.pattern) tiles[j].val.resize(acc);
    }
    std::vector<int64_t> fill(P);
    for (int64_t r = 0; r < nr; ++r) {
        for (int j = 0; j < P; ++j) fill[j] = tiles[j].rowptr[r];
        int j = 0;
        for (int64_t q = rs[r]; q < rs[r + 1]; ++q) {
            while (s_col[q] >= pt.p[j + 1]) ++j;
            int64_t d = fill[j]++;
            tiles[j].col[d] = (int32_t)(s_col[q] - pt.p[j]);
            if (!pt.pattern) {
                // Â_uv = fp32(A_uv) / deg_f(v): v is the ORIGINAL destination of entry e
                const int64_t e = s_pos[q];
                tiles[j].val[d] = g.val[e] / g.deg[g.col[e]];
            }
        }
    }
    return MGGCN_OK;
}

extern "C" int mggcn_partition(mggcn_graph g, int32_t nparts, int32_t rank, uint64_t perm_seed, mggcn_part* out) {
    if (!out) FAIL(MGGCN_EINVAL, "partition: out is NULL");
    *out = nullptr;
    if (!g) FAIL(MGGCN_EINVAL, "partition: NULL graph");
    if (nparts < 1 || nparts > 64) FAIL(MGGCN_EINVAL, "partition: nparts must be in [1, 64]");
    if (rank < 0 || rank >= nparts) FAIL(MGGCN_EINVAL, "partition: rank out of range");
    if (g->n < nparts) FAIL(MGGCN_EINVAL, "partition: n < nparts");
    mggcn_part_s* pt = new (std::nothrow) mggcn_part_s();
    if (!pt) FAIL(MGGCN_ENOMEM, "partition: out of memory");
    try {
        pt->P = nparts;
        pt->rank = rank;
        pt->n = g->n;
        pt->pattern = g->val.empty();
        pt->shared_fb = pt->pattern && g->symmetric;
        // Eq. 13, uniform (reading C14): p(i) = floor(i n / P)
        pt->p.resize(nparts + 1);
        for (int i = 0; i <= nparts; ++i) pt->p[i] = (int64_t)(((__int128)i * g->n) / nparts);
        random_permutation(g->n, perm_seed, pt->perm);
        pt->deg_new.resize(g->n);
        for (int64_t v = 0; v < g->n; ++v) pt->deg_new[pt->perm[v]] = g->deg[v];
        int rc = build_tiles(*g, *pt, true, pt->F);
        if (rc == MGGCN_OK && !pt->shared_fb) rc = build_tiles(*g, *pt, false, pt->B);
        if (rc != MGGCN_OK) {
            delete pt;
            return rc;
        }
        const int64_t lo = pt->p[rank], nr = pt->p[rank + 1] - lo;
        pt->inv_deg.resize(nr);
        for (int64_t r = 0; r < nr; ++r) {
            const float d = pt->deg_new[lo + r];
            pt->inv_deg[r] = d != 0.0f ? 1.0f / d : 0.0f;   // reading C20
        }
    } catch (const std::bad_alloc&) {
        delete pt;
        FAIL(MGGCN_ENOMEM, "partition: out of memory");
    }
    *out = pt;
    return MGGCN_OK;
}

extern "C" int mggcn_part_info(mggcn_part pt, int32_t* nparts, int32_t* rank, int64_t* n, int64_t* p, int64_t* perm,
                               int64_t* tile_nnz) {
    if (!pt) FAIL(MGGCN_EINVAL, "part_info: NULL part");
    if (nparts) *nparts = pt->P;
    if (rank) *rank = pt->rank;
    if (n) *n = pt->n;
    if (p) std::memcpy(p, pt->p.data(), sizeof(int64_t) * (size_t)(pt->P + 1));
    if (perm) std::memcpy(perm, pt->perm.data(), sizeof(int64_t) * (size_t)pt->n);
    if (tile_nnz)
        for (int j = 0; j < pt->P; ++j) {
            tile_nnz[j] = pt->F[j].rowptr.back();
            tile_nnz[pt->P + j] = pt->tileB(j).rowptr.back();
        }
    return MGGCN_OK;
}

extern "C" int mggcn_part_export_tile(mggcn_part pt, int32_t dir, int32_t j, int32_t* rowptr, int32_t* colidx,
                                      float* vals) {
    if (!pt) FAIL(MGGCN_EINVAL, "export_tile: NULL part");
    if ((dir != 0 && dir != 1) || j < 0 || j >= pt->P) FAIL(MGGCN_EINVAL, "export_tile: bad dir / j");
    const HostTile& t = dir == 0 ? pt->F[j] : pt->tileB(j);
    const int64_t nnz = t.rowptr.back();
    if (rowptr) std::memcpy(rowptr, t.rowptr.data(), sizeof(int32_t) * (size_t)(t.nrows + 1));
    if (colidx) std::memcpy(colidx, t.col.data(), sizeof(int32_t) * (size_t)nnz);
    if (vals) {
        if (!pt->pattern) {
            std::memcpy(vals, t.val.data(), sizeof(float) * (size_t)nnz);
        } else {
            // implied value Â'_uv = 1 / deg_f(v); v = the row (fwd) or the column (bwd)
            const int64_t lo = pt->p[pt->rank];
            for (int64_t r = 0; r < t.nrows; ++r)
                for (int64_t q = t.rowptr[r]; q < t.rowptr[r + 1]; ++q) {
                    const int64_t v = dir == 0 ? lo + r : t.col0 + t.col[q];
                    vals[q] = 1.0f / pt->deg_new[v];
                }
        }
    }
    return MGGCN_OK;
}

extern "C" int mggcn_part_inv_deg(mggcn_part pt, float* inv_deg) {
    if (!pt || !inv_deg) FAIL(MGGCN_EINVAL, "part_inv_deg: NULL argument");
    std::memcpy(inv_deg, pt->inv_deg.data(), sizeof(float) * pt->inv_deg.size());
    return MGGCN_OK;
}

extern "C" void mggcn_part_free(mggcn_part pt) { delete pt; }
