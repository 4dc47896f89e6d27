// dense_plan.cpp — host-side choice of the dense blocks of a stage tile (see
// dense.cu).  The stage product C_i (+)= A_ij · H_j is a sum over
// the tile's entries; this splits the entries into dense 128 x 32 blocks (run
// on the tensor cores) and a residual CSR (run by the gather kernel).  Every
// entry lands in exactly one of the two, so the product is unchanged up to
// the order of the fp32 additions.
//
//   1. columns ranked by entry count (descending, ties by id); chunks of 32
//      consecutive ranks; only the leading chunks whose total count could fill
//      one dense block are candidates;
//   2. rows ranked by their entry count in candidate columns (descending, ties
//      by id); groups of 128 consecutive ranks;
//   3. block (group, chunk) is dense when it holds >= thr * 128 * 32 entries
//      whose value is exact in bf16 (pattern-only graphs: multiplicities <= 256);
//   4. dense entries are written, as bf16, into the block's A image in the
//      K-major SWIZZLE_64B layout the MMA reads (64-B rows, 16-B chunk j of
//      row i stored at chunk j ^ ((i >> 1) & 3)); the rest form `resid`.
#include <algorithm>
#include <array>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <numeric>

#include "internal.h"

namespace {
constexpr int TM = 128, TK = 32;
constexpr int64_t kSMs = 148;   // B200 SMs (work-item segment length only)

inline bool bf16_exact(float v) {
    uint32_t b;
    std::memcpy(&b, &v, 4);
    return v != 0.f && (b & 0xFFFFu) == 0 && std::isfinite(v);
}
}  // namespace

// (global scope, like HostTile and DenseHost in internal.h)
void plan_dense(const HostTile& t, double thr, double min_frac, int64_t min_rows, int64_t min_entries,
                DenseHost& d) {
    d = DenseHost();
    const int64_t nr = t.nrows, nc = t.ncols;
    if (thr <= 0 || nr == 0 || nc == 0 || t.rowptr.empty() || t.rowptr[nr] == 0) return;
    // ... and only for tiles of >= min_entries entries (and min_rows rows): a dense launch
    // costs a fixed ~15 us (B images, the persistent kernel's ramp, the fix-up), and the gathers
    // it replaces are cheap when the gathered block sits in L2.  At P = 8 the Reddit-shaped
    // 1.2 M-entry local tile loses with blocks (+0.045 ms per wide SpMM) while its 6 M-entry
    // 5-block stage group gains (-0.075 ms); SOLO rank 0 with >= 3 M entries: Reddit-shaped
    // P = 8 3.70 -> 3.45 ms, P = 4 unchanged (5.58 ms, every tile >= 4.9 M), Proteins-shaped
    // P = 8 1.46 -> 1.45 ms, while all tiles with blocks lose at P = 8 (Proteins 1.70 ms)
    // (profiles/r02_dense_solo_ab.jsonl)
    if (nr < min_rows || (int64_t)t.rowptr[nr] < min_entries) return;
    const int64_t min_cnt = std::max<int64_t>(1, (int64_t)std::ceil(thr * TM * TK));
    const bool pat = t.val.empty();
    auto ok = [&](int64_t e) { return pat || bf16_exact(t.val[e]); };

    // 1. column ranks
    std::vector<int32_t> colcnt(nc, 0);
    for (int64_t e = 0; e < t.rowptr[nr]; ++e)
        if (ok(e)) ++colcnt[t.col[e]];
    std::vector<int32_t> cols;
    for (int64_t c = 0; c < nc; ++c)
        if (colcnt[c] > 0) cols.push_back((int32_t)c);
    std::sort(cols.begin(), cols.end(), [&](int32_t a, int32_t b) {
        return colcnt[a] != colcnt[b] ? colcnt[a] > colcnt[b] : a < b;
    });
    int64_t ncand = 0;
    for (int64_t q = 0; q * TK < (int64_t)cols.size(); ++q) {
        int64_t s = 0;
        for (int64_t i = q * TK; i < std::min<int64_t>((q + 1) * TK, cols.size()); ++i) s += colcnt[cols[i]];
        if (s < min_cnt) break;
        ++ncand;
    }
    if (ncand == 0) return;
    const int64_t ngr_max = (nr + TM - 1) / TM;
    ncand = std::min<int64_t>(ncand, std::max<int64_t>(1, ((int64_t)1 << 28) / ngr_max));   // counter array cap
    std::vector<int32_t> crank(nc, -1);
    for (int64_t i = 0; i < std::min<int64_t>(ncand * TK, cols.size()); ++i) crank[cols[i]] = (int32_t)i;

    // 2. row ranks
    std::vector<int32_t> rowcnt(nr, 0);
    for (int64_t r = 0; r < nr; ++r)
        for (int64_t e = t.rowptr[r]; e < t.rowptr[r + 1]; ++e)
            if (crank[t.col[e]] >= 0 && ok(e)) ++rowcnt[r];
    std::vector<int32_t> rows;
    for (int64_t r = 0; r < nr; ++r)
        if (rowcnt[r] > 0) rows.push_back((int32_t)r);
    std::sort(rows.begin(), rows.end(), [&](int32_t a, int32_t b) {
        return rowcnt[a] != rowcnt[b] ? rowcnt[a] > rowcnt[b] : a < b;
    });
    const int64_t ngr = ((int64_t)rows.size() + TM - 1) / TM;
    std::vector<int32_t> rpos(nr, -1);
    for (size_t i = 0; i < rows.size(); ++i) rpos[rows[i]] = (int32_t)i;

    // 3. block counts and the dense choice
    std::vector<int32_t> cnt((size_t)ngr * ncand, 0);
    for (int64_t r = 0; r < nr; ++r) {
        if (rpos[r] < 0) continue;
        const int64_t g = rpos[r] / TM;
        for (int64_t e = t.rowptr[r]; e < t.rowptr[r + 1]; ++e) {
            const int32_t cr = crank[t.col[e]];
            if (cr >= 0 && ok(e)) ++cnt[(size_t)g * ncand + cr / TK];
        }
    }
    std::vector<int32_t> chunk_new(ncand, -1);
    std::vector<int32_t> grp_orig;
    int32_t ntiles = 0;
    int64_t blk_entries = 0;
    d.grp_beg.push_back(0);
    for (int64_t g = 0; g < ngr; ++g) {
        int32_t nt = 0;
        for (int64_t q = 0; q < ncand; ++q) {
            int32_t& c = cnt[(size_t)g * ncand + q];
            if (c >= min_cnt) {
                blk_entries += c;
                if (chunk_new[q] < 0) chunk_new[q] = 0;   // used; numbered below
                c = ntiles + nt;                           // block index
                ++nt;
            } else {
                c = -1;
            }
        }
        if (nt > 0) {
            grp_orig.push_back((int32_t)g);
            ntiles += nt;
            d.grp_beg.push_back(ntiles);
        }
    }
    // 3b. worth it only when the blocks take most of the tile: the gathers they replace are the
    // L2-resident hub rows, so a tile whose gather is bound by the misses of its long tail
    // (Products-shaped: 27 % of the entries in blocks at thr 0.03) gains nothing
    // (profiles/r02_dense_probe_*.jsonl)
    if (ntiles == 0 || (double)blk_entries < min_frac * (double)t.rowptr[nr]) {
        d = DenseHost();
        return;
    }
    int32_t nch = 0;
    for (int64_t q = 0; q < ncand; ++q)
        if (chunk_new[q] == 0) chunk_new[q] = nch++;
    d.n_groups = (int64_t)grp_orig.size();
    d.n_tiles = ntiles;
    d.n_chunks = nch;
    d.tile_chunk.resize(ntiles);
    for (int64_t g = 0; g < ngr; ++g)
        for (int64_t q = 0; q < ncand; ++q) {
            const int32_t ti = cnt[(size_t)g * ncand + q];
            if (ti >= 0) d.tile_chunk[ti] = chunk_new[q];
        }
    d.chunk_cols.assign((size_t)nch * TK, -1);
    for (int64_t q = 0; q < ncand; ++q)
        if (chunk_new[q] >= 0)
            for (int k = 0; k < TK; ++k) {
                const int64_t i = q * TK + k;
                if (i < (int64_t)cols.size()) d.chunk_cols[(size_t)chunk_new[q] * TK + k] = cols[i];
            }
    d.row_flag.assign(nr, 0);
    d.grp_rows.assign((size_t)d.n_groups * TM, -1);
    for (int64_t gi = 0; gi < d.n_groups; ++gi) {
        const int64_t g = grp_orig[gi];
        for (int i = 0; i < TM; ++i) {
            const int64_t pos = g * TM + i;
            if (pos < (int64_t)rows.size()) {
                d.grp_rows[(size_t)gi * TM + i] = rows[pos];
                d.row_flag[rows[pos]] = 1;
            }
        }
    }
    // work items: segments of at most `seg` blocks, seg ~ half the blocks per SM (a hub row
    // group can hold thousands of blocks; one CTA walking it alone would bound the launch)
    int64_t seg = std::max<int64_t>(16, (ntiles + 2 * kSMs - 1) / (2 * kSMs));
    if (const char* e = getenv("MGGCN_DENSE_SEG")) seg = std::max(1, atoi(e));   // experiment hook
    std::vector<std::array<int32_t, 4>> items;
    for (int64_t g = 0; g < d.n_groups; ++g) {
        const int32_t b = d.grp_beg[g], e = d.grp_beg[g + 1];
        if (e - b <= seg) {
            items.push_back({(int32_t)g, b, e, -1});
            continue;
        }
        const int32_t ns = (int32_t)((e - b + seg - 1) / seg);
        d.splits.insert(d.splits.end(), {(int32_t)g, (int32_t)d.n_slots, ns, 0});
        for (int32_t k = 0; k < ns; ++k) {
            const int32_t sb = b + (int32_t)(k * (int64_t)(e - b) / ns), se = b + (int32_t)((k + 1) * (int64_t)(e - b) / ns);
            items.push_back({(int32_t)g, sb, se, (int32_t)(d.n_slots + k)});
        }
        d.n_slots += ns;
        ++d.n_splits;
    }
    std::stable_sort(items.begin(), items.end(), [](const std::array<int32_t, 4>& a, const std::array<int32_t, 4>& b) {
        return a[2] - a[1] > b[2] - b[1];
    });
    d.n_items = (int64_t)items.size();
    // LPT: items (longest first) go to the least-loaded of kSMs bins, one bin per CTA of the
    // persistent launch (a strided walk of the sorted list gave the SMs 48-87 % tensor-pipe
    // activity, profiles/r02_dense_ncu.md); cost = blocks + 2 (the chain drains and stores)
    const int64_t nb = std::min<int64_t>(kSMs, d.n_items);
    std::vector<std::vector<int32_t>> bins(nb);
    std::vector<std::pair<int64_t, int64_t>> heap;   // (load, bin), min-heap
    for (int64_t b = 0; b < nb; ++b) heap.push_back({0, b});
    auto cmp = [](const std::pair<int64_t, int64_t>& x, const std::pair<int64_t, int64_t>& y) { return x > y; };
    for (int64_t i = 0; i < d.n_items; ++i) {
        std::pop_heap(heap.begin(), heap.end(), cmp);
        auto& top = heap.back();
        bins[top.second].push_back((int32_t)i);
        top.first += (items[i][2] - items[i][1]) + 2;
        std::push_heap(heap.begin(), heap.end(), cmp);
    }
    d.bin_beg.push_back(0);
    for (int64_t b = 0; b < nb; ++b) {
        for (int32_t i : bins[b]) d.work.insert(d.work.end(), items[i].begin(), items[i].end());
        d.bin_beg.push_back((int32_t)(d.work.size() / 4));
    }
    d.n_bins = nb;

    // 4. A images and the residual tile
    d.A.assign((size_t)ntiles * TM * TK, 0);
    HostTile& o = d.resid;
    o.nrows = nr;
    o.ncols = nc;
    o.col0 = t.col0;
    o.rowptr.assign(nr + 1, 0);
    o.col.reserve(t.col.size());
    if (!pat) o.val.reserve(t.val.size());
    for (int64_t r = 0; r < nr; ++r) {
        const int64_t g = rpos[r] >= 0 ? rpos[r] / TM : -1;
        const int i = rpos[r] >= 0 ? rpos[r] % TM : 0;
        for (int64_t e = t.rowptr[r]; e < t.rowptr[r + 1]; ++e) {
            const int32_t cr = crank[t.col[e]];
            const int32_t ti = (g >= 0 && cr >= 0 && ok(e)) ? cnt[(size_t)g * ncand + cr / TK] : -1;
            if (ti >= 0) {
                const float v = pat ? 1.f : t.val[e];
                uint32_t b;
                std::memcpy(&b, &v, 4);
                const int k = cr % TK;
                const int byte = i * 64 + ((((2 * k) >> 4) ^ ((i >> 1) & 3)) << 4) + ((2 * k) & 15);
                d.A[(size_t)ti * TM * TK + byte / 2] = (uint16_t)(b >> 16);
                ++d.nnz;
            } else {
                o.col.push_back(t.col[e]);
                if (!pat) o.val.push_back(t.val[e]);
            }
        }
        o.rowptr[r + 1] = (int32_t)o.col.size();
    }
    d.active = true;
}
