// Host check of plan_dense (csrc/dense_plan.cpp): on a tile with a dense 700 x 700 core
// (30 % density, values 1..3) plus a ring, the dense blocks (A images decoded from their
// SWIZZLE_64B layout through grp_rows / chunk_cols) plus the residual CSR must reproduce
// the tile exactly, every block must belong to exactly one work item, and the rows of the
// groups must be flagged.  Exit 0 on success.  Built and run by tests/test_dense_plan_host.py.
#include "internal.h"
#include <cstdio>
#include <cstdlib>
#include <random>
#include <cstring>
#include <map>
#include <algorithm>
#include <cmath>
int main(int argc, char** argv) {
    const double thr = argc > 1 ? atof(argv[1]) : 0.05;
    const unsigned seed = argc > 2 ? atoi(argv[2]) : 1;
    HostTile t; int n = 1500; t.nrows = n; t.ncols = n;
    std::mt19937 rng(seed);
    std::vector<std::vector<int>> adj(n);
    for (int i = 0; i < 700; ++i) for (int j = 0; j < 700; ++j) if (i != j && (rng() % 100) < 30) adj[i].push_back(j);
    for (int i = 0; i < n; ++i) { adj[i].push_back((i + 1) % n); }
    t.rowptr.push_back(0);
    for (int i = 0; i < n; ++i) { std::sort(adj[i].begin(), adj[i].end()); adj[i].erase(std::unique(adj[i].begin(), adj[i].end()), adj[i].end());
        for (int c : adj[i]) { t.col.push_back(c); t.val.push_back(1.f + (rng() % 3)); } t.rowptr.push_back(t.col.size()); }
    DenseHost d; plan_dense(t, thr, 0.0, 0, 0, d);
    printf("active %d groups %ld tiles %ld chunks %ld nnz %ld items %ld splits %ld slots %ld resid %d total %zu\n", d.active, d.n_groups, d.n_tiles, d.n_chunks, d.nnz, d.n_items, d.n_splits, d.n_slots, d.active ? d.resid.rowptr.back() : -1, t.col.size());
    // reconstruct dense matrix from A images
    std::vector<double> M((size_t)n * n, 0), R((size_t)n * n, 0);
    for (int r = 0; r < n; ++r) for (int e = t.rowptr[r]; e < t.rowptr[r+1]; ++e) M[(size_t)r*n + t.col[e]] += t.val[e];
    const HostTile& res = d.active ? d.resid : t;   // inactive: the tile stays whole
    for (int r = 0; r < n; ++r) for (int e = res.rowptr[r]; e < res.rowptr[r+1]; ++e) R[(size_t)r*n + res.col[e]] += res.val[e];
    // items cover groups
    std::map<int,int> cover;
    for (int64_t i = 0; i < d.n_items; ++i) { int g = d.work[4*i], b = d.work[4*i+1], e = d.work[4*i+2];
        for (int tt = b; tt < e; ++tt) cover[tt]++;
        for (int tt = b; tt < e; ++tt) { int c = d.tile_chunk[tt];
            for (int slot = 0; slot < 128; ++slot) { int row = d.grp_rows[g*128+slot]; 
                for (int k = 0; k < 32; ++k) { int byte = slot*64 + ((((2*k)>>4) ^ ((slot>>1)&3))<<4) + ((2*k)&15);
                    uint16_t h = d.A[(size_t)tt*4096 + byte/2]; uint32_t b32 = (uint32_t)h << 16; float v; memcpy(&v,&b32,4);
                    int col = d.chunk_cols[c*32+k];
                    if (v != 0) { if (row < 0 || col < 0) { printf("bad\n"); return 1; } R[(size_t)row*n+col] += v; } } } } }
    if ((int64_t)cover.size() != d.n_tiles) { printf("cover %zu\n", cover.size()); return 1; }
    if (d.active && (d.bin_beg.empty() || d.bin_beg.front() != 0 || d.bin_beg.back() != d.n_items ||
                     (int64_t)d.bin_beg.size() != d.n_bins + 1)) { printf("bins\n"); return 1; }
    for (auto& kv : cover) if (kv.second != 1) { printf("dup cover\n"); return 1; }
    double err = 0; for (size_t i = 0; i < M.size(); ++i) err = std::max(err, std::abs(M[i]-R[i]));
    int nflag = 0; for (auto f : d.row_flag) nflag += f;
    printf("max err %g flagged rows %d\n", err, nflag);
    return err != 0;
}
