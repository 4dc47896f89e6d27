// internal.h — shared host-side structures of libmggcn (not part of the ABI).
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "../../include/mggcn.h"

namespace mggcn {

// Thread-local error message behind mggcn_last_error().
void set_error(const std::string& msg);

struct Error {
    int code;
    std::string msg;
};

inline int64_t round_up(int64_t x, int64_t a) { return (x + a - 1) / a * a; }

}  // namespace mggcn

// Host copy of A plus the weighted in-degree of Eq. 2.
struct mggcn_graph_s {
    int64_t n = 0, nnz = 0;
    std::vector<int64_t> rowptr;
    std::vector<int32_t> col;
    std::vector<float> val;      // empty => A_uv = 1 (pattern-only)
    std::vector<float> deg;      // fp32(sum_u A_uv), fp64 summation in CSR order
    bool symmetric = false;      // multiset symmetric (and, if weighted, A_uv == A_vu)
};

// One column tile of this rank's row block (Eq. 14-15), int32 local indices.
struct HostTile {
    int64_t nrows = 0, ncols = 0, col0 = 0;
    std::vector<int32_t> rowptr;   // nrows + 1
    std::vector<int32_t> col;      // local column ids, ascending within a row
    std::vector<float> val;        // Â'_uv per entry; empty if pattern-only
};

// Dense blocks of one stage tile (dense_plan.cpp, run by dense.cu): rows and
// columns ranked by entry count, cut into 128-row groups x 32-column chunks;
// a block with >= thr * 128 * 32 entries (values exact in bf16) goes to the
// tensor cores, everything else stays in `resid` for the CSR gather kernel.
struct DenseHost {
    bool active = false;
    HostTile resid;                     // the tile minus the dense blocks' entries
    int64_t n_groups = 0, n_tiles = 0, n_chunks = 0, nnz = 0;
    std::vector<int32_t> grp_rows;      // n_groups * 128, -1 = empty slot
    std::vector<uint8_t> row_flag;      // nrows: 1 = the row is in a group (gets a dense product)
    std::vector<int32_t> grp_beg;       // n_groups + 1
    // work items {group, first block, end block, partial slot (-1: the item is the whole group
    // and adds into the output)}, longest first; groups longer than the segment length are cut
    // into several items whose 128 x N products go to partial slots, summed in item order per
    // group by the fix-up (splits: {group, first slot, slots, 0})
    std::vector<int32_t> work;          // n_items * 4
    std::vector<int32_t> splits;        // n_splits * 4 (last: 0)
    int64_t n_items = 0, n_splits = 0, n_slots = 0;
    std::vector<int32_t> bin_beg;       // n_bins + 1: CTA b runs work items [bin_beg[b], bin_beg[b+1])
    int64_t n_bins = 0;
    std::vector<int32_t> tile_chunk;    // n_tiles
    std::vector<int32_t> chunk_cols;    // n_chunks * 32, -1 = empty slot
    std::vector<uint16_t> A;            // n_tiles * 128 * 32 bf16, K-major SWIZZLE_64B image per block
};
// thr <= 0, a tile of fewer than min_rows rows or min_entries entries, nothing dense, or the blocks holding < min_frac
// of the entries => d.active = false.
void plan_dense(const HostTile& t, double thr, double min_frac, int64_t min_rows, int64_t min_entries,
                DenseHost& d);

// One rank's 1D partition of the permuted graph.
struct mggcn_part_s {
    int32_t P = 1, rank = 0;
    int64_t n = 0;
    bool pattern = true;           // unit weights: values implied by inv_deg
    bool shared_fb = false;        // B tiles == F tiles (pattern + symmetric)
    std::vector<int64_t> p;        // P + 1
    std::vector<int64_t> perm;     // perm[old] = new
    std::vector<float> deg_new;    // deg of every vertex in NEW ids
    std::vector<HostTile> F, B;    // F: rows of Â'^T; B: rows of Â' (empty if shared_fb)
    std::vector<float> inv_deg;    // own rows
    int64_t nrows() const { return p[rank + 1] - p[rank]; }
    const HostTile& tileB(int j) const { return shared_fb ? F[j] : B[j]; }
};
