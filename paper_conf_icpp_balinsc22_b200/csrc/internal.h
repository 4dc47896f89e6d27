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
