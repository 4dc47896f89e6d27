// kernels.cuh — launch interface of the sm_100a kernels (internal).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>

namespace mggcn {

// process-wide count of kernel launches issued by this library
void count_launches(int n);
// test hook (mggcn_debug_comm_delay): one thread spinning on %globaltimer for ns nanoseconds
cudaError_t launch_spin(uint64_t ns, cudaStream_t s);

// ------------------------------------------------------------------ SpMM
// One stage of the staged SpMM: out_i (+)= T_ij · B_j for one
// tile T (CSR, local indices).  Work is pre-cut on the host into items
// {row, beg, end, slot}: rows with <= kSplit entries are one item written
// directly (slot = -1); longer rows (R-MAT hubs) are cut into kSplit-entry
// segments whose partial sums go to `partial[slot]` and are combined in
// segment order by a fix-up kernel (deterministic, no float atomics).
constexpr int kSplit = 2048;      // longest segment
constexpr int kSplitMin = 128;    // shortest segment (small tiles, e.g. Reddit-shaped at P = 8)

// Segment length of a tile with nnz entries: the longest work item is one warp
// walking a segment, so a short stage (a small tile) needs short segments or
// its hub segments become the stage's critical path; ~nnz / (4 x 2368 warps),
// a power of two in [kSplitMin, kSplit].  MGGCN_SPMM_SPLIT overrides.
inline int split_for(int64_t nnz) {
    int s = kSplit;
    while (s > kSplitMin && (int64_t)s * 4 * 2368 > nnz) s >>= 1;
    return s;
}

// ------------------------------------------------------------ dense tiles
// Dense blocks of a stage tile run on the tensor cores (dense.cu; chosen by
// plan_dense, dense_plan.cpp): kDenseM output rows (a row group, rows in
// degree order) x kDenseK columns (a column chunk, columns in degree order).
constexpr int kDenseM = 128;
constexpr int kDenseK = 32;
constexpr int kDenseMaxN = 256;    // features per launch (wider operands: 256-column windows)
// default density threshold of a dense block (entries / (128 x 32)); MGGCN_DENSE_THR overrides, 0 = off
constexpr double kDenseThrDefault = 0.04;
// a tile uses blocks only if they hold >= this share of its entries; MGGCN_DENSE_MINFRAC overrides
constexpr double kDenseMinFracDefault = 0.5;
// ... and only in tiles of at least this many rows (MGGCN_DENSE_MIN_ROWS overrides)
constexpr int64_t kDenseMinRowsDefault = 0;
// ... holding at least this many coalesced entries (MGGCN_DENSE_MIN_ENTRIES overrides)
constexpr int64_t kDenseMinEntriesDefault = 3000000;
struct DenseTiles {
    int64_t n_groups = 0, n_tiles = 0, n_chunks = 0;
    int64_t n_items = 0, n_splits = 0, n_slots = 0, n_bins = 0;
    int64_t nnz = 0;                   // entries (coalesced) covered by the blocks
    int pieces = 3;                    // bf16 pieces of the B operand (2: hi + mid, 3: + lo)
    const int32_t* grp_rows = nullptr;   // [n_groups][kDenseM] output row of each slot, -1 = none
    const uint8_t* row_flag = nullptr;   // [nrows] 1 = row of a group: the gather kernel adds to its output
    const int4* work = nullptr;          // [n_items] {group, first block, end block, partial slot or -1}
    const int32_t* bin_beg = nullptr;    // [n_bins + 1] CTA b of the launch runs items [bin_beg[b], bin_beg[b+1])
    const int4* splits = nullptr;        // [n_splits] {group, first slot, slots, 0}: groups cut into items
    float* partial = nullptr;            // scratch: [n_slots][kDenseM][N]
    const int32_t* tile_chunk = nullptr; // [n_tiles] column chunk of each block
    const int32_t* chunk_cols = nullptr; // [n_chunks][kDenseK] column of each chunk slot, -1 = none
    const uint8_t* A = nullptr;          // [n_tiles][kDenseM x kDenseK bf16], K-major SWIZZLE_64B image
    uint8_t* bimg = nullptr;             // scratch: [n_chunks][pieces][N][kDenseK bf16]
};
// out[rows of the groups][0, width) (+)= dense blocks · B (B row stride ldb, width <= kDenseMaxN,
// % 4 == 0); first: store (the stage's first write) instead of add
cudaError_t launch_dense(const DenseTiles& d, const float* B, int64_t ldb, float* out, int64_t ldo, int width,
                         bool first, cudaStream_t s);
size_t dense_bimg_bytes(int64_t n_chunks, int pieces);
size_t dense_partial_floats(int64_t n_slots);
int dense_stages_for(int N, int pieces);

struct SpmmTile {
    const int4* items = nullptr;   // {row, beg, end, slot}
    int64_t n_items = 0;
    int64_t n_items_nz = 0;        // items[0, n_items_nz) are hub segments and non-empty rows, the rest empty rows
    const int4* splits = nullptr;  // {row, first_slot, nslots, 0}
    int64_t n_splits = 0;
    int64_t n_slots = 0;
    int64_t split = kSplit;        // segment length of this tile (split_for); short segments
                                   // (a small tile) => many per row => block-per-row fix-up
    const int32_t* col = nullptr;
    const float* val = nullptr;    // nullptr => pattern-only (value 1)
    int64_t nnz = 0, nrows = 0, ncols = 0;
    // L2 priority classes: when set, col[e] = (cls << 24) | column, where cls
    // is the 1/8-octave class of the column's rank by reuse count in this tile
    // (hot_class_of); launch_spmm gathers the rows of the classes that fit its
    // L2 budget with evict_last and the rest with evict_first.
    bool hot_enc = false;
    // dense blocks of the tile (n_groups == 0: none); the CSR above then holds the residual entries
    DenseTiles dense;
};

// default evict_last budget of the L2 priority classes (MGGCN_SPMM_HOT_MB overrides)
constexpr int kHotDefaultMB = 0;

// 1/8-octave class of rank r (0 = most reused column): 8*floor(log2(r+1)) + the
// next 3 bits of r+1; monotone in r, < 200 for r < 2^24.
inline int hot_class_of(int64_t r) {
    const uint64_t x = (uint64_t)r + 1;
    int e = 63 - __builtin_clzll(x);
    const int f = e >= 3 ? (int)((x >> (e - 3)) & 7) : (int)((x << (3 - e)) & 7);
    return 8 * e + f;
}

// SPMM_YIELD (host-side only): oversubscribe the grid (kYieldBlocks x the resident
// blocks) so blocks retire throughout the launch and a collective kernel on a
// higher-priority stream (NCCL broadcast / all-reduce) gets SMs within a few
// microseconds instead of waiting for a persistent grid to drain.
enum SpmmFlags : int { SPMM_ACCUM = 1, SPMM_LAST = 2, SPMM_RELU = 4, SPMM_YIELD = 8 };
constexpr int kYieldBlocks = 4;

// width: columns to compute (multiple of 4, <= ldb, <= ldo); B and out 16-B aligned.
// rowscale (nullable): multiplies the finished row on the LAST stage.
cudaError_t launch_spmm(const SpmmTile& t, const float* B, int64_t ldb, float* out, int64_t ldo, float* partial,
                        const float* rowscale, int width, int flags, cudaStream_t s);
// the two halves of launch_spmm, in this order: the tile's dense blocks (no-op without them),
// then the gather of the residual CSR with the stage epilogue
cudaError_t launch_spmm_dense(const SpmmTile& t, const float* B, int64_t ldb, float* out, int64_t ldo, int width,
                              int flags, cudaStream_t s);
cudaError_t launch_spmm_gather(const SpmmTile& t, const float* B, int64_t ldb, float* out, int64_t ldo,
                               float* partial, const float* rowscale, int width, int flags, cudaStream_t s);

// ------------------------------------------------------------------ GEMM
// tcgen05 (kind::tf32) GEMM with TMA-staged operands and TMEM accumulators.
// op 0: C = A·B   (A M x K row-major, B K x N row-major)     [Eq. 5, S-order T·W]
// op 1: C = A·B^T (A M x K, B N x K)                         [Eq. 11]
// op 2: C = A^T·B (A K x M, B K x N), split-K partials       [Eq. 10]
// The fp32 operands are split into tf32 hi + lo in shared memory and the
// product is hi·hi + hi·lo + lo·hi (3xTF32) unless GEMM_TF32X1.
enum GemmFlags : int {
    GEMM_RELU = 1,     // C = max(C, 0)
    GEMM_MASK = 2,     // C = C * [C_old > 0]  (ReLU' of Eq. 8 read from the buffer being overwritten)
    GEMM_SCALE = 4,    // C *= rowscale[row]   (inv_deg pre-scale for the next pattern SpMM)
    GEMM_TF32X1 = 16,
};

struct GemmPlan {
    int op = 0;
    int64_t M = 0, N = 0, K = 0;
    int BN = 0, m_tiles = 0, n_tiles = 0, k_chunks = 1;
    int64_t k_chunk_len = 0;
    CUtensorMap tmA, tmB, tmB2, tmC;
    float* C = nullptr;
    int64_t ldc = 0;
    float* partial = nullptr;   // op 2: [k_chunks][M][N]
    const float* rowscale = nullptr;
    int flags = 0;
    int grid = 0;
    int variant = 0;            // op 2: 1 = MN-major operands straight from TMA (no transpose)
    uint32_t desc_mn[3] = {1, 2048, 512};   // op 2 variant 1: layout type, LBO, SBO (bytes)
};

// Row GEMM (op 0 and op 1 of the comment above): C = A · B^T with B given
// pre-split (launch_split_weights) as tf32 hi / lo copies in K-major [N x K]
// layout, row stride ldb.  Pointers 16-B aligned, lda / ldb multiples of 4.
int gemm_plan_rows(GemmPlan& p, int64_t M, int64_t N, int64_t K, const float* A, int64_t lda, const float* Bhi,
                   const float* Blo, int64_t ldb, float* C, int64_t ldc, int flags);
// Weight-gradient GEMM (op 2): partial[kc] = A^T B over K chunks; caller sets
// p.partial and reduces with launch_splitk_reduce.
int gemm_plan_wgrad(GemmPlan& p, int64_t M, int64_t N, int64_t K, const float* A, int64_t lda, const float* B,
                    int64_t ldb, int flags, size_t* partial_floats);
size_t gemm_wgrad_partial_floats(int64_t M, int64_t N, int64_t K);
// W (din x dout, stride ldw) -> T = W^T hi/lo ([dout x din], stride ldt) and
// S = W hi/lo ([din x dout], stride ldw); either pair may be null.
cudaError_t launch_split_weights(const float* W, int64_t din, int64_t dout, int64_t ldw, float* t_hi, float* t_lo,
                                 int64_t ldt, float* s_hi, float* s_lo, int x1, cudaStream_t s);
cudaError_t gemm_launch(const GemmPlan& p, cudaStream_t s);
// op 2 second pass: C[m][n] (ldc) = sum_kc partial[kc][m][n], in kc order.
cudaError_t launch_splitk_reduce(const float* partial, int k_chunks, int64_t M, int64_t N, float* C, int64_t ldc,
                                 cudaStream_t s);

// ------------------------------------------------------------------ misc
// Softmax-CE forward + backward fused (Eq. 19 in place):
// Z (n x C, ld) holds logits on entry and dLoss/dZ on exit (times
// rowscale[row] if non-null; times [Z > 0] if relu_last).  Per-block fp64
// partial loss sums into block_partial[grid].
constexpr int kCeBlocks = 2368;          // 16 per SM; fixed so partial sums are reduced in a fixed order
constexpr int kCountBlocks = 296;
cudaError_t launch_softmax_ce(float* Z, int64_t n, int C, int64_t ld, const int32_t* y, const int64_t* ntrain,
                              const float* rowscale, int relu_last, double* block_partial, cudaStream_t s);
cudaError_t launch_sum_partials(const double* partial, int count, double* out, cudaStream_t s);
// |T| = #{y >= 0}: per-block counts into scratch[kCountBlocks], then one ordered sum into *out.
cudaError_t launch_count_labelled(const int32_t* y, int64_t n, int64_t* scratch, int64_t* out, cudaStream_t s);
cudaError_t launch_adam(float* W, const float* g, float* m, float* v, int64_t count, double lr, double b1,
                        double b2, double eps, int64_t t, cudaStream_t s);
// CUDA-graph epochs: the Adam kernel's address, and a re-set of a captured Adam node's
// arguments (bias corrections for step t) in an instantiated graph.
const void* adam_kernel_func();
cudaError_t graph_set_adam(cudaGraphExec_t ex, cudaGraphNode_t node, float* W, const float* g, float* m, float* v,
                           int64_t count, double lr, double b1, double b2, double eps, int64_t t);
// out[i] = sum_r in[r][i] in r order (loopback "all-reduce").
cudaError_t launch_sum_buffers(const float* const* in, int nin, float* out, int64_t count, cudaStream_t s);
cudaError_t launch_sum_i64(const int64_t* in, int nin, int64_t* out, cudaStream_t s);
cudaError_t launch_sum_f64(const double* in, int nin, double* out, cudaStream_t s);
cudaError_t launch_scale_rows(const float* in, int64_t ldi, float* out, int64_t ldo, int64_t n, int width,
                              const float* rowscale, cudaStream_t s);

// ------------------------------------------------------------------- IPC
// (ipc.cu) stream memory operations, allocation base lookup and rank-ordered
// sums over peer buffers mapped with cudaIpcOpenMemHandle.
struct PtrArrayF { const float* p[64]; };
struct PtrArrayD { const double* p[64]; };
struct PtrArrayI { const int64_t* p[64]; };
bool ipc_stream_memops_available();
cudaError_t stream_write_u32(cudaStream_t s, uint32_t* addr, uint32_t value);
cudaError_t stream_wait_u32(cudaStream_t s, const uint32_t* addr, uint32_t value);
int ipc_alloc_base(const void* ptr, void** base, size_t* size);
// 1.5D (c = 2) SpMM finish: the two replicas of
// a row block hold partial sums over disjoint column-block sets; pair_sum adds
// them (a + b, commutative: both copies end bitwise equal) and applies the
// last-stage epilogue (row scale of Eq. 2, ReLU of Eq. 7) to both copies;
// rows_epilogue applies it in place after an NCCL pair all-reduce.
cudaError_t launch_pair_sum_epilogue(float* a, float* b, int64_t rows, int width, int64_t ld, const float* rowscale,
                                     int relu, cudaStream_t s);
cudaError_t launch_rows_epilogue(float* a, int64_t rows, int width, int64_t ld, const float* rowscale, int relu,
                                 cudaStream_t s);
cudaError_t launch_sum_ranks_f32(const float* const* in, int nin, float* out, int64_t count, cudaStream_t s);
cudaError_t launch_sum_ranks_scalar(const double* const* in_d, const int64_t* const* in_i, int nin, double* out_d,
                                    int64_t* out_i, cudaStream_t s);

}  // namespace mggcn
