// spmm.cu — the staged CSR SpMM of MG-GCN on sm_100a (F2/B1 of SURVEY §8a).
//
// One launch = one stage j of the P-stage SpMM of P:705-720 (Fig. 2-3):
//     C_i (+)= A_ij · H_j
// with A_ij a CSR tile (Eq. 14-15) of Â'^T (forward, Eq. 6) or Â' (backward,
// Eq. 9).  HBM/L2-bound gather: each non-zero pulls one dense feature row.
//   - one warp per work item (a row, or a <= split_for(nnz)-entry segment of a hub
//     row); the column indices of 32 entries are fetched by one coalesced
//     128-B load and broadcast with shuffles;
//   - lanes are split into S = 32/G slots x G lanes: each slot gathers one
//     row with 128-bit loads (G float4 chunks, CH per lane), so narrow widths
//     still use all 32 lanes; slots are combined with a fixed xor tree;
//   - U gathers per lane are issued before any FMA (memory-level parallelism);
//   - epilogue fused: accumulate into the previous stage's output (RMW), and
//     on the last stage the 1/deg row scale (Eq. 2 for pattern-only graphs)
//     and ReLU (Eq. 7 / Eq. 18 in place).
#include <cstdio>
#include <cstdlib>

#include "kernels.cuh"

namespace mggcn {

namespace {

#ifndef MGGCN_SPMM_WPB
#define MGGCN_SPMM_WPB 8
#endif
#ifndef MGGCN_SPMM_MINB
#define MGGCN_SPMM_MINB 1
#endif
#ifndef MGGCN_SPMM_U2
#define MGGCN_SPMM_U2 8
#endif
constexpr int kWarpsPerBlock = MGGCN_SPMM_WPB;

__device__ __forceinline__ float4 f4_fma(float a, float4 x, float4 acc) {
    acc.x = fmaf(a, x.x, acc.x);
    acc.y = fmaf(a, x.y, acc.y);
    acc.z = fmaf(a, x.z, acc.z);
    acc.w = fmaf(a, x.w, acc.w);
    return acc;
}

__device__ __forceinline__ float4 f4_add(float4 a, float4 b) {
    return make_float4(a.x + b.x, a.y + b.y, a.z + b.z, a.w + b.w);
}

__device__ __forceinline__ float4 shfl_xor4(float4 v, int off) {
    v.x = __shfl_xor_sync(0xffffffffu, v.x, off);
    v.y = __shfl_xor_sync(0xffffffffu, v.y, off);
    v.z = __shfl_xor_sync(0xffffffffu, v.z, off);
    v.w = __shfl_xor_sync(0xffffffffu, v.w, off);
    return v;
}

#ifndef MGGCN_SPMM_HINT
#define MGGCN_SPMM_HINT 0
#endif

__device__ __forceinline__ uint64_t l2_policy_first() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ uint64_t l2_policy_normal() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ uint64_t l2_policy_last() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}

// the L2 policies are created once per thread (a createpolicy per load would cost an issue slot per gather)
__device__ __forceinline__ int ld_stream_i32(const int32_t* p, uint64_t pol) {
    int v;
#if MGGCN_SPMM_HINT >= 1
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
#else
    (void)pol;
    asm volatile("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(v) : "l"(p));
#endif
    return v;
}

__device__ __forceinline__ float4 ld_gather(const float4* p, uint64_t pol) {
#if MGGCN_SPMM_HINT >= 2
    float4 v;
    asm volatile("ld.global.nc.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%4], %5;"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(pol));
    return v;
#else
    (void)pol;
    return __ldg(p);
#endif
}

// gather with a per-load L2 policy (degree-ranked priority classes)
__device__ __forceinline__ float4 ld_gather_pol(const float4* p, uint64_t pol) {
    float4 v;
    asm volatile("ld.global.nc.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%4], %5;"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(pol));
    return v;
}

__device__ __forceinline__ float ld_stream_f32(const float* p) {
    float v;
    asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
}

// accum: SPMM_ACCUM, or a row that already holds this stage's dense-block product (DenseTiles::row_flag)
__device__ __forceinline__ float4 epilogue(float4 acc, const float4* out_row, int q, int flags, float scale, bool accum) {
    if (accum) acc = f4_add(acc, out_row[q]);
    if (flags & SPMM_LAST) {
        acc.x *= scale; acc.y *= scale; acc.z *= scale; acc.w *= scale;
        if (flags & SPMM_RELU) {
            acc.x = fmaxf(acc.x, 0.f); acc.y = fmaxf(acc.y, 0.f);
            acc.z = fmaxf(acc.z, 0.f); acc.w = fmaxf(acc.w, 0.f);
        }
    }
    return acc;
}

// G lanes per gathered row (1..32), CH float4 chunks per lane, S = 32/G slots.
// Full groups of U entries per slot are issued with no predicates or selects,
// so all U*CH 128-bit gathers of a lane are in flight before the first FMA
// (a select such as `ok ? load : 0` would force a move right after each load
// and serialise them); only the last < U*S entries of a 32-entry chunk take
// the guarded tail path.
template <int CH>
__host__ __device__ constexpr int unroll_for() { return CH == 1 ? 16 : CH == 2 ? MGGCN_SPMM_U2 : CH == 3 ? 5 : 4; }

#ifndef MGGCN_SPMM_MINB_NARROW
#define MGGCN_SPMM_MINB_NARROW MGGCN_SPMM_MINB
#endif
// narrow rows (G * CH <= 16 float4, <= 64 floats per window): short gathers, latency-bound on
// short rows -> optionally more resident warps (fewer registers)
template <int G, int CH>
__host__ __device__ constexpr int minb_for() { return G * CH <= 16 ? MGGCN_SPMM_MINB_NARROW : MGGCN_SPMM_MINB; }

// HOT: the column indices carry L2 priority classes in bits 24..31 (SpmmTile::hot_enc);
// rows of class < hot_T are gathered with evict_last, the others with evict_first,
// so the most reused rows of a block larger than the L2 stay resident.
template <int G, int CH, bool VALS, bool HOT>
__global__ void __launch_bounds__(kWarpsPerBlock * 32, minb_for<G, CH>())
spmm_stage_kernel(const int4* __restrict__ items, int64_t n_items, const int32_t* __restrict__ col,
                  const float* __restrict__ val, const float4* __restrict__ B, int64_t ldb4,
                  float4* __restrict__ out, int64_t ldo4, float4* __restrict__ partial, int64_t ldp4,
                  const float* __restrict__ rowscale, int w4, int flags, uint32_t hot_T,
                  const uint8_t* __restrict__ drow) {
    constexpr int S = 32 / G;
    // U entries per slot per group; U * S <= 32 so a group fits a 32-entry chunk
    constexpr int U = unroll_for<CH>() < G ? unroll_for<CH>() : G;
    const int lane = threadIdx.x & 31;
    const int slot = lane / G, cl = lane % G;
    const uint32_t ldb = (uint32_t)ldb4;
    const uint64_t pf = MGGCN_SPMM_HINT >= 1 ? l2_policy_first() : 0, pl = MGGCN_SPMM_HINT >= 2 ? l2_policy_last() : 0;
    uint64_t ph = 0, pc = 0;
    if (HOT) {
        ph = hot_T > 0 ? l2_policy_last() : l2_policy_normal();
        pc = hot_T > 0 ? l2_policy_first() : l2_policy_normal();
    }
    int qc[CH];
#pragma unroll
    for (int ch = 0; ch < CH; ++ch) {
        const int q = cl + ch * G;
        qc[ch] = q < w4 ? q : 0;      // clamped: always a valid address, result unused
    }
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    // Persistent warps: static stride over the work items (hub segments first).
    // Software-pipelined across items: the descriptor of the item two strides
    // ahead and the first index chunk of the next item are loaded while the
    // current item gathers, so a short row (Products-shaped: ~50 entries, 1-2
    // chunks) does not pay item -> index -> gather as three serial latencies.
    const int4 kNone = make_int4(0, 0, 0, -1);
    int64_t wi = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    int4 it = wi < n_items ? __ldg(items + wi) : kNone;
    int4 itn = wi + nwarps < n_items ? __ldg(items + wi + nwarps) : kNone;
    int cur_c = (it.y + lane < it.z) ? ld_stream_i32(col + it.y + lane, pf) : 0;
    float cur_v = 0.f;
    if (VALS) cur_v = (it.y + lane < it.z) ? ld_stream_f32(val + it.y + lane) : 0.f;
    for (; wi < n_items; wi += nwarps) {
        const int4 it2 = wi + 2 * nwarps < n_items ? __ldg(items + wi + 2 * nwarps) : kNone;
        const float scale = (rowscale && it.w < 0) ? __ldg(rowscale + it.x) : 1.f;
        float4 acc[CH];
#pragma unroll
        for (int c = 0; c < CH; ++c) acc[c] = make_float4(0.f, 0.f, 0.f, 0.f);
        int nxt_c = cur_c;
        float nxt_v = cur_v;
        for (int base = it.y; base < it.z; base += 32) {
            const int cnt = min(32, it.z - base);
            const int my_c = nxt_c;
            const float my_v = nxt_v;
            if (base + 32 < it.z) {       // prefetch the next chunk's indices
                const int e = base + 32 + lane;
                nxt_c = e < it.z ? ld_stream_i32(col + e, pf) : 0;
                if (VALS) nxt_v = e < it.z ? ld_stream_f32(val + e) : 0.f;
            } else {                      // ... or the next item's first chunk
                const int e = itn.y + lane;
                nxt_c = e < itn.z ? ld_stream_i32(col + e, pf) : 0;
                if (VALS) nxt_v = e < itn.z ? ld_stream_f32(val + e) : 0.f;
            }
            int k0 = 0;
            for (; k0 + U * S <= cnt; k0 += U * S) {
                float4 x[U][CH];
                float a[U];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const int k = k0 + u * S + slot;
                    const uint32_t raw = (uint32_t)__shfl_sync(0xffffffffu, my_c, k);
                    a[u] = VALS ? __shfl_sync(0xffffffffu, my_v, k) : 1.f;
                    if (HOT) {
                        const float4* brow = B + (raw & 0xFFFFFFu) * ldb;
                        const uint64_t pol = (raw >> 24) < hot_T ? ph : pc;
#pragma unroll
                        for (int ch = 0; ch < CH; ++ch) x[u][ch] = ld_gather_pol(brow + qc[ch], pol);
                    } else {
                        const float4* brow = B + raw * ldb;
#pragma unroll
                        for (int ch = 0; ch < CH; ++ch) x[u][ch] = ld_gather(brow + qc[ch], pl);
                    }
                }
#pragma unroll
                for (int u = 0; u < U; ++u)
#pragma unroll
                    for (int ch = 0; ch < CH; ++ch) acc[ch] = f4_fma(a[u], x[u][ch], acc[ch]);
            }
            if (k0 < cnt) {   // tail (< U*S entries left): one more unpredicated group; padding lanes
                float4 x[U][CH];  // re-read the chunk's last entry (a row of this very sum) with weight 0
                float a[U];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const int k = k0 + u * S + slot;
                    const int kc = k < cnt ? k : cnt - 1;
                    const uint32_t raw = (uint32_t)__shfl_sync(0xffffffffu, my_c, kc);
                    const float v = VALS ? __shfl_sync(0xffffffffu, my_v, kc) : 1.f;
                    a[u] = k < cnt ? v : 0.f;
                    if (HOT) {
                        const float4* brow = B + (raw & 0xFFFFFFu) * ldb;
                        const uint64_t pol = (raw >> 24) < hot_T ? ph : pc;
#pragma unroll
                        for (int ch = 0; ch < CH; ++ch) x[u][ch] = ld_gather_pol(brow + qc[ch], pol);
                    } else {
                        const float4* brow = B + raw * ldb;
#pragma unroll
                        for (int ch = 0; ch < CH; ++ch) x[u][ch] = ld_gather(brow + qc[ch], pl);
                    }
                }
#pragma unroll
                for (int u = 0; u < U; ++u)
#pragma unroll
                    for (int ch = 0; ch < CH; ++ch) acc[ch] = f4_fma(a[u], x[u][ch], acc[ch]);
            }
        }
        if (it.z <= it.y) {               // empty row: still fetch the next item's first chunk
            const int e = itn.y + lane;
            nxt_c = e < itn.z ? ld_stream_i32(col + e, pf) : 0;
            if (VALS) nxt_v = e < itn.z ? ld_stream_f32(val + e) : 0.f;
        }
        // combine the S slots (fixed xor tree => deterministic)
#pragma unroll
        for (int off = G; off < 32; off <<= 1)
#pragma unroll
            for (int ch = 0; ch < CH; ++ch) acc[ch] = f4_add(acc[ch], shfl_xor4(acc[ch], off));
        if (slot == 0) {
            if (it.w >= 0) {
                float4* prow = partial + (int64_t)it.w * ldp4;
#pragma unroll
                for (int ch = 0; ch < CH; ++ch) {
                    const int q = cl + ch * G;
                    if (q < w4) prow[q] = acc[ch];
                }
            } else {
                float4* orow = out + (int64_t)it.x * ldo4;
                const bool accum = (flags & SPMM_ACCUM) || (drow && __ldg(drow + it.x));
#pragma unroll
                for (int ch = 0; ch < CH; ++ch) {
                    const int q = cl + ch * G;
                    if (q < w4) orow[q] = epilogue(acc[ch], orow, q, flags, scale, accum);
                }
            }
        }
        cur_c = nxt_c;
        cur_v = nxt_v;
        it = itn;
        itn = it2;
    }
}

// Hub rows with few segments: one warp per split row sums the partials in segment order.
__global__ void __launch_bounds__(kWarpsPerBlock * 32)
spmm_fixup_warp_kernel(const int4* __restrict__ splits, int64_t n_splits, const float4* __restrict__ partial,
                       int64_t ldp4, float4* __restrict__ out, int64_t ldo4, const float* __restrict__ rowscale,
                       int w4, int flags, const uint8_t* __restrict__ drow) {
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (warp >= n_splits) return;
    const int4 sp = __ldg(splits + warp);
    float4* orow = out + (int64_t)sp.x * ldo4;
    const float scale = rowscale ? __ldg(rowscale + sp.x) : 1.f;
    const bool accum = (flags & SPMM_ACCUM) || (drow && __ldg(drow + sp.x));
    for (int q = lane; q < w4; q += 32) {
        float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
        for (int s = 0; s < sp.z; ++s) acc = f4_add(acc, partial[(int64_t)(sp.y + s) * ldp4 + q]);
        orow[q] = epilogue(acc, orow, q, flags, scale, accum);
    }
}

// Hub rows with many segments (short segments of small tiles): one block per split row.  Warp w sums segments w, w + 8, ... in order,
// then warp 0 adds the 8 warp sums in warp order and applies the same epilogue
// (a fixed order => deterministic, no float atomics).  w4 <= 128 (windows of at
// most 512 floats).
constexpr int kFixWarps = 8;
__global__ void __launch_bounds__(kFixWarps * 32)
spmm_fixup_kernel(const int4* __restrict__ splits, int64_t n_splits, const float4* __restrict__ partial,
                  int64_t ldp4, float4* __restrict__ out, int64_t ldo4, const float* __restrict__ rowscale, int w4,
                  int flags, const uint8_t* __restrict__ drow) {
    __shared__ float4 red[kFixWarps][128];
    const int64_t sid = blockIdx.x;
    if (sid >= n_splits) return;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int4 sp = __ldg(splits + sid);
    for (int q = lane; q < w4; q += 32) {
        float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll 4
        for (int s = warp; s < sp.z; s += kFixWarps) acc = f4_add(acc, partial[(int64_t)(sp.y + s) * ldp4 + q]);
        red[warp][q] = acc;
    }
    __syncthreads();
    if (warp != 0) return;
    float4* orow = out + (int64_t)sp.x * ldo4;
    const float scale = rowscale ? __ldg(rowscale + sp.x) : 1.f;
    const bool accum = (flags & SPMM_ACCUM) || (drow && __ldg(drow + sp.x));
    for (int q = lane; q < w4; q += 32) {
        float4 acc = red[0][q];
#pragma unroll
        for (int w = 1; w < kFixWarps; ++w) acc = f4_add(acc, red[w][q]);
        orow[q] = epilogue(acc, orow, q, flags, scale, accum);
    }
}

int sm_count() {
    static int n = 0;
    if (n == 0) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}

template <int G, int CH, bool V, bool H>
int64_t persistent_blocks(int64_t n_items, int over) {
    static int per_sm = 0;
    if (per_sm == 0) {
        const char* co = getenv("MGGCN_SPMM_CARVEOUT");
        if (co) cudaFuncSetAttribute(spmm_stage_kernel<G, CH, V, H>, cudaFuncAttributePreferredSharedMemoryCarveout,
                                     atoi(co));
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, spmm_stage_kernel<G, CH, V, H>, kWarpsPerBlock * 32, 0);
        if (per_sm <= 0) per_sm = 1;
    }
    const int64_t need = (n_items + kWarpsPerBlock - 1) / kWarpsPerBlock;
    static int sms_env = -1;   // experiment hook: MGGCN_SPMM_SMS = SMs the persistent grid is sized for
    if (sms_env < 0) {
        const char* e = getenv("MGGCN_SPMM_SMS");
        sms_env = e ? atoi(e) : 0;
    }
    const int64_t cap = (int64_t)per_sm * (sms_env > 0 ? sms_env : sm_count()) * over;
    return need < cap ? need : cap;
}

template <int G, int CH, bool V, bool H>
void launch_one(const SpmmTile& t, const float4* B, int64_t ldb4, float4* out, int64_t ldo4, float4* partial,
                int64_t ldp4, const float* rowscale, int w4, int flags, uint32_t hot_T, cudaStream_t s) {
    // SPMM_YIELD: blocks retire throughout the launch (see kernels.cuh); MGGCN_SPMM_YIELD=k
    // overrides the factor (and with k > 1 applies it to every launch, for measurement)
    static int yenv = -1;
    if (yenv < 0) {
        const char* e = getenv("MGGCN_SPMM_YIELD");
        yenv = e ? atoi(e) : 0;
        if (yenv < 0) yenv = 0;
    }
    const int over = yenv > 1 ? yenv : ((flags & SPMM_YIELD) ? (yenv == 1 ? 1 : kYieldBlocks) : 1);
    const int64_t blocks = persistent_blocks<G, CH, V, H>(t.n_items, over);
    spmm_stage_kernel<G, CH, V, H><<<(unsigned)blocks, kWarpsPerBlock * 32, 0, s>>>(
        t.items, t.n_items, t.col, t.val, B, ldb4, out, ldo4, partial, ldp4, rowscale, w4, flags, hot_T,
        t.dense.row_flag);
}

template <int G, int CH>
cudaError_t launch_gc(const SpmmTile& t, const float4* B, int64_t ldb4, float4* out, int64_t ldo4, float4* partial,
                      int64_t ldp4, const float* rowscale, int w4, int flags, uint32_t hot_T, cudaStream_t s) {
    if (t.val) {
        if (t.hot_enc) launch_one<G, CH, true, true>(t, B, ldb4, out, ldo4, partial, ldp4, rowscale, w4, flags, hot_T, s);
        else launch_one<G, CH, true, false>(t, B, ldb4, out, ldo4, partial, ldp4, rowscale, w4, flags, hot_T, s);
    } else {
        if (t.hot_enc) launch_one<G, CH, false, true>(t, B, ldb4, out, ldo4, partial, ldp4, rowscale, w4, flags, hot_T, s);
        else launch_one<G, CH, false, false>(t, B, ldb4, out, ldo4, partial, ldp4, rowscale, w4, flags, hot_T, s);
    }
    count_launches(1);
    return cudaGetLastError();
}

// (G lanes per row, CH float4 per lane): the instantiated shapes; the
// dispatcher picks the one that covers w4 with the fewest idle lanes.
#define MGGCN_SPMM_SHAPES(X) \
    X(1, 1) X(2, 1) X(4, 1) X(8, 1) X(16, 1) X(32, 1) X(2, 2) X(4, 2) X(8, 2) X(16, 2) X(32, 2) \
    X(4, 3) X(8, 3) X(16, 3) X(32, 3) X(8, 4) X(16, 4) X(32, 4)

cudaError_t dispatch_gc(int w4, const SpmmTile& t, const float4* B, int64_t ldb4, float4* out, int64_t ldo4,
                        float4* partial, int64_t ldp4, const float* rowscale, int flags, uint32_t hot_T, cudaStream_t s) {
    int bg = 0, bc = 0;
    double best = 1e9;
#define MGGCN_PICK(g, c)                                                         \
    if (g * c >= w4) {                                                            \
        const double waste = (double)(g * c - w4) / (g * c) + 1e-3 * (c == 1);    \
        if (waste < best - 1e-9) { best = waste; bg = g; bc = c; }               \
    }
    MGGCN_SPMM_SHAPES(MGGCN_PICK)
#undef MGGCN_PICK
    {   // experiment hook: MGGCN_SPMM_SHAPE="G,CH" forces an instantiated shape that covers w4
        static int fg = -1, fc = 0;
        if (fg < 0) {
            fg = 0;
            if (const char* e = getenv("MGGCN_SPMM_SHAPE")) sscanf(e, "%d,%d", &fg, &fc);
        }
        if (fg > 0 && fg * fc >= w4) { bg = fg; bc = fc; }
    }
#define MGGCN_CALL(g, c) \
    if (bg == g && bc == c) return launch_gc<g, c>(t, B, ldb4, out, ldo4, partial, ldp4, rowscale, w4, flags, hot_T, s);
    MGGCN_SPMM_SHAPES(MGGCN_CALL)
#undef MGGCN_CALL
    return cudaErrorInvalidValue;
}

}  // namespace

cudaError_t launch_spmm_dense(const SpmmTile& tile, const float* B, int64_t ldb, float* out, int64_t ldo, int width,
                              int flags, cudaStream_t s) {
    if (tile.nrows == 0 || tile.dense.n_items == 0) return cudaSuccess;
    for (int c0 = 0; c0 < width; c0 += kDenseMaxN) {
        const int w = width - c0 < kDenseMaxN ? width - c0 : kDenseMaxN;
        cudaError_t e = launch_dense(tile.dense, B + c0, ldb, out + c0, ldo, w, !(flags & SPMM_ACCUM), s);
        if (e != cudaSuccess) return e;
    }
    return cudaSuccess;
}

cudaError_t launch_spmm(const SpmmTile& tile, const float* B, int64_t ldb, float* out, int64_t ldo, float* partial,
                        const float* rowscale, int width, int flags, cudaStream_t s) {
    // Dense blocks (dense.cu) first: they store (first stage) or add their products into the
    // rows of their groups; the gather kernel then adds the residual entries to those rows
    // (DenseTiles::row_flag), writes the others as usual and applies the stage epilogue.
    cudaError_t e = launch_spmm_dense(tile, B, ldb, out, ldo, width, flags, s);
    if (e != cudaSuccess) return e;
    return launch_spmm_gather(tile, B, ldb, out, ldo, partial, rowscale, width, flags, s);
}

cudaError_t launch_spmm_gather(const SpmmTile& tile, const float* B, int64_t ldb, float* out, int64_t ldo,
                               float* partial, const float* rowscale, int width, int flags, cudaStream_t s) {
    if (tile.nrows == 0) return cudaSuccess;
    // a middle stage (accumulating, not the last) skips the tile's empty rows: their sum is
    // zero, so their output read-modify-write is a no-op (the first stage writes every row,
    // the last applies the row scale / ReLU to every row)
    SpmmTile t = tile;
    if ((flags & SPMM_ACCUM) && !(flags & SPMM_LAST)) t.n_items = t.n_items_nz;
    // Column windows of at most `win` floats.  The gathers are bound by the
    // SMs' L2 line rate; when the gathered block B_j is larger
    // than 1.5x the L2, a 128-float window that fits it (n_j * 512 B <= L2) keeps the
    // slice L2-resident: same L2 traffic, 2.4x less DRAM traffic, 2 % faster
    // on Reddit-shaped B (profiles/r01_win_sweep.log).  Narrower windows
    // lose (extra index passes); a block that does not fit even at 128 floats
    // (Products-shaped) is gathered at full width.  MGGCN_SPMM_WIN overrides.
    static int win_env = -1, l2_bytes = 0;
    if (win_env < 0) {
        const char* e = getenv("MGGCN_SPMM_WIN");
        win_env = e ? atoi(e) : 0;
        if (win_env != 0 && (win_env < 4 || win_env > 512 || (win_env & 3))) win_env = 0;
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&l2_bytes, cudaDevAttrL2CacheSize, dev);
    }
    int win = win_env;
    if (win == 0) {
        const int64_t full = t.ncols * (int64_t)width * 4, w128 = t.ncols * 128 * 4;
        // windows pay for their second index pass and launch only when the block is well beyond
        // the L2: Reddit-shaped P = 1 (228 MB, 1.8x L2) gains 2 %, a 149 MB merged stage group
        // (Reddit-shaped P = 8, 5 blocks) loses 6 % (profiles/r02_win_rule.log)
        win = (width > 128 && 2 * full > 3 * (int64_t)l2_bytes && w128 <= (int64_t)l2_bytes) ? 128 : 512;
    }
    // L2 priority classes (tiles with hot_enc): when the gathered window does not
    // fit the L2, the rows of the most reused columns, up to hot_bytes of them,
    // are gathered with evict_last and the rest with evict_first (0 = normal).
    static int64_t hot_bytes = -1;
    static bool hot_force = false;   // MGGCN_SPMM_HOTCLS=2 (tests): classes even for blocks that fit
    if (hot_bytes < 0) {
        const char* hc = getenv("MGGCN_SPMM_HOTCLS");
        hot_force = hc && atoi(hc) == 2;
        const char* e = getenv("MGGCN_SPMM_HOT_MB");
        hot_bytes = (int64_t)((e ? atof(e) : (double)kHotDefaultMB) * 1048576.0);
        if (const char* pm = getenv("MGGCN_L2_PERSIST_MB")) {   // experiment hook: persisting set-aside
            int dev = 0, mx = 0;
            cudaGetDevice(&dev);
            cudaDeviceGetAttribute(&mx, cudaDevAttrMaxPersistingL2CacheSize, dev);
            size_t want = (size_t)(atof(pm) * 1048576.0);
            if (want > (size_t)mx) want = (size_t)mx;
            cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, want);
            size_t got = 0;
            cudaDeviceGetLimit(&got, cudaLimitPersistingL2CacheSize);
            fprintf(stderr, "[mggcn] persisting L2 set-aside %zu B (max %d B)\n", got, mx);
        }
    }
    for (int c0 = 0; c0 < width; c0 += win) {
        const int w = width - c0 < win ? width - c0 : win;
        const int w4 = (w + 3) / 4;
        uint32_t hot_T = 0;
        if (t.hot_enc && hot_bytes > 0 && (hot_force || t.ncols * (int64_t)w4 * 16 > (int64_t)l2_bytes)) {
            const int64_t H = hot_bytes / ((int64_t)w4 * 16);
            hot_T = (uint32_t)hot_class_of(H < t.ncols ? H : t.ncols);
        }
        const float4* Bw = reinterpret_cast<const float4*>(B + c0);
        float4* Ow = reinterpret_cast<float4*>(out + c0);
        float4* Pw = reinterpret_cast<float4*>(partial);
        const int64_t ldb4 = ldb / 4, ldo4 = ldo / 4, ldp4 = w4;
        cudaError_t e;
        if (t.n_items > 0) {
            e = dispatch_gc(w4, t, Bw, ldb4, Ow, ldo4, Pw, ldp4, rowscale, flags, hot_T, s);
            if (e != cudaSuccess) return e;
        }
        if (t.n_splits > 0) {
            // one fix-up launch per stage: a warp per split row for long segments (large tiles,
            // few segments per row), a block per split row for short ones (small tiles: a hub row
            // has hundreds of segments); same-box A/B in profiles/r01_split_sweep.log
            static int fix_env = -1;
            if (fix_env < 0) {
                const char* fe = getenv("MGGCN_FIXUP_BLOCK");   // experiment hook: 0 warp, 1 block
                fix_env = fe ? (atoi(fe) ? 1 : 0) : 2;
            }
            const bool block = fix_env == 2 ? t.split < kSplit : fix_env == 1;
            if (block)
                spmm_fixup_kernel<<<(unsigned)t.n_splits, kFixWarps * 32, 0, s>>>(t.splits, t.n_splits, Pw, ldp4,
                                                                                   Ow, ldo4, rowscale, w4, flags,
                                                                                   t.dense.row_flag);
            else
                spmm_fixup_warp_kernel<<<(unsigned)((t.n_splits + kWarpsPerBlock - 1) / kWarpsPerBlock),
                                         kWarpsPerBlock * 32, 0, s>>>(t.splits, t.n_splits, Pw, ldp4, Ow, ldo4,
                                                                      rowscale, w4, flags, t.dense.row_flag);
            count_launches(1);
            e = cudaGetLastError();
            if (e != cudaSuccess) return e;
        }
    }
    return cudaSuccess;
}

}  // namespace mggcn
