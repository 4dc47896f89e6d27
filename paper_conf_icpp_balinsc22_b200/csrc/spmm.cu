// spmm.cu — the staged CSR SpMM of MG-GCN on sm_100a (F2/B1 of SURVEY §8a).
//
// One launch = one stage j of the P-stage SpMM of P:705-720 (Fig. 2-3):
//     C_i (+)= A_ij · H_j
// with A_ij a CSR tile (Eq. 14-15) of Â'^T (forward, Eq. 6) or Â' (backward,
// Eq. 9).  HBM/L2-bound gather: each non-zero pulls one dense feature row.
//   - one warp per work item (a row, or a <= kSplit-entry segment of a hub
//     row); the column indices of 32 entries are fetched by one coalesced
//     128-B load and broadcast with shuffles;
//   - lanes are split into S = 32/G slots x G lanes: each slot gathers one
//     row with 128-bit loads (G float4 chunks, CH per lane), so narrow widths
//     still use all 32 lanes; slots are combined with a fixed xor tree;
//   - U gathers per lane are issued before any FMA (memory-level parallelism);
//   - epilogue fused: accumulate into the previous stage's output (RMW), and
//     on the last stage the 1/deg row scale (Eq. 2 for pattern-only graphs)
//     and ReLU (Eq. 7 / Eq. 18 in place).
#include "kernels.cuh"

namespace mggcn {

namespace {

constexpr int kWarpsPerBlock = 8;
constexpr int kUnroll = 8;

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

__device__ __forceinline__ int ld_stream_i32(const int32_t* p) {
    int v;
    asm volatile("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}

__device__ __forceinline__ float ld_stream_f32(const float* p) {
    float v;
    asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
}

__device__ __forceinline__ float4 epilogue(float4 acc, const float4* out_row, int q, int flags, float scale) {
    if (flags & SPMM_ACCUM) acc = f4_add(acc, out_row[q]);
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
template <int G, int CH, bool VALS>
__global__ void __launch_bounds__(kWarpsPerBlock * 32)
spmm_stage_kernel(const int4* __restrict__ items, int64_t n_items, const int32_t* __restrict__ col,
                  const float* __restrict__ val, const float4* __restrict__ B, int64_t ldb4,
                  float4* __restrict__ out, int64_t ldo4, float4* __restrict__ partial, int64_t ldp4,
                  const float* __restrict__ rowscale, int w4, int flags) {
    constexpr int S = 32 / G;
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (warp >= n_items) return;
    const int4 it = __ldg(items + warp);
    const int slot = lane / G, cl = lane % G;

    float4 acc[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) acc[c] = make_float4(0.f, 0.f, 0.f, 0.f);

    for (int base = it.y; base < it.z; base += 32) {
        const int cnt = min(32, it.z - base);
        const int my_c = lane < cnt ? ld_stream_i32(col + base + lane) : 0;
        float my_v = 0.f;
        if (VALS) my_v = lane < cnt ? ld_stream_f32(val + base + lane) : 0.f;
        // entries k = step*S + slot, steps of U issued together
        for (int k0 = 0; k0 < cnt; k0 += kUnroll * S) {
            float4 x[kUnroll][CH];
            float a[kUnroll];
#pragma unroll
            for (int u = 0; u < kUnroll; ++u) {
                const int k = k0 + u * S + slot;
                const int c = __shfl_sync(0xffffffffu, my_c, k & 31);
                float v = VALS ? __shfl_sync(0xffffffffu, my_v, k & 31) : 1.f;
                const bool ok = k < cnt;
                a[u] = ok ? v : 0.f;
                const float4* brow = B + (int64_t)c * ldb4;
#pragma unroll
                for (int ch = 0; ch < CH; ++ch) {
                    const int q = cl + ch * G;
                    x[u][ch] = (ok && q < w4) ? __ldg(brow + q) : make_float4(0.f, 0.f, 0.f, 0.f);
                }
            }
#pragma unroll
            for (int u = 0; u < kUnroll; ++u)
#pragma unroll
                for (int ch = 0; ch < CH; ++ch) acc[ch] = f4_fma(a[u], x[u][ch], acc[ch]);
        }
    }
    // combine the S slots (fixed xor tree => deterministic)
#pragma unroll
    for (int off = G; off < 32; off <<= 1)
#pragma unroll
        for (int ch = 0; ch < CH; ++ch) acc[ch] = f4_add(acc[ch], shfl_xor4(acc[ch], off));
    if (slot != 0) return;
    if (it.w >= 0) {
        float4* prow = partial + (int64_t)it.w * ldp4;
#pragma unroll
        for (int ch = 0; ch < CH; ++ch) {
            const int q = cl + ch * G;
            if (q < w4) prow[q] = acc[ch];
        }
        return;
    }
    float4* orow = out + (int64_t)it.x * ldo4;
    const float scale = rowscale ? __ldg(rowscale + it.x) : 1.f;
#pragma unroll
    for (int ch = 0; ch < CH; ++ch) {
        const int q = cl + ch * G;
        if (q < w4) orow[q] = epilogue(acc[ch], orow, q, flags, scale);
    }
}

// Hub rows: sum the segment partials in segment order, then the same epilogue.
__global__ void __launch_bounds__(kWarpsPerBlock * 32)
spmm_fixup_kernel(const int4* __restrict__ splits, int64_t n_splits, const float4* __restrict__ partial,
                  int64_t ldp4, float4* __restrict__ out, int64_t ldo4, const float* __restrict__ rowscale, int w4,
                  int flags) {
    const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (warp >= n_splits) return;
    const int4 sp = __ldg(splits + warp);
    float4* orow = out + (int64_t)sp.x * ldo4;
    const float scale = rowscale ? __ldg(rowscale + sp.x) : 1.f;
    for (int q = lane; q < w4; q += 32) {
        float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
        for (int s = 0; s < sp.z; ++s) acc = f4_add(acc, partial[(int64_t)(sp.y + s) * ldp4 + q]);
        orow[q] = epilogue(acc, orow, q, flags, scale);
    }
}

template <int G, int CH>
cudaError_t launch_gc(const SpmmTile& t, const float4* B, int64_t ldb4, float4* out, int64_t ldo4, float4* partial,
                      int64_t ldp4, const float* rowscale, int w4, int flags, cudaStream_t s) {
    const int64_t blocks = (t.n_items + kWarpsPerBlock - 1) / kWarpsPerBlock;
    if (t.val)
        spmm_stage_kernel<G, CH, true><<<(unsigned)blocks, kWarpsPerBlock * 32, 0, s>>>(
            t.items, t.n_items, t.col, t.val, B, ldb4, out, ldo4, partial, ldp4, rowscale, w4, flags);
    else
        spmm_stage_kernel<G, CH, false><<<(unsigned)blocks, kWarpsPerBlock * 32, 0, s>>>(
            t.items, t.n_items, t.col, t.val, B, ldb4, out, ldo4, partial, ldp4, rowscale, w4, flags);
    count_launches(1);
    return cudaGetLastError();
}

}  // namespace

cudaError_t launch_spmm(const SpmmTile& t, const float* B, int64_t ldb, float* out, int64_t ldo, float* partial,
                        const float* rowscale, int width, int flags, cudaStream_t s) {
    if (t.nrows == 0) return cudaSuccess;
    // column windows of at most 128 float4 (512 floats)
    for (int c0 = 0; c0 < width; c0 += 512) {
        const int w = width - c0 < 512 ? width - c0 : 512;
        const int w4 = (w + 3) / 4;
        const float4* Bw = reinterpret_cast<const float4*>(B + c0);
        float4* Ow = reinterpret_cast<float4*>(out + c0);
        float4* Pw = reinterpret_cast<float4*>(partial);
        const int64_t ldb4 = ldb / 4, ldo4 = ldo / 4, ldp4 = w4;
        cudaError_t e;
        if (t.n_items > 0) {
            if (w4 <= 1) e = launch_gc<1, 1>(t, Bw, ldb4, Ow, ldo4, Pw, ldp4, rowscale, w4, flags, s);
            else if (w4 <= 2) e = launch_gc<2, 1>(t, Bw, ldb4, Ow, ldo4, Pw, ldp4, rowscale, w4, flags, s);
            else if (w4 <= 4) e = launch_gc<4, 1>(t, Bw, ldb4, Ow, ldo4, Pw, ldp4, rowscale, w4, flags, s);
            else if (w4 <= 8) e = launch_gc<8, 1>(t, Bw, ldb4, Ow, ldo4, Pw, ldp4, rowscale, w4, flags, s);
            else if (w4 <= 16) e = launch_gc<16, 1>(t, Bw, ldb4, Ow, ldo4, Pw, ldp4, rowscale, w4, flags, s);
            else if (w4 <= 32) e = launch_gc<32, 1>(t, Bw, ldb4, Ow, ldo4, Pw, ldp4, rowscale, w4, flags, s);
            else if (w4 <= 64) e = launch_gc<32, 2>(t, Bw, ldb4, Ow, ldo4, Pw, ldp4, rowscale, w4, flags, s);
            else if (w4 <= 96) e = launch_gc<32, 3>(t, Bw, ldb4, Ow, ldo4, Pw, ldp4, rowscale, w4, flags, s);
            else e = launch_gc<32, 4>(t, Bw, ldb4, Ow, ldo4, Pw, ldp4, rowscale, w4, flags, s);
            if (e != cudaSuccess) return e;
        }
        if (t.n_splits > 0) {
            const int64_t blocks = (t.n_splits + kWarpsPerBlock - 1) / kWarpsPerBlock;
            spmm_fixup_kernel<<<(unsigned)blocks, kWarpsPerBlock * 32, 0, s>>>(t.splits, t.n_splits, Pw, ldp4, Ow,
                                                                                ldo4, rowscale, w4, flags);
            count_launches(1);
            e = cudaGetLastError();
            if (e != cudaSuccess) return e;
        }
    }
    return cudaSuccess;
}

}  // namespace mggcn
