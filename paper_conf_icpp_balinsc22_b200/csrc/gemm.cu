// gemm.cu — tcgen05 / TMA / TMEM GEMM for the dense products of MG-GCN on
// sm_100a (F1, B2, B3 of SURVEY §8a):
//     Eq. 5   HW  = H · W            op 0 (also the S-order (Â^T H) · W)
//     Eq. 11  H_G = HW_G · W^T        op 1 (+ fused ReLU' mask of Eq. 8, Eq. 21 in place)
//     Eq. 10  W_G = H^T · HW_G        op 2 (tall-skinny, split-K, reading C2)
//
// The paper uses cuBLAS row-major SGEMM and states no precision
// (reading C17).  Here the fp32 operands are staged in shared memory by TMA,
// split in shared memory by 4 "transform" warps into tf32 hi + lo parts (and
// transposed into the K-major SWIZZLE_128B layout when the operand is stored
// K-outer), and one thread issues tcgen05.mma.kind::tf32 for hi·hi + hi·lo +
// lo·hi (3xTF32, ~fp32 accuracy) into a TMEM accumulator; 4 epilogue warps
// drain TMEM with tcgen05.ld, apply the fused epilogue and store.
//
// Warp roles (320 threads, one CTA per SM, persistent over output tiles):
//   warps 0-3 epilogue (TMEM lane quadrants 0-3), warps 4-7 transform,
//   warp 8 TMA producer, warp 9 TMEM allocator + MMA issuer.
// Pipelines (mbarriers): raw[2] TMA -> transform, split[2] transform -> MMA,
// accumulator[2] MMA -> epilogue (double-buffered TMEM, 2 x 128 columns).
#include <cuda.h>

#include <cstdio>
#include <cstdlib>
#include <mutex>

#include "kernels.cuh"

namespace mggcn {

namespace {

constexpr int BM = 128;          // UMMA_M (cta_group::1)
constexpr int BK = 32;           // 32 fp32 = 128 B = one SWIZZLE_128B row
constexpr int kMaxBN = 128;
#ifndef MGGCN_ROW_RAWB
#define MGGCN_ROW_RAWB 0          // 1: B_lo recomputed in smem from the raw W tile; 0: B_lo loaded by TMA (faster: profiles/r01_row_gemm_sweep.log)
#endif
#ifndef MGGCN_ROW_PF
#define MGGCN_ROW_PF 0            // row GEMM: L2 prefetch of the A box this many k blocks ahead (0 = off)
#endif
#ifndef MGGCN_ROW_DBG
#define MGGCN_ROW_DBG 0           // TIMING EXPERIMENTS ONLY (results invalid): 1 no MMAs, 2 no lo split, 4 no TMA loads
#endif
#ifndef MGGCN_ROW_XF_WARPS
#define MGGCN_ROW_XF_WARPS 4
#endif
constexpr int kXfWarps = MGGCN_ROW_XF_WARPS;      // transform (lo split) warps of the row GEMM
constexpr int kXfWarp0 = 4, kTmaWarp = 4 + kXfWarps, kMmaWarp = 5 + kXfWarps;
constexpr int kThreads = (6 + kXfWarps) * 32;
constexpr int kTmemCols = 256;   // 2 accumulators x 128 columns

// shared-memory map (bytes from a 1024-B aligned base)
constexpr int kRawA = 0;                    // 2 x 16 KB
constexpr int kRawB = 2 * 16384;            // 2 x 16 KB
constexpr int kAhi = 4 * 16384;
constexpr int kAlo = 6 * 16384;
constexpr int kBhi = 8 * 16384;
constexpr int kBlo = 10 * 16384;
constexpr int kBars = 12 * 16384;           // 12 mbarriers + TMEM slot
constexpr int kSmemBytes = kBars + 256 + 1024;

struct KParams {
    int M, N, K;
    int BN, m_tiles, n_tiles, k_chunks, k_chunk_len;
    float* C;
    int64_t ldc;
    float* partial;
    const float* rowscale;
    int flags;
    int op2;
    uint32_t desc_mn[3];
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred P1;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
        "@!P1 bra WAIT_%=;\n}\n" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}

__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* tm, int c0, int c1, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
            smem_u32(dst)),
        "l"((uint64_t)tm), "r"(c0), "r"(c1), "r"(smem_u32(bar))
        : "memory");
}

// L2 prefetch of a tensor box (no shared-memory destination, no completion)
__device__ __forceinline__ void tma_prefetch_2d(const CUtensorMap* tm, int c0, int c1) {
    asm volatile("cp.async.bulk.prefetch.tensor.2d.L2.global.tile [%0, {%1, %2}];" ::"l"((uint64_t)tm), "r"(c0), "r"(c1)
                 : "memory");
}

__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// K-major, SWIZZLE_128B shared-memory matrix descriptor (sm_100 format):
// start>>4 [0,14), LBO>>4 [16,30) (unused for swizzled K-major), SBO>>4 [32,46)
// = 1024 B between 8-row groups, version 1 at [46,48), layout 2 = SW128 at [61,64).
__device__ __forceinline__ uint64_t sw128_desc(uint32_t saddr) {
    return (uint64_t)((saddr & 0x3FFFFu) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
           ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}

__device__ __forceinline__ void mma_tf32(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                         uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}

__device__ __forceinline__ void mma_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
                 : "memory");
}

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, float* v) {
    uint32_t r[16];
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
        "%15}, [%16];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
    for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
}

// fp32 -> (hi, lo) with hi exactly representable in tf32 (10-bit mantissa).
__device__ __forceinline__ void split_tf32(float x, float& hi, float& lo, bool x1) {
    if (x1) {
        uint32_t t;
        asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(t) : "f"(x));
        hi = __uint_as_float(t);
        lo = 0.f;
    } else {
        hi = __uint_as_float(__float_as_uint(x) & 0xFFFFE000u);
        lo = x - hi;
    }
}

__device__ __forceinline__ void split4(float4 x, float4& hi, float4& lo, bool x1) {
    split_tf32(x.x, hi.x, lo.x, x1);
    split_tf32(x.y, hi.y, lo.y, x1);
    split_tf32(x.z, hi.z, lo.z, x1);
    split_tf32(x.w, hi.w, lo.w, x1);
}

// Fused epilogue store of 16 accumulator columns [nb, nb+16) of `row`:
// ReLU' mask from the old value (Eq. 8 / Eq. 21 in place), inv_deg row scale,
// ReLU (Eq. 7); 128-bit stores when the 16 columns are all valid.
__device__ __forceinline__ void store_epilogue(const KParams& p, int row, int nb, const float* v, float sc) {
    float* dst = p.C + (int64_t)row * p.ldc + nb;
    if (nb + 16 <= p.N) {
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            float4 o = make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
            if (p.flags & GEMM_MASK) {
                const float4 old = reinterpret_cast<const float4*>(dst)[q];
                o.x = old.x > 0.f ? o.x : 0.f;
                o.y = old.y > 0.f ? o.y : 0.f;
                o.z = old.z > 0.f ? o.z : 0.f;
                o.w = old.w > 0.f ? o.w : 0.f;
            }
            o.x *= sc; o.y *= sc; o.z *= sc; o.w *= sc;
            if (p.flags & GEMM_RELU) {
                o.x = fmaxf(o.x, 0.f); o.y = fmaxf(o.y, 0.f);
                o.z = fmaxf(o.z, 0.f); o.w = fmaxf(o.w, 0.f);
            }
            reinterpret_cast<float4*>(dst)[q] = o;
        }
    } else {
        for (int i = 0; i < 16 && nb + i < p.N; ++i) {
            float o = v[i];
            if ((p.flags & GEMM_MASK) && !(dst[i] > 0.f)) o = 0.f;
            o *= sc;
            if (p.flags & GEMM_RELU) o = fmaxf(o, 0.f);
            dst[i] = o;
        }
    }
}

// ==================================================================== wgrad
// Weight-gradient GEMM (op 2, Eq. 10): partial[kc] = A^T B over one K chunk,
// A [K x M] and B [K x N] both stored K-outer (the feature matrices).
// (MN-major operand descriptors with kind::tf32 produced all-zero
// accumulators on B200 in our tests, so the operands are transposed.)
// K blocks of 16: raw tiles [16 k][M or N] come in by TMA (3 stages, no
// swizzle); 8 warps transpose + split them into K-major SWIZZLE_64B hi / lo
// operand buffers (3 stages) so the transform of block kb+1 overlaps the MMAs
// of block kb; warp 9 issues hi.hi + hi.lo + lo.hi per 8-deep k step; warps
// 0-3 drain the TMEM accumulator into the split-K partial buffer.
constexpr int kWgBK = 16;
constexpr int kWgNR = 5;                         // raw (TMA) stages
constexpr int kWgNS = 2;                         // split (MMA operand) stages
constexpr int kWgRawA = 0;                       // 3 x  8 KB  raw A [16 k][128 m]
constexpr int kWgRawB = kWgNR * 8192;            // 5 x 16 KB  raw B [16 k][<=256 n]
constexpr int kWgSplit = kWgRawB + kWgNR * 16384;  // 2 x 48 KB: A_hi 8K | A_lo 8K | B_hi 16K | B_lo 16K
constexpr int kWgSplitStage = 49152;
constexpr int kWgBars = kWgSplit + kWgNS * kWgSplitStage;
constexpr int kWgSmem = kWgBars + 256 + 1024;
constexpr int kWgXfThreads = 512;                // warps 0-15 transform (0-3 also epilogue)
constexpr int kWgTmaWarp = 16, kWgMmaWarp = 17, kWgThreads = 576;

// K-major SWIZZLE_64B descriptor: rows of 64 B (16 tf32), 8-row atoms 512 B apart.
__device__ __forceinline__ uint64_t sw64_desc(uint32_t saddr) {
    return (uint64_t)((saddr & 0x3FFFFu) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(512 >> 4) << 32) |
           ((uint64_t)1 << 46) | ((uint64_t)4 << 61);
}

// raw[kk][r] (pitch `rows`, kk < 16) -> K-major SW64: element (r, k) at
// r*64 + (((k>>2) ^ ((r>>1)&3)) << 4) + (k&3)*4.  Thread t owns row
// r = t % rows and the k-quads kq = g, g+G, ... (g = t / rows, G = NT / rows);
// the offsets are computed once per kernel, and all shared loads of a k block
// are issued before the first split (ILP).
struct XfPlan {
    bool ok[4];       // k-quad j is owned by this thread
    int ld[4];        // float index of raw[(4 kq) * rows + r]
    int st[4];        // byte offset in the SW64 operand tile
    int rows;
};

__device__ __forceinline__ XfPlan make_xf_plan(int rows, int t, int NT) {
    XfPlan pl;
    pl.rows = rows;
    const int G = NT / rows;
    const int g = t / rows, r = t - g * rows;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        const int kq = g + j * G;
        pl.ok[j] = g < G && kq < 4;
        pl.ld[j] = 4 * kq * rows + r;
        pl.st[j] = r * 64 + ((kq ^ ((r >> 1) & 3)) << 4);
    }
    return pl;
}

__device__ __forceinline__ void transpose_split16(const float* __restrict__ raw, uint8_t* hi, uint8_t* lo,
                                                  const XfPlan& pl, bool x1) {
    float4 a[4];
#pragma unroll
    for (int j = 0; j < 4; ++j)
        if (pl.ok[j]) {
            const float* q = raw + pl.ld[j];
            a[j].x = q[0];
            a[j].y = q[pl.rows];
            a[j].z = q[2 * pl.rows];
            a[j].w = q[3 * pl.rows];
        }
#pragma unroll
    for (int j = 0; j < 4; ++j)
        if (pl.ok[j]) {
            float4 ah, al;
            split4(a[j], ah, al, x1);
            *reinterpret_cast<float4*>(hi + pl.st[j]) = ah;
            if (!x1) *reinterpret_cast<float4*>(lo + pl.st[j]) = al;
        }
}

__global__ void __launch_bounds__(kWgThreads, 1)
gemm_wgrad_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB, const KParams p) {
    extern __shared__ uint8_t smem_dyn[];
    uint8_t* smem = smem_dyn + ((1024u - (smem_u32(smem_dyn) & 1023u)) & 1023u);   // keeps the shared state space
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + kWgBars);
    uint64_t* raw_full = bars + 0;               // [kWgNR]
    uint64_t* raw_empty = bars + kWgNR;          // [kWgNR]
    uint64_t* split_full = bars + 2 * kWgNR;     // [kWgNS]
    uint64_t* split_empty = bars + 2 * kWgNR + kWgNS;
    uint64_t* tmem_full = bars + 2 * kWgNR + 2 * kWgNS;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tmem_full + 1);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const bool x1 = (p.flags & GEMM_TF32X1) != 0;
    const int BN = p.BN;
    const uint32_t tcols = BN > 128 ? 256u : 128u;
    const int tile = blockIdx.x;
    const int nt = tile % p.n_tiles;
    const int mt = (tile / p.n_tiles) % p.m_tiles;
    const int kc = tile / (p.n_tiles * p.m_tiles);
    const int k0 = kc * p.k_chunk_len;
    const int k1 = min(p.K, k0 + p.k_chunk_len);
    const int nkb = (k1 - k0 + kWgBK - 1) / kWgBK;

    if (threadIdx.x == 0) {
        for (int s = 0; s < kWgNR; ++s) {
            mbar_init(raw_full + s, 1);
            mbar_init(raw_empty + s, kWgXfThreads);
        }
        for (int s = 0; s < kWgNS; ++s) {
            mbar_init(split_full + s, kWgXfThreads);
            mbar_init(split_empty + s, 1);
        }
        mbar_init(tmem_full, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == kWgMmaWarp) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                     "r"(tcols));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == kWgTmaWarp) {
        if (lane == 0) {
            const uint32_t bytes = (uint32_t)(BM * kWgBK * 4 + BN * kWgBK * 4);
            int s = 0;
            uint32_t ph = 0;
            for (int kb = 0; kb < nkb; ++kb) {
                mbar_wait(raw_empty + s, ph ^ 1);
                mbar_expect_tx(raw_full + s, bytes);
                tma_load_2d(smem + kWgRawA + s * 8192, &tmA, mt * BM, k0 + kb * kWgBK, raw_full + s);
                tma_load_2d(smem + kWgRawB + s * 16384, &tmB, nt * BN, k0 + kb * kWgBK, raw_full + s);
                if (++s == kWgNR) { s = 0; ph ^= 1; }
            }
        }
    } else if (warp == kWgMmaWarp) {
        if (lane == 0) {
            const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(BN >> 3) << 17) |
                                   ((uint32_t)(BM >> 4) << 24);
            int s = 0;
            uint32_t ph = 0;
            for (int kb = 0; kb < nkb; ++kb) {
                mbar_wait(split_full + s, ph);
                tc_fence_after();
                const uint32_t base = smem_u32(smem + kWgSplit + s * kWgSplitStage);
                const uint64_t ah = sw64_desc(base), al = sw64_desc(base + 8192);
                const uint64_t bh = sw64_desc(base + 16384), bl = sw64_desc(base + 32768);
#pragma unroll
                for (int kk = 0; kk < kWgBK / 8; ++kk) {
                    const uint64_t adv = (uint64_t)((kk * 8 * 4) >> 4);   // 32 B per 8-deep k step
                    if (!x1) {
                        mma_tf32(tmem_base, al + adv, bh + adv, idesc, (kb | kk) ? 1u : 0u);
                        mma_tf32(tmem_base, ah + adv, bl + adv, idesc, 1u);
                        mma_tf32(tmem_base, ah + adv, bh + adv, idesc, 1u);
                    } else {
                        mma_tf32(tmem_base, ah + adv, bh + adv, idesc, (kb | kk) ? 1u : 0u);
                    }
                }
                mma_commit(split_empty + s);
                if (++s == kWgNS) { s = 0; ph ^= 1; }
            }
            mma_commit(tmem_full);
        }
    } else {
        // warps 0-7: transpose + split every k block; then warps 0-3 run the epilogue
        const int t = threadIdx.x;
        const XfPlan pa = make_xf_plan(BM, t, kWgXfThreads), pb = make_xf_plan(BN, t, kWgXfThreads);
        int rs = 0, ss = 0;
        uint32_t rph = 0, sph = 0;
        for (int kb = 0; kb < nkb; ++kb) {
            uint8_t* sp = smem + kWgSplit + ss * kWgSplitStage;
            mbar_wait(raw_full + rs, rph);
            mbar_wait(split_empty + ss, sph ^ 1);
            transpose_split16(reinterpret_cast<const float*>(smem + kWgRawA + rs * 8192), sp, sp + 8192, pa, x1);
            transpose_split16(reinterpret_cast<const float*>(smem + kWgRawB + rs * 16384), sp + 16384, sp + 32768,
                              pb, x1);
            mbar_arrive(raw_empty + rs);     // raw tile consumed (generic reads done)
            fence_proxy_async();
            mbar_arrive(split_full + ss);
            if (++rs == kWgNR) { rs = 0; rph ^= 1; }
            if (++ss == kWgNS) { ss = 0; sph ^= 1; }
        }
        if (warp < 4) {
            mbar_wait(tmem_full, 0);
            tc_fence_after();
            const int row = mt * BM + warp * 32 + lane;
            const int n0 = nt * BN;
            for (int c0 = 0; c0 < BN; c0 += 16) {
                float v[16];
                tmem_ld16(tmem_base + ((uint32_t)(warp * 32) << 16) + (uint32_t)c0, v);
                const int nb = n0 + c0;
                if (row >= p.M || nb >= p.N) continue;
                float* dst = p.partial + ((int64_t)kc * p.M + row) * (int64_t)p.N + nb;
#pragma unroll
                for (int i = 0; i < 16; ++i)
                    if (nb + i < p.N) dst[i] = v[i];
            }
            tc_fence_before();
        }
    }
    __syncthreads();
    if (warp == kWgMmaWarp) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(tcols));
    }
}

// ------------------------------------------------ wgrad, MN-major variant
// Same product and split-K tiling as gemm_wgrad_kernel, but the K-outer
// operands are consumed in place: tcgen05 kind::tf32 accepts MN-major
// shared-memory operands in the 128B-swizzle / 32B-atom layout
// (SWIZZLE_128B_BASE32B: LBO = stride of 32-float MN chunks, SBO = stride of
// 4-row k groups), which TMA writes directly (CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B,
// boxes of 32 MN-contiguous floats x 16 k rows).  No transpose.
// 3xTF32: the MMA reads an fp32 operand as tf32 by ignoring the low 13
// mantissa bits, i.e. as hi = x & 0xFFFFE000 -- so the raw TMA tile IS the hi
// operand and 4 warps only compute lo = x - hi into a separate ring (1xTF32:
// the raw tile is rounded to nearest in place instead).  Rings: 6 raw stages
// (TMA -> MMA, 24 KB) and 2 lo stages; 192 threads: warps 0-3 lo + epilogue,
// warp 4 TMA, warp 5 TMEM allocator + MMA issuer.
constexpr int kMnBK = 16;
// Rings of stages of A 8K (4 boxes) | B nbox_b x 2K: raw (TMA -> MMA) and lo
// (split -> MMA), sized from BN so narrow-N products keep more k blocks of
// the streamed operands in flight (BN = 256: 6 raw + 2 lo stages of 24 KB;
// BN = 64: 10 raw + 4 lo stages of 12 KB).
#ifndef MGGCN_MN_BUDGET
#define MGGCN_MN_BUDGET (8 * 24576)
#endif
#ifndef MGGCN_MN_MAXNR
#define MGGCN_MN_MAXNR 10
#endif
constexpr int kMnBudget = MGGCN_MN_BUDGET;
constexpr int kMnMaxNR = MGGCN_MN_MAXNR, kMnMaxNL = 4;
constexpr int kMnBars = kMnBudget;
constexpr int kMnSmem = kMnBars + 512 + 1024;
__host__ __device__ __forceinline__ int mn_stage_bytes(int BN) { return 8192 + (BN / 32) * 2048; }
__host__ __device__ __forceinline__ int mn_lo_stages(int BN) { return mn_stage_bytes(BN) <= 12288 ? kMnMaxNL : 2; }
__host__ __device__ __forceinline__ int mn_raw_stages(int BN) {
    const int nr = (kMnBudget - mn_lo_stages(BN) * mn_stage_bytes(BN)) / mn_stage_bytes(BN);
    return nr < kMnMaxNR ? nr : kMnMaxNR;
}
#ifndef MGGCN_MN_LO_WARPS
#define MGGCN_MN_LO_WARPS 12
#endif
constexpr int kMnLoWarps = MGGCN_MN_LO_WARPS;    // lo-split warps (0-3 also run the epilogue)
constexpr int kMnThreads = (kMnLoWarps + 2) * 32, kMnTmaWarp = kMnLoWarps, kMnMmaWarp = kMnLoWarps + 1;

__device__ __forceinline__ uint64_t mn_desc(uint32_t saddr, const uint32_t* d) {
    return (uint64_t)((saddr & 0x3FFFFu) >> 4) | ((uint64_t)((d[1] >> 4) & 0x3FFFu) << 16) |
           ((uint64_t)((d[2] >> 4) & 0x3FFFu) << 32) | ((uint64_t)1 << 46) | ((uint64_t)(d[0] & 7u) << 61);
}

__global__ void __launch_bounds__(kMnThreads, 1)
gemm_wgrad_mn_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                     const KParams p) {
    extern __shared__ uint8_t smem_dyn[];
    uint8_t* smem = smem_dyn + ((1024u - (smem_u32(smem_dyn) & 1023u)) & 1023u);
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + kMnBars);
    uint64_t* full = bars;                       // [NR] TMA -> lo warps
    uint64_t* ready = bars + kMnMaxNR;           // [NR] lo warps -> MMA
    uint64_t* empty = bars + 2 * kMnMaxNR;       // [NR] MMA -> TMA
    uint64_t* lo_free = bars + 3 * kMnMaxNR;     // [NL] MMA -> lo warps
    uint64_t* tmem_full = lo_free + kMnMaxNL;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tmem_full + 1);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const bool x1 = (p.flags & GEMM_TF32X1) != 0;
    const int BN = p.BN;
    const uint32_t tcols = BN > 128 ? 256u : BN > 64 ? 128u : 64u;
    const int tile = blockIdx.x;
    const int nt = tile % p.n_tiles;
    const int mt = (tile / p.n_tiles) % p.m_tiles;
    const int kc = tile / (p.n_tiles * p.m_tiles);
    const int k0 = kc * p.k_chunk_len;
    const int k1 = min(p.K, k0 + p.k_chunk_len);
    const int nkb = (k1 - k0 + kMnBK - 1) / kMnBK;
    const int nbox_b = BN / 32;
    const int SB = mn_stage_bytes(BN), NR = mn_raw_stages(BN), NL = mn_lo_stages(BN);
    uint8_t* const lo0 = smem + NR * SB;

    if (threadIdx.x == 0) {
        for (int s = 0; s < NR; ++s) {
            mbar_init(full + s, 1);
            mbar_init(ready + s, kMnLoWarps * 32);
            mbar_init(empty + s, 1);
        }
        for (int s = 0; s < NL; ++s) mbar_init(lo_free + s, 1);
        mbar_init(tmem_full, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == kMnMmaWarp) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                     "r"(tcols));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == kMnTmaWarp) {
        if (lane == 0) {
            const uint32_t bytes = (uint32_t)((4 + nbox_b) * 2048);
            int s = 0;
            uint32_t ph = 0;
            for (int kb = 0; kb < nkb; ++kb) {
                uint8_t* st = smem + s * SB;
                mbar_wait(empty + s, ph ^ 1);
                mbar_expect_tx(full + s, bytes);
                const int kr = k0 + kb * kMnBK;
                for (int j = 0; j < 4; ++j) tma_load_2d(st + j * 2048, &tmA, mt * BM + 32 * j, kr, full + s);
                for (int j = 0; j < nbox_b; ++j)
                    tma_load_2d(st + 8192 + j * 2048, &tmB, nt * BN + 32 * j, kr, full + s);
                if (++s == NR) { s = 0; ph ^= 1; }
            }
        }
    } else if (warp == kMnMmaWarp) {
        if (lane == 0) {
            const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | (1u << 15) | (1u << 16) |
                                   ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
            int s = 0, l = 0;
            uint32_t ph = 0;
            for (int kb = 0; kb < nkb; ++kb) {
                mbar_wait(ready + s, ph);
                tc_fence_after();
                const uint32_t raw = smem_u32(smem + s * SB), lo = smem_u32(lo0 + l * SB);
#pragma unroll
                for (int kk = 0; kk < kMnBK / 8; ++kk) {
                    const uint32_t off = kk * 8 * 128;   // 8 k rows of 128 B
                    const uint64_t ah = mn_desc(raw + off, p.desc_mn), bh = mn_desc(raw + 8192 + off, p.desc_mn);
                    if (!x1) {
                        const uint64_t al = mn_desc(lo + off, p.desc_mn), bl = mn_desc(lo + 8192 + off, p.desc_mn);
                        mma_tf32(tmem_base, al, bh, idesc, (kb | kk) ? 1u : 0u);
                        mma_tf32(tmem_base, ah, bl, idesc, 1u);
                        mma_tf32(tmem_base, ah, bh, idesc, 1u);
                    } else {
                        mma_tf32(tmem_base, ah, bh, idesc, (kb | kk) ? 1u : 0u);
                    }
                }
                mma_commit(empty + s);
                mma_commit(lo_free + l);
                if (++s == NR) { s = 0; ph ^= 1; }
                if (++l == NL) l = 0;
            }
            mma_commit(tmem_full);
        }
    } else {
        // warps 0-3: lo = x - hi of every staged tile (1xTF32: round the tile in place)
        const int t = threadIdx.x;
        const int nA4 = 4 * 2048 / 16, nT4 = nA4 + nbox_b * 2048 / 16;   // float4 counts
        int s = 0, l = 0;
        uint32_t ph = 0, lph = 0;
        for (int kb = 0; kb < nkb; ++kb) {
            uint8_t* st = smem + s * SB;
            uint8_t* lb = lo0 + l * SB;
            mbar_wait(full + s, ph);
            if (!x1) mbar_wait(lo_free + l, lph ^ 1);
            for (int i = t; i < nT4; i += kMnLoWarps * 32) {
                float4* hp = reinterpret_cast<float4*>(st + i * 16);
                float4 hi, lo;
                split4(*hp, hi, lo, x1);
                if (x1) *hp = hi;
                else *reinterpret_cast<float4*>(lb + i * 16) = lo;
            }
            fence_proxy_async();
            mbar_arrive(ready + s);
            if (++s == NR) { s = 0; ph ^= 1; }
            if (++l == NL) { l = 0; lph ^= 1; }
        }
        if (warp < 4) {
            mbar_wait(tmem_full, 0);
            tc_fence_after();
            const int row = mt * BM + warp * 32 + lane;
            const int n0 = nt * BN;
            for (int c0 = 0; c0 < BN; c0 += 16) {
                float v[16];
                tmem_ld16(tmem_base + ((uint32_t)(warp * 32) << 16) + (uint32_t)c0, v);
                const int nb = n0 + c0;
                if (row >= p.M || nb >= p.N) continue;
                float* dst = p.partial + ((int64_t)kc * p.M + row) * (int64_t)p.N + nb;
#pragma unroll
                for (int i = 0; i < 16; ++i)
                    if (nb + i < p.N) dst[i] = v[i];
            }
            tc_fence_before();
        }
    }
    __syncthreads();
    if (warp == kMnMmaWarp) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(tcols));
    }
}

// ===================================================================== rows
// Row GEMM (op 0 / op 1): C[M x N] = A[M x K] · B^T with B given PRE-SPLIT as
// tf32 hi / lo copies in K-major [N x K] layout (the weights; split once per
// step by launch_split_weights).  K blocks of 16 (SWIZZLE_64B operands), 3
// stages: TMA writes raw A and B_hi / B_lo straight into the operand buffers;
// the 4 transform warps split A IN PLACE; BN = N up to 256 so A is staged
// once.  Epilogue: 32-column chunks go TMEM -> registers -> swizzled smem ->
// TMA bulk store (full 128-B lines); the old C values for the ReLU' mask of
// Eq. 8 / Eq. 21 come in by TMA into the same layout.
constexpr int kRowBK = 16;
// shared memory: 2 x 16 KB output chunks [128 rows][32 cols] SW128, 2 x 16 KB
// old-C chunks (mask), then the operand ring: stages of A 8K | A_lo 8K |
// B_hi BN x 64 B | B_lo BN x 64 B, as many as fit the budget (3 for BN = 256,
// 7 for BN = 48): narrow-N products are bound by the A stream, which needs
// more k blocks in flight than the MMAs do.
// Without the mask (forward F1, and B3 when no ReLU' applies) the old-C
// chunks are never loaded, so the ring starts at kRowOld and gets their 32 KB
// too (BN = 256: 3 -> 4 stages, BN = 48: 7 -> 8); MGGCN_ROW_RING=0 keeps the
// short ring for A/B.
constexpr int kRowOut = 0;
constexpr int kRowOld = 2 * 16384;
constexpr int kRowStage0 = 4 * 16384;
constexpr int kRowStageBudget = 160 * 1024;
constexpr int kRowMaxNS = 10;
constexpr int kRowBars = kRowStage0 + kRowStageBudget;
constexpr int kRowSmem = kRowBars + 512 + 1024;
constexpr int GEMM_ROW_LONGRING = 1 << 20;   // internal KParams flag: ring starts at kRowOld

__host__ __device__ __forceinline__ int row_stage_bytes(int BN) { return (16384 + 2 * BN * 64 + 1023) / 1024 * 1024; }
__host__ __device__ __forceinline__ int row_stages(int BN, bool longring = false) {
    const int ns = (kRowStageBudget + (longring ? kRowStage0 - kRowOld : 0)) / row_stage_bytes(BN);
    return ns < kRowMaxNS ? ns : kRowMaxNS;
}

__device__ __forceinline__ void tma_store_2d(const CUtensorMap* tm, int c0, int c1, const void* src) {
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];" ::"l"((uint64_t)tm),
                 "r"(c0), "r"(c1), "r"(smem_u32(src))
                 : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void epi_bar() { asm volatile("bar.sync 1, 128;" ::: "memory"); }

// ---- CTA-pair (cta_group::2) helpers
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// arrive on the barrier at the same shared-memory offset in CTA `rank` of the cluster
__device__ __forceinline__ void mbar_arrive_cluster(uint64_t* bar, uint32_t rank) {
    uint32_t ra;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(smem_u32(bar)), "r"(rank));
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(ra) : "memory");
}
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred P1;\n"
        "WAITC_%=:\n\t"
        "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P1, [%0], %1;\n\t"
        "@!P1 bra WAITC_%=;\n}\n" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void mma_tf32_pair(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                              uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::tf32 [%0], %1, %2, %3, p;\n}\n" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}
// completion of the pair's MMAs arrives on the barrier at this offset in BOTH CTAs
__device__ __forceinline__ void mma_commit_pair(uint64_t* bar) {
    asm volatile(
        "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
            smem_u32(bar)),
        "h"((unsigned short)3)
        : "memory");
}

// byte offset of (row r, 16-B chunk q) in a [128][32 fp32] SWIZZLE_128B tile
__device__ __forceinline__ int sw128_off(int r, int q) { return r * 128 + ((q ^ (r & 7)) << 4); }

// PAIR (opt-in, MGGCN_ROW_PAIR=1): a cluster of two CTAs on one TPC computes a
// 256 x BN tile with tcgen05.mma.cta_group::2 (M = 256): each CTA stages its
// own 128 rows of A and HALF of B (BN/2 rows of W^T), so the per-SM TMA feed
// per k block drops from A 8K + B 2 x 16K to A 8K + B 2 x 8K at BN = 256 (the
// feed, not the MMA rate, bounds the single-CTA kernel:
// profiles/r01_row_gemm_components.log).  Only CTA 0 issues MMAs; CTA 1's
// transform / epilogue warps sync locally and one thread arrives on CTA 0's
// xf / tmem_empty barrier; MMA completion is multicast to both CTAs.  It is
// correct but slower for 3xTF32 (each k step reads the peer's B half three
// times across SMs), so the single-CTA kernel stays the default.
template <bool PAIR>
__global__ void __launch_bounds__(kThreads, 1)
gemm_rows_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmBh,
                 const __grid_constant__ CUtensorMap tmBl, const __grid_constant__ CUtensorMap tmC, const KParams p) {
    extern __shared__ uint8_t smem_dyn[];
    uint8_t* smem = smem_dyn + ((1024u - (smem_u32(smem_dyn) & 1023u)) & 1023u);   // keeps the shared state space
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + kRowBars);
    uint64_t* full = bars + 0;                   // [kRowMaxNS]
    uint64_t* xf = bars + kRowMaxNS;             // [kRowMaxNS]
    uint64_t* empty = bars + 2 * kRowMaxNS;      // [kRowMaxNS]
    uint64_t* tmem_full = bars + 3 * kRowMaxNS;  // [2]
    uint64_t* tmem_empty = tmem_full + 2;        // [2]
    uint64_t* old_full = tmem_full + 4;          // [2]
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tmem_full + 6);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const bool x1 = (p.flags & GEMM_TF32X1) != 0;
    const bool mask = (p.flags & GEMM_MASK) != 0;
    const int BN = p.BN;
    const int BNH = PAIR ? BN / 2 : BN;         // rows of W^T staged by this CTA
    const uint32_t tcols = BN > 128 ? 512u : 256u;
    const bool longring = (p.flags & GEMM_ROW_LONGRING) != 0 && !mask;
    const int NS = row_stages(BNH, longring), SB = row_stage_bytes(BNH);
    uint8_t* const ring = smem + (longring ? kRowOld : kRowStage0);
    const int kBlo = 16384 + BNH * 64;           // B_lo offset within a stage
    const uint32_t crank = PAIR ? cluster_rank() : 0u;
    const int nunits = PAIR ? (int)(gridDim.x / 2) : (int)gridDim.x;    // tile workers (CTA pairs or CTAs)
    const int unit = PAIR ? (int)(blockIdx.x / 2) : (int)blockIdx.x;

    if (threadIdx.x == 0) {
        for (int s = 0; s < NS; ++s) {
            mbar_init(full + s, 1);
            mbar_init(xf + s, kXfWarps * 32 + (PAIR ? 1 : 0));   // PAIR: + one arrival from CTA 1
            mbar_init(empty + s, 1);
        }
        for (int s = 0; s < 2; ++s) {
            mbar_init(tmem_full + s, 1);
            mbar_init(tmem_empty + s, 128 + (PAIR ? 1 : 0));
            mbar_init(old_full + s, 1);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == kMmaWarp) {
        if (PAIR) {
            asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                             smem_u32(tmem_slot)),
                         "r"(tcols));
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
        } else {
            asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                             smem_u32(tmem_slot)),
                         "r"(tcols));
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
        }
    }
    tc_fence_before();
    __syncthreads();
    if (PAIR) cluster_sync_all();                // both CTAs' barriers exist before any remote arrive
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    const int total_tiles = (PAIR ? (p.m_tiles + 1) / 2 : p.m_tiles) * p.n_tiles;
    const int nkb = (p.K + kRowBK - 1) / kRowBK;

    if (warp == kTmaWarp) {
        if (lane == 0) {
            const uint32_t bytes = (uint32_t)(BM * kRowBK * 4 + BNH * kRowBK * 4 * (MGGCN_ROW_RAWB || x1 ? 1 : 2));
            int s = 0;
            uint32_t ph = 0;
            for (int tile = unit; tile < total_tiles; tile += nunits) {
                const int nt = tile % p.n_tiles, mt = PAIR ? (tile / p.n_tiles) * 2 + (int)crank : tile / p.n_tiles;
                const int nb = nt * BN + (int)crank * BNH;   // first W^T row staged here
                for (int kb = 0; kb < nkb; ++kb) {
                    uint8_t* st = ring + s * SB;
                    if (!PAIR && MGGCN_ROW_PF > 0) {   // A streams from DRAM: warm L2 ahead of the ring
                        const int kp = kb + MGGCN_ROW_PF;
                        if (kp < nkb) tma_prefetch_2d(&tmA, kp * kRowBK, mt * BM);
                        else if (tile + (int)gridDim.x < total_tiles)
                            tma_prefetch_2d(&tmA, (kp - nkb) * kRowBK, ((tile + gridDim.x) / p.n_tiles) * BM);
                    }
                    mbar_wait(empty + s, ph ^ 1);
                    if (MGGCN_ROW_DBG & 4) {
                        mbar_arrive(full + s);
                    } else {
                        mbar_expect_tx(full + s, bytes);
                        tma_load_2d(st, &tmA, kb * kRowBK, mt * BM, full + s);
                        tma_load_2d(st + 16384, &tmBh, kb * kRowBK, nb, full + s);
                        if (!MGGCN_ROW_RAWB && !x1) tma_load_2d(st + kBlo, &tmBl, kb * kRowBK, nb, full + s);
                    }
                    if (++s == NS) { s = 0; ph ^= 1; }
                }
            }
        }
    } else if (warp >= kXfWarp0 && warp < kXfWarp0 + kXfWarps) {
        const int t = threadIdx.x - kXfWarp0 * 32;
        int s = 0;
        uint32_t ph = 0;
        for (int tile = unit; tile < total_tiles; tile += nunits) {
            for (int kb = 0; kb < nkb; ++kb) {
                float4* a = reinterpret_cast<float4*>(ring + s * SB);
                mbar_wait(full + s, ph);
                // raw A [0, 512) -> lo at +512; raw B [1024, 1024 + 4 BN) -> lo at +4 BN (float4
                // units, same swizzled offsets).  3xTF32: the MMA reads a raw x as hi = x &
                // 0xFFFFE000 itself, so only lo = x - hi is written (B's lo is recomputed per
                // tile instead of loaded: 40 -> 24 KB of TMA per k block at BN = 256).
                const int nA = BM * 4, nT = nA + (MGGCN_ROW_RAWB ? BNH * 4 : 0);
                for (int c = t; c < ((MGGCN_ROW_DBG & 2) ? 0 : nT); c += kXfWarps * 32) {
                    const int src = c < nA ? c : 1024 + (c - nA);
                    const int dst = src + (c < nA ? nA : BNH * 4);
                    float4 v = a[src], h, l;
                    split4(v, h, l, x1);
                    if (x1) a[src] = h;    // 1xTF32: round to nearest in place
                    else a[dst] = l;
                }
                fence_proxy_async();
                if (PAIR && crank != 0) {   // CTA 1: one release.cluster arrival on CTA 0's barrier
                    asm volatile("bar.sync 2, %0;" ::"n"(kXfWarps * 32) : "memory");
                    if (t == 0) mbar_arrive_cluster(xf + s, 0);
                } else {
                    mbar_arrive(xf + s);
                }
                if (++s == NS) { s = 0; ph ^= 1; }
            }
        }
    } else if (warp == kMmaWarp) {
        if (lane == 0 && crank == 0) {
            const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(BN >> 3) << 17) |
                                   ((uint32_t)((PAIR ? 2 * BM : BM) >> 4) << 24);
            int s = 0;
            uint32_t ph = 0, tc = 0;
            for (int tile = unit; tile < total_tiles; tile += nunits, ++tc) {
                const int acc = tc & 1;
                const uint32_t aph = (tc >> 1) & 1;
                if (PAIR) mbar_wait_cluster(tmem_empty + acc, aph ^ 1);
                else mbar_wait(tmem_empty + acc, aph ^ 1);
                tc_fence_after();
                const uint32_t d_tmem = tmem_base + (uint32_t)(acc * BN);
                for (int kb = 0; kb < nkb; ++kb) {
                    if (PAIR) mbar_wait_cluster(xf + s, ph);
                    else mbar_wait(xf + s, ph);
                    tc_fence_after();
                    const uint32_t base = smem_u32(ring + s * SB);
                    const uint64_t ah = sw64_desc(base), al = sw64_desc(base + 8192);
                    const uint64_t bh = sw64_desc(base + 16384), bl = sw64_desc(base + kBlo);
#pragma unroll
                    for (int kk = 0; kk < ((MGGCN_ROW_DBG & 1) ? 0 : kRowBK / 8); ++kk) {
                        const uint64_t adv = (uint64_t)((kk * 8 * 4) >> 4);
                        if (PAIR) {
                            if (!x1) {
                                mma_tf32_pair(d_tmem, al + adv, bh + adv, idesc, (kb | kk) ? 1u : 0u);
                                mma_tf32_pair(d_tmem, ah + adv, bl + adv, idesc, 1u);
                                mma_tf32_pair(d_tmem, ah + adv, bh + adv, idesc, 1u);
                            } else {
                                mma_tf32_pair(d_tmem, ah + adv, bh + adv, idesc, (kb | kk) ? 1u : 0u);
                            }
                        } else if (!x1) {   // small products first
                            mma_tf32(d_tmem, al + adv, bh + adv, idesc, (kb | kk) ? 1u : 0u);
                            mma_tf32(d_tmem, ah + adv, bl + adv, idesc, 1u);
                            mma_tf32(d_tmem, ah + adv, bh + adv, idesc, 1u);
                        } else {
                            mma_tf32(d_tmem, ah + adv, bh + adv, idesc, (kb | kk) ? 1u : 0u);
                        }
                    }
                    if (PAIR) mma_commit_pair(empty + s);
                    else mma_commit(empty + s);
                    if (++s == NS) { s = 0; ph ^= 1; }
                }
                if (PAIR) mma_commit_pair(tmem_full + acc);
                else mma_commit(tmem_full + acc);
            }
        }
    } else {
        // ---- epilogue warps 0-3: thread = accumulator row (TMEM lane quadrant = warp)
        const int r = warp * 32 + lane;
        const bool leader = threadIdx.x == 0;
        uint32_t tc = 0, chunk_ctr = 0;
        const int nch = (BN + 31) / 32;
        for (int tile = unit; tile < total_tiles; tile += nunits, ++tc) {
            const int nt = tile % p.n_tiles, mt = PAIR ? (tile / p.n_tiles) * 2 + (int)crank : tile / p.n_tiles;
            const int acc = tc & 1;
            const uint32_t aph = (tc >> 1) & 1;
            const int row = mt * BM + r;
            const float sc = ((p.flags & GEMM_SCALE) && row < p.M) ? __ldg(p.rowscale + row) : 1.f;
            const uint32_t c_base = chunk_ctr;
            if (mask && leader)   // prefetch the old values of the first two chunks
                for (int c = 0; c < 2 && c < nch; ++c) {
                    const int b = (c_base + c) & 1;
                    mbar_expect_tx(old_full + b, 16384);
                    tma_load_2d(smem + kRowOld + b * 16384, &tmC, nt * BN + 32 * c, mt * BM, old_full + b);
                }
            mbar_wait(tmem_full + acc, aph);
            tc_fence_after();
            for (int c = 0; c < nch; ++c, ++chunk_ctr) {
                const int b = chunk_ctr & 1;
                uint8_t* ob = smem + kRowOut + b * 16384;
                float v[32];
                const uint32_t ta = tmem_base + ((uint32_t)(warp * 32) << 16) + (uint32_t)(acc * BN + 32 * c);
                tmem_ld16(ta, v);
                tmem_ld16(ta + 16, v + 16);
                if (leader) bulk_wait_read<1>();   // the store that last used `ob` has read it
                if (mask) mbar_wait(old_full + b, (chunk_ctr >> 1) & 1);
                epi_bar();
                const uint8_t* oldb = smem + kRowOld + b * 16384;
#pragma unroll
                for (int q = 0; q < 8; ++q) {
                    float4 o = make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
                    if (mask) {
                        const float4 old = *reinterpret_cast<const float4*>(oldb + sw128_off(r, q));
                        o.x = old.x > 0.f ? o.x : 0.f;
                        o.y = old.y > 0.f ? o.y : 0.f;
                        o.z = old.z > 0.f ? o.z : 0.f;
                        o.w = old.w > 0.f ? o.w : 0.f;
                    }
                    o.x *= sc; o.y *= sc; o.z *= sc; o.w *= sc;
                    if (p.flags & GEMM_RELU) {
                        o.x = fmaxf(o.x, 0.f); o.y = fmaxf(o.y, 0.f);
                        o.z = fmaxf(o.z, 0.f); o.w = fmaxf(o.w, 0.f);
                    }
                    *reinterpret_cast<float4*>(ob + sw128_off(r, q)) = o;
                }
                fence_proxy_async();
                epi_bar();
                if (leader) {
                    tma_store_2d(&tmC, nt * BN + 32 * c, mt * BM, ob);
                    bulk_commit();
                    if (mask && c + 2 < nch) {   // old values of chunk c+2 into the buffer just consumed
                        mbar_expect_tx(old_full + b, 16384);
                        tma_load_2d(smem + kRowOld + b * 16384, &tmC, nt * BN + 32 * (c + 2), mt * BM, old_full + b);
                    }
                }
            }
            tc_fence_before();
            if (PAIR && crank != 0) {       // CTA 1: one arrival on CTA 0's barrier
                epi_bar();
                if (leader) mbar_arrive_cluster(tmem_empty + acc, 0);
            } else {
                mbar_arrive(tmem_empty + acc);
            }
        }
        if (leader) bulk_wait_read<0>();
    }
    __syncthreads();
    if (PAIR) cluster_sync_all();                // the peer's MMAs / arrivals are done
    if (warp == kMmaWarp) {
        tc_fence_after();
        if (PAIR)
            asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(tcols));
        else
            asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(tcols));
    }
}

// tf32 hi/lo split of a small matrix W (din x dout, row stride ldw) into the
// two K-major B layouts: T = W^T ([dout x din], stride ldt; op 0 uses it for
// H·W) and S = W ([din x dout], stride ldw; op 1 uses it for G·W^T).
__global__ void split_weights_kernel(const float* __restrict__ W, int din, int dout, int64_t ldw,
                                     float* __restrict__ t_hi, float* __restrict__ t_lo, int64_t ldt,
                                     float* __restrict__ s_hi, float* __restrict__ s_lo, int x1) {
    const int64_t total = (int64_t)din * dout;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        const int c = (int)(i / dout), k = (int)(i % dout);
        float hi, lo;
        const float w = W[c * ldw + k];
        split_tf32(w, hi, lo, x1 != 0);
        if (!x1) hi = w;   // the raw value: the MMA reads it as tf32 by truncation (= the hi part)
        if (t_hi) {
            t_hi[(int64_t)k * ldt + c] = hi;
            t_lo[(int64_t)k * ldt + c] = lo;
        }
        if (s_hi) {
            s_hi[(int64_t)c * ldw + k] = hi;
            s_lo[(int64_t)c * ldw + k] = lo;
        }
    }
}

// --------------------------------------------------------------- host side
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn get_encode() {
    static EncodeTiledFn fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* f = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<EncodeTiledFn>(f);
    });
    return fn;
}

// 2-D fp32 tensor map: dim0 = contiguous extent, dim1 = rows with stride ld floats.
int encode2d(CUtensorMap* m, const float* base, int64_t dim0, int64_t dim1, int64_t ld, int box0, int box1,
             bool swizzle128) {
    EncodeTiledFn fn = get_encode();
    if (!fn) return -1;
    cuuint64_t dims[2] = {(cuuint64_t)dim0, (cuuint64_t)dim1};
    cuuint64_t strides[1] = {(cuuint64_t)(ld * 4)};
    cuuint32_t box[2] = {(cuuint32_t)box0, (cuuint32_t)box1};
    cuuint32_t es[2] = {1, 1};
    CUresult r = fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims, strides, box, es,
                    CU_TENSOR_MAP_INTERLEAVE_NONE,
                    swizzle128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                    CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? 0 : -2;
}

// as encode2d with an explicit swizzle span (0, 64 or 128 bytes)
int encode2d_sw(CUtensorMap* m, const float* base, int64_t dim0, int64_t dim1, int64_t ld, int box0, int box1,
                int swizzle) {
    EncodeTiledFn fn = get_encode();
    if (!fn) return -1;
    cuuint64_t dims[2] = {(cuuint64_t)dim0, (cuuint64_t)dim1};
    cuuint64_t strides[1] = {(cuuint64_t)(ld * 4)};
    cuuint32_t box[2] = {(cuuint32_t)box0, (cuuint32_t)box1};
    cuuint32_t es[2] = {1, 1};
    const CUtensorMapSwizzle sw = swizzle == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                                  : swizzle == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                                  : CU_TENSOR_MAP_SWIZZLE_NONE;
    CUresult r = fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims, strides, box, es,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? 0 : -2;
}

// as encode2d with an explicit CUtensorMapSwizzle
int encode2d_mode(CUtensorMap* m, const float* base, int64_t dim0, int64_t dim1, int64_t ld, int box0, int box1,
                  CUtensorMapSwizzle sw) {
    EncodeTiledFn fn = get_encode();
    if (!fn) return -1;
    cuuint64_t dims[2] = {(cuuint64_t)dim0, (cuuint64_t)dim1};
    cuuint64_t strides[1] = {(cuuint64_t)(ld * 4)};
    cuuint32_t box[2] = {(cuuint32_t)box0, (cuuint32_t)box1};
    cuuint32_t es[2] = {1, 1};
    CUresult r = fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims, strides, box, es,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? 0 : -2;
}

int num_sms() {
    static int n = 0;
    if (n == 0) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}

cudaError_t launch_wgrad(const GemmPlan& g, const KParams& kp, cudaStream_t s) {
    static bool attr_set = false;
    if (!attr_set) {
        cudaError_t e = cudaFuncSetAttribute(gemm_wgrad_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kWgSmem);
        if (e != cudaSuccess) return e;
        attr_set = true;
    }
    gemm_wgrad_kernel<<<g.grid, kWgThreads, kWgSmem, s>>>(g.tmA, g.tmB, kp);
    count_launches(1);
    return cudaGetLastError();
}

cudaError_t launch_wgrad_mn(const GemmPlan& g, const KParams& kp, cudaStream_t s) {
    static bool attr_set = false;
    if (!attr_set) {
        cudaError_t e =
            cudaFuncSetAttribute(gemm_wgrad_mn_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kMnSmem);
        if (e != cudaSuccess) return e;
        attr_set = true;
    }
    gemm_wgrad_mn_kernel<<<g.grid, kMnThreads, kMnSmem, s>>>(g.tmA, g.tmB, kp);
    count_launches(1);
    return cudaGetLastError();
}

cudaError_t launch_rows(const GemmPlan& g, const KParams& kp, cudaStream_t s) {
    static bool attr_set = false;
    if (!attr_set) {
        cudaError_t e = cudaFuncSetAttribute(gemm_rows_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             kRowSmem);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(gemm_rows_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, kRowSmem);
        if (e != cudaSuccess) return e;
        attr_set = true;
    }
    if (g.variant == 2) {   // CTA pairs (cluster of 2, tcgen05 cta_group::2)
        cudaLaunchConfig_t cfg = {};
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = 2;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.gridDim = dim3((unsigned)g.grid);
        cfg.blockDim = dim3(kThreads);
        cfg.dynamicSmemBytes = kRowSmem;
        cfg.stream = s;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        cudaError_t e = cudaLaunchKernelEx(&cfg, gemm_rows_kernel<true>, g.tmA, g.tmB, g.tmB2, g.tmC, kp);
        count_launches(1);
        return e != cudaSuccess ? e : cudaGetLastError();
    }
    gemm_rows_kernel<false><<<g.grid, kThreads, kRowSmem, s>>>(g.tmA, g.tmB, g.tmB2, g.tmC, kp);
    count_launches(1);
    return cudaGetLastError();
}

}  // namespace

int gemm_plan_rows(GemmPlan& g, int64_t M, int64_t N, int64_t K, const float* A, int64_t lda, const float* Bhi,
                   const float* Blo, int64_t ldb, float* C, int64_t ldc, int flags) {
    if (M <= 0 || N <= 0 || K <= 0 || M >= (1 << 30) || K >= (1 << 30) || N > 65536) return -1;
    if ((lda & 3) || (ldb & 3) || (reinterpret_cast<uintptr_t>(A) & 15) || (reinterpret_cast<uintptr_t>(Bhi) & 15) ||
        (reinterpret_cast<uintptr_t>(Blo) & 15))
        return -1;
    g = GemmPlan();
    g.op = 0;
    g.M = M; g.N = N; g.K = K;
    g.n_tiles = (int)((N + 255) / 256);
    // one N tile: multiple of 16 (MMA N); several: multiple of 32 so the 32-column
    // epilogue chunks never spill into the neighbouring tile
    g.BN = g.n_tiles == 1 ? (int)((N + 15) / 16 * 16) : (int)(((N + g.n_tiles - 1) / g.n_tiles + 31) / 32 * 32);
    g.m_tiles = (int)((M + BM - 1) / BM);
    g.C = C;
    g.ldc = ldc;
    g.flags = flags;
    g.k_chunks = 1;
    g.k_chunk_len = (K + BK - 1) / BK * BK;
    if ((ldc & 3) || (reinterpret_cast<uintptr_t>(C) & 15)) return -1;
    // CTA pairs (cta_group::2, M = 256) when B is wide: each CTA of a pair stages half of B
    static int pair_env = -1;
    if (pair_env < 0) {
        // default off: correct, but 1.5-1.8x SLOWER for 3xTF32 -- the pair's MMAs read the peer
        // CTA's half of B three times per k step (hi, lo, hi) over the SM-to-SM path
        // (profiles/r01_row_gemm_pair.log)
        const char* e = getenv("MGGCN_ROW_PAIR");
        pair_env = e ? atoi(e) : 0;
    }
    const bool pair = pair_env != 0 && g.BN >= 128 && g.m_tiles >= 2;
    g.variant = pair ? 2 : 0;
    const int bbox = pair ? g.BN / 2 : g.BN;
    int rc = encode2d_sw(&g.tmA, A, K, M, lda, 16, BM, 64);
    if (!rc) rc = encode2d_sw(&g.tmB, Bhi, K, N, ldb, 16, bbox, 64);
    if (!rc) rc = encode2d_sw(&g.tmB2, Blo, K, N, ldb, 16, bbox, 64);
    if (!rc) rc = encode2d_sw(&g.tmC, C, N, M, ldc, 32, BM, 128);   // epilogue store / old-value load
    if (rc) return rc;
    if (pair) {
        const int total = ((g.m_tiles + 1) / 2) * g.n_tiles;      // 256-row pair tiles
        const int pairs = num_sms() / 2;
        g.grid = 2 * (total < pairs ? total : pairs);
    } else {
        const int total = g.m_tiles * g.n_tiles;
        g.grid = total < num_sms() ? total : num_sms();
    }
    return 0;
}

int gemm_plan_wgrad(GemmPlan& g, int64_t M, int64_t N, int64_t K, const float* A, int64_t lda, const float* B,
                    int64_t ldb, int flags, size_t* partial_floats) {
    if (M <= 0 || N <= 0 || K <= 0 || M >= (1 << 30) || K >= (1 << 30) || N > 65536) return -1;
    if ((lda & 3) || (ldb & 3) || (reinterpret_cast<uintptr_t>(A) & 15) || (reinterpret_cast<uintptr_t>(B) & 15))
        return -1;
    g = GemmPlan();
    g.op = 2;
    g.M = M; g.N = N; g.K = K;
    g.n_tiles = (int)((N + 255) / 256);
    g.BN = (int)(((N + g.n_tiles - 1) / g.n_tiles + 15) / 16 * 16);
    g.m_tiles = (int)((M + BM - 1) / BM);
    g.flags = flags;
    const int mn = g.m_tiles * g.n_tiles;
    int want = num_sms() / mn;   // one wave: (M, N, K-chunk) tiles <= #SMs (1 CTA / SM)
    const int64_t kblocks = (K + BK - 1) / BK;
    if (want > kblocks) want = (int)kblocks;
    if (want < 1) want = 1;
    g.k_chunk_len = (kblocks + want - 1) / want * BK;
    g.k_chunks = (int)((K + g.k_chunk_len - 1) / g.k_chunk_len);
    if (partial_floats) *partial_floats = (size_t)g.k_chunks * (size_t)M * (size_t)N;
    // A is K x M (M contiguous), B is K x N (N contiguous)
    static int variant = -1, tsw = 0;
    static uint32_t dmn[3] = {1, 2048, 512};
    if (variant < 0) {
        const char* e = getenv("MGGCN_WGRAD");
        variant = (e && e[0] == 'x') ? 0 : 1;     // default: MN-major operands (no transpose)
        if (const char* d = getenv("MGGCN_WG_DESC")) sscanf(d, "%u,%u,%u", &dmn[0], &dmn[1], &dmn[2]);
        if (const char* t = getenv("MGGCN_WG_TMASW")) tsw = atoi(t);
    }
    g.variant = variant;
    int rc;
    if (variant == 1) {
        // boxes of 32 MN-contiguous floats x 16 k rows, 128B swizzle with 32B atoms
        g.BN = (int)(((N + g.n_tiles - 1) / g.n_tiles + 31) / 32 * 32);
        for (int i = 0; i < 3; ++i) g.desc_mn[i] = dmn[i];
        const CUtensorMapSwizzle sw = tsw == 1 ? CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B_FLIP_8B
                                      : tsw == 2 ? CU_TENSOR_MAP_SWIZZLE_128B_ATOM_64B
                                      : tsw == 3 ? CU_TENSOR_MAP_SWIZZLE_128B
                                                 : CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B;
        rc = encode2d_mode(&g.tmA, A, M, K, lda, 32, 16, sw);
        if (!rc) rc = encode2d_mode(&g.tmB, B, N, K, ldb, 32, 16, sw);
    } else {
        // raw boxes {M or N, 16 K}, transposed in smem
        rc = encode2d(&g.tmA, A, M, K, lda, BM, 16, false);
        if (!rc) rc = encode2d(&g.tmB, B, N, K, ldb, g.BN, 16, false);
    }
    if (rc) return rc;
    g.grid = g.m_tiles * g.n_tiles * g.k_chunks;   // one CTA per tile
    return 0;
}

size_t gemm_wgrad_partial_floats(int64_t M, int64_t N, int64_t K) {
    const int n_tiles = (int)((N + 255) / 256);
    const int m_tiles = (int)((M + BM - 1) / BM);
    const int mn = m_tiles * n_tiles;
    int want = num_sms() / mn;   // one wave: (M, N, K-chunk) tiles <= #SMs (1 CTA / SM)
    const int64_t kblocks = (K + BK - 1) / BK;
    if (want > kblocks) want = (int)kblocks;
    if (want < 1) want = 1;
    const int64_t len = (kblocks + want - 1) / want * BK;
    return (size_t)((K + len - 1) / len) * (size_t)M * (size_t)N;
}

cudaError_t gemm_launch(const GemmPlan& g, cudaStream_t s) {
    KParams kp;
    kp.M = (int)g.M; kp.N = (int)g.N; kp.K = (int)g.K;
    kp.BN = g.BN; kp.m_tiles = g.m_tiles; kp.n_tiles = g.n_tiles;
    kp.k_chunks = g.k_chunks; kp.k_chunk_len = (int)g.k_chunk_len;
    kp.C = g.C; kp.ldc = g.ldc; kp.partial = g.partial; kp.rowscale = g.rowscale;
    kp.flags = g.flags; kp.op2 = g.op == 2;
    static const bool longring = [] {
        const char* e = getenv("MGGCN_ROW_RING");
        return !(e && atoi(e) == 0);
    }();
    if (g.op != 2 && g.variant != 2 && longring) kp.flags |= GEMM_ROW_LONGRING;
    for (int i = 0; i < 3; ++i) kp.desc_mn[i] = g.desc_mn[i];

    if (g.op == 2) return g.variant == 1 ? launch_wgrad_mn(g, kp, s) : launch_wgrad(g, kp, s);
    return launch_rows(g, kp, s);
}

cudaError_t launch_split_weights(const float* W, int64_t din, int64_t dout, int64_t ldw, float* t_hi, float* t_lo,
                                 int64_t ldt, float* s_hi, float* s_lo, int x1, cudaStream_t s) {
    const int64_t total = din * dout;
    int blocks = (int)((total + 255) / 256);
    if (blocks > 1184) blocks = 1184;
    if (blocks < 1) blocks = 1;
    split_weights_kernel<<<blocks, 256, 0, s>>>(W, (int)din, (int)dout, ldw, t_hi, t_lo, ldt, s_hi, s_lo, x1);
    count_launches(1);
    return cudaGetLastError();
}

}  // namespace mggcn
