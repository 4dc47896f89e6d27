// dense.cu — the dense-tile part of the staged SpMM (F2/B1 of SURVEY §8a) on
// the sm_100a tensor cores.
//
// The stage product C_i (+)= A_ij · H_j (Eq. 6 / Eq. 9) is a sum
// over the tile's non-zeros; how the sum is split is free.  An R-MAT tile
// ordered by degree has a dense corner (hub rows x hub columns): on the
// Reddit-shaped graph 2/3 of the coalesced non-zeros lie in 128 x 32 blocks of
// >= 5 % density.  Gathered, every such non-zero costs one 1 KB feature row
// from L2 (the gathers run at the L2 line rate); as a dense block
// the same rows are read once per 128 output rows and multiplied on the
// tensor cores.  plan_dense (dense_plan.cpp) picks the blocks on the host; this
// file runs them:
//
//   dense_bimg_kernel   B image of every used column chunk: the chunk's 32
//                       source rows of H_j, split into bf16 pieces
//                       (hi + mid + lo = the fp32 value to ~2^-24), transposed
//                       into the K-major SWIZZLE_64B layout the MMA reads;
//   dense_tile_kernel   per work item (a row group of 128 output rows, or a
//                       segment of a long one; items binned per CTA on the host):
//                       for every dense block, one bulk copy of its A image (the
//                       block's entries as bf16, pre-swizzled on the host; values
//                       are small integer multiplicities, exact in bf16) and one
//                       of the chunk's B image, then tcgen05.mma.kind::f16 (BF16
//                       in, FP32 accumulate in TMEM) per piece; every 8 blocks the
//                       accumulator chain is drained into fp32 registers (reading
//                       C32), and the epilogue stores / adds the 128 x N result
//                       into the output rows (or a segment's partial);
//   dense_fixup_kernel  segments of one row group, summed in order into the rows.
//
// The residual non-zeros (everything not in a dense block) stay in the CSR
// gather kernel (spmm.cu), which runs after this one with SPMM_ACCUM and
// applies the stage epilogue (row scale of Eq. 2, ReLU of Eq. 7).
//
// Warp roles (320 threads, one CTA per SM, persistent over work items):
//   warps 0-7 epilogue (TMEM lane quadrant w % 4, columns 128 (w / 4) ..), warp 8
//   bulk-copy producer, warp 9 TMEM allocator + MMA issuer.
#include <cstdio>
#include <cstdlib>

#include "kernels.cuh"

namespace mggcn {

namespace {

constexpr int kDnEpiWarps = 8;                     // 2 per TMEM lane quadrant, 128 columns each
constexpr int kDnThreads = (kDnEpiWarps + 2) * 32;
#ifndef MGGCN_DENSE_BPOL
#define MGGCN_DENSE_BPOL 0    // L2 policy of the B-image loads: 0 evict_first (default: the next gather kernel keeps the L2), 1 evict_normal, 2 evict_last
#endif
constexpr int kDnProdWarp = kDnEpiWarps, kDnMmaWarp = kDnEpiWarps + 1;
constexpr int kDnMaxStages = 16;                    // narrow N: many small stages cover the latency
constexpr int kDnABytes = kDenseM * kDenseK * 2;   // 8 KB: 128 rows x 64 B
constexpr int kDnSmemMax = 232448;                 // sm_100 opt-in shared memory per block
constexpr int kDnBarBytes = 512;
constexpr int kDenseDrain = 8;                      // blocks per accumulation chain (MGGCN_DENSE_DRAIN)

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

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

// 1-D bulk copy global -> shared, completion on an mbarrier (bytes % 16 == 0)
__device__ __forceinline__ void bulk_load(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint64_t pol) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
        : "memory");
}

__device__ __forceinline__ uint64_t policy_first() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ uint64_t policy_normal() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ uint64_t policy_last() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}

__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// K-major SWIZZLE_64B shared-memory descriptor (sm_100 format): rows of 64 B
// (32 bf16), 8-row atoms 512 B apart (SBO), LBO unused (1), version 1,
// layout type 4 = SWIZZLE_64B.
__device__ __forceinline__ uint64_t sw64_desc(uint32_t saddr) {
    return (uint64_t)((saddr & 0x3FFFFu) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(512 >> 4) << 32) |
           ((uint64_t)1 << 46) | ((uint64_t)4 << 61);
}

__device__ __forceinline__ void mma_bf16(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                         uint32_t accumulate) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}

__device__ __forceinline__ void mma_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
                 : "memory");
}

// 32 lanes x 32 columns (one 32-bit word per column) from TMEM; the caller waits
__device__ __forceinline__ void tmem_ld32_nowait(uint32_t taddr, uint32_t* r) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
        "%15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// fp32 -> bf16 bits, round to nearest even
__device__ __forceinline__ uint32_t bf16_bits(float x) {
    uint16_t h;
    asm("cvt.rn.bf16.f32 %0, %1;" : "=h"(h) : "f"(x));
    return h;
}
__device__ __forceinline__ float bf16_val(uint32_t b) { return __uint_as_float(b << 16); }

// ------------------------------------------------------------ B images
// One block per used column chunk c: rows src = chunk_cols[32c + k] of B
// (width valid columns from column 0 of the window; -1 = zero row) ->
// image[c][piece][n][k] (n < N output features, k < 32), K-major SW64: element
// (n, k) of a piece at byte n*64 + (((2k >> 4) ^ ((n >> 1) & 3)) << 4) + (2k & 15).
// The fp32 value x is split as hi = bf16(x), mid = bf16(x - hi), lo = bf16(x - hi - mid)
// (each difference exact in fp32), so hi + mid + lo = x to ~2^-24 relative.
__global__ void __launch_bounds__(256)
dense_bimg_kernel(const int32_t* __restrict__ chunk_cols, const float* __restrict__ B, int64_t ldb, int width, int N,
                  int pieces, uint8_t* __restrict__ bimg) {
    extern __shared__ float tile[];   // [32][N + 1]
    const int c = blockIdx.x;
    const int ldt = N + 1;
    const int n4 = N / 4;
    for (int idx = threadIdx.x; idx < 32 * n4; idx += blockDim.x) {
        const int k = idx / n4, q = idx - k * n4;
        const int src = __ldg(chunk_cols + (int64_t)c * kDenseK + k);
        float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
        if (src >= 0 && 4 * q < width) v = __ldg(reinterpret_cast<const float4*>(B + (int64_t)src * ldb) + q);
        float* t = tile + k * ldt + 4 * q;
        t[0] = v.x; t[1] = v.y; t[2] = v.z; t[3] = v.w;
    }
    __syncthreads();
    uint8_t* base = bimg + (size_t)c * pieces * N * 64;
    for (int idx = threadIdx.x; idx < N * 4; idx += blockDim.x) {
        const int n = idx >> 2, j = idx & 3;
        uint32_t w[3][4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            uint32_t h2[3][2];
#pragma unroll
            for (int e = 0; e < 2; ++e) {
                const float x = tile[(8 * j + 2 * i + e) * ldt + n];
                const uint32_t h = bf16_bits(x);
                const float r1 = x - bf16_val(h);
                const uint32_t mbits = bf16_bits(r1);
                const float r2 = r1 - bf16_val(mbits);
                h2[0][e] = h;
                h2[1][e] = mbits;
                h2[2][e] = bf16_bits(r2);
            }
#pragma unroll
            for (int p = 0; p < 3; ++p) w[p][i] = h2[p][0] | (h2[p][1] << 16);
        }
        const int off = n * 64 + ((j ^ ((n >> 1) & 3)) << 4);
        for (int p = 0; p < pieces; ++p)
            *reinterpret_cast<uint4*>(base + (size_t)p * N * 64 + off) = make_uint4(w[p][0], w[p][1], w[p][2], w[p][3]);
    }
}

struct DnParams {
    const int32_t* grp_rows;
    const int4* work;
    const int32_t* bin_beg;
    float* partial;
    const int32_t* tile_chunk;
    const uint8_t* A;
    const uint8_t* bimg;
    float* out;
    int64_t ldo;
    int first;
    int n_items;
    int N, width, pieces, stages;
    int drain;      // blocks per TMEM accumulation chain
    int stack;      // bf16 pieces stacked along N in one MMA (B = [hi; mid; lo] rows, N_mma = stack x N <= 256)
};

// ------------------------------------------------------------ tiles
template <int PIECES>
__global__ void __launch_bounds__(kDnThreads, 1) dense_tile_kernel(const DnParams p) {
    extern __shared__ uint8_t smem_dyn[];
    uint8_t* smem = smem_dyn + ((1024u - (smem_u32(smem_dyn) & 1023u)) & 1023u);
    const int N = p.N, S = p.stages;
    const uint32_t b_bytes = (uint32_t)(p.pieces * N * 64);
    const uint32_t stage_bytes = (uint32_t)kDnABytes + b_bytes;   // multiple of 1024 (N % 16 == 0)
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + S * stage_bytes);
    uint64_t* full = bars;                   // [S] producer -> MMA (tx bytes)
    uint64_t* empty = bars + kDnMaxStages;   // [S] MMA commit -> producer
    uint64_t* accf = bars + 2 * kDnMaxStages;       // [2] MMA -> epilogue
    uint64_t* acce = bars + 2 * kDnMaxStages + 2;   // [2] epilogue (128 threads) -> MMA
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * kDnMaxStages + 4);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    // Narrow N: the MMA issue, not the tensor work, bounds a block (6 tcgen05.mma of N = 48 take
    // ~550 of ~690 cycles), so `stack` consecutive pieces, stored contiguously in the B image, go
    // into ONE MMA of N_mma = stack x N whose accumulator holds each piece in its own N-column
    // range; the drain sums the ranges in fp32.  An accumulator is accw = stack x N columns.
    const int accw = p.stack * N;
    const uint32_t tcols = accw <= 128 ? 256u : 512u;   // two accumulators of accw columns

    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(full + s, 1);
            mbar_init(empty + s, 1);
        }
        for (int a = 0; a < 2; ++a) {
            mbar_init(accf + a, 1);
            mbar_init(acce + a, kDnEpiWarps * 32);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == kDnMmaWarp) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                     "r"(tcols));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    const int w_end = __ldg(p.bin_beg + blockIdx.x + 1);   // this CTA's bin of work items (host LPT)

    if (warp == kDnProdWarp) {
        if (lane == 0) {
#if MGGCN_DENSE_BPOL == 2
            const uint64_t pa = policy_first(), pb = policy_last();
#elif MGGCN_DENSE_BPOL == 1
            const uint64_t pa = policy_first(), pb = policy_normal();
#else
            const uint64_t pa = policy_first(), pb = policy_first();
#endif
            int s = 0;
            uint32_t ph = 0;
            for (int w = __ldg(p.bin_beg + blockIdx.x); w < w_end; ++w) {
                const int4 it = __ldg(p.work + w);
                for (int t = it.y; t < it.z; ++t) {
                    const int c = __ldg(p.tile_chunk + t);
                    mbar_wait(empty + s, ph ^ 1);
                    mbar_expect_tx(full + s, stage_bytes);
                    uint8_t* st = smem + (size_t)s * stage_bytes;
                    bulk_load(st, p.A + (size_t)t * kDnABytes, kDnABytes, full + s, pa);
                    bulk_load(st + kDnABytes, p.bimg + (size_t)c * b_bytes, b_bytes, full + s, pb);
                    if (++s == S) { s = 0; ph ^= 1; }
                }
            }
        }
    } else if (warp == kDnMmaWarp) {
        if (lane == 0) {
            // kind::f16: F32 accumulator (bit 4), A and B BF16 (bits 7-9, 10-12 = 1), both K-major,
            // N >> 3 at bit 17, M >> 4 at bit 24
            auto idesc_n = [](int n) {
                return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(n >> 3) << 17) |
                       ((uint32_t)(kDenseM >> 4) << 24);
            };
            // MMA q of a k step covers pieces [q0, q0 + nq) with N_mma = nq x N (nq = stack, the last
            // one the remainder); its D range starts at column 0 (the first piece's range) -- the
            // stacked pieces land in ranges 0, N, 2N, and a remainder MMA adds into range 0
            const int stack = p.stack;
            const int nmma = (PIECES + stack - 1) / stack;
            const uint32_t idesc0 = idesc_n(stack * N);
            const uint32_t idesc1 = idesc_n((PIECES - stack) * N > 0 ? (PIECES - stack < stack ? PIECES - stack : stack) * N : N);
            int s = 0, a = 0;
            uint32_t ph = 0, aph = 0;
            for (int w = __ldg(p.bin_beg + blockIdx.x); w < w_end; ++w) {
                const int4 it = __ldg(p.work + w);
                const int t0 = it.y, t1 = it.z;
                uint32_t d = 0;
                int tc = 0;   // block index inside the current accumulation chain
                for (int t = t0; t < t1; ++t) {
                    if (tc == 0) {   // a new chain: wait until the epilogue drained this accumulator
                        mbar_wait(acce + a, aph ^ 1);
                        tc_fence_after();
                        d = tmem_base + (uint32_t)(a * accw);
                    }
                    mbar_wait(full + s, ph);
                    tc_fence_after();
                    const uint32_t sa = smem_u32(smem + (size_t)s * stage_bytes);
                    const uint64_t ad = sw64_desc(sa);
                    const uint64_t bd0 = sw64_desc(sa + kDnABytes);
                    const uint64_t bd1 = sw64_desc(sa + kDnABytes + (uint32_t)(stack * N * 64));
#pragma unroll
                    for (int kk = 0; kk < kDenseK / 16; ++kk) {
                        const uint64_t adv = (uint64_t)((kk * 32) >> 4);   // 16 bf16 = 32 B per k step
                        mma_bf16(d, ad + adv, bd0 + adv, idesc0, (tc > 0 || kk > 0) ? 1u : 0u);
                        if (nmma > 1) {
                            mma_bf16(d, ad + adv, bd1 + adv, idesc1, 1u);
                            for (int q = 2; q < nmma; ++q)   // stack 1: the third piece
                                mma_bf16(d, ad + adv, sw64_desc(sa + kDnABytes + (uint32_t)(q * N * 64)) + adv, idesc1,
                                         1u);
                        }
                    }
                    mma_commit(empty + s);
                    if (++s == S) { s = 0; ph ^= 1; }
                    if (++tc == p.drain || t + 1 == t1) {   // chain done: hand the accumulator over
                        mma_commit(accf + a);
                        if (++a == 2) { a = 0; aph ^= 1; }
                        tc = 0;
                    }
                }
            }
        }
    } else {
        // epilogue: warp w drains TMEM lane quadrant w % 4 (one output row per thread), columns
        // [128 h, 128 h + 128) with h = w / 4.  The tensor core's fp32 accumulation loses low
        // bits at every MMA into a long chain (error ~ chain length: 1.1e-6 of max|C| after
        // 323 blocks, 1.2e-7 after 8; profiles/r02_dense_chain.jsonl), so the MMA warp closes a
        // chain every p.drain blocks and the drained accumulators are summed here in IEEE fp32
        // registers, in chain order (deterministic).
        int a = 0;
        uint32_t aph = 0;
        const int quad = warp & 3, h = warp >> 2;
        const int slot = quad * 32 + lane;
        const int cb = h * 128;                       // first column of this warp
        for (int w = __ldg(p.bin_beg + blockIdx.x); w < w_end; ++w) {
            const int4 it = __ldg(p.work + w);
            const int row = __ldg(p.grp_rows + (int64_t)it.x * kDenseM + slot);
            const int nchains = (it.z - it.y + p.drain - 1) / p.drain;
            float run[128];
#pragma unroll
            for (int i = 0; i < 128; ++i) run[i] = 0.f;
            for (int ch = 0; ch < nchains; ++ch) {
                mbar_wait(accf + a, aph);
                tc_fence_after();
#pragma unroll
                for (int cc = 0; cc < 4; ++cc) {
                    if (cb + cc * 32 < N) {
                        const uint32_t ta = tmem_base + ((uint32_t)(quad * 32) << 16) + (uint32_t)(a * accw + cb + cc * 32);
                        // the stacked pieces' ranges (hi, mid, lo), one at a time into the running sum
                        for (int j = 0; j < p.stack; ++j) {
                            uint32_t v[32];
                            tmem_ld32_nowait(ta + (uint32_t)(j * N), v);
                            tmem_wait_ld();
#pragma unroll
                            for (int i = 0; i < 32; ++i) run[cc * 32 + i] += __uint_as_float(v[i]);
                        }
                    }
                }
                tc_fence_before();
                mbar_arrive(acce + a);
                if (++a == 2) { a = 0; aph ^= 1; }
            }
            if (it.w >= 0) {   // a segment of a split group: its partial (summed by the fix-up)
                float* prow = p.partial + ((int64_t)it.w * kDenseM + slot) * N + cb;
#pragma unroll
                for (int q = 0; q < 32; ++q)
                    if (cb + 4 * q < N)
                        reinterpret_cast<float4*>(prow)[q] =
                            make_float4(run[4 * q], run[4 * q + 1], run[4 * q + 2], run[4 * q + 3]);
            } else if (row >= 0) {
                float* orow = p.out + (int64_t)row * p.ldo + cb;
#pragma unroll
                for (int q = 0; q < 32; ++q)
                    if (cb + 4 * q < p.width) {   // width % 4 == 0
                        float4* o4 = reinterpret_cast<float4*>(orow) + q;
                        float4 o = p.first ? make_float4(0.f, 0.f, 0.f, 0.f) : *o4;
                        o.x += run[4 * q];
                        o.y += run[4 * q + 1];
                        o.z += run[4 * q + 2];
                        o.w += run[4 * q + 3];
                        *o4 = o;
                    }
            }
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == kDnMmaWarp) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(tcols));
    }
}

// Split groups: out[row] += sum over the group's partial slots in slot order (deterministic).
// Block (s, r4): rows 4 r4 .. 4 r4 + 3 of split s, 64 threads per row (float4 columns).
__global__ void __launch_bounds__(256)
dense_fixup_kernel(const int4* __restrict__ splits, const int32_t* __restrict__ grp_rows,
                   const float* __restrict__ partial, int N, int width, float* __restrict__ out, int64_t ldo,
                   int first) {
    const int4 sp = __ldg(splits + blockIdx.x);
    const int i = blockIdx.y * 4 + (threadIdx.x >> 6);
    const int q = threadIdx.x & 63;
    const int row = __ldg(grp_rows + (int64_t)sp.x * kDenseM + i);
    if (row < 0 || 4 * q >= width) return;
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int k = 0; k < sp.z; ++k) {
        const float4 v = __ldg(reinterpret_cast<const float4*>(partial + ((int64_t)(sp.y + k) * kDenseM + i) * N) + q);
        acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
    float4* o = reinterpret_cast<float4*>(out + (int64_t)row * ldo) + q;
    float4 x = first ? make_float4(0.f, 0.f, 0.f, 0.f) : *o;
    x.x += acc.x; x.y += acc.y; x.z += acc.z; x.w += acc.w;
    *o = x;
}

}  // namespace

int dense_stages_for(int N, int pieces) {
    const int stage = kDnABytes + pieces * N * 64;
    int s = (kDnSmemMax - 1024 - kDnBarBytes) / stage;
    if (s > kDnMaxStages) s = kDnMaxStages;
    return s;
}

size_t dense_bimg_bytes(int64_t n_chunks, int pieces) { return (size_t)n_chunks * pieces * kDenseMaxN * 64; }
size_t dense_partial_floats(int64_t n_slots) { return (size_t)n_slots * kDenseM * kDenseMaxN; }

cudaError_t launch_dense(const DenseTiles& d, const float* B, int64_t ldb, float* out, int64_t ldo, int width,
                         bool first, cudaStream_t s) {
    if (d.n_items == 0 || width <= 0) return cudaSuccess;
    if (width > kDenseMaxN || (width & 3) || !d.bimg || (d.n_splits && !d.partial)) return cudaErrorInvalidValue;
    const int N = (width + 15) / 16 * 16;
    const int pieces = d.pieces;
    const size_t bsm = sizeof(float) * 32 * (N + 1);
    dense_bimg_kernel<<<(unsigned)d.n_chunks, 256, bsm, s>>>(d.chunk_cols, B, ldb, width, N, pieces, d.bimg);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    const int S = dense_stages_for(N, pieces);
    const size_t smem = 1024 + (size_t)S * (kDnABytes + pieces * N * 64) + kDnBarBytes;
    static bool attr = false;
    if (!attr) {
        e = cudaFuncSetAttribute(dense_tile_kernel<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, kDnSmemMax);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(dense_tile_kernel<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, kDnSmemMax);
        if (e != cudaSuccess) return e;
        attr = true;
    }
    DnParams p;
    p.grp_rows = d.grp_rows;
    p.work = d.work;
    p.bin_beg = d.bin_beg;
    p.partial = d.partial;
    p.tile_chunk = d.tile_chunk;
    p.A = d.A;
    p.bimg = d.bimg;
    p.out = out;
    p.ldo = ldo;
    p.first = first ? 1 : 0;
    p.n_items = (int)d.n_items;
    p.N = N;
    p.width = width;
    p.pieces = pieces;
    p.stages = S;
    static int drain_env = -1;
    if (drain_env < 0) {
        const char* de = getenv("MGGCN_DENSE_DRAIN");
        drain_env = de ? atoi(de) : 0;
        if (drain_env < 0) drain_env = 0;
    }
    p.drain = drain_env > 0 ? drain_env : kDenseDrain;
    static int stack_env = -1;   // MGGCN_DENSE_STACK=1: one MMA per piece (experiment hook)
    if (stack_env < 0) {
        const char* se = getenv("MGGCN_DENSE_STACK");
        stack_env = se ? atoi(se) : 0;
    }
    int stack = kDenseMaxN / N < pieces ? kDenseMaxN / N : pieces;
    if (stack < 1) stack = 1;
    if (stack_env > 0 && stack_env < stack) stack = stack_env;
    p.stack = stack;
    const int grid = (int)d.n_bins;
    if (pieces == 2) dense_tile_kernel<2><<<grid, kDnThreads, smem, s>>>(p);
    else dense_tile_kernel<3><<<grid, kDnThreads, smem, s>>>(p);
    count_launches(2);
    e = cudaGetLastError();
    if (e != cudaSuccess || d.n_splits == 0) return e;
    dense_fixup_kernel<<<dim3((unsigned)d.n_splits, kDenseM / 4), 256, 0, s>>>(d.splits, d.grp_rows, d.partial, N,
                                                                              width, out, ldo, first ? 1 : 0);
    count_launches(1);
    return cudaGetLastError();
}

}  // namespace mggcn
