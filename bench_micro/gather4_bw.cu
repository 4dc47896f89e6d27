// gather4_bw.cu — is TMA tile::gather4 staging a faster way to gather feature rows?
//
// The SpMM (csrc/spmm.cu) gathers one feature row per non-zero with direct
// LDG.128s.  north_star asks for "TMA/shared-memory staging of the broadcast
// block"; round 1 measured 1-D cp.async.bulk (one 1 KB row per op: issue-bound
// at 6.5 TB/s).  This measures the sm_100 tensor-map gather,
// cp.async.bulk.tensor.2d...tile::gather4 (4 rows of up to 256 elements per
// instruction), against the LDG gather of gather_bw.cu, on the same random
// row indices and table sizes:
//   ldg     : warp per 32 indices, 16 LDG.128 per lane in flight (the SpMM's shape)
//   gather4 : 1 producer thread per CTA issues gather4 ops (4 rows x ROWB bytes)
//             into an NS-stage shared-memory ring (full/empty mbarriers); 4
//             consumer warps sum every stage from shared memory
// Output: one JSON line per (mode, row bytes, table MB).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gather4_bw gather4_bw.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %s\n", cudaGetErrorString(e), #x); exit(1);} } while (0)

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int CH, int U>
__global__ void __launch_bounds__(256) ldg_gather(const float4* __restrict__ tab, const int* __restrict__ idx,
                                                  size_t n_idx, int ld4, float* out) {
    const int lane = threadIdx.x & 31;
    const size_t warp = (blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5;
    const size_t nw = ((size_t)gridDim.x * blockDim.x) >> 5;
    float4 acc[CH];
    for (int c = 0; c < CH; ++c) acc[c] = make_float4(0, 0, 0, 0);
    for (size_t base = warp * 32; base < n_idx; base += nw * 32) {
        const int my = idx[base + lane];
#pragma unroll 1
        for (int k0 = 0; k0 < 32; k0 += U) {
            float4 x[U][CH];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint32_t r = (uint32_t)__shfl_sync(0xffffffffu, my, k0 + u);
#pragma unroll
                for (int c = 0; c < CH; ++c) x[u][c] = __ldg(tab + r * (uint32_t)ld4 + lane + 32 * c);
            }
#pragma unroll
            for (int u = 0; u < U; ++u)
#pragma unroll
                for (int c = 0; c < CH; ++c) {
                    acc[c].x += x[u][c].x; acc[c].y += x[u][c].y; acc[c].z += x[u][c].z; acc[c].w += x[u][c].w;
                }
        }
    }
    float s = 0;
    for (int c = 0; c < CH; ++c) s += acc[c].x + acc[c].y + acc[c].z + acc[c].w;
    if (s == 12345.f) *out = s;
}

// ROWB bytes per gathered row (box dim 0 = ROWB / 4 floats); a stage = 4 rows.
// 32 stages: lane i of the producer warp owns stage i and issues its gather4
// ops (indices of 32 groups loaded by one coalesced int4 load per lane), so up
// to 32 gather4 ops per CTA are in flight.
template <int ROWB>
__global__ void __launch_bounds__(160) gather4_kernel(const __grid_constant__ CUtensorMap tm,
                                                      const int4* __restrict__ idx4, size_t n_groups, float* out) {
    constexpr int NS = 32, STAGE = 4 * ROWB;
    extern __shared__ __align__(1024) uint8_t ring[];
    __shared__ __align__(8) uint64_t full[NS], empty[NS];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        for (int s = 0; s < NS; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&full[s])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 4;" ::"r"(smem_u32(&empty[s])));
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const size_t step = (size_t)gridDim.x * NS;
    if (warp == 4) {   // producer warp
        uint32_t batch = 0;
        for (size_t base = (size_t)blockIdx.x * NS; base < n_groups; base += step, ++batch) {
            const size_t g = base + lane;
            const int4 r = g < n_groups ? idx4[g] : make_int4(0, 0, 0, 0);
            if (batch > 0)
                asm volatile("{\n\t.reg .pred P1;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t@!P1 bra W_%=;\n}\n"
                             ::"r"(smem_u32(&empty[lane])), "r"((batch - 1) & 1) : "memory");
            if (g < n_groups) {
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&full[lane])),
                             "r"(STAGE) : "memory");
                asm volatile(
                    "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
                    " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(smem_u32(ring + lane * STAGE)),
                    "l"(reinterpret_cast<uint64_t>(&tm)), "r"(0), "r"(r.x), "r"(r.y), "r"(r.z), "r"(r.w),
                    "r"(smem_u32(&full[lane])) : "memory");
            }
        }
        return;
    }
    // consumers: 128 threads sum every stage (STAGE / 16 float4)
    float4 acc = make_float4(0, 0, 0, 0);
    uint32_t batch = 0;
    for (size_t base = (size_t)blockIdx.x * NS; base < n_groups; base += step, ++batch) {
        for (int j = 0; j < NS && base + j < n_groups; ++j) {
            asm volatile("{\n\t.reg .pred P1;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t@!P1 bra W_%=;\n}\n"
                         ::"r"(smem_u32(&full[j])), "r"(batch & 1) : "memory");
            const float4* st = reinterpret_cast<const float4*>(ring + j * STAGE);
#pragma unroll
            for (int q = threadIdx.x; q < STAGE / 16; q += 128) {
                const float4 v = st[q];
                acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
            }
            __syncwarp();
            if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty[j])) : "memory");
        }
    }
    if (acc.x + acc.y + acc.z + acc.w == 12345.f) *out = acc.x;
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                             const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

template <int ROWB>
double run_gather4(EncodeFn enc, float* tab, size_t rows, const int* didx, size_t n_idx, int sms, float* out,
                   int ctas_per_sm) {
    CUtensorMap tm;
    cuuint64_t dims[2] = {(cuuint64_t)(ROWB / 4), (cuuint64_t)rows};
    cuuint64_t strides[1] = {(cuuint64_t)1024};   // table rows are 1 KB apart (256 floats)
    cuuint32_t box[2] = {(cuuint32_t)(ROWB / 4), 1};
    cuuint32_t es[2] = {1, 1};
    CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, tab, dims, strides, box, es,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) { printf("encode failed %d\n", (int)r); exit(1); }
    const int smem = 32 * 4 * ROWB;
    CK(cudaFuncSetAttribute(gather4_kernel<ROWB>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    const size_t ng = n_idx / 4;
    cudaEvent_t a, b;
    CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
    gather4_kernel<ROWB><<<sms * ctas_per_sm, 160, smem>>>(tm, reinterpret_cast<const int4*>(didx), ng, out);
    CK(cudaGetLastError());
    CK(cudaEventRecord(a));
    for (int i = 0; i < 3; ++i) gather4_kernel<ROWB><<<sms * ctas_per_sm, 160, smem>>>(tm, reinterpret_cast<const int4*>(didx), ng, out);
    CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
    float ms; CK(cudaEventElapsedTime(&ms, a, b));
    return (double)ng * 4 * ROWB * 3 / (ms * 1e-3) / 1e9;
}

int main() {
    int dev = 0, sms = 0;
    CK(cudaGetDevice(&dev));
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
    EncodeFn enc = (EncodeFn)fn;
    float* out; CK(cudaMalloc(&out, 4));
    const size_t n_idx = 64u << 20;
    std::vector<int> h(n_idx);
    for (size_t rows : {29120ul, 116483ul, 232965ul, 2449029ul}) {
        const size_t bytes = rows * 1024;
        float* tab; CK(cudaMalloc(&tab, bytes)); CK(cudaMemset(tab, 0, bytes));
        uint64_t s = 88172645463325252ull;
        for (size_t i = 0; i < n_idx; ++i) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; h[i] = (int)(s % rows); }
        int* didx; CK(cudaMalloc(&didx, n_idx * 4)); CK(cudaMemcpy(didx, h.data(), n_idx * 4, cudaMemcpyHostToDevice));
        // LDG baseline (1 KB rows, the SpMM's wide shape; 512 B rows = a 128-float column window)
        for (int rowb : {1024, 512}) {
            int per_sm = 0;
            cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
            float ms = 0;
            if (rowb == 1024) {
                CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, ldg_gather<2, 8>, 256, 0));
                ldg_gather<2, 8><<<sms * per_sm, 256>>>((const float4*)tab, didx, n_idx, 64, out);
                CK(cudaEventRecord(a));
                for (int i = 0; i < 3; ++i) ldg_gather<2, 8><<<sms * per_sm, 256>>>((const float4*)tab, didx, n_idx, 64, out);
            } else {
                CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, ldg_gather<1, 16>, 256, 0));
                ldg_gather<1, 16><<<sms * per_sm, 256>>>((const float4*)tab, didx, n_idx, 64, out);
                CK(cudaEventRecord(a));
                for (int i = 0; i < 3; ++i) ldg_gather<1, 16><<<sms * per_sm, 256>>>((const float4*)tab, didx, n_idx, 64, out);
            }
            CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
            CK(cudaEventElapsedTime(&ms, a, b));
            printf("{\"mode\": \"ldg\", \"row_bytes\": %d, \"table_MB\": %.1f, \"GBps\": %.1f}\n", rowb,
                   bytes / 1048576.0, (double)n_idx * rowb * 3 / (ms * 1e-3) / 1e9);
        }
        for (int cps : {1, 2, 3}) {
            if (cps == 1)
                printf("{\"mode\": \"gather4\", \"row_bytes\": 1024, \"ctas_per_sm\": 1, \"table_MB\": %.1f, \"GBps\": %.1f}\n",
                       bytes / 1048576.0, run_gather4<1024>(enc, tab, rows, didx, n_idx, sms, out, 1));
            printf("{\"mode\": \"gather4\", \"row_bytes\": 512, \"ctas_per_sm\": %d, \"table_MB\": %.1f, \"GBps\": %.1f}\n",
                   cps, bytes / 1048576.0, run_gather4<512>(enc, tab, rows, didx, n_idx, sms, out, cps));
        }
        fflush(stdout);
        CK(cudaFree(tab)); CK(cudaFree(didx));
    }
    return 0;
}
