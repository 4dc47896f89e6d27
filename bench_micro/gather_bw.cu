// gather_bw.cu — B200 memory-system ceilings for the SpMM roofline.
// Measures, with CUDA events, the bandwidth of:
//   stream   : sequential float4 read of a buffer (HBM if > L2, L2 if small)
//   gather   : random whole-row gathers (row = W floats) from a table of R rows,
//              each warp gathering rows like the SpMM kernel (16 x LDG.128 in flight per lane)
// Usage: gather_bw  (prints one line per case)
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %s\n", cudaGetErrorString(e), #x); exit(1);} } while (0)

__global__ void stream_read(const float4* __restrict__ a, size_t n4, float* out) {
    float4 acc = make_float4(0, 0, 0, 0);
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x) {
        float4 v = __ldg(a + i);
        acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
    if (acc.x + acc.y + acc.z + acc.w == 12345.f) *out = acc.x;
}

// each warp: for its entries, lanes own CH float4 of a W4-float4 row (W4 = 32*CH), U entries in flight
template <int CH, int U>
__global__ void __launch_bounds__(256) gather_rows(const float4* __restrict__ tab, const int* __restrict__ idx,
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
                for (int c = 0; c < CH; ++c) { acc[c].x += x[u][c].x; acc[c].y += x[u][c].y; acc[c].z += x[u][c].z; acc[c].w += x[u][c].w; }
        }
    }
    float s = 0;
    for (int c = 0; c < CH; ++c) s += acc[c].x + acc[c].y + acc[c].z + acc[c].w;
    if (s == 12345.f) *out = s;
}


// same gather through shared memory with 1-D bulk async copies (the TMA
// engine): per warp a 2-stage ring of 32 row slots; lane i issues
// cp.async.bulk of row idx[k+i] (1 KB) into slot i, completion on the
// stage's mbarrier; the warp then sums the 32 rows from shared memory.
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int WARPS>
__global__ void __launch_bounds__(WARPS * 32) gather_bulk(const float4* __restrict__ tab, const int* __restrict__ idx,
                                                           size_t n_idx, int ld4, float* out) {
    extern __shared__ __align__(128) uint8_t sm[];
    const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
    uint8_t* ring = sm + (size_t)wl * 2 * 32 * 1024;
    __shared__ uint64_t bars[WARPS][2];
    if (lane == 0) {
        for (int s = 0; s < 2; ++s)
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bars[wl][s])));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    const size_t warp = (blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5;
    const size_t nw = ((size_t)gridDim.x * blockDim.x) >> 5;
    float4 acc0 = make_float4(0, 0, 0, 0), acc1 = acc0;
    uint32_t ph[2] = {0, 0};
    auto issue = [&](size_t base, int s) {
        if (lane == 0)
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&bars[wl][s])),
                         "r"(32 * 1024) : "memory");
        __syncwarp();
        const int r = idx[base + lane];
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 1024, [%2];" ::
                     "r"(smem_u32(ring + s * 32768 + lane * 1024)), "l"(tab + (size_t)r * ld4),
                     "r"(smem_u32(&bars[wl][s])) : "memory");
    };
    auto consume = [&](int s) {
        asm volatile("{\n\t.reg .pred P1;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t@!P1 bra W_%=;\n}\n"
                     ::"r"(smem_u32(&bars[wl][s])), "r"(ph[s]) : "memory");
        ph[s] ^= 1;
        const float4* rows = reinterpret_cast<const float4*>(ring + s * 32768);
#pragma unroll 8
        for (int k = 0; k < 32; ++k) {
            const float4 a = rows[k * 64 + lane], b = rows[k * 64 + lane + 32];
            acc0.x += a.x; acc0.y += a.y; acc0.z += a.z; acc0.w += a.w;
            acc1.x += b.x; acc1.y += b.y; acc1.z += b.z; acc1.w += b.w;
        }
        __syncwarp();
    };
    int s = 0;
    size_t base = warp * 32;
    if (base < n_idx) issue(base, 0);
    for (; base < n_idx; base += nw * 32) {
        const size_t nxt = base + nw * 32;
        if (nxt < n_idx) issue(nxt, s ^ 1);
        consume(s);
        s ^= 1;
    }
    float t = acc0.x + acc0.y + acc0.z + acc0.w + acc1.x + acc1.y + acc1.z + acc1.w;
    if (t == 12345.f) *out = t;
}

int main() {
    int dev = 0, sms = 0, l2 = 0;
    CK(cudaGetDevice(&dev));
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    CK(cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev));
    printf("{\"sms\": %d, \"l2_bytes\": %d}\n", sms, l2);
    float* out; CK(cudaMalloc(&out, 4));
    cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
    // ---- stream reads
    for (size_t mb : {32ul, 64ul, 1024ul, 4096ul}) {
        size_t bytes = mb << 20, n4 = bytes / 16;
        float4* buf; CK(cudaMalloc(&buf, bytes)); CK(cudaMemset(buf, 0, bytes));
        int reps = mb <= 64 ? 200 : 10;
        stream_read<<<sms * 8, 512>>>(buf, n4, out);
        CK(cudaEventRecord(a));
        for (int r = 0; r < reps; ++r) stream_read<<<sms * 8, 512>>>(buf, n4, out);
        CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
        float ms; CK(cudaEventElapsedTime(&ms, a, b));
        printf("{\"case\": \"stream_read\", \"MB\": %zu, \"GBps\": %.1f}\n", mb, bytes * (double)reps / (ms * 1e-3) / 1e9);
        CK(cudaFree(buf));
    }
    // ---- random row gathers (1 KB rows, like width-256 SpMM)
    const size_t n_idx = 64u << 20;
    std::vector<int> h(n_idx);
    for (size_t rows : {8192ul, 32768ul, 65536ul, 120000ul, 232965ul, 2449029ul}) {
        const int ld4 = 64;  // 256 floats
        size_t bytes = rows * ld4 * 16;
        float4* tab; CK(cudaMalloc(&tab, bytes)); CK(cudaMemset(tab, 0, bytes));
        uint64_t s = 88172645463325252ull;
        for (size_t i = 0; i < n_idx; ++i) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; h[i] = (int)(s % rows); }
        int* didx; CK(cudaMalloc(&didx, n_idx * 4)); CK(cudaMemcpy(didx, h.data(), n_idx * 4, cudaMemcpyHostToDevice));
        int per_sm = 0; CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, gather_rows<2, 8>, 256, 0));
        gather_rows<2, 8><<<sms * per_sm, 256>>>(tab, didx, n_idx, ld4, out);
        CK(cudaEventRecord(a));
        for (int r = 0; r < 3; ++r) gather_rows<2, 8><<<sms * per_sm, 256>>>(tab, didx, n_idx, ld4, out);
        CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
        float ms; CK(cudaEventElapsedTime(&ms, a, b));
        printf("{\"case\": \"gather_1KB_rows\", \"table_MB\": %.1f, \"GBps\": %.1f, \"rows_per_s\": %.3e}\n",
               bytes / 1048576.0, n_idx * 1024.0 * 3 / (ms * 1e-3) / 1e9, n_idx * 3 / (ms * 1e-3));
        // bulk-copy (TMA engine) variant: 3 warps x 64 KB ring per CTA, 1 CTA / SM
        CK(cudaFuncSetAttribute(gather_bulk<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, 3 * 65536));
        gather_bulk<3><<<sms, 96, 3 * 65536>>>(tab, didx, n_idx, ld4, out);
        CK(cudaGetLastError());
        CK(cudaEventRecord(a));
        for (int r = 0; r < 3; ++r) gather_bulk<3><<<sms, 96, 3 * 65536>>>(tab, didx, n_idx, ld4, out);
        CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
        CK(cudaEventElapsedTime(&ms, a, b));
        printf("{\"case\": \"gather_1KB_rows_bulk_async\", \"table_MB\": %.1f, \"GBps\": %.1f, \"rows_per_s\": %.3e}\n",
               bytes / 1048576.0, n_idx * 1024.0 * 3 / (ms * 1e-3) / 1e9, n_idx * 3 / (ms * 1e-3));
        CK(cudaFree(tab)); CK(cudaFree(didx));
    }
    return 0;
}
