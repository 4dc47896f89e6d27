// dsmem_gather.cu — can a cluster-distributed hot-row cache lift the SpMM's
// gather rate above the per-SM L2 port?  (SpMM roofline probe.)
//
// Gathers 512-B rows (a 128-float column window, like the width-256 Reddit
// SpMM at MGGCN_SPMM_WIN = 128) for a stream of indices of which a fraction x
// hit a "hot set".  The hot set is held in the shared memory of the C CTAs of
// a thread-block cluster (each CTA H rows); a hot entry is read with
// ld.shared::cluster from its owner CTA (mapa), a cold one with ld.global.nc.
// Both loads are issued predicated (no select after the load), so U rows per
// lane stay in flight.  mode 0 = every entry from global memory (the hot rows
// are then L1/L2 hits), mode 1 = hot entries from distributed shared memory.
//
// Usage: dsmem_gather      prints one JSON line per case
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %s:%d\n", cudaGetErrorString(e), #x, __LINE__); exit(1);} } while (0)

constexpr int kLd4 = 32;            // 128 floats per row = 32 float4
constexpr int kRowBytes = kLd4 * 16;
constexpr int kThreads = 512;
constexpr int kU = 16;

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ float4 ld_mixed(int hot, uint32_t caddr, const float4* g) {
    float4 v;
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "@p ld.shared::cluster.v4.f32 {%0, %1, %2, %3}, [%5];\n\t"
                 "@!p ld.global.nc.v4.f32 {%0, %1, %2, %3}, [%6];\n}"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(hot), "r"(caddr), "l"(g));
    return v;
}

__device__ __forceinline__ void cluster_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// idx >= 0: global row; idx < 0: hot id h = -idx-1 -> owner CTA h / H, slot h % H
template <int MODE>
__global__ void __launch_bounds__(kThreads, 1) gather_mixed(const float4* __restrict__ tab, const int* __restrict__ idx,
                                                            size_t n_idx, int H, float* out) {
    extern __shared__ __align__(128) float4 hot[];
    uint32_t crank, csize;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(crank));
    asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(csize));
    const int lane = threadIdx.x & 31;
    if (MODE == 1) {
        // stage this CTA's share of the hot set: hot id h lives in table row h
        for (int i = threadIdx.x; i < H * kLd4; i += blockDim.x)
            hot[i] = __ldg(tab + (size_t)(crank * H + i / kLd4) * kLd4 + i % kLd4);
        cluster_sync();
    }
    const uint32_t hot_base = smem_u32(hot) + lane * 16;
    const size_t warp = (blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5;
    const size_t nw = ((size_t)gridDim.x * blockDim.x) >> 5;
    float4 acc = make_float4(0, 0, 0, 0);
    for (size_t base = warp * 32; base < n_idx; base += nw * 32) {
        const int my = idx[base + lane];
#pragma unroll 1
        for (int k0 = 0; k0 < 32; k0 += kU) {
            float4 x[kU];
#pragma unroll
            for (int u = 0; u < kU; ++u) {
                const int e = __shfl_sync(0xffffffffu, my, k0 + u);
                if (MODE == 0) {
                    const uint32_t r = e >= 0 ? (uint32_t)e : (uint32_t)(-e - 1);
                    x[u] = __ldg(tab + r * (uint32_t)kLd4 + lane);
                } else {
                    const int h = -e - 1;
                    const int hot_e = e < 0;
                    const uint32_t owner = hot_e ? (uint32_t)h / (uint32_t)H : crank;
                    const uint32_t slot = hot_e ? (uint32_t)h % (uint32_t)H : 0;
                    uint32_t caddr;
                    asm("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(caddr) : "r"(hot_base + slot * kRowBytes), "r"(owner));
                    x[u] = ld_mixed(hot_e, caddr, tab + (uint32_t)(hot_e ? 0 : e) * (uint32_t)kLd4 + lane);
                }
            }
#pragma unroll
            for (int u = 0; u < kU; ++u) { acc.x += x[u].x; acc.y += x[u].y; acc.z += x[u].z; acc.w += x[u].w; }
        }
    }
    if (MODE == 1) cluster_sync();   // peers may still read this CTA's hot rows
    const float s = acc.x + acc.y + acc.z + acc.w;
    if (s == 12345.f) *out = s;
}

int main() {
    int dev = 0, sms = 0;
    CK(cudaGetDevice(&dev));
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    float* out; CK(cudaMalloc(&out, 4));
    cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
    const size_t n_idx = 32u << 20;
    std::vector<int> h(n_idx);
    const int smem = 192 * 1024, H = smem / kRowBytes;
    CK(cudaFuncSetAttribute(gather_mixed<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    CK(cudaFuncSetAttribute(gather_mixed<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    CK(cudaFuncSetAttribute(gather_mixed<1>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
    int* didx; CK(cudaMalloc(&didx, n_idx * 4));
    // ---- SM scaling of plain LDG gathers (mode 0, no hot rows) from an L2-resident table:
    // linear in the number of SMs => a per-SM (L1 fill) limit; flat => a shared L2 limit
    if (getenv("SM_SWEEP")) {
        const size_t rows = 60000;
        float4* tab; CK(cudaMalloc(&tab, rows * kRowBytes)); CK(cudaMemset(tab, 0, rows * kRowBytes));
        uint64_t s = 88172645463325252ull;
        for (size_t i = 0; i < n_idx; ++i) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; h[i] = (int)(s % rows); }
        CK(cudaMemcpy(didx, h.data(), n_idx * 4, cudaMemcpyHostToDevice));
        for (int g : {18, 37, 74, 111, 148}) {
            gather_mixed<0><<<g, kThreads, smem>>>(tab, didx, n_idx, H, out);
            CK(cudaDeviceSynchronize());
            CK(cudaEventRecord(a));
            for (int r = 0; r < 3; ++r) gather_mixed<0><<<g, kThreads, smem>>>(tab, didx, n_idx, H, out);
            CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
            float ms; CK(cudaEventElapsedTime(&ms, a, b));
            const double gbs = n_idx * (double)kRowBytes * 3 / (ms * 1e-3) / 1e9;
            printf("{\"sm_sweep\": %d, \"table_MB\": %.1f, \"GBps\": %.1f, \"GBps_per_sm\": %.1f, \"B_per_clk_per_sm_at_1965\": %.1f}\n",
                   g, rows * kRowBytes / 1048576.0, gbs, gbs / g, gbs / g / 1.965);
            fflush(stdout);
        }
        CK(cudaFree(tab));
        return 0;
    }
    for (size_t rows : {60000ul, 232965ul}) {
        float4* tab; CK(cudaMalloc(&tab, rows * kRowBytes)); CK(cudaMemset(tab, 0, rows * kRowBytes));
        for (int C : {1, 2, 4, 8, 16}) {
            for (double x : {0.0, 0.1, 0.2, 0.3, 0.5, 1.0}) {
                const int nhot = C * H;
                uint64_t s = 88172645463325252ull ^ (uint64_t)(x * 1000) ^ ((uint64_t)C << 40);
                for (size_t i = 0; i < n_idx; ++i) {
                    s ^= s << 13; s ^= s >> 7; s ^= s << 17;
                    const double u = (double)(s >> 11) * (1.0 / 9007199254740992.0);
                    s ^= s << 13; s ^= s >> 7; s ^= s << 17;
                    h[i] = u < x ? -(int)(s % nhot) - 1 : (int)(nhot + s % (rows - nhot));
                }
                CK(cudaMemcpy(didx, h.data(), n_idx * 4, cudaMemcpyHostToDevice));
                for (int mode = 0; mode < 2; ++mode) {
                    cudaLaunchConfig_t cfg = {};
                    cudaLaunchAttribute at[1];
                    at[0].id = cudaLaunchAttributeClusterDimension;
                    at[0].val.clusterDim.x = mode ? C : 1; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
                    cfg.blockDim = dim3(kThreads); cfg.dynamicSmemBytes = smem; cfg.attrs = at; cfg.numAttrs = 1;
                    int ncl = 0;
                    cfg.gridDim = dim3(sms);
                    if (mode) {
                        if (cudaOccupancyMaxActiveClusters(&ncl, (void*)gather_mixed<1>, &cfg) != cudaSuccess || ncl <= 0) {
                            cudaGetLastError();
                            printf("{\"rows\": %zu, \"C\": %d, \"x\": %.2f, \"mode\": 1, \"skip\": \"no cluster occupancy\"}\n", rows, C, x);
                            continue;
                        }
                        cfg.gridDim = dim3(ncl * C);
                    }
                    auto launch = [&]() {
                        if (mode) CK(cudaLaunchKernelEx(&cfg, gather_mixed<1>, (const float4*)tab, (const int*)didx, n_idx, H, out));
                        else CK(cudaLaunchKernelEx(&cfg, gather_mixed<0>, (const float4*)tab, (const int*)didx, n_idx, H, out));
                    };
                    launch();
                    CK(cudaDeviceSynchronize());
                    CK(cudaEventRecord(a));
                    for (int r = 0; r < 5; ++r) launch();
                    CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
                    float ms; CK(cudaEventElapsedTime(&ms, a, b));
                    printf("{\"rows\": %zu, \"table_MB\": %.1f, \"C\": %d, \"hot_rows\": %d, \"x\": %.2f, \"mode\": %d, "
                           "\"grid\": %u, \"GBps\": %.1f}\n", rows, rows * kRowBytes / 1048576.0, C, nhot, x, mode,
                           cfg.gridDim.x, n_idx * (double)kRowBytes * 5 / (ms * 1e-3) / 1e9);
                    fflush(stdout);
                }
            }
            if (C == 1) continue;
        }
        CK(cudaFree(tab));
    }
    return 0;
}
