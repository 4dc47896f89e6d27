// misc.cu — loss layer, Adam and small reductions (sm_100a).
//
// Softmax cross-entropy: P:1244-1246 ("softmax cross-entropy loss [9]"),
// forward and backward fused into one warp-per-row pass whose gradient
// overwrites the logits in place (Eq. 19: AHW_G -> AHWB).  Adam: P:1244 with
// ref [23] (Kingma & Ba), reading C6.  All reductions run in a fixed order
// (no floating-point atomics) so results are bitwise reproducible.
#include <atomic>
#include <cmath>

#include "kernels.cuh"

namespace mggcn {

namespace {

__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}
__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}
__device__ __forceinline__ double warp_sum_d(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

constexpr int kCeWarps = 8;

// Each warp owns a fixed, strided set of rows; per-warp fp64 loss sums are
// combined in warp order, giving one partial per block (deterministic).
__global__ void __launch_bounds__(kCeWarps * 32)
softmax_ce_kernel(float* __restrict__ Z, int64_t n, int C, int64_t ld, const int32_t* __restrict__ y,
                  const int64_t* __restrict__ ntrain, const float* __restrict__ rowscale, int relu_last,
                  double* __restrict__ block_partial) {
    __shared__ double wsum[kCeWarps];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int64_t gw = (int64_t)blockIdx.x * kCeWarps + wid, nw = (int64_t)gridDim.x * kCeWarps;
    const float inv_nt = 1.0f / (float)(*ntrain > 0 ? *ntrain : 1);
    double lsum = 0.0;
    for (int64_t r = gw; r < n; r += nw) {
        float* z = Z + r * ld;
        const int lab = y[r];
        if (lab < 0) {
            for (int c = lane; c < C; c += 32) z[c] = 0.f;
            continue;
        }
        float mx = -INFINITY;
        for (int c = lane; c < C; c += 32) mx = fmaxf(mx, z[c]);
        mx = warp_max(mx);
        float s = 0.f;
        for (int c = lane; c < C; c += 32) s += expf(z[c] - mx);
        s = warp_sum(s);
        const float lse = mx + logf(s);
        const float zy = z[lab];   // every lane reads the same address
        if (lane == 0) lsum += (double)lse - (double)zy;
        const float sc = inv_nt * (rowscale ? rowscale[r] : 1.f);
        for (int c = lane; c < C; c += 32) {
            const float zc = z[c];
            float g = expf(zc - lse) - (c == lab ? 1.f : 0.f);
            if (relu_last && !(zc > 0.f)) g = 0.f;
            z[c] = g * sc;
        }
    }
    if (lane == 0) wsum[wid] = lsum;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < kCeWarps; ++w) t += wsum[w];
        block_partial[blockIdx.x] = t;
    }
}

// Vectorised variant for C <= 256: a row is held by a group of G lanes, CH
// float4 per lane, so a warp works on 32/G rows at once and U row groups are
// loaded before any arithmetic (one read and one write of each row, all loads
// in flight together).  Same arithmetic per row as softmax_ce_kernel: fp32
// max, sum of exp(z - max), lse = max + log(sum), gradient (exp(z - lse) -
// [c == y]) * inv_nt * rowscale (Eq. 19), loss lse - z_y summed in fp64; the
// group sums use a fixed xor tree and the per-row losses are added in a fixed
// order (lane-group, then iteration, then warp), so results are deterministic.
template <int G, int CH>
__device__ __forceinline__ float group_max(float v) {
#pragma unroll
    for (int o = G / 2; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}
template <int G>
__device__ __forceinline__ float group_sum(float v) {
#pragma unroll
    for (int o = G / 2; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

template <int G, int CH, int U>
__global__ void __launch_bounds__(kCeWarps * 32)
softmax_ce_vec_kernel(float* __restrict__ Z, int64_t n, int C, int64_t ld, const int32_t* __restrict__ y,
                      const int64_t* __restrict__ ntrain, const float* __restrict__ rowscale, int relu_last,
                      double* __restrict__ block_partial) {
    constexpr int R = 32 / G;          // rows per warp step
    __shared__ double wsum[kCeWarps];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int sub = lane / G, gl = lane % G;
    const int64_t gw = (int64_t)blockIdx.x * kCeWarps + wid, nw = (int64_t)gridDim.x * kCeWarps;
    const float inv_nt = 1.0f / (float)(*ntrain > 0 ? *ntrain : 1);
    double lsum = 0.0;
    for (int64_t r0 = gw * (R * U); r0 < n; r0 += nw * (R * U)) {
        float4 x[U][CH];
        int lab[U];
        float sc[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t r = r0 + u * R + sub;
            const bool ok = r < n;
            const float4* zr = reinterpret_cast<const float4*>(Z + (ok ? r : 0) * ld);
#pragma unroll
            for (int ch = 0; ch < CH; ++ch) {
                const int q = gl + ch * G;
                x[u][ch] = (4 * q < C) ? zr[q] : make_float4(0.f, 0.f, 0.f, 0.f);
            }
            lab[u] = ok ? y[r] : -1;
            sc[u] = ok && rowscale ? rowscale[r] : 1.f;
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t r = r0 + u * R + sub;
            float mx = -INFINITY;
#pragma unroll
            for (int ch = 0; ch < CH; ++ch) {
                const int c = 4 * (gl + ch * G);
                if (c + 0 < C) mx = fmaxf(mx, x[u][ch].x);
                if (c + 1 < C) mx = fmaxf(mx, x[u][ch].y);
                if (c + 2 < C) mx = fmaxf(mx, x[u][ch].z);
                if (c + 3 < C) mx = fmaxf(mx, x[u][ch].w);
            }
            mx = group_max<G, CH>(mx);
            float sm = 0.f;
#pragma unroll
            for (int ch = 0; ch < CH; ++ch) {
                const int c = 4 * (gl + ch * G);
                if (c + 0 < C) sm += expf(x[u][ch].x - mx);
                if (c + 1 < C) sm += expf(x[u][ch].y - mx);
                if (c + 2 < C) sm += expf(x[u][ch].z - mx);
                if (c + 3 < C) sm += expf(x[u][ch].w - mx);
            }
            sm = group_sum<G>(sm);
            const float lse = mx + logf(sm);
            const int l = lab[u];
            // z_y from the lane that holds column l
            float zy = 0.f;
            const int ql = l >= 0 ? l >> 2 : 0;
            if (l >= 0 && gl == ql % G) {
#pragma unroll
                for (int ch = 0; ch < CH; ++ch)
                    if (ch == ql / G) {
                        const float4 v = x[u][ch];
                        zy = (l & 3) == 0 ? v.x : (l & 3) == 1 ? v.y : (l & 3) == 2 ? v.z : v.w;
                    }
            }
            zy = group_sum<G>(zy);       // one non-zero term: exact
            if (r >= n) continue;
            if (gl == 0 && l >= 0) lsum += (double)lse - (double)zy;
            const float s2 = inv_nt * sc[u];
            float* zr = Z + r * ld;
#pragma unroll
            for (int ch = 0; ch < CH; ++ch) {
                const int q = gl + ch * G, c = 4 * q;
                if (c >= C) continue;
                float o[4] = {x[u][ch].x, x[u][ch].y, x[u][ch].z, x[u][ch].w};
#pragma unroll
                for (int e = 0; e < 4; ++e) {
                    const float zc = o[e];
                    float g = expf(zc - lse) - (c + e == l ? 1.f : 0.f);
                    if (relu_last && !(zc > 0.f)) g = 0.f;
                    o[e] = l >= 0 ? g * s2 : 0.f;
                }
                if (c + 4 <= C) {
                    reinterpret_cast<float4*>(zr)[q] = make_float4(o[0], o[1], o[2], o[3]);
                } else {
                    for (int e = 0; c + e < C; ++e) zr[c + e] = o[e];
                }
            }
        }
    }
    // fixed-order reduction: lane-group leaders' sums in lane order, then warps
    lsum = warp_sum_d(lsum);
    if (lane == 0) wsum[wid] = lsum;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < kCeWarps; ++w) t += wsum[w];
        block_partial[blockIdx.x] = t;
    }
}

__global__ void sum_partials_kernel(const double* __restrict__ p, int count, double* __restrict__ out) {
    // one warp, strided lane sums then fixed xor tree
    double t = 0.0;
    for (int i = threadIdx.x; i < count; i += 32) t += p[i];
    t = warp_sum_d(t);
    if (threadIdx.x == 0) *out = t;
}

__global__ void count_labelled_kernel(const int32_t* __restrict__ y, int64_t n, int64_t* __restrict__ out) {
    __shared__ long long ws[32];
    long long c = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        c += y[i] >= 0 ? 1 : 0;
    for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
    if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = c;
    __syncthreads();
    if (threadIdx.x == 0) {
        long long t = 0;
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += ws[w];
        out[blockIdx.x] = t;
    }
}

// Adam (Kingma & Ba, Alg. 1): bias-corrected, eps outside the sqrt.
__global__ void adam_kernel(float* __restrict__ W, const float* __restrict__ g, float* __restrict__ m,
                            float* __restrict__ v, int64_t count, double lr, double b1, double b2, double eps,
                            double c1, double c2) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x) {
        const double gi = g[i];
        const double mi = b1 * (double)m[i] + (1.0 - b1) * gi;
        const double vi = b2 * (double)v[i] + (1.0 - b2) * gi * gi;
        m[i] = (float)mi;
        v[i] = (float)vi;
        W[i] = (float)((double)W[i] - lr * (mi / c1) / (sqrt(vi / c2) + eps));
    }
}

struct PtrArray {
    const float* p[64];
};

__global__ void sum_buffers_kernel(PtrArray in, int nin, float* __restrict__ out, int64_t count) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x) {
        float t = in.p[0][i];
        for (int r = 1; r < nin; ++r) t += in.p[r][i];
        out[i] = t;
    }
}

__global__ void sum_i64_kernel(const int64_t* in, int nin, int64_t* out) {
    int64_t t = 0;
    for (int r = 0; r < nin; ++r) t += in[r];
    *out = t;
}

__global__ void sum_f64_kernel(const double* in, int nin, double* out) {
    double t = 0;
    for (int r = 0; r < nin; ++r) t += in[r];
    *out = t;
}

__global__ void scale_rows_kernel(const float* __restrict__ in, int64_t ldi, float* __restrict__ out, int64_t ldo,
                                  int64_t n, int width, const float* __restrict__ rowscale) {
    const int64_t total = n * width;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = i / width;
        const int c = (int)(i % width);
        out[r * ldo + c] = in[r * ldi + c] * (rowscale ? rowscale[r] : 1.f);
    }
}

__global__ void splitk_reduce_kernel(const float* __restrict__ partial, int k_chunks, int64_t M, int64_t N,
                                     float* __restrict__ C, int64_t ldc) {
    const int64_t total = M * N;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        float t = 0.f;
        for (int k = 0; k < k_chunks; ++k) t += partial[(int64_t)k * total + i];
        C[(i / N) * ldc + (i % N)] = t;
    }
}

// 1.5D pair finish: v = (a + b) [* rowscale[r]] [max(., 0)], written to a
// (and b when given).  float4 over the first ceil(width / 4) * 4 columns
// (ld is a multiple of 4; padding columns stay 0 + 0 = 0).
__global__ void pair_epilogue_kernel(float4* __restrict__ a, float4* __restrict__ b, int64_t rows, int w4,
                                     int64_t ld4, const float* __restrict__ rowscale, int relu) {
    const int64_t total = rows * w4;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = i / w4;
        const int64_t o = r * ld4 + (i - r * w4);
        float4 v = a[o];
        if (b) {
            const float4 u = b[o];
            v.x += u.x; v.y += u.y; v.z += u.z; v.w += u.w;
        }
        if (rowscale) {
            const float sc = rowscale[r];
            v.x *= sc; v.y *= sc; v.z *= sc; v.w *= sc;
        }
        if (relu) {
            v.x = fmaxf(v.x, 0.f); v.y = fmaxf(v.y, 0.f); v.z = fmaxf(v.z, 0.f); v.w = fmaxf(v.w, 0.f);
        }
        a[o] = v;
        if (b) b[o] = v;
    }
}

}  // namespace

cudaError_t launch_softmax_ce(float* Z, int64_t n, int C, int64_t ld, const int32_t* y, const int64_t* ntrain,
                              const float* rowscale, int relu_last, double* block_partial, cudaStream_t s) {
    // row-group shapes: G lanes x CH float4 per lane cover C columns (ld is a multiple of 4)
#define MGGCN_CE(G, CH, U) \
    softmax_ce_vec_kernel<G, CH, U><<<kCeBlocks, kCeWarps * 32, 0, s>>>(Z, n, C, ld, y, ntrain, rowscale, relu_last, \
                                                                        block_partial)
    if ((ld & 3) == 0 && (reinterpret_cast<uintptr_t>(Z) & 15) == 0 && C <= 256) {
        if (C <= 16) MGGCN_CE(4, 1, 4);
        else if (C <= 32) MGGCN_CE(8, 1, 4);
        else if (C <= 64) MGGCN_CE(16, 1, 4);
        else if (C <= 128) MGGCN_CE(32, 1, 4);
        else MGGCN_CE(32, 2, 2);
    } else {
        softmax_ce_kernel<<<kCeBlocks, kCeWarps * 32, 0, s>>>(Z, n, C, ld, y, ntrain, rowscale, relu_last,
                                                              block_partial);
    }
#undef MGGCN_CE
    count_launches(1);
    return cudaGetLastError();
}

__global__ void spin_kernel(uint64_t ns) {
    uint64_t t0, t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    do {
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    } while (t - t0 < ns);
}

cudaError_t launch_spin(uint64_t ns, cudaStream_t s) {
    spin_kernel<<<1, 1, 0, s>>>(ns);
    count_launches(1);
    return cudaGetLastError();
}

cudaError_t launch_sum_partials(const double* partial, int count, double* out, cudaStream_t s) {
    sum_partials_kernel<<<1, 32, 0, s>>>(partial, count, out);
    count_launches(1);
    return cudaGetLastError();
}

cudaError_t launch_count_labelled(const int32_t* y, int64_t n, int64_t* scratch, int64_t* out, cudaStream_t s) {
    count_labelled_kernel<<<kCountBlocks, 512, 0, s>>>(y, n, scratch);
    count_launches(1);
    sum_i64_kernel<<<1, 1, 0, s>>>(scratch, kCountBlocks, out);
    count_launches(1);
    return cudaGetLastError();
}

static int adam_blocks(int64_t count) {
    int blocks = (int)((count + 255) / 256);
    if (blocks > 1184) blocks = 1184;
    if (blocks < 1) blocks = 1;
    return blocks;
}

cudaError_t launch_adam(float* W, const float* g, float* m, float* v, int64_t count, double lr, double b1, double b2,
                        double eps, int64_t t, cudaStream_t s) {
    const double c1 = 1.0 - std::pow(b1, (double)t), c2 = 1.0 - std::pow(b2, (double)t);
    adam_kernel<<<adam_blocks(count), 256, 0, s>>>(W, g, m, v, count, lr, b1, b2, eps, c1, c2);
    count_launches(1);
    return cudaGetLastError();
}

// Captured epochs (mggcn_epoch_capture): Adam's bias corrections depend on the
// step count t, a kernel argument, so every replay re-sets the Adam node's
// arguments for its own t before the graph is launched.
const void* adam_kernel_func() { return reinterpret_cast<const void*>(&adam_kernel); }

cudaError_t graph_set_adam(cudaGraphExec_t ex, cudaGraphNode_t node, float* W, const float* g, float* m, float* v,
                           int64_t count, double lr, double b1, double b2, double eps, int64_t t) {
    double c1 = 1.0 - std::pow(b1, (double)t), c2 = 1.0 - std::pow(b2, (double)t);
    void* args[] = {&W, &g, &m, &v, &count, &lr, &b1, &b2, &eps, &c1, &c2};
    cudaKernelNodeParams p = {};
    p.func = const_cast<void*>(adam_kernel_func());
    p.gridDim = dim3((unsigned)adam_blocks(count));
    p.blockDim = dim3(256);
    p.sharedMemBytes = 0;
    p.kernelParams = args;
    p.extra = nullptr;
    return cudaGraphExecKernelNodeSetParams(ex, node, &p);
}

cudaError_t launch_sum_buffers(const float* const* in, int nin, float* out, int64_t count, cudaStream_t s) {
    if (nin < 1 || nin > 64) return cudaErrorInvalidValue;
    PtrArray a{};
    for (int i = 0; i < nin; ++i) a.p[i] = in[i];
    int blocks = (int)((count + 255) / 256);
    if (blocks > 1184) blocks = 1184;
    if (blocks < 1) blocks = 1;
    sum_buffers_kernel<<<blocks, 256, 0, s>>>(a, nin, out, count);
    count_launches(1);
    return cudaGetLastError();
}

cudaError_t launch_sum_i64(const int64_t* in, int nin, int64_t* out, cudaStream_t s) {
    sum_i64_kernel<<<1, 1, 0, s>>>(in, nin, out);
    count_launches(1);
    return cudaGetLastError();
}

cudaError_t launch_sum_f64(const double* in, int nin, double* out, cudaStream_t s) {
    sum_f64_kernel<<<1, 1, 0, s>>>(in, nin, out);
    count_launches(1);
    return cudaGetLastError();
}

cudaError_t launch_scale_rows(const float* in, int64_t ldi, float* out, int64_t ldo, int64_t n, int width,
                              const float* rowscale, cudaStream_t s) {
    int64_t total = n * width;
    int blocks = (int)((total + 255) / 256);
    if (blocks > 4736) blocks = 4736;
    if (blocks < 1) blocks = 1;
    scale_rows_kernel<<<blocks, 256, 0, s>>>(in, ldi, out, ldo, n, width, rowscale);
    count_launches(1);
    return cudaGetLastError();
}

cudaError_t launch_splitk_reduce(const float* partial, int k_chunks, int64_t M, int64_t N, float* C, int64_t ldc,
                                 cudaStream_t s) {
    int64_t total = M * N;
    int blocks = (int)((total + 255) / 256);
    if (blocks > 1184) blocks = 1184;
    if (blocks < 1) blocks = 1;
    splitk_reduce_kernel<<<blocks, 256, 0, s>>>(partial, k_chunks, M, N, C, ldc);
    count_launches(1);
    return cudaGetLastError();
}

}  // namespace mggcn

namespace mggcn {
static std::atomic<long long> g_launches{0};
void count_launches(int n) { g_launches.fetch_add(n, std::memory_order_relaxed); }
}  // namespace mggcn

extern "C" int64_t mggcn_kernel_launch_count(void) { return (int64_t)mggcn::g_launches.load(); }

namespace mggcn {

static cudaError_t launch_pair(float* a, float* b, int64_t rows, int width, int64_t ld, const float* rowscale,
                               int relu, cudaStream_t s) {
    if (rows <= 0) return cudaSuccess;
    if ((ld & 3) || (reinterpret_cast<uintptr_t>(a) & 15) || (reinterpret_cast<uintptr_t>(b) & 15))
        return cudaErrorInvalidValue;
    const int w4 = (width + 3) / 4;
    const int64_t total = rows * w4;
    int64_t blocks = (total + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    pair_epilogue_kernel<<<(unsigned)blocks, 256, 0, s>>>(reinterpret_cast<float4*>(a), reinterpret_cast<float4*>(b),
                                                          rows, w4, ld / 4, rowscale, relu);
    count_launches(1);
    return cudaGetLastError();
}

cudaError_t launch_pair_sum_epilogue(float* a, float* b, int64_t rows, int width, int64_t ld, const float* rowscale,
                                     int relu, cudaStream_t s) {
    return launch_pair(a, b, rows, width, ld, rowscale, relu, s);
}

cudaError_t launch_rows_epilogue(float* a, int64_t rows, int width, int64_t ld, const float* rowscale, int relu,
                                 cudaStream_t s) {
    return launch_pair(a, nullptr, rows, width, ld, rowscale, relu, s);
}

}  // namespace mggcn
