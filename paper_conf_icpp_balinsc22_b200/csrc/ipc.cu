// ipc.cu — SM-free block exchange over CUDA IPC (copy-engine
// variant): peers' workspaces are mapped with cudaIpcOpenMemHandle, feature
// blocks are PULLED by each receiver with cudaMemcpyAsync (copy engines over
// NVLink / NVSwitch, no SMs taken from the SpMM), and cross-process ordering
// uses monotone 32-bit sequence flags in device memory driven by the stream
// memory operations cuStreamWriteValue32 / cuStreamWaitValue32 (no host
// round trips).  Sums over ranks (W_G, |T|, loss) read every rank's partial in
// rank order, so all ranks obtain bitwise identical results.
#include <cuda.h>

#include <mutex>

#include "kernels.cuh"

namespace mggcn {

namespace {

typedef CUresult (*WaitValue32Fn)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
typedef CUresult (*WriteValue32Fn)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
typedef CUresult (*GetAddressRangeFn)(CUdeviceptr*, size_t*, CUdeviceptr);

struct DriverFns {
    WaitValue32Fn wait = nullptr;
    WriteValue32Fn write = nullptr;
    GetAddressRangeFn range = nullptr;
};

const DriverFns& drv() {
    static DriverFns f;
    static std::once_flag once;
    std::call_once(once, [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuStreamWaitValue32", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            f.wait = reinterpret_cast<WaitValue32Fn>(p);
        if (cudaGetDriverEntryPoint("cuStreamWriteValue32", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            f.write = reinterpret_cast<WriteValue32Fn>(p);
        if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            f.range = reinterpret_cast<GetAddressRangeFn>(p);
    });
    return f;
}

__global__ void sum_ranks_f32_kernel(PtrArrayF in, int nin, float* __restrict__ out, int64_t count) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x) {
        float t = in.p[0][i];
        for (int r = 1; r < nin; ++r) t += in.p[r][i];
        out[i] = t;
    }
}

__global__ void sum_ranks_scalar_kernel(PtrArrayD in_d, PtrArrayI in_i, int nin, double* out_d, int64_t* out_i) {
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        double t = 0;
        int64_t ti = 0;
        for (int r = 0; r < nin; ++r) {
            if (out_d) t += in_d.p[r][0];
            if (out_i) ti += in_i.p[r][0];
        }
        if (out_d) *out_d = t;
        if (out_i) *out_i = ti;
    }
}

}  // namespace

bool ipc_stream_memops_available() {
    const DriverFns& f = drv();
    return f.wait && f.write;
}

cudaError_t stream_write_u32(cudaStream_t s, uint32_t* addr, uint32_t value) {
    const DriverFns& f = drv();
    if (!f.write) return cudaErrorNotSupported;
    return f.write(reinterpret_cast<CUstream>(s), reinterpret_cast<CUdeviceptr>(addr), value, 0) == CUDA_SUCCESS
               ? cudaSuccess
               : cudaErrorUnknown;
}

// Waits until (int32)(*addr - value) >= 0 (CU_STREAM_WAIT_VALUE_GEQ, wrap-around safe).
cudaError_t stream_wait_u32(cudaStream_t s, const uint32_t* addr, uint32_t value) {
    const DriverFns& f = drv();
    if (!f.wait) return cudaErrorNotSupported;
    return f.wait(reinterpret_cast<CUstream>(s), reinterpret_cast<CUdeviceptr>(const_cast<uint32_t*>(addr)), value,
                  0 /* CU_STREAM_WAIT_VALUE_GEQ */) == CUDA_SUCCESS
               ? cudaSuccess
               : cudaErrorUnknown;
}

int ipc_alloc_base(const void* ptr, void** base, size_t* size) {
    const DriverFns& f = drv();
    if (!f.range) return -1;
    CUdeviceptr b = 0;
    size_t sz = 0;
    if (f.range(&b, &sz, reinterpret_cast<CUdeviceptr>(ptr)) != CUDA_SUCCESS) return -1;
    *base = reinterpret_cast<void*>(b);
    *size = sz;
    return 0;
}

cudaError_t launch_sum_ranks_f32(const float* const* in, int nin, float* out, int64_t count, cudaStream_t s) {
    if (nin < 1 || nin > 64) return cudaErrorInvalidValue;
    PtrArrayF a{};
    for (int i = 0; i < nin; ++i) a.p[i] = in[i];
    int blocks = (int)((count + 255) / 256);
    if (blocks > 1184) blocks = 1184;
    if (blocks < 1) blocks = 1;
    sum_ranks_f32_kernel<<<blocks, 256, 0, s>>>(a, nin, out, count);
    count_launches(1);
    return cudaGetLastError();
}

cudaError_t launch_sum_ranks_scalar(const double* const* in_d, const int64_t* const* in_i, int nin, double* out_d,
                                    int64_t* out_i, cudaStream_t s) {
    if (nin < 1 || nin > 64) return cudaErrorInvalidValue;
    PtrArrayD a{};
    PtrArrayI b{};
    for (int i = 0; i < nin; ++i) {
        a.p[i] = in_d ? in_d[i] : nullptr;
        b.p[i] = in_i ? in_i[i] : nullptr;
    }
    sum_ranks_scalar_kernel<<<1, 32, 0, s>>>(a, b, nin, out_d, out_i);
    count_launches(1);
    return cudaGetLastError();
}

}  // namespace mggcn
