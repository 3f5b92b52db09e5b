// Small host-side helpers shared by the kernel instantiation units.
#pragma once
#include <atomic>
#include <cuda_runtime.h>

namespace winrs {

// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) once per (kernel, device).
template <class KernelPtr>
inline cudaError_t ensure_smem_attr(KernelPtr k, size_t smem, std::atomic<unsigned long long>& done) {
    if (smem <= 48 * 1024) return cudaSuccess;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    const unsigned long long bit = 1ull << (dev & 63);
    if (done.load(std::memory_order_acquire) & bit) return cudaSuccess;
    e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess) done.fetch_or(bit, std::memory_order_acq_rel);
    return e;
}

}  // namespace winrs
