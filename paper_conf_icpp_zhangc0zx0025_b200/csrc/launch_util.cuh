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

// Launch with a 1-D thread-block cluster of `cluster` CTAs (cluster split).
template <class Kernel, class... Args>
inline cudaError_t launch_cluster(Kernel k, unsigned grid, unsigned block, size_t smem, cudaStream_t stream,
                                  int cluster, Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(block);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = (unsigned)cluster;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k, args...);
}

}  // namespace winrs
