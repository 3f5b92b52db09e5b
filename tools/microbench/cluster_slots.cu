// How many thread-block clusters of size cs can be co-resident on this GPU
// with one 227 KB-smem CTA per SM (the FP16 BFC kernel's footprint):
// cudaOccupancyMaxActiveClusters for cs = 1..8 (and 16, non-portable).
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k(int* p) {
    extern __shared__ int s[];
    if (p) p[blockIdx.x] = s[threadIdx.x];
}

int main() {
    const int smem = 227 * 1024;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    for (int cs : {1, 2, 3, 4, 5, 6, 7, 8, 10, 12, 16}) {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(cs * 64);
        cfg.blockDim = dim3(320);
        cfg.dynamicSmemBytes = smem;
        cudaLaunchAttribute a[1];
        a[0].id = cudaLaunchAttributeClusterDimension;
        a[0].val.clusterDim.x = cs;
        a[0].val.clusterDim.y = 1;
        a[0].val.clusterDim.z = 1;
        cfg.attrs = a;
        cfg.numAttrs = 1;
        int n = -1;
        cudaError_t e = cudaOccupancyMaxActiveClusters(&n, k, &cfg);
        printf("cluster %2d: max active clusters %3d -> %3d SMs (%s)\n", cs, n, n * cs, cudaGetErrorString(e));
    }
    return 0;
}
