// Block-group (bucket) reduction: dW = sum_{z<Z} bucket_z with FP32 Kahan
// summation in fixed z order (§3 P@17126 "launch a reduction kernel
// to sum all nabla W buckets"; §5.2 P@39101 "The reduction kernel sums all
// partition results using FP32 Kahan summation").  Bucket 0 is dW itself,
// buckets 1..Z-1 are contiguous in the workspace (P@15661).
//
// HBM-bound: reads Z*|dW|*4 bytes and writes |dW|*4 bytes.  128-bit loads,
// grid sized to a multiple of the SM count, deterministic (no atomics).
#include <cuda_runtime.h>
#include <stdint.h>

namespace winrs {

struct Kahan4 {
    float4 s, c;
};

__device__ __forceinline__ void kahan_add(float& s, float& c, float x) {
    const float y = x - c;
    const float t = s + y;
    c = (t - s) - y;
    s = t;
}

__global__ void __launch_bounds__(256)
bucket_reduce_kernel(float* __restrict__ dW, const float* __restrict__ ws, long long n, int Z) {
    const long long n4 = n >> 2;
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += stride) {
        float4 s = reinterpret_cast<const float4*>(dW)[i];
        float4 c = make_float4(0.f, 0.f, 0.f, 0.f);
        for (int z = 1; z < Z; ++z) {
            const float4 x = __ldcs(reinterpret_cast<const float4*>(ws + (long long)(z - 1) * n) + i);
            kahan_add(s.x, c.x, x.x);
            kahan_add(s.y, c.y, x.y);
            kahan_add(s.z, c.z, x.z);
            kahan_add(s.w, c.w, x.w);
        }
        reinterpret_cast<float4*>(dW)[i] = s;
    }
    // scalar tail (n % 4 elements)
    for (long long i = (n4 << 2) + (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        float s = dW[i], c = 0.f;
        for (int z = 1; z < Z; ++z) kahan_add(s, c, ws[(long long)(z - 1) * n + i]);
        dW[i] = s;
    }
}

cudaError_t launch_bucket_reduce(float* dW, const float* ws, long long n, int Z, int num_sms,
                                 cudaStream_t stream) {
    if (Z <= 1) return cudaSuccess;
    const long long n4 = (n + 3) / 4;
    long long blocks = (n4 + 255) / 256;
    const long long cap = (long long)num_sms * 8;
    if (blocks > cap) blocks = cap - cap % num_sms;
    if (blocks < 1) blocks = 1;
    bucket_reduce_kernel<<<(unsigned)blocks, 256, 0, stream>>>(dW, ws, n, Z);
    return cudaGetLastError();
}

}  // namespace winrs
