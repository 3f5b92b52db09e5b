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
#include <stdlib.h>

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

// The bucket loads of a group of ZB are issued together (they are independent)
// and then added in z order, so a thread waits for one memory latency per ZB
// buckets instead of one per bucket; small dW uses one float per thread so
// the grid still covers the SMs.  The summation order is unchanged.
#ifndef WINRS_REDUCE_ZB
#define WINRS_REDUCE_ZB 8   // layer times with the reduction (tools/ab_reduce_zb.sh): VGG conv1_2 (Z = 336)
#endif                      // 652 / 761 / 660 us at ZB = 8 / 16 / 32 -- deeper batches did not pay
template <class V> constexpr int zbatch() { return sizeof(V) == 4 ? WINRS_REDUCE_ZB : (WINRS_REDUCE_ZB < 16 ? WINRS_REDUCE_ZB : 16); }

template <class V>
__device__ __forceinline__ void kahan_v(V& s, V& c, const V& x);
template <>
__device__ __forceinline__ void kahan_v<float4>(float4& s, float4& c, const float4& x) {
    kahan_add(s.x, c.x, x.x);
    kahan_add(s.y, c.y, x.y);
    kahan_add(s.z, c.z, x.z);
    kahan_add(s.w, c.w, x.w);
}
template <>
__device__ __forceinline__ void kahan_v<float>(float& s, float& c, const float& x) {
    kahan_add(s, c, x);
}
template <class V> __device__ __forceinline__ V vzero();
template <> __device__ __forceinline__ float4 vzero<float4>() { return make_float4(0.f, 0.f, 0.f, 0.f); }
template <> __device__ __forceinline__ float vzero<float>() { return 0.f; }

// V = float4: i indexes float4 groups of the first n/4*4 elements; V = float: all n elements.
template <class V>
__global__ void __launch_bounds__(256)
bucket_reduce_kernel(float* __restrict__ dW, const float* __restrict__ ws, long long n, int Z) {
    constexpr int W = sizeof(V) / 4;
    constexpr int ZB = zbatch<V>();
    // Launched as a programmatic dependent of the BFC kernel: wait until that
    // grid has completed and its bucket writes are visible (a no-op otherwise).
    asm volatile("griddepcontrol.wait;" ::: "memory");
    const long long nv = n / W;
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nv; i += stride) {
        V s = reinterpret_cast<const V*>(dW)[i];
        V c = vzero<V>();
        for (int z0 = 1; z0 < Z; z0 += ZB) {
            V x[ZB];
#pragma unroll
            for (int j = 0; j < ZB; ++j)
                if (z0 + j < Z) x[j] = __ldcs(reinterpret_cast<const V*>(ws + (long long)(z0 + j - 1) * n) + i);
#pragma unroll
            for (int j = 0; j < ZB; ++j)
                if (z0 + j < Z) kahan_v<V>(s, c, x[j]);
        }
        reinterpret_cast<V*>(dW)[i] = s;
    }
    if (W > 1) {   // scalar tail (n % 4 elements)
        for (long long i = nv * W + (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
            float s = dW[i], c = 0.f;
            for (int z = 1; z < Z; ++z) kahan_add(s, c, ws[(long long)(z - 1) * n + i]);
            dW[i] = s;
        }
    }
}

cudaError_t launch_bucket_reduce(float* dW, const float* ws, long long n, int Z, int num_sms,
                                 cudaStream_t stream) {
    if (Z <= 1) return cudaSuccess;
    const long long cap = (long long)num_sms * 8;
    // one float per thread while a float4 per thread would leave SMs idle
    const bool scalar = (n / 4 + 255) / 256 < num_sms;
    const long long items = scalar ? n : n / 4 + (n % 4 ? 1 : 0);
    long long blocks = (items + 255) / 256;
    if (blocks > cap) blocks = cap - cap % num_sms;
    if (blocks < 1) blocks = 1;
    // Programmatic stream serialisation: the reduction is scheduled once every
    // CTA of the BFC kernel ahead of it has started (griddepcontrol.launch_dependents
    // in the tc kernels; kernels without it trigger at exit) and waits on the
    // device, so its launch latency overlaps the BFC kernel's tail.
    // WINRS_PDL=0 launches it plainly (A/B).
    static const bool pdl = [] { const char* v = getenv("WINRS_PDL"); return !(v && v[0] == '0'); }();
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.gridDim = dim3((unsigned)blocks);
    cfg.blockDim = dim3(256);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = stream;
    cfg.attrs = attr;
    cfg.numAttrs = pdl ? 1 : 0;
    if (scalar)
        return cudaLaunchKernelEx(&cfg, bucket_reduce_kernel<float>, dW, ws, n, Z);
    return cudaLaunchKernelEx(&cfg, bucket_reduce_kernel<float4>, dW, ws, n, Z);
}

}  // namespace winrs
