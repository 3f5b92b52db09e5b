// Fused block-group reduction + cross-rank all-reduce over peer memory
// (DESIGN.md §8.1).
//
// The data-parallel BFC ends with two reductions of the same |dW| tensor: the
// block-group (bucket) reduction inside a rank (§3 P@17126: "launch a
// reduction kernel to sum all nabla W buckets"; §5.2 P@39101: FP32 Kahan
// summation) and the sum over the ranks' batch shards.  This kernel does both
// in one persistent, cooperative launch over peer-mapped buffers (CUDA IPC:
// other processes on the same node, NVLink peers or, in the tests, processes
// sharing one GPU):
//   phase 1  every element: Kahan sum of the Z buckets in z order (exactly the
//            arithmetic of bucket_reduce_kernel) -> this rank's staging buffer;
//   barrier  all CTAs of all ranks (flag words written with st.release.sys,
//            polled with ld.acquire.sys);
//   phase 2  rank r owns the element slice r: sum of the W staging buffers in
//            rank order 0..W-1 (FP32), stored into every rank's dW;
//   barrier  so that every rank's dW is complete when its kernel returns.
// The result is deterministic and identical on every rank; it equals the
// unfused path "bucket reduction, then an FP32 sum over ranks in rank order"
// bit for bit.  A rank that never arrives makes the spin time out (~20 s) and
// trap: the launch fails instead of hanging.
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include "registry.h"

namespace winrs {

// PeerArgs (registry.h): each rank's staging buffer (|dW| floats), dW, and
// flag block ([0, AR_MAX) barrier A, [AR_MAX, 2 AR_MAX) barrier B, then the
// rank's own CTA arrival counter).

namespace {

__device__ __forceinline__ void kahan_add(float& s, float& c, float x) {
    const float y = x - c;
    const float t = s + y;
    c = (t - s) - y;
    s = t;
}

__device__ __forceinline__ unsigned int ld_acquire_sys(const unsigned int* p) {
    unsigned int v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(unsigned int* p, unsigned int v) {
    asm volatile("st.release.sys.global.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}

// Grid-wide + cross-rank barrier.  counter: this rank's local arrival counter
// (reset by the last CTA); slot: 0 (A) or AR_MAX (B).
__device__ void rank_barrier(const PeerArgs& pa, unsigned int* counter, int slot, int rank, int world,
                             unsigned int epoch) {
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence_system();
        const unsigned int arrived = atomicAdd(counter, 1u) + 1;
        if (arrived == gridDim.x) {          // last CTA of this rank: publish to every rank
            atomicExch(counter, 0u);
            __threadfence_system();
            for (int q = 0; q < world; ++q) st_release_sys(pa.flags[q] + slot + rank, epoch);
        }
        const unsigned int* mine = pa.flags[rank] + slot;
        long long t0 = clock64();
        for (int q = 0; q < world; ++q) {
            while (ld_acquire_sys(mine + q) != epoch) {
                if (clock64() - t0 > 40000000000LL) __trap();   // ~20 s: a rank never arrived
            }
        }
    }
    __syncthreads();
}

__global__ void __launch_bounds__(256)
fused_reduce_allreduce_kernel(const float* __restrict__ dW_local, const float* __restrict__ ws, long long n, int Z,
                              PeerArgs pa, unsigned int* counter, int rank, int world, unsigned int epoch) {
    const long long stride = (long long)gridDim.x * blockDim.x;
    const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    // ---- phase 1: bucket reduction (float4 body + scalar tail, z order, Kahan)
    const long long n4 = n / 4;
    float* stage = pa.stage[rank];
    for (long long i = tid; i < n4; i += stride) {
        float4 s = reinterpret_cast<const float4*>(dW_local)[i];
        float4 c = make_float4(0.f, 0.f, 0.f, 0.f);
        for (int z = 1; z < Z; ++z) {
            const float4 x = __ldcs(reinterpret_cast<const float4*>(ws + (long long)(z - 1) * n) + i);
            kahan_add(s.x, c.x, x.x);
            kahan_add(s.y, c.y, x.y);
            kahan_add(s.z, c.z, x.z);
            kahan_add(s.w, c.w, x.w);
        }
        reinterpret_cast<float4*>(stage)[i] = s;
    }
    for (long long i = n4 * 4 + tid; i < n; i += stride) {
        float s = dW_local[i], c = 0.f;
        for (int z = 1; z < Z; ++z) kahan_add(s, c, ws[(long long)(z - 1) * n + i]);
        stage[i] = s;
    }
    rank_barrier(pa, counter, 0, rank, world, epoch);
    // ---- phase 2: this rank's slice, summed over ranks in order, stored to every rank
    const long long lo = n4 * rank / world, hi = n4 * (rank + 1) / world;
    for (long long i = lo + tid; i < hi; i += stride) {
        float4 s = __ldcg(reinterpret_cast<const float4*>(pa.stage[0]) + i);
        for (int q = 1; q < world; ++q) {
            const float4 x = __ldcg(reinterpret_cast<const float4*>(pa.stage[q]) + i);
            s.x += x.x;
            s.y += x.y;
            s.z += x.z;
            s.w += x.w;
        }
        for (int q = 0; q < world; ++q) __stcg(reinterpret_cast<float4*>(pa.dW[q]) + i, s);
    }
    if (rank == world - 1) {   // scalar tail: the last rank
        for (long long i = n4 * 4 + tid; i < n; i += stride) {
            float s = __ldcg(pa.stage[0] + i);
            for (int q = 1; q < world; ++q) s += __ldcg(pa.stage[q] + i);
            for (int q = 0; q < world; ++q) __stcg(pa.dW[q] + i, s);
        }
    }
    rank_barrier(pa, counter, AR_MAX, rank, world, epoch);
}

}  // namespace

cudaError_t launch_fused_reduce_allreduce(const float* dW_local, const float* ws, long long n, int Z,
                                          const PeerArgs& pa, unsigned int* counter, int rank, int world,
                                          unsigned int epoch, int num_sms, cudaStream_t stream) {
    // persistent cooperative grid: every CTA resident (the barriers spin)
    int per_sm = 0;
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fused_reduce_allreduce_kernel, 256, 0);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) return cudaErrorLaunchOutOfResources;
    long long want = (n / 4 + 255) / 256;
    const long long cap = (long long)num_sms * (per_sm < 2 ? per_sm : 2);
    if (want > cap) want = cap;
    if (want < 1) want = 1;
    PeerArgs a = pa;
    void* args[] = {(void*)&dW_local, (void*)&ws, (void*)&n, (void*)&Z, (void*)&a, (void*)&counter,
                    (void*)&rank, (void*)&world, (void*)&epoch};
    return cudaLaunchCooperativeKernel((const void*)fused_reduce_allreduce_kernel, dim3((unsigned)want), dim3(256),
                                       args, 0, stream);
}

}  // namespace winrs
