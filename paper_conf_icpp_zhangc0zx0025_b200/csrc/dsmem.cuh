// Deterministic cluster reduction of a staged output tile through distributed
// shared memory: rank r of a cs-CTA cluster sums its row slice
// of the cs partial tiles in fixed rank order 0..cs-1.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace winrs {

// Sum over ranks 0..cs-1 (cs <= 8) of the float4 at shared-window offset
// `saddr` of each rank.  All remote loads are issued before the first add, so
// the cs DSMEM round trips overlap instead of serialising on the adds; the
// adds then run in rank order (bitwise reproducible).
// Ranks stride * q + offset (a CTA pair's halves reduce separately).
__device__ __forceinline__ float4 dsmem_sum4(uint32_t saddr, int cs, int stride = 1, int offset = 0) {
    float4 v[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
        if (q < cs) {
            uint32_t remote;
            asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(saddr), "r"(stride * q + offset));
            asm volatile("ld.shared::cluster.v4.f32 {%0, %1, %2, %3}, [%4];"
                         : "=f"(v[q].x), "=f"(v[q].y), "=f"(v[q].z), "=f"(v[q].w) : "r"(remote) : "memory");
        }
    }
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
    for (int q = 0; q < 8; ++q) {
        if (q < cs) { acc.x += v[q].x; acc.y += v[q].y; acc.z += v[q].z; acc.w += v[q].w; }
    }
    return acc;
}

__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

}  // namespace winrs
