// Microbenchmark (round 2): tcgen05.mma kind::f16 rate on sm_100a as a
// function of operand layout (K-major SWIZZLE_NONE vs SWIZZLE_128B), N,
// A-from-TMEM (TS) and cta_group::2 (M = 256 over an SM pair).  One CTA (or
// CTA pair) per SM, one thread issues `per` MMAs round-robin over `nd`
// accumulators (the alpha-batched EWM pattern), commits, waits; reports
// cycles per MMA and MAC/clk/SM.  Timing only: operand contents are junk.
// Build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a mma_rate2.cu -o /tmp/mma_rate2
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t a, uint32_t lbo, uint32_t sbo, uint32_t layout) {
    return (uint64_t)((a >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) | ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) |
           (1ull << 46) | ((uint64_t)layout << 61);
}
__device__ __forceinline__ uint32_t cta_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}

// MODE 0: SS cta_group::1; 1: TS cta_group::1; 2: SS cta_group::2 (M = 256)
template <int MODE, int N, int layout, int fixa, int nd, int MN = 0>
__global__ void __launch_bounds__(128, 1) kmma(unsigned long long* out, int iters) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint64_t bar;
    __shared__ uint32_t tbase;
    const int warp = threadIdx.x / 32;
    constexpr bool PAIR = MODE == 2;
    const uint32_t rank = PAIR ? cta_rank() : 0;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    for (int i = threadIdx.x; i < 128 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = 0x3c003c00u;
    if (warp == 0) {
        if (PAIR) {
            asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" :: "r"(su(&tbase)));
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
        } else {
            asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" :: "r"(su(&tbase)));
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
        }
    }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (PAIR) asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    asm volatile("tcgen05.fence::after_thread_sync;");
    constexpr int M = PAIR ? 256 : 128;
    const uint32_t idesc = (1u << 4) | ((uint32_t)MN << 15) | ((uint32_t)MN << 16) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
    // no swizzle K-major: core matrices 8 rows x 16 B, LBO (K) = 128, SBO (8-row groups) = 256.
    // SW128 K-major: 8-row atoms of 128 B rows (1 KB), SBO = 1024, K step = +32 B inside the atom.
    const uint32_t lbo = MN ? 2048 : (layout == 0 ? 128 : 16), sbo = layout == 0 ? 256 : 1024;
    if (threadIdx.x == 0 && rank == 0) {
        const uint32_t a0 = su(sm), b0 = su(sm + 64 * 1024);
        uint32_t ph = 0;
        long long t0 = clock64();
        const uint64_t ad0 = desc(a0, lbo, sbo, layout), bd0 = desc(b0, lbo, sbo, layout);
        const int ndd = MODE == 1 && nd * N > 256 ? (256 / N > 0 ? 256 / N : 1) : nd;
        for (int it = 0; it < iters; ++it) {
#pragma unroll
            for (int x = 0; x < 64; ++x) {
                // A slab: 128 rows x K16 = 4 KB (none) / a 32-B column of a 16 KB atom block (SW128)
                const uint32_t aoff = fixa ? 0 : (layout == 0 ? (x & 7) * 4096 : (x & 3) * 16384 + ((x >> 2) & 3) * 32);
                const uint32_t boff = layout == 0 ? (x & 3) * 8192 : ((x >> 2) & 3) * 32;
                const uint64_t ad = ad0 + ((aoff & 0xFFFF) >> 4);
                const uint64_t bd = bd0 + (boff >> 4);
                const uint32_t d = tbase + (uint32_t)((x & (ndd - 1)) * N);
                if constexpr (MODE == 1) {
                    const uint32_t at = tbase + 256 + (uint32_t)((x & 7) * 8);
                    asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}\n"
                                 :: "r"(d), "r"(at), "l"(bd), "r"(idesc), "r"(1));
                } else if constexpr (MODE == 2) {
                    asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n}\n"
                                 :: "r"(d), "l"(ad), "l"(bd), "r"(idesc), "r"(1));
                } else {
                    asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n"
                                 :: "r"(d), "l"(ad), "l"(bd), "r"(idesc), "r"(1));
                }
            }
            if (PAIR)
                asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                             :: "r"(su(&bar)), "h"((uint16_t)1));
            else
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(su(&bar)));
            asm volatile("{\n.reg .pred P;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n@!P bra W;\n}\n"
                         :: "r"(su(&bar)), "r"(ph));
            ph ^= 1;
        }
        long long t1 = clock64();
        out[blockIdx.x] = (unsigned long long)(t1 - t0);
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (PAIR) asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    if (warp == 0) {
        if (PAIR) asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" :: "r"(tbase));
        else asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(tbase));
    }
}

template <int MODE, int N, int layout, int nd, int fixa, int MN = 0>
void run(const char* name) {
    const int per = 64;
    unsigned long long* d;
    cudaMalloc(&d, 8 * 148);
    cudaMemset(d, 0, 8 * 148);
    const int smem = 128 * 1024 + 1024;
    cudaFuncSetAttribute(kmma<MODE, N, layout, fixa, nd, MN>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    const int iters = 100;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(148);
    cfg.blockDim = dim3(128);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = MODE == 2 ? 2 : 1;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, kmma<MODE, N, layout, fixa, nd, MN>, d, iters);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    unsigned long long h[148];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double avg = 0;
    int cnt = 0;
    for (int i = 0; i < 148; ++i)
        if (h[i]) { avg += h[i]; ++cnt; }
    avg /= cnt ? cnt : 1;
    const double cyc = avg / iters / per;
    const int M = MODE == 2 ? 256 : 128;
    const double mac_per_sm = (double)M * N * 16 / cyc / (MODE == 2 ? 2 : 1);
    printf("%-14s %s %-6s N=%3d nd=%d fixA=%d per=%2d: %7.1f cyc/MMA %7.0f MAC/clk/SM  %s\n", name, MN ? "MN" : "K ",
           layout == 0 ? "none" : "sw128", N, nd, fixa, per, cyc, mac_per_sm, cudaGetErrorString(e));
    cudaFree(d);
}

template <int MODE, int L>
void sweep(const char* name) {
    run<MODE, 16, L, 8, 0>(name);
    run<MODE, 32, L, 8, 0>(name);
    run<MODE, 64, L, 8, 0>(name);
    run<MODE, 64, L, 8, 1>(name);
    run<MODE, 128, L, 2, 0>(name);
    run<MODE, 128, L, 4, 0>(name);
    run<MODE, 256, L, 1, 0>(name);
    run<MODE, 256, L, 2, 0>(name);
}

int main() {
    run<0, 64, 2, 8, 0, 1>("SS cg1 M128");
    run<0, 128, 2, 4, 0, 1>("SS cg1 M128");
    run<0, 256, 2, 2, 0, 1>("SS cg1 M128");
    run<0, 64, 2, 8, 0, 0>("SS cg1 M128");
    run<0, 128, 2, 4, 0, 0>("SS cg1 M128");
    run<0, 256, 2, 2, 0, 0>("SS cg1 M128");
    return 0;
}
