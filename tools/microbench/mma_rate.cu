// Microbenchmark: tcgen05.mma kind::f16 (M=128, K=16) issue/complete rate on
// sm_100a for SS operands in the K-major no-swizzle layout (LBO/SBO as in
// bfc_f16.cuh) vs N.  One CTA per SM, one thread issues `iters` x `per` MMAs,
// commits to an mbarrier after each group and waits; reports cycles per MMA.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t a, uint32_t lbo, uint32_t sbo, uint32_t layout) {
    return (uint64_t)((a >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) | ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) |
           (1ull << 46) | ((uint64_t)layout << 61);
}

template <int N, bool TS = false, int M = 128>
__global__ void __launch_bounds__(128, 1) k(unsigned long long* out, int iters, int per, uint32_t lbo, uint32_t sbo, int layout) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint64_t bar;
    __shared__ uint32_t tbase;
    const int warp = threadIdx.x / 32;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    for (int i = threadIdx.x; i < 64 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = 0x3c003c00u;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" :: "r"(smem_u32(&tbase)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t idesc = (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
    if (threadIdx.x == 0) {
        const uint32_t a0 = smem_u32(sm), b0 = smem_u32(sm + 32 * 1024);
        uint32_t ph = 0;
        long long t0 = clock64();
        for (int it = 0; it < iters; ++it) {
            for (int x = 0; x < per; ++x) {
                const uint64_t ad = desc(a0 + (x & 7) * 4096, lbo, sbo, layout);
                const uint64_t bd = desc(b0 + (x & 7) * 2048, lbo, sbo, layout);
                const uint32_t d = tbase + (uint32_t)((x * N) & 255);
                if constexpr (TS) {
                    const uint32_t at = tbase + 256 + (uint32_t)((x & 7) * 8);   // A (128 x 16 f16) in TMEM
                    asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}\n"
                                 :: "r"(d), "r"(at), "l"(bd), "r"(idesc), "r"(1));
                } else {
                    asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n"
                                 :: "r"(d), "l"(ad), "l"(bd), "r"(idesc), "r"(1));
                }
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(smem_u32(&bar)));
            asm volatile("{\n.reg .pred P;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n@!P bra W;\n}\n"
                         :: "r"(smem_u32(&bar)), "r"(ph));
            ph ^= 1;
        }
        long long t1 = clock64();
        out[blockIdx.x] = (unsigned long long)(t1 - t0);
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(tbase));
}

template <int N, bool TS = false, int M = 128>
void run(int per, uint32_t lbo, uint32_t sbo, int layout, const char* name) {
    unsigned long long* d;
    cudaMalloc(&d, 8 * 148);
    cudaFuncSetAttribute(k<N, TS, M>, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024 + 1024);
    const int iters = 200;
    k<N, TS, M><<<148, 128, 64 * 1024 + 1024>>>(d, iters, per, lbo, sbo, layout);
    cudaError_t e = cudaDeviceSynchronize();
    unsigned long long h[148];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < 148; ++i) avg += h[i];
    avg /= 148;
    const double cyc = avg / iters / per;
    printf("%-28s N=%3d per=%2d: %7.1f cycles/MMA  -> %6.0f MAC/clk/SM (%s)\n", name, N, per, cyc,
           (double)M * N * 16 / cyc, cudaGetErrorString(e));
    cudaFree(d);
}

int main() {
    for (int per : {8, 32}) {
        run<64>(per, 128, 256, 0, "SS noswz M128");
        run<64, false, 64>(per, 128, 256, 0, "SS noswz M64");
        run<128>(per, 128, 256, 0, "SS noswz M128");
        run<128, false, 64>(per, 128, 256, 0, "SS noswz M64");
    }
    return 0;
}
