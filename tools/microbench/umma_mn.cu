// Layout probe: one tcgen05.mma kind::f16 (M=128, N=128, K=16) with both
// operands MN-major in the 128-byte-swizzled canonical layout (atoms of
// 64 MN elements x 8 K rows = 1 KB; 16-byte chunk c of row r stored at
// chunk c ^ r).  Tries descriptor (LBO, SBO) assignments and reports which
// reproduces the CPU product.  Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t a, uint32_t lbo, uint32_t sbo, uint32_t layout) {
    return (uint64_t)((a >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) | ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) |
           (1ull << 46) | ((uint64_t)layout << 61);
}
constexpr int M = 128, N = 128, K = 16;
// byte offset of element (mn, k) in an MN-major SW128 tile whose MN atoms are
// `mn_stride` bytes apart and K atoms `k_stride` bytes apart
__host__ __device__ inline uint32_t off(int mn, int k, uint32_t mn_stride, uint32_t k_stride) {
    const int r = k % 8, c = (mn % 64) / 8;
    return (mn / 64) * mn_stride + (k / 8) * k_stride + r * 128 + ((c ^ r) * 16) + (mn % 8) * 2;
}

__global__ void k(const __half* A, const __half* B, float* D, uint32_t lbo, uint32_t sbo, uint32_t layout,
                  uint32_t amn, uint32_t ak, int mn_major) {
    extern __shared__ __align__(1024) uint8_t sm[];
    uint64_t& bar = *reinterpret_cast<uint64_t*>(sm + 16384);
    uint32_t& tbase = *reinterpret_cast<uint32_t*>(sm + 16384 + 8);
    if (threadIdx.x == 0 && (su(sm) & 1023)) printf("smem base not 1K aligned: %u\n", su(sm));
    uint8_t* sa = sm;
    uint8_t* sb = sm + 8192;
    for (int i = threadIdx.x; i < M * K; i += blockDim.x) {
        const int m = i / K, kk = i % K;
        *reinterpret_cast<__half*>(sa + off(m, kk, amn, ak)) = A[i];
        *reinterpret_cast<__half*>(sb + off(m, kk, amn, ak)) = B[i];
    }
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" :: "r"(su(&tbase)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t idesc = (1u << 4) | ((uint32_t)mn_major << 15) | ((uint32_t)mn_major << 16) | ((uint32_t)(N >> 3) << 17) |
                           ((uint32_t)(M >> 4) << 24);
    if (threadIdx.x == 0) {
        const uint64_t ad = desc(su(sa), lbo, sbo, layout), bd = desc(su(sb), lbo, sbo, layout);
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n"
                     :: "r"(tbase), "l"(ad), "l"(bd), "r"(idesc), "r"(0));
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(su(&bar)));
        asm volatile("{\n.reg .pred P;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n@!P bra W;\n}\n" :: "r"(su(&bar)));
    }
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    // warp w reads TMEM lanes 32w..32w+31 (rows m), columns n
    const int w = threadIdx.x / 32, lane = threadIdx.x % 32;
    for (int n0 = 0; n0 < N; n0 += 8) {
        uint32_t r[8];
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
                     : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                     : "r"(tbase + ((uint32_t)(32 * w) << 16) + n0));
        asm volatile("tcgen05.wait::ld.sync.aligned;");
        for (int i = 0; i < 8; ++i) D[(32 * w + lane) * N + n0 + i] = __uint_as_float(r[i]);
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" :: "r"(tbase));
}

int main() {
    __half hA[M * K], hB[N * K];
    float ref[M * N];
    for (int i = 0; i < M * K; ++i) hA[i] = __float2half((float)((i * 7 + 3) % 11 - 5));
    for (int i = 0; i < N * K; ++i) hB[i] = __float2half((float)((i * 5 + 1) % 9 - 4));
    for (int m = 0; m < M; ++m)
        for (int n = 0; n < N; ++n) {
            float s = 0;
            for (int kk = 0; kk < K; ++kk) s += __half2float(hA[m * K + kk]) * __half2float(hB[n * K + kk]);
            ref[m * N + n] = s;
        }
    __half *dA, *dB;
    float* dD;
    cudaMalloc(&dA, sizeof(hA));
    cudaMalloc(&dB, sizeof(hB));
    cudaMalloc(&dD, sizeof(ref));
    cudaMemcpy(dA, hA, sizeof(hA), cudaMemcpyHostToDevice);
    cudaMemcpy(dB, hB, sizeof(hB), cudaMemcpyHostToDevice);
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 20000);
    struct V { uint32_t lbo, sbo, layout, amn, ak; const char* name; } vs[] = {
        {1024, 2048, 2, 1024, 2048, "SW128 lbo=MNstride(1K) sbo=Kstride(2K)"},
        {2048, 1024, 2, 1024, 2048, "SW128 lbo=Kstride(2K) sbo=MNstride(1K)"},
        {2048, 1024, 2, 2048, 1024, "SW128 lbo=MNstride(2K) sbo=Kstride(1K)"},
        {1024, 2048, 2, 2048, 1024, "SW128 lbo=Kstride(1K) sbo=MNstride(2K)"},
        {1024, 2048, 1, 1024, 2048, "layout1 lbo=MN sbo=K"},
        {2048, 1024, 1, 1024, 2048, "layout1 lbo=K sbo=MN"},
    };
    for (auto& v : vs) {
        cudaMemset(dD, 0, sizeof(ref));
        k<<<1, 128, 20000>>>(dA, dB, dD, v.lbo, v.sbo, v.layout, v.amn, v.ak, 1);
        cudaError_t e = cudaDeviceSynchronize();
        float hD[M * N];
        cudaMemcpy(hD, dD, sizeof(hD), cudaMemcpyDeviceToHost);
        double err = 0;
        for (int i = 0; i < M * N; ++i) err = fmax(err, fabs(hD[i] - ref[i]));
        printf("%-44s max|err| = %g  (%s)\n", v.name, err, cudaGetErrorString(e));
        if (e != cudaSuccess) return 1;
    }
    return 0;
}
