// Probe (round 2): tcgen05.mma kind::tf32 with MN-major SW128 operands of
// 32-bit elements (128-byte rows = 32 MN elements, 8 K rows per 1 KB atom),
// and the 3xTF32 split D = Ah.Bh + Ah.Bl + Al.Bh (hi = x with the low 13
// mantissa bits cleared, lo = x - hi) against an FP64 host product; then the
// issue rate of M=128 x N=64 x K=8 SS tf32 MMAs (64 per commit, 148 CTAs).
// Build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a tf32_probe.cu -o tf32_probe.bin
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t addr, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46) | (2ull << 61);
}
// D f32 (bit 4), A/B tf32 (2 at bits 7 and 10), A and B MN-major (15, 16), N>>3 @17, M>>4 @24
constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | (1u << 15) | (1u << 16) | ((64u >> 3) << 17) |
                           ((128u >> 4) << 24);
constexpr uint32_t IDESC_K = (1u << 4) | (2u << 7) | (2u << 10) | ((64u >> 3) << 17) | ((128u >> 4) << 24);
__device__ int g_kmajor;

__device__ __forceinline__ void mma(uint32_t d, uint64_t a, uint64_t b, uint32_t acc) {
    const uint32_t id = g_kmajor ? IDESC_K : IDESC;
    asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n"
                 :: "r"(d), "l"(a), "l"(b), "r"(id), "r"(acc));
}
// K-major, no swizzle: core matrices of 8 rows x 16 B (4 fp32 of K); LBO = 128 (K), SBO = 256 (8 rows)
__device__ __forceinline__ uint32_t offk(int mn, int k) {
    return (uint32_t)((mn >> 3) * 256 + (k >> 2) * 128 + (mn & 7) * 16 + (k & 3) * 4);
}
__device__ __forceinline__ uint64_t desck(uint32_t addr) {
    return (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)((128 >> 4) & 0x3FFF) << 16) |
           ((uint64_t)((256 >> 4) & 0x3FFF) << 32) | (1ull << 46);
}
__device__ __forceinline__ uint32_t hi_bits(float x) { return __float_as_uint(x) & 0xFFFFE000u; }

// element (mn, k) of an MN-major SW128 32-bit operand with MN atoms of 32 elements lbo bytes apart
__device__ __forceinline__ uint32_t off32(int mn, int k, int lbo) {
    return (uint32_t)((mn >> 5) * lbo + k * 128 + ((((mn >> 2) & 7) ^ (k & 7)) << 4) + (mn & 3) * 4);
}

// mode 0: plain tf32 (hi only); mode 1: 3xTF32
__global__ void probe(const float* A, const float* B, float* D, int mode) {
    const bool km = mode >= 2;
    if (threadIdx.x == 0) g_kmajor = km;
    __shared__ __align__(1024) uint8_t sa[2][4096];   // [hi/lo] 128 x 8 fp32
    __shared__ __align__(1024) uint8_t sb[2][2048];   // [hi/lo] 64 x 8
    __shared__ uint32_t tbase;
    __shared__ __align__(8) uint64_t bar;
    const int warp = threadIdx.x >> 5, t = threadIdx.x & 31;
    for (int i = threadIdx.x; i < 128 * 8; i += blockDim.x) {
        const int m = i / 8, k = i % 8;
        const float x = A[m * 8 + k];
        const float h = __uint_as_float(hi_bits(x));
        const uint32_t o = km ? offk(m, k) : off32(m, k, 1024);
        *reinterpret_cast<float*>(sa[0] + o) = x;      // the MMA reads the top 19 bits
        *reinterpret_cast<float*>(sa[1] + o) = x - h;
    }
    for (int i = threadIdx.x; i < 64 * 8; i += blockDim.x) {
        const int n = i / 8, k = i % 8;
        const float x = B[n * 8 + k];
        const float h = __uint_as_float(hi_bits(x));
        const uint32_t o = km ? offk(n, k) : off32(n, k, 1024);
        *reinterpret_cast<float*>(sb[0] + o) = x;
        *reinterpret_cast<float*>(sb[1] + o) = x - h;
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 64;" :: "r"(su(&tbase)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tm = tbase;
    if (warp == 0) {
        uint32_t pred;
        asm volatile("{\n.reg .pred p;\nelect.sync _|p, 0xffffffff;\nselp.u32 %0, 1, 0, p;\n}\n" : "=r"(pred));
        if (pred) {
            const uint64_t ah = km ? desck(su(sa[0])) : desc(su(sa[0]), 1024, 1024);
            const uint64_t al = km ? desck(su(sa[1])) : desc(su(sa[1]), 1024, 1024);
            const uint64_t bh = km ? desck(su(sb[0])) : desc(su(sb[0]), 1024, 1024);
            const uint64_t bl = km ? desck(su(sb[1])) : desc(su(sb[1]), 1024, 1024);
            mma(tm, ah, bh, 0);
            if (mode & 1) {
                mma(tm, ah, bl, 1);
                mma(tm, al, bh, 1);
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(su(&bar)) : "memory");
        }
        __syncwarp();
    }
    asm volatile("{\n.reg .pred P;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n@!P bra W_%=;\n}\n" :: "r"(su(&bar)) : "memory");
    asm volatile("tcgen05.fence::after_thread_sync;");
    const int q = warp & 3;
    for (int c0 = 0; c0 < 64; c0 += 8) {
        uint32_t r[8];
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
                     : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                     : "r"(tm + ((uint32_t)(32 * q) << 16) + c0));
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        for (int j = 0; j < 8; ++j) D[(32 * q + t) * 64 + c0 + j] = __uint_as_float(r[j]);
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 64;" :: "r"(tm));
}

__global__ void rate(unsigned long long* out, int iters) {
    __shared__ __align__(1024) uint8_t sa[4096];
    __shared__ __align__(1024) uint8_t sb[2048];
    __shared__ uint32_t tbase;
    __shared__ __align__(8) uint64_t bar;
    const int warp = threadIdx.x >> 5;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 64;" :: "r"(su(&tbase)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tm = tbase;
    if (warp == 0) {
        const uint64_t a = desc(su(sa), 1024, 1024), b = desc(su(sb), 1024, 1024);
        long long t0 = clock64();
        uint32_t ph = 0;
        for (int it = 0; it < iters; ++it) {
            uint32_t pred;
            asm volatile("{\n.reg .pred p;\nelect.sync _|p, 0xffffffff;\nselp.u32 %0, 1, 0, p;\n}\n" : "=r"(pred));
            if (pred) {
                for (int j = 0; j < 64; ++j) mma(tm, a, b, 1);
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(su(&bar)) : "memory");
            }
            __syncwarp();
            asm volatile("{\n.reg .pred P;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n@!P bra W_%=;\n}\n" :: "r"(su(&bar)), "r"(ph) : "memory");
            ph ^= 1;
        }
        long long t1 = clock64();
        if (threadIdx.x == 0) out[blockIdx.x] = (unsigned long long)(t1 - t0);
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 64;" :: "r"(tm));
}

int main() {
    static float A[128 * 8], B[64 * 8], D[128 * 64];
    srand(1);
    for (auto& v : A) v = (float)rand() / RAND_MAX * 2.f - 1.f;
    for (auto& v : B) v = (float)rand() / RAND_MAX * 2.f - 1.f;
    float *dA, *dB, *dD;
    cudaMalloc(&dA, sizeof(A));
    cudaMalloc(&dB, sizeof(B));
    cudaMalloc(&dD, sizeof(D));
    cudaMemcpy(dA, A, sizeof(A), cudaMemcpyHostToDevice);
    cudaMemcpy(dB, B, sizeof(B), cudaMemcpyHostToDevice);
    for (int mode = 0; mode < 4; ++mode) {
        probe<<<1, 128>>>(dA, dB, dD, mode);
        cudaError_t e = cudaMemcpy(D, dD, sizeof(D), cudaMemcpyDeviceToHost);
        double maxerr = 0, maxref = 0;
        for (int m = 0; m < 128; ++m)
            for (int n = 0; n < 64; ++n) {
                double ref = 0;
                for (int k = 0; k < 8; ++k) ref += (double)A[m * 8 + k] * (double)B[n * 8 + k];
                maxerr = fmax(maxerr, fabs(D[m * 64 + n] - ref));
                maxref = fmax(maxref, fabs(ref));
            }
        printf("%s %s (%s): max|err| / max|ref| = %.3e   D[0][0..2] = %g %g %g\n", (mode & 1) ? "3xTF32" : "1xTF32",
               mode >= 2 ? "K-major none" : "MN-major SW128", cudaGetErrorString(e), maxerr / maxref, D[0], D[1], D[2]);
    }
    unsigned long long* d;
    cudaMalloc(&d, 8 * 148);
    rate<<<148, 128>>>(d, 4);
    rate<<<148, 128>>>(d, 50);
    cudaError_t e = cudaDeviceSynchronize();
    unsigned long long h[148];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double avg = 0;
    for (auto v : h) avg += v;
    avg /= 148;
    printf("SS tf32 M128 N64 K8 (%s): %.1f cycles / MMA\n", cudaGetErrorString(e), avg / (50 * 64));
    return 0;
}
