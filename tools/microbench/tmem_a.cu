// Microbenchmark / probe (round 2): the A operand of tcgen05.mma taken from
// TMEM, filled from a TMA-style SW128 operand slab with ldmatrix.trans +
// tcgen05.st.16x256b — the data path of the WINRS_TC2_ITM=2 kernel variant.
//   part 1: the 16x256b fragment layout (which lane / column each thread's
//           registers land in), read back with 32x32b loads;
//   part 2: A (128 channels x 16 images, K-major in TMEM) built from an
//           MN-major SW128 slab (rows = images, 128 B = 64 channels, chunk
//           j stored at j ^ (row & 7)) by 4 warps (lane quarters), B (16 x 64)
//           MN-major SW128 in shared memory; D = A B in TMEM compared with the
//           host product.
// Build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a tmem_a.cu -o tmem_a.bin
#include <cstdint>
#include <cstdio>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void st16x256(uint32_t taddr, uint32_t r0, uint32_t r1, uint32_t r2, uint32_t r3) {
    asm volatile("tcgen05.st.sync.aligned.16x256b.x1.b32 [%0], {%1, %2, %3, %4};"
                 :: "r"(taddr), "r"(r0), "r"(r1), "r"(r2), "r"(r3) : "memory");
}
__device__ __forceinline__ void ld32x32x8(uint32_t taddr, uint32_t* r) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                 : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void ldsm_x4_t(uint32_t addr, uint32_t& a, uint32_t& b, uint32_t& c, uint32_t& d) {
    asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0, %1, %2, %3}, [%4];"
                 : "=r"(a), "=r"(b), "=r"(c), "=r"(d) : "r"(addr));
}

__global__ void probe_layout(uint32_t* out) {
    __shared__ uint32_t tbase;
    const int warp = threadIdx.x >> 5, t = threadIdx.x & 31;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" :: "r"(su(&tbase)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tm = tbase;
    if (warp == 0) {
        // zero lanes 0..31, cols 0..7, then one 16x256b store of tags at lane 0
        uint32_t z = 0;
        asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1, %1, %1, %1, %1, %1, %1, %1};" :: "r"(tm), "r"(z) : "memory");
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        st16x256(tm, (t << 8) | 0x10, (t << 8) | 0x11, (t << 8) | 0x12, (t << 8) | 0x13);
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        uint32_t r[8];
        ld32x32x8(tm, r);
        for (int j = 0; j < 8; ++j) out[t * 8 + j] = r[j];
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" :: "r"(tm));
}

// X slab: 2 atoms (channels 0-63, 64-127) x 16 image rows, MN-major SW128.
// B: 16 K rows x 64 n, MN-major SW128.  A[m][k] = X[image k][channel m].
__global__ void probe_mma(const __half* Xlin, const __half* Blin, float* D) {
    __shared__ __align__(1024) uint8_t xs[4096];
    __shared__ __align__(1024) uint8_t bs[2048];
    __shared__ uint32_t tbase;
    __shared__ __align__(8) uint64_t bar;
    const int warp = threadIdx.x >> 5, t = threadIdx.x & 31;
    // swizzled fill (what the TMA would write)
    for (int i = threadIdx.x; i < 16 * 128; i += blockDim.x) {
        const int img = i / 128, ch = i % 128, atom = ch / 64, c = ch % 64;
        const int off = atom * 2048 + (img >> 3) * 1024 + (img & 7) * 128 + ((((c >> 3) ^ (img & 7))) << 4) + (c & 7) * 2;
        *reinterpret_cast<__half*>(xs + off) = Xlin[img * 128 + ch];
    }
    for (int i = threadIdx.x; i < 16 * 64; i += blockDim.x) {
        const int k = i / 64, n = i % 64;
        const int off = (k >> 3) * 1024 + (k & 7) * 128 + ((((n >> 3) ^ (k & 7))) << 4) + (n & 7) * 2;
        *reinterpret_cast<__half*>(bs + off) = Blin[k * 64 + n];
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" :: "r"(su(&tbase)));
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
    const uint32_t acol = 64;   // A at columns 64..71, D at 0..63
    {
        // warp q: lanes 32q..32q+31 = channels 32q..; two 16-lane halves
        const int q = warp & 3;
        for (int hf = 0; hf < 2; ++hf) {
            const int ch0 = 32 * q + 16 * hf;          // first channel of the 16
            const int atom = ch0 / 64, o0 = (ch0 % 64) / 8;
            // ldmatrix.x4.trans: matrix i gets row addresses from threads 8i..8i+7
            const int i = t >> 3, rho = t & 7;
            const int oct = o0 + (i >> 1);                                  // channel octet
            const int img = 4 * (rho >> 1) + (rho & 1) + 2 * (i & 1);     // image permutation
            const uint32_t addr = su(xs) + atom * 2048 + (img >> 3) * 1024 + (img & 7) * 128 + ((oct ^ (img & 7)) << 4);
            uint32_t r0, r1, r2, r3;
            ldsm_x4_t(addr, r0, r1, r2, r3);
            const uint32_t ta = tm + ((uint32_t)(32 * q + 16 * hf) << 16) + acol;
            st16x256(ta, r0, r1, r2, r3);
        }
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    if (warp == 0) {
        const uint64_t bdesc = (uint64_t)((su(bs) >> 4) & 0x3FFF) | ((uint64_t)((8192 >> 4) & 0x3FFF) << 16) |
                               ((uint64_t)((1024 >> 4) & 0x3FFF) << 32) | (1ull << 46) | (2ull << 61);
        // D f32, A f16 K-major (TMEM), B f16 MN-major, N = 64, M = 128
        const uint32_t idesc = (1u << 4) | (1u << 16) | ((uint32_t)(64 >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
        uint32_t pred;
        asm volatile("{\n.reg .pred p;\nelect.sync _|p, 0xffffffff;\nselp.u32 %0, 1, 0, p;\n}\n" : "=r"(pred));
        if (pred) {
            asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
                         "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}\n"
                         :: "r"(tm), "r"(tm + acol), "l"(bdesc), "r"(idesc), "r"(0u));
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(su(&bar)) : "memory");
        }
        __syncwarp();
    }
    asm volatile("{\n.reg .pred P;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n@!P bra W_%=;\n}\n"
                 :: "r"(su(&bar)) : "memory");
    asm volatile("tcgen05.fence::after_thread_sync;");
    {
        const int q = warp & 3;
        for (int c0 = 0; c0 < 64; c0 += 8) {
            uint32_t r[8];
            ld32x32x8(tm + ((uint32_t)(32 * q) << 16) + c0, r);
            for (int j = 0; j < 8; ++j) D[(32 * q + t) * 64 + c0 + j] = __uint_as_float(r[j]);
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" :: "r"(tm));
}

int main() {
    uint32_t* d;
    cudaMalloc(&d, 32 * 8 * 4);
    probe_layout<<<1, 32>>>(d);
    uint32_t h[256];
    cudaError_t e = cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    printf("16x256b layout (%s): lane: col0..7 = thread<<8 | reg (0 = untouched)\n", cudaGetErrorString(e));
    for (int l = 0; l < 16; ++l) {
        printf("lane %2d:", l);
        for (int j = 0; j < 8; ++j) printf(" t%02d.r%d", h[l * 8 + j] >> 8, (h[l * 8 + j] & 0xff) - 0x10);
        printf("\n");
    }
    int stray = 0;
    for (int l = 16; l < 32; ++l)
        for (int j = 0; j < 8; ++j) stray += h[l * 8 + j] != 0;
    printf("lanes 16..31 written: %d cells\n", stray);

    __half Xh[16 * 128], Bh[16 * 64];
    float X[16 * 128], B[16 * 64];
    for (int i = 0; i < 16; ++i)
        for (int c = 0; c < 128; ++c) { X[i * 128 + c] = (float)((c * 3 + i * 5) % 9 - 4); Xh[i * 128 + c] = __float2half(X[i * 128 + c]); }
    for (int k = 0; k < 16; ++k)
        for (int n = 0; n < 64; ++n) { B[k * 64 + n] = (float)((2 * k + 7 * n) % 5 - 2); Bh[k * 64 + n] = __float2half(B[k * 64 + n]); }
    __half *dX, *dB;
    float* dD;
    cudaMalloc(&dX, sizeof(Xh));
    cudaMalloc(&dB, sizeof(Bh));
    cudaMalloc(&dD, 128 * 64 * 4);
    cudaMemcpy(dX, Xh, sizeof(Xh), cudaMemcpyHostToDevice);
    cudaMemcpy(dB, Bh, sizeof(Bh), cudaMemcpyHostToDevice);
    cudaMemset(dD, 0, 128 * 64 * 4);
    probe_mma<<<1, 128>>>(dX, dB, dD);
    static float D[128 * 64];
    e = cudaMemcpy(D, dD, sizeof(D), cudaMemcpyDeviceToHost);
    int bad = 0;
    for (int m = 0; m < 128; ++m)
        for (int n = 0; n < 64; ++n) {
            float ref = 0;
            for (int k = 0; k < 16; ++k) ref += X[k * 128 + m] * B[k * 64 + n];
            if (D[m * 64 + n] != ref) {
                if (bad < 8) printf("mismatch m=%d n=%d got %g ref %g\n", m, n, D[m * 64 + n], ref);
                ++bad;
            }
        }
    printf("A-from-TMEM MMA (%s): %d mismatches of %d\n", cudaGetErrorString(e), bad, 128 * 64);
    return 0;
}
