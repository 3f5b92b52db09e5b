// Microbenchmark: per-SM fill rate of a shared-memory ring from an NHWC fp16
// tensor, as the FP16 BFC kernel loads its raw chunks (ResNet-50 layer-3
// shape, N=64 14x14 C=256; a chunk = 16 depth entries x (r=2 dY columns +
// alpha=4 X columns) x 128 channels = 24 KB):
//   tma   one warp issues 4-D TMA boxes [128 ch][cols][1][8 images] (as now)
//   cpa   W producer warps issue 16-byte cp.async (LDGSTS) for the same bytes
// One CTA per SM; consumers release each stage immediately, so the number is
// the producer-side ceiling.  Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -lcuda
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#ifndef OOB
#define OOB 0
#endif
#ifndef NIMG
#define NIMG 64
#endif

constexpr int N = NIMG, H = 14, W = 14, C = 256, STAGES = 4, CH = 128, KC = 16;
constexpr int COLS_Y = 2, COLS_X = 4;
constexpr int RAW_Y = KC * COLS_Y * CH * 2, RAW_X = KC * COLS_X * CH * 2, RAW = RAW_Y + RAW_X;

__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void wait(uint64_t* b, uint32_t ph) {
    asm volatile("{\n.reg .pred P;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n@!P bra W_%=;\n}\n"
                 :: "r"(su(b)), "r"(ph) : "memory");
}

template <int MODE, int PW, int NB = 8, int NOISE = 0, int POLL = 0>
__global__ void __launch_bounds__(32 * (PW + 1 + NOISE), 1) k(const __grid_constant__ CUtensorMap tm, const __half* X,
                                                     unsigned long long* out, int iters) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint64_t full[STAGES], empty[STAGES];
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(su(&full[s])), "r"(MODE == 0 ? 1 : PW * 32));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(&empty[s])));
        }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    long long t0 = clock64();
    if (warp < PW) {
        for (int it = 0; it < iters; ++it) {
            const int s = it % STAGES;
            wait(&empty[s], ((it / STAGES) & 1) ^ 1);
            uint8_t* raw = sm + s * RAW;
            // depth entries of this chunk: images n0..n0+15 (2 boxes of 8), row h, unit u
            const int blk = (blockIdx.x * 131 + it) % (N / KC * H * 3);
            const int n0 = (blk % (N / KC)) * KC, h = (blk / (N / KC)) % H, u = blk / (N / KC) / H;
            if (MODE == 0) {
                if (lane == 0)
                    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su(&full[s])), "r"(RAW) : "memory");
                __syncwarp();
                if (lane < 2 * (KC / NB)) {
                    const int b = (lane >> 1) * NB;
                    const bool y = (lane & 1) == 0;
                    uint8_t* dst = y ? raw + b * COLS_Y * CH * 2 : raw + RAW_Y + b * COLS_X * CH * 2;
                    asm volatile(
                        "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];"
                        :: "r"(su(dst)), "l"((uint64_t)&tm), "r"(0), "r"(u * 2 + (y ? 0 : 1) - OOB), "r"(h), "r"(n0 + b),
                           "r"(su(&full[s])) : "memory");
                }
            } else {
                // 16-byte pieces: [depth][col][ch/8]
                constexpr int PIECES = RAW / 16;
                for (int p = warp * 32 + lane; p < PIECES; p += PW * 32) {
                    const bool y = p < RAW_Y / 16;
                    const int q = y ? p : p - RAW_Y / 16;
                    const int cols = y ? COLS_Y : COLS_X;
                    const int c8 = q % (CH / 8), col = (q / (CH / 8)) % cols, d = q / (CH / 8) / cols;
                    const __half* src = X + ((((size_t)(n0 + d) * H + h) * W + (u * 2 + col)) * C + c8 * 8);
                    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(su(raw + p * 16)), "l"(src) : "memory");
                }
                asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" :: "r"(su(&full[s])) : "memory");
            }
        }
    } else if (warp > PW && POLL) {   // extra consumer warps polling the full barriers (as the transformers do)
        for (int it = 0; it < iters; ++it) wait(&full[it % STAGES], (it / STAGES) & 1);
    } else if (warp > PW) {   // smem noise: STS.128 + LDS.128 traffic like the transformers
        uint4* q = reinterpret_cast<uint4*>(sm + STAGES * RAW) + (warp - PW - 1) * 32 * 8;
        uint4 a = make_uint4(lane, 1, 2, 3);
        for (int it = 0; it < iters * 20; ++it) {
#pragma unroll
            for (int j = 0; j < 8; ++j) { q[(j * 32 + lane) % 256] = a; a.x += q[((j + 3) * 32 + lane) % 256].y; }
#ifdef FENCE
            if (it % FENCE == 0) asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
#endif
        }
        if (a.x == 12345) out[0] = 0;
    } else if (lane == 0) {
        for (int it = 0; it < iters; ++it) {
            const int s = it % STAGES;
            wait(&full[s], (it / STAGES) & 1);
            asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(su(&empty[s])) : "memory");
        }
        out[blockIdx.x] = clock64() - t0;
    }
}

__global__ void fill(uint32_t* p, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
        uint32_t x = (uint32_t)i * 2654435761u;
        x ^= x >> 13; x *= 0x5bd1e995u; x ^= x >> 15;
        p[i] = x & 0x3bff3bffu;   // finite fp16 pairs
    }
}

typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                        const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                        CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

template <int MODE, int PW, int NB = 8, int NOISE = 0, int POLL = 0>
void run(const CUtensorMap& tm, const __half* X, const char* name) {
    unsigned long long* d;
    cudaMalloc(&d, 8 * 148);
    const int smem = STAGES * RAW + (NOISE ? NOISE * 32 * 8 * 16 : 0);
    cudaFuncSetAttribute(k<MODE, PW, NB, NOISE, POLL>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    const int iters = 2000;
    k<MODE, PW, NB, NOISE, POLL><<<148, 32 * (PW + 1 + NOISE), smem>>>(tm, X, d, iters);   // warm
    k<MODE, PW, NB, NOISE, POLL><<<148, 32 * (PW + 1 + NOISE), smem>>>(tm, X, d, iters);
    cudaError_t e = cudaDeviceSynchronize();
    unsigned long long h[148];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < 148; ++i) avg += h[i];
    avg /= 148;
    printf("%-10s NB=%d NOISE=%d POLL=%d PW=%d: %7.1f cycles/chunk  %6.1f B/cycle/SM  (%s)\n", name, NB, NOISE, POLL, PW, avg / iters, RAW * iters / avg,
           cudaGetErrorString(e));
    cudaFree(d);
}

int main() {
    __half* X;
    cudaMalloc(&X, (size_t)N * H * W * C * 2);
    cudaMemset(X, 0, (size_t)N * H * W * C * 2);
    if (getenv("RANDOM_FILL")) fill<<<1024, 256>>>((uint32_t*)X, (size_t)N * H * W * C / 2);
    cudaDeviceSynchronize();
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
    Enc enc = (Enc)p;
    // one map; dY boxes use COLS_Y columns by loading a COLS_X box into a smaller slot would
    // overflow, so use a box of COLS_Y columns for both (bytes per chunk scaled below).
    CUtensorMap tm;
    const cuuint64_t dims[4] = {C, W, H, N};
    const cuuint64_t str[3] = {(cuuint64_t)C * 2, (cuuint64_t)W * C * 2, (cuuint64_t)H * W * C * 2};
    const cuuint32_t box[4] = {CH, 3, 1, 8};   // 3 columns: the average of the 2- and 4-column boxes
    const cuuint32_t es[4] = {1, 1, 1, 1};
    CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 4, X, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("encode %d\n", (int)r);
    CUtensorMap tm16 = tm, tm4 = tm;
    const cuuint32_t box16[4] = {CH, 3, 1, 16}, box4[4] = {CH, 3, 1, 4};
    enc(&tm16, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 4, X, dims, str, box16, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
        CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    enc(&tm4, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 4, X, dims, str, box4, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
        CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    run<0, 1, 8>(tm, X, "tma");
    run<0, 1, 16>(tm16, X, "tma");
    run<0, 1, 4>(tm4, X, "tma");
    run<0, 1, 8, 8>(tm, X, "tma");
    run<0, 1, 8, 14>(tm, X, "tma");
    run<0, 1, 16, 14>(tm16, X, "tma");
    run<0, 1, 8, 14, 1>(tm, X, "tma");
    run<0, 1, 16, 14, 1>(tm16, X, "tma");
    return 0;
}
