// Microbenchmark (round 2): per-SM TMA fill rate for the box shapes of the
// second-generation tensor-core kernel (bfc_tc2.cuh) on the ResNet-50 layer-3
// shape (N=64, 14x14, C=K=256 fp16, NHWC; 12.8 MB, L2-resident after the
// first touch).  One CTA per SM (grid G), warp 0 / one elected lane issues
// each stage's boxes into an S-stage ring, the same warp waits for the data
// and re-arms; consumers do nothing.  Reports bytes/clk/SM and chip GB/s.
//   mode 0: tc2 stage  = 2 X boxes {64c,16n,1,4w} + 2 dY boxes {64k,16n,1,2w}, SW128   (24 KB)
//   mode 1: X boxes only                                                            (16 KB)
//   mode 2: round-1 style 256-B rows: X {128c,4w,1,16n} + dY {128k,2w,1,16n}, no swizzle (24 KB)
//   mode 3: tc2 stage, two units per stage (X overlap): X {64c,8n,1,6w} x2 + dY {64k,8n,1,4w} x2 (20 KB)
// Build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a tma_rate3.cu -o tma_rate3.bin -lcuda
#include <cstdint>
#include <cstdio>
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

constexpr int N = 64, H = 14, W = 14, C = 256, S = 6;

__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void tma4(uint32_t dst, const CUtensorMap* m, uint64_t* bar, int c0, int c1, int c2, int c3) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];"
        :: "r"(dst), "l"(reinterpret_cast<uint64_t>(m)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(su(bar)) : "memory");
}
__device__ __forceinline__ bool elect_one() {
    uint32_t pred;
    asm volatile("{\n.reg .pred p;\nelect.sync _|p, 0xffffffff;\nselp.u32 %0, 1, 0, p;\n}\n" : "=r"(pred));
    return pred != 0;
}
__device__ __forceinline__ void wait(uint64_t* b, uint32_t ph) {
    asm volatile("{\n.reg .pred P;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n@!P bra W_%=;\n}\n"
                 :: "r"(su(b)), "r"(ph) : "memory");
}

template <int MODE>
__global__ void __launch_bounds__(32, 1) k(const __grid_constant__ CUtensorMap tmX, const __grid_constant__ CUtensorMap tmY,
                                           unsigned long long* out, int iters) {
    extern __shared__ uint8_t smr[];
    uint8_t* sm = smr + ((1024 - (su(smr) & 1023)) & 1023);
    __shared__ uint64_t full[S];
    constexpr int STAGE = 24 * 1024;
    constexpr uint32_t BYTES = MODE == 1 ? 16384 : MODE == 3 ? 20480 : 24576;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(&full[s])));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncwarp();
    const uint32_t base = su(sm);
    auto issue = [&](int it) {
        const int s = it % S;
        const int blk = (blockIdx.x * 131 + it) % (N / 16 * H * 6);
        const int n0 = (blk % (N / 16)) * 16, h = (blk / (N / 16)) % H, u = blk / (N / 16) / H;
        const int w0 = 2 * u;
        const uint32_t st = base + s * STAGE;
        if (elect_one()) {
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su(&full[s])), "r"(BYTES) : "memory");
            if (MODE == 0 || MODE == 1) {
                tma4(st, &tmX, &full[s], 0, n0, h, w0 - 1);
                tma4(st + 8192, &tmX, &full[s], 64, n0, h, w0 - 1);
                if (MODE == 0) {
                    tma4(st + 16384, &tmY, &full[s], 0, n0, h, w0);
                    tma4(st + 20480, &tmY, &full[s], 64, n0, h, w0);
                }
            } else if (MODE == 2) {
                tma4(st, &tmX, &full[s], 0, w0 - 1, h, n0);
                tma4(st + 16384, &tmY, &full[s], 0, w0, h, n0);
            } else {
                tma4(st, &tmX, &full[s], 0, n0 / 2, h, w0 - 1);
                tma4(st + 6144, &tmX, &full[s], 64, n0 / 2, h, w0 - 1);
                tma4(st + 12288, &tmY, &full[s], 0, n0 / 2, h, w0);
                tma4(st + 16384, &tmY, &full[s], 64, n0 / 2, h, w0);
            }
        }
        __syncwarp();
    };
    for (int it = 0; it < S; ++it) issue(it);
    long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
        wait(&full[it % S], (it / S) & 1);
        issue(it + S);
    }
    for (int it = iters; it < iters + S; ++it) wait(&full[it % S], (it / S) & 1);
    long long t1 = clock64();
    if (threadIdx.x == 0) out[blockIdx.x] = (unsigned long long)(t1 - t0);
}

typedef CUresult (*EncFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                          const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                          CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncFn enc() {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
    return (EncFn)p;
}

// dims order {C, N, H, W} (tc2) or {C, W, H, N} (round 1)
static void map(CUtensorMap* m, void* p, bool tc2, int bc, int bn, int bw) {
    const cuuint64_t d_tc2[4] = {C, N, H, W}, d_r1[4] = {C, W, H, N};
    const cuuint64_t s_tc2[3] = {(cuuint64_t)H * W * C * 2, (cuuint64_t)W * C * 2, (cuuint64_t)C * 2};
    const cuuint64_t s_r1[3] = {(cuuint64_t)C * 2, (cuuint64_t)W * C * 2, (cuuint64_t)H * W * C * 2};
    const cuuint32_t box_tc2[4] = {(cuuint32_t)bc, (cuuint32_t)bn, 1, (cuuint32_t)bw};
    const cuuint32_t box_r1[4] = {(cuuint32_t)bc, (cuuint32_t)bw, 1, (cuuint32_t)bn};
    const cuuint32_t es[4] = {1, 1, 1, 1};
    CUresult r = enc()(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 4, p, tc2 ? d_tc2 : d_r1, tc2 ? s_tc2 : s_r1,
                       tc2 ? box_tc2 : box_r1, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                       tc2 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                       CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) printf("encode failed %d\n", (int)r);
}

template <int MODE>
void run(int grid, void* X, void* Y) {
    CUtensorMap mX, mY;
    if (MODE == 2) { map(&mX, X, false, 128, 16, 4); map(&mY, Y, false, 128, 16, 2); }
    else if (MODE == 3) { map(&mX, X, true, 64, 8, 6); map(&mY, Y, true, 64, 8, 4); }
    else { map(&mX, X, true, 64, 16, 4); map(&mY, Y, true, 64, 16, 2); }
    unsigned long long* d;
    cudaMalloc(&d, 8 * 148);
    const int smem = S * 24 * 1024 + 1024;
    cudaFuncSetAttribute(k<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    const int iters = 400;
    k<MODE><<<grid, 32, smem>>>(mX, mY, d, 50);
    k<MODE><<<grid, 32, smem>>>(mX, mY, d, iters);
    cudaError_t e = cudaDeviceSynchronize();
    unsigned long long h[148];
    cudaMemcpy(h, d, 8 * grid, cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < grid; ++i) avg += h[i];
    avg /= grid;
    const double bytes = (MODE == 1 ? 16384.0 : MODE == 3 ? 20480.0 : 24576.0) * (iters + S);
    printf("mode %d grid %3d: %6.1f cycles/stage  %5.1f B/clk/SM  %6.0f GB/s chip (@1.965GHz)  %s\n", MODE, grid,
           avg / (iters + S), bytes / avg, bytes / avg * grid * 1.965, cudaGetErrorString(e));
    cudaFree(d);
}

int main() {
    void *X, *Y;
    cudaMalloc(&X, (size_t)N * H * W * C * 2);
    cudaMalloc(&Y, (size_t)N * H * W * C * 2);
    cudaMemset(X, 0, (size_t)N * H * W * C * 2);
    cudaMemset(Y, 0, (size_t)N * H * W * C * 2);
    for (int g : {96, 148}) {
        run<0>(g, X, Y);
        run<1>(g, X, Y);
        run<2>(g, X, Y);
        run<3>(g, X, Y);
    }
    run<0>(8, X, Y);
    run<0>(1, X, Y);
    return 0;
}
