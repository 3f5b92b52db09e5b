// Microbenchmark: per-SM throughput of FFMA (3-reg), FFMA2 (fma.rn.f32x2),
// HFMA2 and FADD2 on sm_100a.  Each thread runs independent chains; reports
// flop/clk/SM.  Used to size the transform/EWM design.
#include <cstdio>
#include <cuda_runtime.h>
#include <cuda_fp16.h>

constexpr int ITERS = 4096;
constexpr int CH = 8;   // independent chains per thread

__global__ void k_ffma(float* out, float a, float b) {
    float x[CH];
#pragma unroll
    for (int i = 0; i < CH; ++i) x[i] = threadIdx.x + i;
    for (int it = 0; it < ITERS; ++it)
#pragma unroll
        for (int i = 0; i < CH; ++i) x[i] = fmaf(x[i], a, b);
    float s = 0;
#pragma unroll
    for (int i = 0; i < CH; ++i) s += x[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void k_ffma_outer(float* out, float a0, float a1) {
    // outer-product style: acc[i][j] += a[i]*b[j] with a, b varying (3 distinct regs)
    float acc[4][4] = {};
    float a[4], b[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) { a[i] = a0 + i + threadIdx.x; b[i] = a1 - i; }
    for (int it = 0; it < ITERS / 2; ++it) {
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
        a[it & 3] += 1e-7f;
    }
    float s = 0;
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) s += acc[i][j];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__device__ __forceinline__ float2 ffma2(float2 a, float2 b, float2 c) {
    unsigned long long ra = *reinterpret_cast<unsigned long long*>(&a);
    unsigned long long rb = *reinterpret_cast<unsigned long long*>(&b);
    unsigned long long rc = *reinterpret_cast<unsigned long long*>(&c);
    unsigned long long d;
    asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(ra), "l"(rb), "l"(rc));
    return *reinterpret_cast<float2*>(&d);
}

__global__ void k_ffma2(float* out, float a, float b) {
    float2 x[CH];
#pragma unroll
    for (int i = 0; i < CH; ++i) x[i] = make_float2(threadIdx.x + i, i);
    const float2 A = make_float2(a, a), B = make_float2(b, b);
    for (int it = 0; it < ITERS; ++it)
#pragma unroll
        for (int i = 0; i < CH; ++i) x[i] = ffma2(x[i], A, B);
    float s = 0;
#pragma unroll
    for (int i = 0; i < CH; ++i) s += x[i].x + x[i].y;
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void k_ffma2_outer(float* out, float a0, float a1) {
    // outer product with packed FMA: acc[i][j..j+1] += {a_i,a_i} * {b_j,b_j+1}
    float2 acc[8][4];
    float2 aa[8], bb[4];
#pragma unroll
    for (int i = 0; i < 8; ++i) { aa[i] = make_float2(a0 + i + threadIdx.x, a0 + i + threadIdx.x); }
#pragma unroll
    for (int j = 0; j < 4; ++j) bb[j] = make_float2(a1 - j, a1 + j);
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = make_float2(0.f, 0.f);
    for (int it = 0; it < ITERS / 4; ++it) {
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) acc[i][j] = ffma2(aa[i], bb[j], acc[i][j]);
        aa[it & 7].x += 1e-7f;
    }
    float s = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) s += acc[i][j].x + acc[i][j].y;
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void k_ffma_outer8(float* out, float a0, float a1) {
    // 8x8 outer product, plain FFMA (like the GEMM inner loop)
    float acc[8][8];
    float a[8], b[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) { a[i] = a0 + i + threadIdx.x; b[i] = a1 - i; }
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;
    for (int it = 0; it < ITERS / 4; ++it) {
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
            for (int j = 0; j < 8; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
        a[it & 7] += 1e-7f;
    }
    float s = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) s += acc[i][j];
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void k_hfma2(float* out, float a, float b) {
    __half2 x[CH];
#pragma unroll
    for (int i = 0; i < CH; ++i) x[i] = __floats2half2_rn(threadIdx.x * 1e-3f + i, i);
    const __half2 A = __floats2half2_rn(a, a), B = __floats2half2_rn(b, b);
    for (int it = 0; it < ITERS; ++it)
#pragma unroll
        for (int i = 0; i < CH; ++i) x[i] = __hfma2(x[i], A, B);
    float s = 0;
#pragma unroll
    for (int i = 0; i < CH; ++i) s += __low2float(x[i]) + __high2float(x[i]);
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <class K>
double run(K kern, const char* name, double flop_per_iter_per_thread, int threads, int blocks_per_sm) {
    int dev = 0, sms = 0, clk = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
    float* out;
    cudaMalloc(&out, sizeof(float) * sms * blocks_per_sm * threads);
    kern<<<sms * blocks_per_sm, threads>>>(out, 0.999f, 1e-3f);
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    cudaEventRecord(a);
    for (int r = 0; r < 5; ++r) kern<<<sms * blocks_per_sm, threads>>>(out, 0.999f, 1e-3f);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    const double flops = 5.0 * sms * blocks_per_sm * threads * flop_per_iter_per_thread * ITERS;
    const double tf = flops / (ms * 1e-3) / 1e12;
    const double per_clk_sm = flops / (ms * 1e-3) / (clk * 1e3) / sms;
    printf("%-12s threads=%d x %d/SM: %8.2f TFLOP/s  %7.1f flop/clk/SM (at %d MHz nominal)\n", name, threads,
           blocks_per_sm, tf, per_clk_sm, clk / 1000);
    cudaFree(out);
    return tf;
}

int main() {
    for (int bps : {1, 2, 4}) {
        run(k_ffma, "FFMA", 2.0 * CH, 256, bps);
        run(k_ffma_outer, "FFMA-outer", 2.0 * 16 / 2, 256, bps);
        run(k_ffma2, "FFMA2", 4.0 * CH, 256, bps);
        run(k_ffma2_outer, "FFMA2-outer", 4.0 * 32 / 4, 256, bps);
        run(k_ffma_outer8, "FFMA-outer8", 2.0 * 64 / 4, 256, bps);
        run(k_hfma2, "HFMA2", 4.0 * CH, 256, bps);
    }
    return 0;
}
