// Scalar / packed arithmetic used by the generated Winograd transforms.
//
// The same generated code (winograd_generated.cuh) is instantiated for
//   float  — FP32 transforms in the kernels (§5.2 P@38729: "FT, IT
//            and OT are temporarily computed in FP32"),
//   F2     — two independent FP32 lanes packed in one 64-bit register pair,
//            lowered to FFMA2 / FMUL2 / FADD2 on sm_100a (same IEEE FP32 RN
//            result per lane, half the issue slots; constants fold into the
//            instruction's immediate operand),
//   double — the host FP64 emulator (winrs_debug_emulate).
#pragma once
#include <stdint.h>

#if defined(__CUDACC__)
#define WV_HD __host__ __device__ __forceinline__
#else
#define WV_HD inline
#endif

namespace winrs {

template <class T> WV_HD T wc(int num, int den);
template <> WV_HD float wc<float>(int num, int den) { return static_cast<float>(num) / static_cast<float>(den); }
template <> WV_HD double wc<double>(int num, int den) { return static_cast<double>(num) / static_cast<double>(den); }
template <class T> WV_HD T wzero() { return T(0); }

WV_HD float wadd(float a, float b) { return a + b; }
WV_HD float wsub(float a, float b) { return a - b; }
WV_HD float wneg(float a) { return -a; }
WV_HD float wmul(float c, float a) { return c * a; }
#if defined(__CUDA_ARCH__)
WV_HD float wfma(float c, float a, float acc) { return __fmaf_rn(c, a, acc); }
#else
WV_HD float wfma(float c, float a, float acc) { return c * a + acc; }
#endif

WV_HD double wadd(double a, double b) { return a + b; }
WV_HD double wsub(double a, double b) { return a - b; }
WV_HD double wneg(double a) { return -a; }
WV_HD double wmul(double c, double a) { return c * a; }
WV_HD double wfma(double c, double a, double acc) { return c * a + acc; }

// Two packed FP32 lanes.
struct F2 {
    float x, y;
};
template <> WV_HD F2 wc<F2>(int num, int den) {
    const float v = static_cast<float>(num) / static_cast<float>(den);
    return F2{v, v};
}
template <> WV_HD F2 wzero<F2>() { return F2{0.f, 0.f}; }

#if defined(__CUDA_ARCH__)
__device__ __forceinline__ uint64_t f2_bits(F2 a) {
    uint64_t r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a.x), "f"(a.y));
    return r;
}
__device__ __forceinline__ F2 f2_from(uint64_t r) {
    F2 a;
    asm("mov.b64 {%0, %1}, %2;" : "=f"(a.x), "=f"(a.y) : "l"(r));
    return a;
}
__device__ __forceinline__ F2 wadd(F2 a, F2 b) {
    uint64_t d;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(f2_bits(a)), "l"(f2_bits(b)));
    return f2_from(d);
}
__device__ __forceinline__ F2 wsub(F2 a, F2 b) {
    uint64_t d;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(f2_bits(a)), "l"(f2_bits(b)));
    return f2_from(d);
}
__device__ __forceinline__ F2 wmul(F2 c, F2 a) {
    uint64_t d;
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(f2_bits(c)), "l"(f2_bits(a)));
    return f2_from(d);
}
__device__ __forceinline__ F2 wfma(F2 c, F2 a, F2 acc) {
    uint64_t d;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(f2_bits(c)), "l"(f2_bits(a)), "l"(f2_bits(acc)));
    return f2_from(d);
}
__device__ __forceinline__ F2 wneg(F2 a) { return F2{-a.x, -a.y}; }
#else
inline F2 wadd(F2 a, F2 b) { return F2{a.x + b.x, a.y + b.y}; }
inline F2 wsub(F2 a, F2 b) { return F2{a.x - b.x, a.y - b.y}; }
inline F2 wmul(F2 c, F2 a) { return F2{c.x * a.x, c.y * a.y}; }
inline F2 wfma(F2 c, F2 a, F2 acc) { return F2{c.x * a.x + acc.x, c.y * a.y + acc.y}; }
inline F2 wneg(F2 a) { return F2{-a.x, -a.y}; }
#endif

}  // namespace winrs
