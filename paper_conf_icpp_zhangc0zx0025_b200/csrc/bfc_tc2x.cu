// Instantiations and launch of the xi-split FP16 / BF16 tensor-core kernel
// (bfc_tc2x.cuh): tile = 128 k x (128 / F) c x F filter rows per CTA pair,
// cluster = 2 x csplit CTAs.
#include <cuda.h>
#include <cuda_runtime.h>
#include "bfc_tc2x.cuh"
#include "launch_util.cuh"
#include "registry.h"
#include "tc2_maps.cuh"

namespace winrs {
namespace tc2 {

template <int F, bool BF>
cudaError_t launch_x(const Geometry& g, const void* X, const void* dY, float* dW, float* ws, cudaStream_t stream) {
    using L = LayX<F>;
    const long long grid = num_ctas(g);
    if (grid <= 0) return cudaSuccess;
    Args a;
    a.g = g;
    a.dW = dW;
    a.ws = ws;
    a.nb = images_per_box(g);
    if (a.nb == 0 || g.a0 != 4 || g.n0 != 3 || g.r0 != 2 || g.a1 != 0 || g.cg != 2 || g.fhs != F || g.csplit > 4)
        return cudaErrorInvalidValue;
    const bool nd = g.T > 1 || g.D > 1;
    CUtensorMap mX4, mX2, mY;
    if (!make_maps(g, X, dY, BF, &mX4, &mY, 8)) return cudaErrorInvalidValue;
    // x1, x2 only (the e = 0 half): box {64, 8, 1, 1, 2}
    if (!make_map(&mX2, X, nd ? g.D : g.N, nd ? g.Nb : 1, g.H, g.W, g.C, g.C, 2, 8, BF)) return cudaErrorInvalidValue;
    static std::atomic<unsigned long long> done{0};
    auto k = bfc_tc2x_kernel<F, BF>;
    cudaError_t e = ensure_smem_attr(k, (size_t)L::BYTES, done);
    if (e != cudaSuccess) return e;
    return launch_cluster(k, (unsigned)grid, (unsigned)tc2_threads<true>(), (size_t)L::BYTES, stream, 2 * g.csplit, a,
                          mX4, mX2, mY);
}

}  // namespace tc2

#define WINRS_TC2X_ENTRY(DT, BF, PFX, F)                                                                  \
    {DT, 4, 3, 2, 0, 0, 0, 128, ::winrs::tc2::MROWS / F, ::winrs::tc2::tc2_threads<true>(), 1, 1,         \
     (size_t)::winrs::tc2::LayX<F>::BYTES, &::winrs::tc2::launch_x<F, BF>, PFX "_O4(3,2)_v2x_128x" #F "fh", \
     F, 2, 2}

#ifdef WINRS_TC2_TRACE
// this translation unit's copy of the trace buffer (bfc_tc2.cu: winrs_tc2_trace)
extern "C" __attribute__((visibility("default"))) int winrs_tc2x_trace(int cta, long long* out) {
    if (cta >= 0) return (int)cudaMemcpyToSymbol(tc2::g_tc2_trace_cta, &cta, sizeof(int));
    return (int)cudaMemcpyFromSymbol(out, tc2::g_tc2_trace, sizeof(tc2::g_tc2_trace));
}
#endif

const KernelEntry* tc2x_entries(int* n) {
    static const KernelEntry e[] = {
        WINRS_TC2X_ENTRY(1, false, "f16tc", 1),
        WINRS_TC2X_ENTRY(1, false, "f16tc", 2),
        WINRS_TC2X_ENTRY(2, true, "bf16tc", 1),
        WINRS_TC2X_ENTRY(2, true, "bf16tc", 2),
    };
    *n = sizeof(e) / sizeof(e[0]);
    return e;
}

}  // namespace winrs
