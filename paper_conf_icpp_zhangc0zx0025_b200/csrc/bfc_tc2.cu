// Instantiations, TMA tensor maps and launch of the second-generation
// FP16 / BF16 tensor-core kernel (bfc_tc2.cuh).
#include <cuda.h>
#include <cuda_runtime.h>
#include <mutex>
#include "bfc_tc2.cuh"
#include "tc2_maps.cuh"
#include "launch_util.cuh"
#include "registry.h"

namespace winrs {
namespace tc2 {

template <int F, int NK, bool BF, int CG, bool TA = false>
cudaError_t launch(const Geometry& g, const void* X, const void* dY, float* dW, float* ws, cudaStream_t stream) {
    using L = Lay<F, NK, CG, TA>;
    const long long grid = num_ctas(g);
    if (grid <= 0) return cudaSuccess;
    Args a;
    a.g = g;
    a.dW = dW;
    a.ws = ws;
    a.nb = images_per_box(g);
    if (a.nb == 0 || g.a0 != 4 || g.n0 != 3 || g.r0 != 2 || g.a1 != 0) return cudaErrorInvalidValue;
    CUtensorMap mX, mY;
    if (!make_maps(g, X, dY, BF, &mX, &mY, TA ? 8 : KC)) return cudaErrorInvalidValue;
    static std::atomic<unsigned long long> done{0};
    auto k = bfc_tc2_kernel<F, NK, BF, CG, TA>;
    cudaError_t e = ensure_smem_attr(k, (size_t)L::BYTES, done);
    if (e != cudaSuccess) return e;
    const int cluster = CG * g.csplit;
    constexpr unsigned NTH = (unsigned)tc2_threads<TA>();
    if (cluster <= 1) {
        k<<<(unsigned)grid, NTH, L::BYTES, stream>>>(a, mX, mY);
        return cudaGetLastError();
    }
    if (cluster > 8) {   // 16-CTA clusters (a pair per rank of an 8-way depth split): non-portable size
        static std::atomic<unsigned long long> np{0};
        int dev = 0;
        cudaGetDevice(&dev);
        if (!(np.load() & (1ull << (dev & 63)))) {
            e = cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
            if (e != cudaSuccess) return e;
            np.fetch_or(1ull << (dev & 63));
        }
    }
    return launch_cluster(k, (unsigned)grid, NTH, (size_t)L::BYTES, stream, cluster, a, mX, mY);
}

// The swapped CTA pair (bfc_tc2s_kernel): tile = 256 k x 128 c x 1 filter row.
template <bool BF>
cudaError_t launch_sw(const Geometry& g, const void* X, const void* dY, float* dW, float* ws, cudaStream_t stream) {
    using L = LaySw;
    const long long grid = num_ctas(g);
    if (grid <= 0) return cudaSuccess;
    Args a;
    a.g = g;
    a.dW = dW;
    a.ws = ws;
    a.nb = images_per_box(g);
    if (a.nb == 0 || g.a0 != 4 || g.n0 != 3 || g.r0 != 2 || g.a1 != 0 || g.cg != 2 || g.fhs != 1)
        return cudaErrorInvalidValue;
    CUtensorMap mX, mY;
    if (!make_maps(g, X, dY, BF, &mX, &mY)) return cudaErrorInvalidValue;
    static std::atomic<unsigned long long> done{0};
    auto k = bfc_tc2s_kernel<BF>;
    cudaError_t e = ensure_smem_attr(k, (size_t)L::BYTES, done);
    if (e != cudaSuccess) return e;
    const int cluster = 2 * g.csplit;
    if (cluster > 8) {
        static std::atomic<unsigned long long> np{0};
        int dev = 0;
        cudaGetDevice(&dev);
        if (!(np.load() & (1ull << (dev & 63)))) {
            e = cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
            if (e != cudaSuccess) return e;
            np.fetch_or(1ull << (dev & 63));
        }
    }
    return launch_cluster(k, (unsigned)grid, (unsigned)NTHREADS, (size_t)L::BYTES, stream, cluster, a, mX, mY);
}

}  // namespace tc2

// tile = NK k columns x (128 / F) c rows x F filter rows (one CTA), or for a
// cta_group::2 pair (CG = 2) 256 c rows (F = 1) or 4 filter rows (F = 2).
#define WINRS_TC2_ENTRY(DT, BF, PFX, F, NK, CG)                                                          \
    {DT, 4, 3, 2, 0, 0, 0, NK, (F == 1 ? ::winrs::tc2::MROWS * CG : ::winrs::tc2::MROWS / F),            \
     ::winrs::tc2::NTHREADS, 1, 1, (size_t)::winrs::tc2::Lay<F, NK, CG>::BYTES,                          \
     &::winrs::tc2::launch<F, NK, BF, CG>,                                                                \
     PFX "_O4(3,2)_v2" #CG "_" #NK "x" #F "fh", (F == 1 ? 1 : F * CG), CG, 0}
// Xhat in TMEM (TA): single CTA, NK = 64
#define WINRS_TC2T_ENTRY(DT, BF, PFX, F)                                                                  \
    {DT, 4, 3, 2, 0, 0, 0, 64, ::winrs::tc2::MROWS / F, ::winrs::tc2::tc2_threads<true>(), 1, 1,          \
     (size_t)::winrs::tc2::Lay<F, 64, 1, true>::BYTES, &::winrs::tc2::launch<F, 64, BF, 1, true>,              \
     PFX "_O4(3,2)_v2t_64x" #F "fh", F, 1, 1}

#ifdef WINRS_TC2_TRACE
extern "C" __attribute__((visibility("default"))) int winrs_tc2_trace(int cta, long long* out) {
    if (cta >= 0) return (int)cudaMemcpyToSymbol(tc2::g_tc2_trace_cta, &cta, sizeof(int));
    return (int)cudaMemcpyFromSymbol(out, tc2::g_tc2_trace, sizeof(tc2::g_tc2_trace));
}
#endif

const KernelEntry* tc2_entries(int* n) {
    // tile = NK k columns x (128 / F) c rows x F filter rows
    static const KernelEntry e[] = {
        WINRS_TC2_ENTRY(1, false, "f16tc", 1, 128, 1),
        WINRS_TC2_ENTRY(1, false, "f16tc", 1, 64, 1),
        WINRS_TC2_ENTRY(1, false, "f16tc", 2, 128, 1),
        WINRS_TC2_ENTRY(1, false, "f16tc", 2, 64, 1),
        WINRS_TC2_ENTRY(1, false, "f16tc", 1, 128, 2),
        WINRS_TC2_ENTRY(1, false, "f16tc", 2, 128, 2),
        WINRS_TC2_ENTRY(2, true, "bf16tc", 1, 128, 1),
        WINRS_TC2_ENTRY(2, true, "bf16tc", 1, 64, 1),
        WINRS_TC2_ENTRY(2, true, "bf16tc", 2, 128, 1),
        WINRS_TC2_ENTRY(2, true, "bf16tc", 2, 64, 1),
        WINRS_TC2_ENTRY(2, true, "bf16tc", 1, 128, 2),
        WINRS_TC2_ENTRY(2, true, "bf16tc", 2, 128, 2),
        // swapped CTA pair: 256 k x 128 c (What rows split, the Xhat side shared)
        {1, 4, 3, 2, 0, 0, 0, 256, 128, ::winrs::tc2::NTHREADS, 1, 1, (size_t)::winrs::tc2::LaySw::BYTES,
         &::winrs::tc2::launch_sw<false>, "f16tc_O4(3,2)_v2s_256x128", 1, 2, 0},
        {2, 4, 3, 2, 0, 0, 0, 256, 128, ::winrs::tc2::NTHREADS, 1, 1, (size_t)::winrs::tc2::LaySw::BYTES,
         &::winrs::tc2::launch_sw<true>, "bf16tc_O4(3,2)_v2s_256x128", 1, 2, 0},
        WINRS_TC2T_ENTRY(1, false, "f16tc", 1),
        WINRS_TC2T_ENTRY(1, false, "f16tc", 2),
        WINRS_TC2T_ENTRY(2, true, "bf16tc", 1),
        WINRS_TC2T_ENTRY(2, true, "bf16tc", 2),
    };
    *n = sizeof(e) / sizeof(e[0]);
    return e;
}

}  // namespace winrs
