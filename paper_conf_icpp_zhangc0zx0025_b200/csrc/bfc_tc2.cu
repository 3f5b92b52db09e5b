// Instantiations, TMA tensor maps and launch of the second-generation
// FP16 / BF16 tensor-core kernel (bfc_tc2.cuh).
#include <cuda.h>
#include <cuda_runtime.h>
#include <mutex>
#include "bfc_tc2.cuh"
#include "launch_util.cuh"
#include "registry.h"

namespace winrs {
namespace tc2 {

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn encode_fn() {
    static EncodeTiledFn fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<EncodeTiledFn>(p);
    });
    return fn;
}

// 16-bit channels-last tensor as the 5-D TMA map {Ch, A, B, H, W} (A inner
// image axis, B outer: 2-D [N][H][W][Ch] -> A = N, B = 1; N-D [Nb][D][H][W][Ch]
// -> A = D, B = Nb), pixel stride ld >= Ch elements; box {64, bn, 1, 1, bw}
// with the 128-byte swizzle: every (col, image) is one 128-byte row of a UMMA
// MN-major SW128 atom.  Out-of-bounds elements (padding, depth taps outside
// [0, D), masked columns, channel tails, past-the-end images) read as zero.
static bool make_map(CUtensorMap* m, const void* base, int A, int B, int H, int W, int Ch, int ld, int bw, int bn, bool bf) {
    EncodeTiledFn fn = encode_fn();
    if (!fn) return false;
    const cuuint64_t dims[5] = {(cuuint64_t)Ch, (cuuint64_t)A, (cuuint64_t)B, (cuuint64_t)H, (cuuint64_t)W};
    const cuuint64_t img = (cuuint64_t)H * W * ld * 2;
    const cuuint64_t strides[4] = {img, img * A, (cuuint64_t)W * ld * 2, (cuuint64_t)ld * 2};
    const cuuint32_t box[5] = {64u, (cuuint32_t)bn, 1u, 1u, (cuuint32_t)bw};
    const cuuint32_t es[5] = {1u, 1u, 1u, 1u, 1u};
    return fn(m, bf ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 5, const_cast<void*>(base),
              dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
              CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}
// The X and dY maps of a plan (2-D or N-D).
// xbn: images per X box (TA kernels: 8, two boxes per stage and atom).
static bool make_maps(const Geometry& g, const void* X, const void* dY, bool bf, CUtensorMap* mX, CUtensorMap* mY,
                      int xbn = KC) {
    const bool nd = g.T > 1 || g.D > 1;
    return make_map(mX, X, nd ? g.D : g.N, nd ? g.Nb : 1, g.H, g.W, g.C, g.C, 4, xbn, bf) &&
           make_map(mY, dY, nd ? g.Do : g.N, nd ? g.Nb : 1, g.Ho, g.Wo, g.K, g.ldy, 2, KC, bf);
}

// Images per TMA box: one box per stage and atom, so the box's [cols][images]
// rows are exactly a column-major run of 16-row operand atoms (N % 16 == 0;
// N-D: Do % 16 == 0, 16 depth slices of one batch image).
static int images_per_box(const Geometry& g) {
    const bool nd = g.T > 1 || g.D > 1;
    return (nd ? g.Do : g.N) % KC == 0 ? KC : 0;
}

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
