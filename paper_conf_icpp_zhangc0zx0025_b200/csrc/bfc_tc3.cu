// Instantiations, TMA tensor maps and launch of the FP32 tensor-core kernel
// (bfc_tc3.cuh: Omega_4(3,2), 3xTF32 split on tcgen05 kind::tf32).
#include <cuda.h>
#include <cuda_runtime.h>
#include <mutex>
#include "bfc_tc3.cuh"
#include "launch_util.cuh"
#include "registry.h"

namespace winrs {
namespace tc3 {

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

// FP32 channels-last tensor as the 5-D map {Ch, A, B, H, W} (as bfc_tc2.cu:
// 2-D A = N, B = 1; N-D A = D or Do, B = Nb), pixel stride ld elements, box
// {bc, 8 images, 1, 1, bw}, no swizzle (the FT warps re-lay the operands
// K-major); out-of-bounds elements read as zero.
static bool make_map(CUtensorMap* m, const void* base, int A, int B, int H, int W, int Ch, int ld, int bc, int bw) {
    EncodeTiledFn fn = encode_fn();
    if (!fn) return false;
    const cuuint64_t dims[5] = {(cuuint64_t)Ch, (cuuint64_t)A, (cuuint64_t)B, (cuuint64_t)H, (cuuint64_t)W};
    const cuuint64_t img = (cuuint64_t)H * W * ld * 4;
    const cuuint64_t strides[4] = {img, img * A, (cuuint64_t)W * ld * 4, (cuuint64_t)ld * 4};
    const cuuint32_t box[5] = {(cuuint32_t)bc, (cuuint32_t)KT, 1u, 1u, (cuuint32_t)bw};
    const cuuint32_t es[5] = {1u, 1u, 1u, 1u, 1u};
    return fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 5, const_cast<void*>(base), dims, strides, box, es,
              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

template <int F, int NK>
cudaError_t launch(const Geometry& g, const void* X, const void* dY, float* dW, float* ws, cudaStream_t stream) {
    using L = Lay3<F, NK>;
    const long long grid = num_ctas(g);
    if (grid <= 0) return cudaSuccess;
    const bool nd = g.T > 1 || g.D > 1;
    if ((nd ? g.Do : g.N) % KT != 0 || g.a0 != 4 || g.n0 != 3 || g.r0 != 2 || g.a1 != 0 || g.cg != 1)
        return cudaErrorInvalidValue;
    Args a;
    a.g = g;
    a.dW = dW;
    a.ws = ws;
    a.nb = KT;
    CUtensorMap mX, mY;
    if (!make_map(&mX, X, nd ? g.D : g.N, nd ? g.Nb : 1, g.H, g.W, g.C, g.C, L::BC, 4) ||
        !make_map(&mY, dY, nd ? g.Do : g.N, nd ? g.Nb : 1, g.Ho, g.Wo, g.K, g.ldy, NK, 2))
        return cudaErrorInvalidValue;
    static std::atomic<unsigned long long> done{0};
    auto k = bfc_tc3_kernel<F, NK>;
    cudaError_t e = ensure_smem_attr(k, (size_t)L::BYTES, done);
    if (e != cudaSuccess) return e;
    if (g.csplit <= 1) {
        k<<<(unsigned)grid, NTHREADS, L::BYTES, stream>>>(a, mX, mY);
        return cudaGetLastError();
    }
    return launch_cluster(k, (unsigned)grid, (unsigned)NTHREADS, (size_t)L::BYTES, stream, g.csplit, a, mX, mY);
}

}  // namespace tc3

// tile = NK k x (128 / F) c x F filter rows; fhs > 0 marks the tcgen05
// kernels, tf32 = 1 the FP32 (3xTF32) ones.
#define WINRS_TC3_ENTRY(F, NK)                                                                             \
    {0, 4, 3, 2, 0, 0, 0, NK, ::winrs::tc2::MROWS / F, ::winrs::tc2::NTHREADS, 1, 1,                       \
     (size_t)::winrs::tc3::Lay3<F, NK>::BYTES, &::winrs::tc3::launch<F, NK>,                              \
     "f32tc_O4(3,2)_v3_" #NK "x" #F "fh", F, 1, 0, 1}

const KernelEntry* tc3_entries(int* n) {
    static const KernelEntry e[] = {
        WINRS_TC3_ENTRY(1, 128),
        WINRS_TC3_ENTRY(2, 128),
        WINRS_TC3_ENTRY(1, 64),
        WINRS_TC3_ENTRY(2, 64),
    };
    *n = sizeof(e) / sizeof(e[0]);
    return e;
}

}  // namespace winrs
