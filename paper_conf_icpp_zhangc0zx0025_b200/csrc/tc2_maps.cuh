// TMA tensor maps of the tc2 / tc2x kernels (bfc_tc2.cuh, bfc_tc2x.cuh):
// 16-bit channels-last X and dY as 5-D maps with the 128-byte swizzle.
#pragma once
#include <atomic>
#include <cuda.h>
#include <cuda_runtime.h>
#include <mutex>
#include "bfc_tc2.cuh"

#ifndef WINRS_TMA_L2PROMO
#define WINRS_TMA_L2PROMO CU_TENSOR_MAP_L2_PROMOTION_L2_256B   // L2 sector promotion of the X / dY boxes (A/B knob)
#endif

namespace winrs {
namespace tc2 {

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

inline EncodeTiledFn encode_fn() {
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
inline bool make_map(CUtensorMap* m, const void* base, int A, int B, int H, int W, int Ch, int ld, int bw, int bn, bool bf) {
    EncodeTiledFn fn = encode_fn();
    if (!fn) return false;
    const cuuint64_t dims[5] = {(cuuint64_t)Ch, (cuuint64_t)A, (cuuint64_t)B, (cuuint64_t)H, (cuuint64_t)W};
    const cuuint64_t img = (cuuint64_t)H * W * ld * 2;
    const cuuint64_t strides[4] = {img, img * A, (cuuint64_t)W * ld * 2, (cuuint64_t)ld * 2};
    const cuuint32_t box[5] = {64u, (cuuint32_t)bn, 1u, 1u, (cuuint32_t)bw};
    const cuuint32_t es[5] = {1u, 1u, 1u, 1u, 1u};
    return fn(m, bf ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 5, const_cast<void*>(base),
              dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
              WINRS_TMA_L2PROMO, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}
// The X and dY maps of a plan (2-D or N-D).
// xbn: images per X box (TA kernels: 8, two boxes per stage and atom).
inline bool make_maps(const Geometry& g, const void* X, const void* dY, bool bf, CUtensorMap* mX, CUtensorMap* mY,
                      int xbn = KC) {
    const bool nd = g.T > 1 || g.D > 1;
    return make_map(mX, X, nd ? g.D : g.N, nd ? g.Nb : 1, g.H, g.W, g.C, g.C, 4, xbn, bf) &&
           make_map(mY, dY, nd ? g.Do : g.N, nd ? g.Nb : 1, g.Ho, g.Wo, g.K, g.ldy, 2, KC, bf);
}

// Images per TMA box: one box per stage and atom, so the box's [cols][images]
// rows are exactly a column-major run of 16-row operand atoms (N % 16 == 0;
// N-D: Do % 16 == 0, 16 depth slices of one batch image).
inline int images_per_box(const Geometry& g) {
    const bool nd = g.T > 1 || g.D > 1;
    return (nd ? g.Do : g.N) % KC == 0 ? KC : 0;
}

// Stream-K chain flags / ticket counters (bfc_tc2x.cu): a fresh epoch tag per
// launch and the device's flag region for that epoch (regions rotate, so launches
// in flight on different streams do not share one); nullptr if allocation failed.
unsigned int sk_next_epoch();
unsigned int* sk_flags_region(int dev, unsigned int epoch);

}  // namespace tc2
}  // namespace winrs
