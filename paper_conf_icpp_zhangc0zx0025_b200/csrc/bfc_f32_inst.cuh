// Instantiation helper for the FP32 fused kernels (included by the
// bfc_f32_part*.cu translation units, which are compiled in parallel).
#pragma once
#include "bfc_f32.cuh"
#include "launch_util.cuh"
#include "registry.h"

namespace winrs {
namespace f32k {

template <int A0, int N0, int R0, int A1, int N1, int R1, int BN, int BM, typename TI = float>
cudaError_t launch(const Geometry& g, const void* X, const void* dY, float* dW, float* ws,
                   cudaStream_t stream) {
    static std::atomic<unsigned long long> done{0};
    auto k = bfc_f32_kernel<A0, N0, R0, A1, N1, R1, BN, BM, TI>;
    constexpr size_t sm = smem_bytes<A0, N0, R0, A1, N1, R1, BN, BM>();
    cudaError_t e = ensure_smem_attr(k, sm, done);
    if (e != cudaSuccess) return e;
    const long long grid = num_ctas(g);
    if (grid <= 0) return cudaSuccess;
    if (g.csplit <= 1) {
        k<<<(unsigned)grid, NTOT, sm, stream>>>(g, static_cast<const TI*>(X), static_cast<const TI*>(dY), dW, ws);
        return cudaGetLastError();
    }
    return launch_cluster(k, (unsigned)grid, NTOT, sm, stream, g.csplit, g, static_cast<const TI*>(X),
                          static_cast<const TI*>(dY), dW, ws);
}

}  // namespace f32k
}  // namespace winrs

#define WINRS_F32_ENTRY(A0, N0, R0, A1, N1, R1, BN, BM)                                         \
    {0, A0, N0, R0, A1, N1, R1, BN, BM, ::winrs::f32k::NTOT, 1, 1,                                  \
     ::winrs::f32k::smem_bytes<A0, N0, R0, A1, N1, R1, BN, BM>(),                                \
     &::winrs::f32k::launch<A0, N0, R0, A1, N1, R1, BN, BM>,                                     \
     "f32_O" #A0 "(" #N0 "," #R0 ")+O" #A1 "(" #N1 "," #R1 ")_" #BN "x" #BM}
// FP16 / BF16 inputs on the FP32 CUDA-core pipeline (the alpha = 16 widths, R26):
// cc16 = 1 marks them for the planner's time model.
#define WINRS_C16_ENTRY(DT, TI, PFX, A0, N0, R0, A1, N1, R1, BN, BM)                                    \
    {DT, A0, N0, R0, A1, N1, R1, BN, BM, ::winrs::f32k::NTOT, 1, 1,                                       \
     ::winrs::f32k::smem_bytes<A0, N0, R0, A1, N1, R1, BN, BM>(),                                     \
     &::winrs::f32k::launch<A0, N0, R0, A1, N1, R1, BN, BM, TI>,                                      \
     PFX "cc_O" #A0 "(" #N0 "," #R0 ")+O" #A1 "(" #N1 "," #R1 ")_" #BN "x" #BM, 0, 0, 0, 0, 1}
