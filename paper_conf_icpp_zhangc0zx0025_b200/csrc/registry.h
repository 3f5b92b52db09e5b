// Registry of compiled fused-kernel instantiations.  The planner only ever
// chooses a (kernel pair, CTA tile) that is present here, so every plan is
// runnable; there is no fallback path.
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include "winrs_internal.h"

namespace winrs {

typedef cudaError_t (*LaunchFn)(const Geometry& g, const void* X, const void* dY, float* dW,
                                float* ws, cudaStream_t stream);

struct KernelEntry {
    int dtype;                 // 0 = FP32 CUDA-core, 1 = FP16 tensor-core
    int a0, n0, r0;            // bulk kernel Omega_a0(n0, r0)
    int a1, n1, r1;            // residual kernel (a1 == 0: none)
    int bn, bm;                // CTA tile B_N (k) x B_M (c)
    int threads;
    int occ;                   // planner's CTAs/SM hint
    int csplit_ok;             // kernel supports the thread-block-cluster depth split
    size_t smem;               // dynamic shared memory bytes
    LaunchFn launch;
    const char* name;
    int fhs;                   // filter rows per tile (fh group; 0 = 1: one row); > 0 marks the
                               // second-generation tcgen05 kernels (bfc_tc2.cuh), which need N % 16 == 0
    int cg;                    // CTAs per UMMA: 2 = cta_group::2 pair (0 = 1)
    int ta;                    // 1: tc2 kernel with the transformed X operand in TMEM (bfc_tc2.cuh TA);
                               // 2: the same with the four xi split over a CTA pair (bfc_tc2x.cuh);
                               // 3: those pairs on the stream-K schedule
    int tf32;                  // 1: FP32 inputs on the tensor cores, 3xTF32 split (bfc_tc3.cuh)
    int cc16;                  // 1: FP16 / BF16 inputs on the FP32 CUDA-core pipeline (bfc_f32.cuh, TI = 16-bit)
};

// All entries (FP32 and FP16), terminated by count.
const KernelEntry* kernel_entries(int* count);

// Allocates the stream-K chain-flag regions of device `dev` (bfc_tc2x.cu), once.
cudaError_t sk_prepare(int dev);

cudaError_t launch_bucket_reduce(float* dW, const float* ws, long long n, int Z, int num_sms,
                                 cudaStream_t stream);

// Fused bucket reduction + cross-rank all-reduce over peer memory (allreduce.cu).
constexpr int AR_MAX = 8;
struct PeerArgs {
    float* stage[AR_MAX];
    float* dW[AR_MAX];
    unsigned int* flags[AR_MAX];
};
cudaError_t launch_fused_reduce_allreduce(const float* dW_local, const float* ws, long long n, int Z,
                                          const PeerArgs& pa, unsigned int* counter, int rank, int world,
                                          unsigned int epoch, int num_sms, cudaStream_t stream);

}  // namespace winrs
