// Instantiations and launch of the xi-split FP16 / BF16 tensor-core kernel
// (bfc_tc2x.cuh): tile = 128 k x (128 / F) c x F filter rows per CTA pair,
// cluster = 2 x csplit CTAs.
#include <cuda.h>
#include <cuda_runtime.h>
#include "bfc_tc2x.cuh"
#include "launch_util.cuh"
#include "registry.h"
#include "tc2_maps.cuh"
#include <atomic>
#include <mutex>

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
    if (!make_map(&mX2, X, nd ? g.D : g.N, nd ? g.Nb : 1, g.H, g.W, g.C, g.C, LayX<F>::BAL ? 3 : 2, 8, BF))
        return cudaErrorInvalidValue;
    if (LayX<F>::BAL) mX4 = mX2;   // balanced split: both halves load three columns
    static std::atomic<unsigned long long> done{0};
    auto k = bfc_tc2x_kernel<F, BF>;
    cudaError_t e = ensure_smem_attr(k, (size_t)L::BYTES, done);
    if (e != cudaSuccess) return e;
    return launch_cluster(k, (unsigned)grid, (unsigned)tc2_threads<true>(), (size_t)L::BYTES, stream, 2 * g.csplit, a,
                          mX4, mX2, mY);
}

// Stream-K pairs (SK): the chain flags live in a library-owned, zero-initialised
// per-device buffer (no workspace); each launch tags its flag values with a fresh
// epoch so values left by an earlier launch never match a waiter.
// SK_REGIONS independent flag / ticket regions per device, used in rotation (one per
// launch): launches that overlap on different streams use different regions (up to
// SK_REGIONS in flight); launches on one stream are serialised anyway.
constexpr int SK_REGIONS = 8;
constexpr size_t SK_REGION_WORDS = SK_MAX_TILES + 64;   // flags, ticket counters, 256-byte aligned
static unsigned int* sk_flags_for_device(int dev) {
    static std::mutex mu;
    static unsigned int* bufs[64] = {};
    std::lock_guard<std::mutex> lk(mu);
    if (dev < 0 || dev >= 64) return nullptr;
    if (!bufs[dev]) {
        void* p = nullptr;
        if (cudaMalloc(&p, SK_REGIONS * SK_REGION_WORDS * sizeof(unsigned int)) != cudaSuccess) return nullptr;
        if (cudaMemset(p, 0, SK_REGIONS * SK_REGION_WORDS * sizeof(unsigned int)) != cudaSuccess) return nullptr;
        if (cudaDeviceSynchronize() != cudaSuccess) return nullptr;
        bufs[dev] = static_cast<unsigned int*>(p);
    }
    return bufs[dev];
}

unsigned int* sk_flags_region(int dev, unsigned int epoch) {
    unsigned int* base = sk_flags_for_device(dev);
    return base ? base + (size_t)(epoch % SK_REGIONS) * SK_REGION_WORDS : nullptr;
}

// One epoch counter for every instantiation (f16 / bf16, F = 1 / 2): the flags and
// the ticket counter are shared, so two launches must never carry the same tag.
unsigned int sk_next_epoch() {
    static std::atomic<unsigned int> epoch{0};
    return (epoch.fetch_add(1) % 0xFFFFFEu) + 1u;   // 24-bit tag, never 0
}

template <int F, bool BF>
cudaError_t launch_sk(const Geometry& g, const void* X, const void* dY, float* dW, float* ws, cudaStream_t stream) {
    using L = LayX<F>;
    const long long tiles = num_tiles(g);
    if (tiles <= 0) return cudaSuccess;
    Args a;
    a.g = g;
    a.dW = dW;
    a.ws = ws;
    a.nb = images_per_box(g);
    if (a.nb == 0 || g.a0 != 4 || g.n0 != 3 || g.r0 != 2 || g.a1 != 0 || g.cg != 2 || g.fhs != F || g.csplit != 1 ||
        tiles > SK_MAX_TILES || g.bands * g.seg_cols * g.fhg > 4096)
        return cudaErrorInvalidValue;
    const bool nd = g.T > 1 || g.D > 1;
    CUtensorMap mX4, mX2, mY;
    if (!make_maps(g, X, dY, BF, &mX4, &mY, 8)) return cudaErrorInvalidValue;
    if (!make_map(&mX2, X, nd ? g.D : g.N, nd ? g.Nb : 1, g.H, g.W, g.C, g.C, LayX<F>::BAL ? 3 : 2, 8, BF))
        return cudaErrorInvalidValue;
    if (LayX<F>::BAL) mX4 = mX2;   // balanced split: both halves load three columns
    auto k = bfc_tc2x_kernel<F, BF, true>;
    static std::atomic<unsigned long long> done{0};
    cudaError_t e = ensure_smem_attr(k, (size_t)L::BYTES, done);
    if (e != cudaSuccess) return e;
    int dev = 0;
    if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
    a.sk_epoch = sk_next_epoch();
    a.sk_flags = sk_flags_region(dev, a.sk_epoch);
    if (!a.sk_flags) return cudaErrorMemoryAllocation;
    // pairs: the co-resident 2-CTA clusters (one wave; the chain itself only waits for
    // lower, already running pairs -- ticketed in the kernel -- so residency is not
    // required for progress)
    cudaLaunchConfig_t cfg = {};
    cfg.blockDim = dim3((unsigned)tc2_threads<true>());
    cfg.dynamicSmemBytes = (size_t)L::BYTES;
    cfg.stream = stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = 2;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    static int max_pairs[64] = {};
    if (dev < 64 && max_pairs[dev] == 0) {
        cfg.gridDim = dim3(2);
        int n = 0;
        if ((e = cudaOccupancyMaxActiveClusters(&n, k, &cfg)) != cudaSuccess) return e;
        max_pairs[dev] = n > 0 ? n : 1;
    }
    int P = dev < 64 ? max_pairs[dev] : 1;
    // a.sk_pairs <= the chunk count, so that every pair has work
    long long chunks = 0;
    for (int bi = 0; bi < g.bands * g.seg_cols * g.fhg; ++bi) {
        int hs, he, wf, units;
        const int sc = bi / g.fhg;
        group_rows(g, sc / g.seg_cols, (bi % g.fhg) * g.fhs, &hs, &he);
        seg_units(g, sc % g.seg_cols, &wf, &units);
        chunks += (long long)g.kblocks * g.cblocks * g.ftiles * (((long long)(he > hs ? he - hs : 0) * units * g.N + KC - 1) / KC);
    }
    if (chunks <= 0) return cudaSuccess;
    if (P > chunks) P = (int)chunks;
    a.sk_pairs = P;
    cfg.gridDim = dim3((unsigned)(2 * P));
    return cudaLaunchKernelEx(&cfg, k, a, mX4, mX2, mY);
}

}  // namespace tc2

cudaError_t sk_prepare(int dev) { return tc2::sk_flags_region(dev, 0) ? cudaSuccess : cudaErrorMemoryAllocation; }

#define WINRS_TC2K_ENTRY(DT, BF, PFX, F)                                                                  \
    {DT, 4, 3, 2, 0, 0, 0, 128, ::winrs::tc2::MROWS / F, ::winrs::tc2::tc2_threads<true>(), 1, 1,         \
     (size_t)::winrs::tc2::LayX<F>::BYTES, &::winrs::tc2::launch_sk<F, BF>, PFX "_O4(3,2)_v2k_128x" #F "fh", \
     F, 2, 3}

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
        // stream-K pairs (one launch of all co-resident pairs over the concatenated tile depths)
        WINRS_TC2K_ENTRY(1, false, "f16tc", 1),
        WINRS_TC2K_ENTRY(1, false, "f16tc", 2),
        WINRS_TC2K_ENTRY(2, true, "bf16tc", 1),
        WINRS_TC2K_ENTRY(2, true, "bf16tc", 2),
    };
    *n = sizeof(e) / sizeof(e[0]);
    return e;
}

}  // namespace winrs
