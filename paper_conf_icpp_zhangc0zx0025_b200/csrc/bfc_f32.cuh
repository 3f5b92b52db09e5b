// FP32 CUDA-core fused WinRS BFC kernel for sm_100a.
//
// One CTA computes one B_N x B_M x n0 tile of one dW bucket (§5.1
// P@28778-29449, Algorithm 3): it walks its segment's depth d = (row h,
// unit u, image n) in chunks of BD entries (the paper steps n by 8, line 25),
// and per chunk
//   1. stages raw dY units (r x B_N) and X windows (alpha x B_M) into shared
//      memory with cp.async (16-byte, zero-filled outside the map: the width
//      padding of P@33854 and the masked tail unit of DESIGN.md R6),
//   2. runs the filter transform G w (FT) and input transform D^T x (IT) in
//      FP32 (generated straight-line code, +/- row pairing P@38072),
//   3. runs the alpha-batched B_N x B_M x BD GEMM (EWM, footnote 2 P@18784)
//      into register accumulators v[xi][k][c] (eq. (6): everything stays in
//      the Winograd domain until the end of the main loop, P@29449).
// After the main loop the OT (A^T v) runs once per tile through shared
// memory in rounds (P@36150 "Result Output") and the tile is written to the
// CTA's bucket.  CTAs of a band's last column segment then run a second
// phase over the residual Omega_a1 units and add into the same bucket.
//
// Differences from the paper's design: cp.async
// zero-fill replaces texture -1 masking; 4-wide interleaved register tiles
// replace the "contrapuntal" offsets; the residual kernel is fused into the
// same launch instead of a separate block group.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include "winrs_internal.h"
#include "winograd_generated.cuh"

namespace winrs {
namespace f32k {

constexpr int NT = 256;   // threads per CTA (8 warps)
constexpr int BD = 8;     // depth entries per chunk

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void cp_async16(void* dst, const void* src, bool valid) {
    const int sz = valid ? 16 : 0;   // src-size 0 => the 16 bytes are zero-filled
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n"
                 :: "r"(smem_u32(dst)), "l"(src), "r"(sz) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N_>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" :: "n"(N_) : "memory"); }

// Thread layout of the batched GEMM for a given alpha and CTA tile.
template <int ALPHA, int BN, int BM>
struct GemmLayout {
    static constexpr int TPX = NT / ALPHA;                 // threads per Winograd point xi
    // threads along k (TPK) x along c (TPC); register tile TM x TN in 4-wide groups
    static constexpr int TPK = (TPX >= 128) ? 16 : 8;
    static constexpr int TPC = TPX / TPK;
    static constexpr int TM = BN / TPK;
    static constexpr int TN = BM / TPC;
    static_assert(TPX * ALPHA == NT, "alpha must divide the thread count");
    static_assert(TPK * TPC == TPX, "bad thread split");
    static_assert(TM % 4 == 0 && TN % 4 == 0 && TM >= 4 && TN >= 4, "register tile must be 4-wide groups");
    static constexpr int GM = TM / 4, GN = TN / 4;       // 4-wide groups per thread
};

// Shared-memory footprint of one phase (pipeline buffers or the OT staging,
// whichever is larger) in floats.
template <int ALPHA, int RR, int BN, int BM>
struct PhaseSmem {
    static constexpr int rawG = 2 * BD * RR * BN;
    static constexpr int rawX = 2 * BD * ALPHA * BM;
    static constexpr int Gt = ALPHA * BD * BN;
    static constexpr int Xt = ALPHA * BD * BM;
    static constexpr int pipe = rawG + rawX + Gt + Xt;
    static constexpr int ot = ALPHA * (GemmLayout<ALPHA, BN, BM>::TPK * 4) * BM;   // one round
    static constexpr int floats = pipe > ot ? pipe : ot;
};

// One phase: the main loop over `units` units of width RR starting at dY
// column w_first, for dW columns [fw0, fw0 + NN), then the OT and the bucket
// write (store, or add when `accumulate`).
template <int ALPHA, int NN, int RR, int BN, int BM>
__device__ __forceinline__ void run_phase(const Geometry& g, const float* __restrict__ X,
                                          const float* __restrict__ dY, float* __restrict__ bucket,
                                          const CtaCoord& cc, int hs, int he, int w_first, int units,
                                          int fw0, bool accumulate, float* smem) {
    using WT = Wino<ALPHA, NN, RR>;
    using L = GemmLayout<ALPHA, BN, BM>;
    using SM = PhaseSmem<ALPHA, RR, BN, BM>;
    float* rawG = smem;                       // [2][BD][RR][BN]
    float* rawX = rawG + SM::rawG;            // [2][BD][ALPHA][BM]
    float* Gt = rawX + SM::rawX;              // [ALPHA][BD][BN]
    float* Xt = Gt + SM::Gt;                  // [ALPHA][BD][BM]

    const int tid = threadIdx.x;
    const int k_base = cc.kb * BN, c_base = cc.cb * BM;
    const int rows = he - hs;
    const long long depth = (long long)(rows > 0 ? rows : 0) * units * g.N;
    const int nchunks = (int)((depth + BD - 1) / BD);

    // ---- loader: 32 threads per depth entry of a chunk
    constexpr int TPD = NT / BD;
    const int ld_d = tid / TPD, ld_l = tid % TPD;
    auto issue = [&](int chunk, int buf) {
        const long long d = (long long)chunk * BD + ld_d;
        const bool dv = d < depth;
        int n = 0, h = hs, u = 0;
        if (dv) {
            n = (int)(d % g.N);
            const long long t = d / g.N;
            u = (int)(t % units);
            h = hs + (int)(t / units);
        }
        const int w0 = w_first + u * RR;
        const float* gsrc = dY + (((long long)n * g.Ho + h) * g.Wo + w0) * g.K + k_base;
        const int xrow = h + cc.fh - g.pad;
        const int xcol0 = w0 + fw0 - g.pad;
        const float* xsrc = X + (((long long)n * g.H + xrow) * g.W) * g.C + c_base;
        float* gdst = rawG + ((buf * BD + ld_d) * RR) * BN;
        float* xdst = rawX + ((buf * BD + ld_d) * ALPHA) * BM;
        constexpr int GV = RR * (BN / 4);
        for (int q = ld_l; q < GV; q += TPD) {
            const int i = q / (BN / 4), v4 = q % (BN / 4);
            const int kk = k_base + v4 * 4;
            const bool ok = dv && (w0 + i < g.Wo) && (kk < g.K);
            cp_async16(gdst + i * BN + v4 * 4, ok ? (const void*)(gsrc + (long long)i * g.K + v4 * 4) : (const void*)dY, ok);
        }
        constexpr int XV = ALPHA * (BM / 4);
        for (int q = ld_l; q < XV; q += TPD) {
            const int t = q / (BM / 4), v4 = q % (BM / 4);
            const int col = xcol0 + t;
            const int ccn = c_base + v4 * 4;
            const bool ok = dv && col >= 0 && col < g.W && ccn < g.C;
            cp_async16(xdst + t * BM + v4 * 4, ok ? (const void*)(xsrc + (long long)col * g.C + v4 * 4) : (const void*)X, ok);
        }
    };

    // ---- accumulators
    float v[L::TM][L::TN];
#pragma unroll
    for (int i = 0; i < L::TM; ++i)
#pragma unroll
        for (int j = 0; j < L::TN; ++j) v[i][j] = 0.f;
    const int xi = tid / L::TPX;
    const int tl = tid % L::TPX;
    const int tk = tl / L::TPC, tc = tl % L::TPC;

    if (nchunks > 0) {
        issue(0, 0);
        cp_async_commit();
    }
    for (int ch = 0; ch < nchunks; ++ch) {
        const int buf = ch & 1;
        if (ch + 1 < nchunks) {
            issue(ch + 1, buf ^ 1);
            cp_async_commit();
            cp_async_wait<1>();
        } else {
            cp_async_wait<0>();
        }
        __syncthreads();
        // ---- transforms (FP32), raw[buf] -> Gt / Xt
        {
            const float* rg = rawG + buf * BD * RR * BN;
            for (int p = tid; p < BD * BN; p += NT) {
                const int d = p / BN, k = p % BN;
                float w[RR], o[ALPHA];
#pragma unroll
                for (int i = 0; i < RR; ++i) w[i] = rg[(d * RR + i) * BN + k];
                WT::ft(w, o);
#pragma unroll
                for (int x = 0; x < ALPHA; ++x) Gt[(x * BD + d) * BN + k] = o[x];
            }
            const float* rx = rawX + buf * BD * ALPHA * BM;
            for (int p = tid; p < BD * BM; p += NT) {
                const int d = p / BM, c = p % BM;
                float xv[ALPHA], o[ALPHA];
#pragma unroll
                for (int t = 0; t < ALPHA; ++t) xv[t] = rx[(d * ALPHA + t) * BM + c];
                WT::it(xv, o);
#pragma unroll
                for (int x = 0; x < ALPHA; ++x) Xt[(x * BD + d) * BM + c] = o[x];
            }
        }
        __syncthreads();
        // ---- alpha-batched GEMM: v[xi] += Gt[xi]^T Xt[xi]
        {
            const float* ga = Gt + xi * BD * BN;
            const float* xb = Xt + xi * BD * BM;
#pragma unroll
            for (int d = 0; d < BD; ++d) {
                float a[L::TM], b[L::TN];
#pragma unroll
                for (int gm = 0; gm < L::GM; ++gm) {
                    const float4 t = *reinterpret_cast<const float4*>(ga + d * BN + (gm * L::TPK + tk) * 4);
                    a[gm * 4 + 0] = t.x; a[gm * 4 + 1] = t.y; a[gm * 4 + 2] = t.z; a[gm * 4 + 3] = t.w;
                }
#pragma unroll
                for (int gn = 0; gn < L::GN; ++gn) {
                    const float4 t = *reinterpret_cast<const float4*>(xb + d * BM + (gn * L::TPC + tc) * 4);
                    b[gn * 4 + 0] = t.x; b[gn * 4 + 1] = t.y; b[gn * 4 + 2] = t.z; b[gn * 4 + 3] = t.w;
                }
#pragma unroll
                for (int i = 0; i < L::TM; ++i)
#pragma unroll
                    for (int j = 0; j < L::TN; ++j) v[i][j] = fmaf(a[i], b[j], v[i][j]);
            }
        }
    }
    __syncthreads();   // pipeline buffers are free from here on

    // ---- OT in rounds (one 4-wide k-group of every thread per round)
    float* As = smem;   // [ALPHA][TPK*4][BM]
    constexpr int KR = L::TPK * 4;   // k rows per round
#pragma unroll
    for (int gm = 0; gm < L::GM; ++gm) {
        // stage: k_local = tk*4 + e (global k = (gm*TPK + tk)*4 + e)
#pragma unroll
        for (int e = 0; e < 4; ++e)
#pragma unroll
            for (int gn = 0; gn < L::GN; ++gn) {
                float4 t;
                t.x = v[gm * 4 + e][gn * 4 + 0]; t.y = v[gm * 4 + e][gn * 4 + 1];
                t.z = v[gm * 4 + e][gn * 4 + 2]; t.w = v[gm * 4 + e][gn * 4 + 3];
                *reinterpret_cast<float4*>(As + (xi * KR + tk * 4 + e) * BM + (gn * L::TPC + tc) * 4) = t;
            }
        __syncthreads();
        for (int p = tid; p < KR * BM; p += NT) {
            const int kl = p / BM, c = p % BM;
            const int kg = k_base + gm * KR + kl, cg = c_base + c;
            float vv[ALPHA], y[NN];
#pragma unroll
            for (int x = 0; x < ALPHA; ++x) vv[x] = As[(x * KR + kl) * BM + c];
            WT::ot(vv, y);
            if (kg < g.K && cg < g.C) {
                float* dst = bucket + (((long long)kg * g.R + cc.fh) * g.S + fw0) * g.C + cg;
#pragma unroll
                for (int j = 0; j < NN; ++j) {
                    if (accumulate) dst[(long long)j * g.C] += y[j];
                    else dst[(long long)j * g.C] = y[j];
                }
            }
        }
        __syncthreads();
    }
}

// The fused launch: every CTA runs the Omega_a0 phase over its segment, and
// CTAs of a band's last column segment also run the residual Omega_a1 phase.
template <int A0, int N0, int R0, int A1, int N1, int R1, int BN, int BM>
__global__ void __launch_bounds__(NT, 1)
bfc_f32_kernel(const Geometry g, const float* __restrict__ X, const float* __restrict__ dY,
               float* __restrict__ dW, float* __restrict__ ws) {
    extern __shared__ __align__(16) float smem[];
    const CtaCoord cc = decode_cta(g, blockIdx.x);
    const int seg = cc.band * g.seg_cols + cc.col;
    float* bucket = seg == 0 ? dW : ws + (long long)(seg - 1) * g.dw_elems;
    int hs, he;
    band_rows(g, cc.band, cc.fh, &hs, &he);
    int w_first, units;
    seg_units(g, cc.col, &w_first, &units);
    const int fw0 = cc.ft * N0;
    run_phase<A0, N0, R0, BN, BM>(g, X, dY, bucket, cc, hs, he, w_first, units, fw0, false, smem);
    if constexpr (A1 != 0) {
        if (has_residual(g, cc.col)) {
            static_assert(N0 % N1 == 0, "residual n1 must divide n0");
#pragma unroll 1
            for (int j = 0; j < N0 / N1; ++j)
                run_phase<A1, N1, R1, BN, BM>(g, X, dY, bucket, cc, hs, he, g.res_col0, g.k1,
                                              fw0 + j * N1, true, smem);
        }
    }
}

template <int A0, int N0, int R0, int A1, int N1, int R1, int BN, int BM>
constexpr size_t smem_bytes() {
    size_t a = PhaseSmem<A0, R0, BN, BM>::floats;
    size_t b = A1 ? PhaseSmem<(A1 ? A1 : A0), (R1 ? R1 : R0), BN, BM>::floats : 0;
    return 4 * (a > b ? a : b);
}

}  // namespace f32k
}  // namespace winrs
