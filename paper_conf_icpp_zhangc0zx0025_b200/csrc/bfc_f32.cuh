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
#include "winrs_vec.cuh"

namespace winrs {
namespace f32k {

// Packed FP32 pair helpers: ptxas folds pk2(a, a) into the scalar-broadcast
// operand form of FFMA2, so the outer product acc[i][j..j+1] += a_i * b[j..j+1]
// issues one FFMA2 per two FMAs with no extra moves.
__device__ __forceinline__ uint64_t pk2(float lo, float hi) {
    uint64_t r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(lo), "f"(hi));
    return r;
}
__device__ __forceinline__ float2 up2(uint64_t r) {
    float2 f;
    asm("mov.b64 {%0, %1}, %2;" : "=f"(f.x), "=f"(f.y) : "l"(r));
    return f;
}
__device__ __forceinline__ uint64_t ffma2(uint64_t a, uint64_t b, uint64_t c) {
    uint64_t d;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
    return d;
}

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

// Output staging tile in shared memory: [n0][B_N][B_M + 4] floats (row pad
// keeps the float4 staging stores conflict-free).
template <int BM> __host__ __device__ constexpr int out_ld() { return BM + 4; }

// One phase: the main loop over this CTA's chunk range of the depth of
// `units` units of width RR starting at dY column w_first, for dW columns
// [fw0, fw0 + NN), then the OT into the output staging tile at column offset
// j_off (store, or add when `accumulate`).
template <int ALPHA, int NN, int RR, int BN, int BM>
__device__ __forceinline__ void run_phase(const Geometry& g, const float* __restrict__ X,
                                          const float* __restrict__ dY, float* __restrict__ Out,
                                          const CtaCoord& cc, int hs, int he, int w_first, int units,
                                          int fw0, int j_off, bool accumulate, int rank, float* smem) {
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
    int c_lo, c_hi;   // this cluster rank's share of the chunks
    split_chunks((int)((depth + BD - 1) / BD), rank, g.csplit, &c_lo, &c_hi);
    const int nchunks = c_hi - c_lo;

    // ---- loader: 32 threads per depth entry of a chunk
    constexpr int TPD = NT / BD;
    const int ld_d = tid / TPD, ld_l = tid % TPD;
    auto issue = [&](int chunk, int buf) {
        const long long d = (long long)(c_lo + chunk) * BD + ld_d;
        const bool dv = d < depth;
        int n = 0, h = hs, u = 0;
        if (dv) {
            n = (int)(d % g.N);
            const long long t = d / g.N;
            u = (int)(t % units);
            h = hs + (int)(t / units);
        }
        const int w0 = w_first + u * RR;
        const float* gsrc = dY + (((long long)n * g.Ho + h) * g.Wo + w0) * g.ldy + k_base;
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
            cp_async16(gdst + i * BN + v4 * 4, ok ? (const void*)(gsrc + (long long)i * g.ldy + v4 * 4) : (const void*)dY, ok);
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

    // ---- accumulators: pairs along c, FFMA2
    uint64_t v2[L::TM][L::TN / 2];
#pragma unroll
    for (int i = 0; i < L::TM; ++i)
#pragma unroll
        for (int j = 0; j < L::TN / 2; ++j) v2[i][j] = 0ull;
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
        // ---- transforms (FP32, packed f32x2 over channel pairs), raw[buf] -> Gt / Xt
        {
            const float* rg = rawG + buf * BD * RR * BN;
            for (int p = tid; p < BD * (BN / 2); p += NT) {
                const int d = p / (BN / 2), k = 2 * (p % (BN / 2));
                F2 w[RR], o[ALPHA];
#pragma unroll
                for (int i = 0; i < RR; ++i) {
                    const float2 t = *reinterpret_cast<const float2*>(rg + (d * RR + i) * BN + k);
                    w[i] = F2{t.x, t.y};
                }
                WT::ft(w, o);
#pragma unroll
                for (int x = 0; x < ALPHA; ++x)
                    *reinterpret_cast<float2*>(Gt + (x * BD + d) * BN + k) = make_float2(o[x].x, o[x].y);
            }
            const float* rx = rawX + buf * BD * ALPHA * BM;
            for (int p = tid; p < BD * (BM / 2); p += NT) {
                const int d = p / (BM / 2), c = 2 * (p % (BM / 2));
                F2 xv[ALPHA], o[ALPHA];
#pragma unroll
                for (int t = 0; t < ALPHA; ++t) {
                    const float2 q = *reinterpret_cast<const float2*>(rx + (d * ALPHA + t) * BM + c);
                    xv[t] = F2{q.x, q.y};
                }
                WT::it(xv, o);
#pragma unroll
                for (int x = 0; x < ALPHA; ++x)
                    *reinterpret_cast<float2*>(Xt + (x * BD + d) * BM + c) = make_float2(o[x].x, o[x].y);
            }
        }
        __syncthreads();
        // ---- alpha-batched GEMM: v[xi] += Gt[xi]^T Xt[xi]
        {
            const float* ga = Gt + xi * BD * BN;
            const float* xb = Xt + xi * BD * BM;
#pragma unroll
            for (int d = 0; d < BD; ++d) {
                float a[L::TM];
                uint64_t b2[L::TN / 2];
#pragma unroll
                for (int gm = 0; gm < L::GM; ++gm) {
                    const float4 t = *reinterpret_cast<const float4*>(ga + d * BN + (gm * L::TPK + tk) * 4);
                    a[gm * 4 + 0] = t.x; a[gm * 4 + 1] = t.y; a[gm * 4 + 2] = t.z; a[gm * 4 + 3] = t.w;
                }
#pragma unroll
                for (int gn = 0; gn < L::GN; ++gn) {
                    const float4 t = *reinterpret_cast<const float4*>(xb + d * BM + (gn * L::TPC + tc) * 4);
                    b2[gn * 2 + 0] = pk2(t.x, t.y);
                    b2[gn * 2 + 1] = pk2(t.z, t.w);
                }
#pragma unroll
                for (int i = 0; i < L::TM; ++i) {
                    const uint64_t aa = pk2(a[i], a[i]);
#pragma unroll
                    for (int j = 0; j < L::TN / 2; ++j) v2[i][j] = ffma2(aa, b2[j], v2[i][j]);
                }
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
                const float2 lo = up2(v2[gm * 4 + e][gn * 2 + 0]), hi = up2(v2[gm * 4 + e][gn * 2 + 1]);
                float4 t;
                t.x = lo.x; t.y = lo.y; t.z = hi.x; t.w = hi.y;
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
            float* o = Out + ((long long)j_off * BN + gm * KR + kl) * out_ld<BM>() + c;
#pragma unroll
            for (int j = 0; j < NN; ++j) {
                float* dst = o + (long long)j * BN * out_ld<BM>();
                *dst = accumulate ? *dst + y[j] : y[j];
            }
        }
        __syncthreads();
    }
}

// Writes the staged output tile [n0][B_N][B_M] to the bucket.  With a cluster
// split, rank r first waits for every rank's partial tile, sums the rows
// [r*rows/cs, (r+1)*rows/cs) over ranks 0..cs-1 in order through distributed
// shared memory (deterministic), and writes them.
template <int N0, int BN, int BM>
__device__ __forceinline__ void write_out(const Geometry& g, float* __restrict__ bucket, const CtaCoord& cc,
                                          int fw0, int rank, const float* Out) {
    const int k_base = cc.kb * BN, c_base = cc.cb * BM;
    constexpr int C4 = BM / 4;
    constexpr int ROWS = N0 * BN;
    int r_lo = 0, r_hi = ROWS;
    if (g.csplit > 1) {
        asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
        r_lo = ROWS * rank / g.csplit;
        r_hi = ROWS * (rank + 1) / g.csplit;
    }
    const uint32_t out_s = static_cast<uint32_t>(__cvta_generic_to_shared(Out));
    for (int p = r_lo * C4 + threadIdx.x; p < r_hi * C4; p += NT) {
        const int row = p / C4, c4 = p % C4;
        const int j = row / BN, kl = row % BN;
        const int kg = k_base + kl, cg = c_base + c4 * 4;
        const uint32_t off = (uint32_t)(((row) * out_ld<BM>() + c4 * 4) * 4);
        float4 acc;
        if (g.csplit > 1) {
            acc = make_float4(0.f, 0.f, 0.f, 0.f);
            for (int q = 0; q < g.csplit; ++q) {
                uint32_t remote;
                asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(out_s + off), "r"(q));
                float4 v;
                asm volatile("ld.shared::cluster.v4.f32 {%0, %1, %2, %3}, [%4];"
                             : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(remote) : "memory");
                acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
            }
        } else {
            acc = *reinterpret_cast<const float4*>(Out + row * out_ld<BM>() + c4 * 4);
        }
        if (kg < g.K && cg < g.C)
            *reinterpret_cast<float4*>(bucket + (((long long)kg * g.R + cc.fh) * g.S + fw0 + j) * g.C + cg) = acc;
    }
    if (g.csplit > 1)   // peers may still be reading this CTA's tile
        asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// The fused launch: every CTA runs the Omega_a0 phase over its segment, and
// CTAs of a band's last column segment also run the residual Omega_a1 phase.
template <int A0, int N0, int R0, int A1, int N1, int R1, int BN, int BM>
constexpr size_t pipe_floats() {
    size_t a = PhaseSmem<A0, R0, BN, BM>::floats;
    size_t b = A1 ? PhaseSmem<(A1 ? A1 : A0), (R1 ? R1 : R0), BN, BM>::floats : 0;
    return a > b ? a : b;
}
template <int A0, int N0, int R0, int A1, int N1, int R1, int BN, int BM>
constexpr size_t smem_bytes() {
    return 4 * (pipe_floats<A0, N0, R0, A1, N1, R1, BN, BM>() + (size_t)N0 * BN * out_ld<BM>());
}

// The fused launch: every CTA runs the Omega_a0 phase over its segment (its
// cluster rank's share of the depth), CTAs of a band's last column segment
// also run the residual Omega_a1 phase into the same staged tile, then the
// tile (summed over the cluster) is written to the segment's bucket.
template <int A0, int N0, int R0, int A1, int N1, int R1, int BN, int BM>
__global__ void __launch_bounds__(NT, 1)
bfc_f32_kernel(const Geometry g, const float* __restrict__ X, const float* __restrict__ dY,
               float* __restrict__ dW, float* __restrict__ ws) {
    extern __shared__ __align__(16) float smem[];
    float* Out = smem + pipe_floats<A0, N0, R0, A1, N1, R1, BN, BM>();
    const int rank = (int)(blockIdx.x % g.csplit);
    const CtaCoord cc = decode_cta(g, blockIdx.x / g.csplit);
    const int seg = cc.band * g.seg_cols + cc.col;
    float* bucket = seg == 0 ? dW : ws + (long long)(seg - 1) * g.dw_elems;
    int hs, he;
    band_rows(g, cc.band, cc.fh, &hs, &he);
    int w_first, units;
    seg_units(g, cc.col, &w_first, &units);
    const int fw0 = cc.ft * N0;
    run_phase<A0, N0, R0, BN, BM>(g, X, dY, Out, cc, hs, he, w_first, units, fw0, 0, false, rank, smem);
    if constexpr (A1 != 0) {
        if (has_residual(g, cc.col)) {
            static_assert(N0 % N1 == 0, "residual n1 must divide n0");
#pragma unroll 1
            for (int j = 0; j < N0 / N1; ++j)
                run_phase<A1, N1, R1, BN, BM>(g, X, dY, Out, cc, hs, he, g.res_col0, g.k1, fw0 + j * N1, j * N1,
                                              true, rank, smem);
        }
    }
    __syncthreads();
    write_out<N0, BN, BM>(g, bucket, cc, fw0, rank, Out);
}

}  // namespace f32k
}  // namespace winrs
