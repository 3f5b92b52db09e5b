// FP32 CUDA-core fused WinRS BFC kernel for sm_100a.
//
// One CTA computes one B_N x B_M x n0 tile of one dW bucket (§5.1
// P@28778-29449, Algorithm 3): it walks its segment's depth d = (row h,
// unit u, image n) in chunks of BD entries (the paper steps n by 8, line 25).
// Warp-specialised (B200): warpgroup 0 (128 threads, few registers) loads and
// transforms chunks into a 2-stage transformed-tile ring while warpgroups 1-2
// (256 threads, setmaxnreg-raised register budget) run the batched GEMM, so
// the FMA pipe is not idle during loads / transforms (the paper overlaps them
// by software pipelining inside every warp, P@36703).  Per chunk
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
//
// TI (input element type): float, or __half / __nv_bfloat16 for the FP16 /
// BF16 plans whose kernel pair has no tensor-core kernel (the alpha = 16
// widths, R26): 16-bit inputs are staged as they are and widened to
// FP32 when the transforms read them; transforms, EWM and OT stay FP32.
#pragma once
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include "dsmem.cuh"
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

constexpr int NT = 256;   // GEMM threads (warpgroups 1-2)
constexpr int NP = 128;   // loader / transformer threads (warpgroup 0)
constexpr int NTOT = NT + NP;
// Depth entries per chunk (BD) and cp.async raw ring stages (SR) are chosen
// per instantiation (pipe_cfg below) so that the largest alpha = 16 tiles fit
// the 227 KB of shared memory; the paper steps n by 8 (Algorithm 3 line 25).
constexpr int S_T = 2;    // transformed-tile ring stages
constexpr int REG_P = 88, REG_G = 208;   // setmaxnreg budgets: 128*88 + 256*208 <= 64K

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void cp_async16(void* dst, const void* src, bool valid) {
    const int sz = valid ? 16 : 0;   // src-size 0 => the 16 bytes are zero-filled
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n"
                 :: "r"(smem_u32(dst)), "l"(src), "r"(sz) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
// Two consecutive raw elements widened to FP32.
__device__ __forceinline__ float2 ld2f(const float* p) { return *reinterpret_cast<const float2*>(p); }
__device__ __forceinline__ float2 ld2f(const __half* p) { return __half22float2(*reinterpret_cast<const __half2*>(p)); }
__device__ __forceinline__ float2 ld2f(const __nv_bfloat16* p) {
    return __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(p));
}
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
template <int ALPHA, int RR, int BN, int BM, int SR, int BD>
struct PhaseSmem {
    static constexpr int rawG = SR * BD * RR * BN;
    static constexpr int rawX = SR * BD * ALPHA * BM;
    static constexpr int Gt1 = ALPHA * BD * BN;       // one stage
    static constexpr int Xt1 = ALPHA * BD * BM;
    static constexpr int Gt = S_T * Gt1;
    static constexpr int Xt = S_T * Xt1;
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
// mbarrier ring of transformed tiles, shared by both roles across phases.
struct TRing {
    uint64_t t_full[S_T], t_empty[S_T];
};

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n.reg .pred P;\nWAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1, %2;\n"
        "@!P bra WAIT_%=;\n}\n" :: "r"(smem_u32(bar)), "r"(parity), "r"(1000000) : "memory");
}

// Per-job chunk geometry shared by both roles.
struct PhaseCtx {
    int hs, he, w_first, units, fw0, j_off, rank;
    bool accumulate;
};

// This cluster rank's depth range [d_lo, d_hi) (split in units of g.chunk = 8
// entries, the emulator's granularity) and its number of BD-entry chunks.
template <int BD>
__device__ __forceinline__ void phase_chunks(const Geometry& g, const PhaseCtx& P, long long* d_lo, long long* d_hi,
                                             int* nchunks) {
    const int rows = P.he - P.hs;
    const long long depth = (long long)(rows > 0 ? rows : 0) * P.units * g.N;
    int lo, hi;
    split_chunks((int)((depth + g.chunk - 1) / g.chunk), P.rank, g.csplit, &lo, &hi);
    *d_lo = (long long)lo * g.chunk;
    *d_hi = depth < (long long)hi * g.chunk ? depth : (long long)hi * g.chunk;
    *nchunks = *d_hi > *d_lo ? (int)((*d_hi - *d_lo + BD - 1) / BD) : 0;
}

// ================= warpgroup 0: cp.async loads + FP32 transforms of one job =================
template <int ALPHA, int NN, int RR, int BN, int BM, int S_RAW, int BD, typename TI = float>
__device__ __forceinline__ void producer_phase(const Geometry& g, const TI* __restrict__ X,
                                               const TI* __restrict__ dY, const CtaCoord& cc, const PhaseCtx& P,
                                               float* smem, TRing& ring, int& tcount) {
    using WT = Wino<ALPHA, NN, RR>;
    using SM = PhaseSmem<ALPHA, RR, BN, BM, S_RAW, BD>;
    constexpr int VE = 16 / (int)sizeof(TI);  // elements per 16-byte copy
    TI* rawG = reinterpret_cast<TI*>(smem);   // [S_RAW][BD][RR][BN] (16-bit inputs use half the region)
    TI* rawX = rawG + SM::rawG;               // [S_RAW][BD][ALPHA][BM]
    float* Gt = smem + SM::rawG + SM::rawX;   // [S_T][ALPHA][BD][BN]
    float* Xt = Gt + SM::Gt;                  // [S_T][ALPHA][BD][BM]
    const int k_base = cc.kb * BN, c_base = cc.cb * BM;
    long long d_lo, d_hi;
    int nchunks;
    phase_chunks<BD>(g, P, &d_lo, &d_hi, &nchunks);
    const int ptid = threadIdx.x;
    constexpr int TPD = NP / BD;   // threads per depth entry of a chunk
    const int ld_d = ptid / TPD, ld_l = ptid % TPD;
    // This thread's depth entry d = (h, u, n) (n fastest), walked incrementally:
    // issue() is called for chunks 0, 1, 2, ... in order, each advancing d by BD.
    long long d = d_lo + ld_d;
    int n = 0, u = 0, h = P.hs;
    {
        const int d32 = (int)d;   // depth < 2^31 (planner: rows*units*N)
        if (d < d_hi) {
            n = d32 % g.N;
            const int t = d32 / g.N;
            u = t % P.units;
            h = P.hs + t / P.units;
        }
    }
    auto issue = [&](int buf) {
        const bool dv = d < d_hi;
        const int w0 = P.w_first + u * RR;
        const TI* gsrc = dY + (((long long)n * g.Ho + h) * g.Wo + w0) * g.ldy + k_base;
        // filter row fh = (depth tap fh / Rh, height tap fh % Rh); for an N-D plan
        // image n = (batch n / Do, dY depth slice n % Do) reads X slice
        // (n % Do) + t - pad, zero outside [0, D) (PAPER.md P@17805)
        const int xrow = h + cc.fh % g.Rh - g.pad;
        const int xcol0 = w0 + P.fw0 - g.pad;
        long long ximg = n;
        bool dok = true;
        if (g.T > 1 || g.D > 1) {
            const int dd = n % g.Do + cc.fh / g.Rh - g.pad;
            dok = dd >= 0 && dd < g.D;
            ximg = (long long)(n / g.Do) * g.D + dd;
        }
        const TI* xsrc = X + ((ximg * g.H + xrow) * g.W) * g.C + c_base;
        TI* gdst = rawG + ((buf * BD + ld_d) * RR) * BN;
        TI* xdst = rawX + ((buf * BD + ld_d) * ALPHA) * BM;
        constexpr int GV = RR * (BN / VE);
#pragma unroll
        for (int it = 0; it < (GV + TPD - 1) / TPD; ++it) {
            const int q = ld_l + it * TPD;
            if (GV % TPD == 0 || q < GV) {
                const int i = q / (BN / VE), v4 = q % (BN / VE);
                const bool ok = dv && (w0 + i < g.Wo) && (k_base + v4 * VE < g.K);
                cp_async16(gdst + i * BN + v4 * VE,
                           ok ? (const void*)(gsrc + (long long)i * g.ldy + v4 * VE) : (const void*)dY, ok);
            }
        }
        constexpr int XV = ALPHA * (BM / VE);
#pragma unroll
        for (int it = 0; it < (XV + TPD - 1) / TPD; ++it) {
            const int q = ld_l + it * TPD;
            if (XV % TPD == 0 || q < XV) {
                const int t = q / (BM / VE), v4 = q % (BM / VE);
                const int col = xcol0 + t;
                const bool ok = dv && dok && col >= 0 && col < g.W && c_base + v4 * VE < g.C;
                cp_async16(xdst + t * BM + v4 * VE,
                           ok ? (const void*)(xsrc + (long long)col * g.C + v4 * VE) : (const void*)X, ok);
            }
        }
        // advance to this thread's entry of the next chunk
        d += BD;
        n += BD;
        while (n >= g.N) {
            n -= g.N;
            if (++u == P.units) { u = 0; ++h; }
        }
    };
    for (int c = 0; c < S_RAW - 1; ++c) {
        if (c < nchunks) issue(c);
        cp_async_commit();
    }
    for (int ch = 0; ch < nchunks; ++ch) {
        // the slot of chunk ch+S_RAW-1 was read by every thread's transform of ch-1
        __syncwarp();   // converged warp at the named barrier
        asm volatile("barrier.sync 1, %0;" :: "n"(NP) : "memory");
        if (ch + S_RAW - 1 < nchunks) issue((ch + S_RAW - 1) % S_RAW);
        cp_async_commit();
        cp_async_wait<S_RAW - 1>();                                   // this thread's copies of chunk ch
        __syncwarp();   // converged warp at the named barrier
        asm volatile("barrier.sync 1, %0;" :: "n"(NP) : "memory");       // everyone's copies of chunk ch
        const int ts = tcount % S_T;
        mbar_wait(&ring.t_empty[ts], ((tcount / S_T) & 1) ^ 1);
        const int buf = ch % S_RAW;
        float* Gs = Gt + ts * SM::Gt1;
        float* Xs = Xt + ts * SM::Xt1;
        const TI* rg = rawG + buf * BD * RR * BN;
        for (int p = ptid; p < BD * (BN / 2); p += NP) {
            const int d = p / (BN / 2), k = 2 * (p % (BN / 2));
            F2 w[RR], o[ALPHA];
#pragma unroll
            for (int i = 0; i < RR; ++i) {
                const float2 t = ld2f(rg + (d * RR + i) * BN + k);
                w[i] = F2{t.x, t.y};
            }
            WT::ft(w, o);
#pragma unroll
            for (int x = 0; x < ALPHA; ++x)
                *reinterpret_cast<float2*>(Gs + (x * BD + d) * BN + k) = make_float2(o[x].x, o[x].y);
        }
        const TI* rx = rawX + buf * BD * ALPHA * BM;
        for (int p = ptid; p < BD * (BM / 2); p += NP) {
            const int d = p / (BM / 2), c = 2 * (p % (BM / 2));
            F2 xv[ALPHA], o[ALPHA];
#pragma unroll
            for (int t = 0; t < ALPHA; ++t) {
                const float2 q = ld2f(rx + (d * ALPHA + t) * BM + c);
                xv[t] = F2{q.x, q.y};
            }
            WT::it(xv, o);
#pragma unroll
            for (int x = 0; x < ALPHA; ++x)
                *reinterpret_cast<float2*>(Xs + (x * BD + d) * BM + c) = make_float2(o[x].x, o[x].y);
        }
        __syncwarp();
        if ((ptid & 31) == 0) mbar_arrive(&ring.t_full[ts]);
        ++tcount;
    }
    cp_async_wait<0>();
}

// ================= warpgroups 1-2: alpha-batched GEMM + OT of one job =================
template <int ALPHA, int NN, int RR, int BN, int BM, int S_RAW, int BD>
__device__ __forceinline__ void gemm_phase(const Geometry& g, float* __restrict__ Out, const CtaCoord& cc,
                                           const PhaseCtx& P, float* smem, TRing& ring, int& tcount) {
    using WT = Wino<ALPHA, NN, RR>;
    using L = GemmLayout<ALPHA, BN, BM>;
    using SM = PhaseSmem<ALPHA, RR, BN, BM, S_RAW, BD>;
    float* Gt = smem + SM::rawG + SM::rawX;   // [S_T][ALPHA][BD][BN]
    float* Xt = Gt + SM::Gt;                  // [S_T][ALPHA][BD][BM]
    long long d_lo, d_hi;
    int nchunks;
    phase_chunks<BD>(g, P, &d_lo, &d_hi, &nchunks);
    const int gtid = threadIdx.x - NP;
    const int xi = gtid / L::TPX;
    const int tl = gtid % L::TPX;
    const int tk = tl / L::TPC, tc = tl % L::TPC;
    uint64_t v2[L::TM][L::TN / 2];   // accumulators: pairs along c, FFMA2
#pragma unroll
    for (int i = 0; i < L::TM; ++i)
#pragma unroll
        for (int j = 0; j < L::TN / 2; ++j) v2[i][j] = 0ull;
    for (int ch = 0; ch < nchunks; ++ch) {
        const int ts = tcount % S_T;
        mbar_wait(&ring.t_full[ts], (tcount / S_T) & 1);
        const float* ga = Gt + ts * SM::Gt1 + xi * BD * BN;
        const float* xb = Xt + ts * SM::Xt1 + xi * BD * BM;
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
        __syncwarp();
        if ((gtid & 31) == 0) mbar_arrive(&ring.t_empty[ts]);
        ++tcount;
    }
    // All of this job's ring writes are done (the producer only fills chunks of
    // this job, each consumed above), so the ring memory can hold the OT staging.
    __syncwarp();   // converged warp at the named barrier
    asm volatile("barrier.sync 2, %0;" :: "n"(NT) : "memory");

    // ---- OT in rounds (one 4-wide k-group of every thread per round)
    float* As = smem;   // [ALPHA][TPK*4][BM]
    constexpr int KR = L::TPK * 4;   // k rows per round
#pragma unroll
    for (int gm = 0; gm < L::GM; ++gm) {
#pragma unroll
        for (int e = 0; e < 4; ++e)
#pragma unroll
            for (int gn = 0; gn < L::GN; ++gn) {
                const float2 lo = up2(v2[gm * 4 + e][gn * 2 + 0]), hi = up2(v2[gm * 4 + e][gn * 2 + 1]);
                float4 t;
                t.x = lo.x; t.y = lo.y; t.z = hi.x; t.w = hi.y;
                *reinterpret_cast<float4*>(As + (xi * KR + tk * 4 + e) * BM + (gn * L::TPC + tc) * 4) = t;
            }
        __syncwarp();   // converged warp at the named barrier
        asm volatile("barrier.sync 2, %0;" :: "n"(NT) : "memory");
        for (int p = gtid; p < KR * BM; p += NT) {
            const int kl = p / BM, c = p % BM;
            float vv[ALPHA], y[NN];
#pragma unroll
            for (int x = 0; x < ALPHA; ++x) vv[x] = As[(x * KR + kl) * BM + c];
            WT::ot(vv, y);
            float* o = Out + ((long long)P.j_off * BN + gm * KR + kl) * out_ld<BM>() + c;
#pragma unroll
            for (int j = 0; j < NN; ++j) {
                float* dst = o + (long long)j * BN * out_ld<BM>();
                *dst = P.accumulate ? *dst + y[j] : y[j];
            }
        }
        __syncwarp();   // converged warp at the named barrier
        asm volatile("barrier.sync 2, %0;" :: "n"(NT) : "memory");
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
    for (int p = r_lo * C4 + threadIdx.x; p < r_hi * C4; p += NTOT) {
        const int row = p / C4, c4 = p % C4;
        const int j = row / BN, kl = row % BN;
        const int kg = k_base + kl, cg = c_base + c4 * 4;
        const uint32_t off = (uint32_t)(((row) * out_ld<BM>() + c4 * 4) * 4);
        float4 acc;
        if (g.csplit > 1) {
            acc = dsmem_sum4(out_s + off, g.csplit);
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
template <int A0, int N0, int R0, int A1, int N1, int R1, int BN, int BM, int SR, int BD>
constexpr size_t pipe_floats_cfg() {
    size_t a = PhaseSmem<A0, R0, BN, BM, SR, BD>::floats;
    size_t b = A1 ? PhaseSmem<(A1 ? A1 : A0), (R1 ? R1 : R0), BN, BM, SR, BD>::floats : 0;
    return a > b ? a : b;
}
template <int A0, int N0, int R0, int A1, int N1, int R1, int BN, int BM, int SR, int BD>
constexpr size_t smem_bytes_cfg() {
    return 4 * (pipe_floats_cfg<A0, N0, R0, A1, N1, R1, BN, BM, SR, BD>() + (size_t)N0 * BN * out_ld<BM>()) + 64;
}
constexpr size_t SMEM_LIMIT = 227 * 1024;
// Pipeline configuration: 0 = (SR 3, BD 8), 1 = (2, 8), 2 = (3, 4), 3 = (2, 4),
// the first whose footprint fits.
template <int A0, int N0, int R0, int A1, int N1, int R1, int BN, int BM>
constexpr int pipe_cfg() {
    return smem_bytes_cfg<A0, N0, R0, A1, N1, R1, BN, BM, 3, 8>() <= SMEM_LIMIT   ? 0
           : smem_bytes_cfg<A0, N0, R0, A1, N1, R1, BN, BM, 2, 8>() <= SMEM_LIMIT ? 1
           : smem_bytes_cfg<A0, N0, R0, A1, N1, R1, BN, BM, 3, 4>() <= SMEM_LIMIT ? 2
                                                                                  : 3;
}
template <int A0, int N0, int R0, int A1, int N1, int R1, int BN, int BM>
struct Cfg {
    static constexpr int id = pipe_cfg<A0, N0, R0, A1, N1, R1, BN, BM>();
    static constexpr int SR = (id == 0 || id == 2) ? 3 : 2;
    static constexpr int BD = id < 2 ? 8 : 4;
};
template <int A0, int N0, int R0, int A1, int N1, int R1, int BN, int BM>
constexpr size_t pipe_floats() {
    using C = Cfg<A0, N0, R0, A1, N1, R1, BN, BM>;
    return pipe_floats_cfg<A0, N0, R0, A1, N1, R1, BN, BM, C::SR, C::BD>();
}
template <int A0, int N0, int R0, int A1, int N1, int R1, int BN, int BM>
constexpr size_t smem_bytes() {
    using C = Cfg<A0, N0, R0, A1, N1, R1, BN, BM>;
    static_assert(smem_bytes_cfg<A0, N0, R0, A1, N1, R1, BN, BM, C::SR, C::BD>() <= SMEM_LIMIT,
                  "tile does not fit shared memory");
    return smem_bytes_cfg<A0, N0, R0, A1, N1, R1, BN, BM, C::SR, C::BD>();
}

// The fused launch: every CTA runs the Omega_a0 phase over its segment (its
// cluster rank's share of the depth), CTAs of a band's last column segment
// also run the residual Omega_a1 phase into the same staged tile, then the
// tile (summed over the cluster) is written to the segment's bucket.
template <int A0, int N0, int R0, int A1, int N1, int R1, int BN, int BM, typename TI = float>
__global__ void __launch_bounds__(NTOT, 1)
bfc_f32_kernel(const Geometry g, const TI* __restrict__ X, const TI* __restrict__ dY,
               float* __restrict__ dW, float* __restrict__ ws) {
    extern __shared__ __align__(16) float smem[];
    float* Out = smem + pipe_floats<A0, N0, R0, A1, N1, R1, BN, BM>();
    TRing& ring = *reinterpret_cast<TRing*>(Out + (size_t)N0 * BN * out_ld<BM>());
    if (threadIdx.x == 0) {
        for (int s = 0; s < S_T; ++s) {
            mbar_init(&ring.t_full[s], NP / 32);
            mbar_init(&ring.t_empty[s], NT / 32);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    using C = Cfg<A0, N0, R0, A1, N1, R1, BN, BM>;
    int tcount = 0;   // transformed-ring position (both roles advance it identically, per thread)
    const int rank = (int)(blockIdx.x % g.csplit);
    const CtaCoord cc = decode_cta(g, blockIdx.x / g.csplit);
    const int seg = cc.band * g.seg_cols + cc.col;
    float* bucket = seg == 0 ? dW : ws + (long long)(seg - 1) * g.dw_elems;
    int hs, he;
    band_rows(g, cc.band, cc.fh, &hs, &he);
    int w_first, units;
    seg_units(g, cc.col, &w_first, &units);
    const int fw0 = cc.ft * N0;
    const PhaseCtx P0{hs, he, w_first, units, fw0, 0, rank, false};
    const bool resid = A1 != 0 && has_residual(g, cc.col);
    static_assert(A1 == 0 || N0 % N1 == 0, "residual n1 must divide n0");
    constexpr int NJ1 = A1 ? N0 / (N1 ? N1 : 1) : 0;
    if (threadIdx.x < NP) {
        // the transformer warpgroup hands registers to the GEMM warpgroups
        asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" :: "n"(REG_P));
        producer_phase<A0, N0, R0, BN, BM, C::SR, C::BD, TI>(g, X, dY, cc, P0, smem, ring, tcount);
        __syncwarp();   // converged warp at the named barrier
        asm volatile("barrier.sync 3, %0;" :: "n"(NTOT) : "memory");   // job boundary (ring reused by the OT)
        if constexpr (A1 != 0) {
            if (resid) {
#pragma unroll 1
                for (int j = 0; j < NJ1; ++j) {
                    const PhaseCtx P1{hs, he, g.res_col0, g.k1, fw0 + j * N1, j * N1, rank, true};
                    producer_phase<(A1 ? A1 : A0), (N1 ? N1 : N0), (R1 ? R1 : R0), BN, BM, C::SR, C::BD, TI>(
                        g, X, dY, cc, P1, smem, ring, tcount);
                    __syncwarp();   // converged warp at the named barrier
                    asm volatile("barrier.sync 3, %0;" :: "n"(NTOT) : "memory");
                }
            }
        }
    } else {
        asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" :: "n"(REG_G));
        gemm_phase<A0, N0, R0, BN, BM, C::SR, C::BD>(g, Out, cc, P0, smem, ring, tcount);
        __syncwarp();   // converged warp at the named barrier
        asm volatile("barrier.sync 3, %0;" :: "n"(NTOT) : "memory");
        if constexpr (A1 != 0) {
            if (resid) {
#pragma unroll 1
                for (int j = 0; j < NJ1; ++j) {
                    const PhaseCtx P1{hs, he, g.res_col0, g.k1, fw0 + j * N1, j * N1, rank, true};
                    gemm_phase<(A1 ? A1 : A0), (N1 ? N1 : N0), (R1 ? R1 : R0), BN, BM, C::SR, C::BD>(g, Out, cc, P1, smem, ring,
                                                                                     tcount);
                    __syncwarp();   // converged warp at the named barrier
                    asm volatile("barrier.sync 3, %0;" :: "n"(NTOT) : "memory");
                }
            }
        }
    }
    __syncthreads();
    write_out<N0, BN, BM>(g, bucket, cc, fw0, rank, Out);
}

}  // namespace f32k
}  // namespace winrs
