// Third-generation fused BFC kernel: FP32 inputs on the tensor cores
// (B200 design, reading R25).
//
// The Omega_4(3,2) decomposition of the tc2 kernels (bfc_tc2.cuh: the same
// segments, filter-row groups, cluster depth split and epilogue) with FP32
// operands.  The EWM is a dense contraction, so it runs on tcgen05
// (kind::tf32) instead of the CUDA cores, with FP32-class accuracy from the
// 3xTF32 split: every transformed operand x = hi + lo, hi = x with the 13 low
// mantissa bits cleared (what the tensor core reads from the FP32 word), lo =
// x - hi exactly; v += Xh.Wh + Xh.Wl + Xl.Wh drops only the Xl.Wl term
// (~2^-22 relative).  Probed on B200 (tools/microbench/tf32_probe.cu): 1xTF32
// 5.5e-4, 3xTF32 5.0e-7 relative error on an 8-term dot product; kind::tf32
// takes K-major operands only.
//
// One stage = 8 depth entries (KT, the tf32 UMMA K): TMA lands the raw FP32
// tiles without swizzle (X: [col 4][image 8][128 channel rows], dY: [col 2]
// [image 8][64 k]); the FT warps transform them (IT: x1+x2, x2-x1, x0-x2,
// x3-x1; FT: w0+w1, w0-w1, w0, w1, in FP32) and store hi / lo operands
// K-major (core matrices of 8 rows x 4 depth entries, 16 B rows) -- the
// transpose the tf32 MMA needs happens in the same pass.  12 MMAs per stage
// (4 xi x 3 products, M = 128, N = 64, K = 8) accumulate in TMEM; the
// epilogue (OT, bucket or cluster staging) is tc2's.
//
// Warp roles (352 threads, one CTA per SM): warps 0 and 10 TMA producers
// (even / odd stages), warp 1 TMEM allocator + MMA issuer, warps 2-9 two
// groups of four FT warps taking alternate stages (warp q of a group: A rows
// 32q..32q+31 and a quarter of the dY items), then the epilogue.
#pragma once
#include "bfc_tc2.cuh"

namespace winrs {
namespace tc3 {

using tc2::Args;
using tc2::Bars;
using tc2::ImgCoord;
using tc2::ImgTracker;
using tc2::MROWS;
using tc2::NSOUT;
using tc2::NTHREADS;
using tc2::PW2;

constexpr int KT = 8;      // depth entries per stage = kind::tf32 UMMA K

// NK: k columns per tile (UMMA N): 64, or 128 (the MMAs' A reads -- A_hi is
// read twice per xi -- amortised over twice the columns; 2 operand stages).
template <int F, int NK>
struct Lay3 {
    static constexpr int BC = MROWS / F;                       // channels per fh slot
    // Two rings (the raw TMA tiles are 20 KB, the hi / lo operands 48 KB, so
    // separate rings give the TMA 4 stages of latency hiding next to 3
    // operand stages instead of 3 combined ones):
    //   raw  [SR]: X [fh slot][col 4][img 8][BC] fp32 (16 KB) + dY [col 2][img 8][64 k] (4 KB)
    //   op   [SO]: A [hi, lo][xi 4] K-major slabs 128 x 8 (32 KB) + B [hi, lo][xi 4] 64 x 8 (16 KB)
    static constexpr int XSLOT = 4 * KT * BC * 4;              // raw X of one fh slot
    static constexpr int OFF_X = 0;
    static constexpr int OFF_Y = 4 * KT * MROWS * 4;           // 16 KB
    static constexpr int RAW = OFF_Y + 2 * KT * NK * 4;        // 20 KB
    static constexpr int ASLAB = MROWS * KT * 4;               // 4 KB
    static constexpr int BSLAB = NK * KT * 4;                  // 2 KB
    static constexpr int OFF_A = 0;                            // within an operand stage
    static constexpr int OFF_B = 2 * 4 * ASLAB;                // 32 KB
    static constexpr int OP = OFF_B + 2 * 4 * BSLAB;           // 48 KB
    static constexpr int LIMIT = 227 * 1024 - 1024 - 512;
    static constexpr int SO = NK == 64 ? 3 : 2;
    static constexpr int SR = (LIMIT - SO * OP) / RAW > 6 ? 6 : (LIMIT - SO * OP) / RAW;   // 4
    static constexpr int OP_OFF = SR * RAW;
    static constexpr int RING = OP_OFF + SO * OP;
    static constexpr int OUT = NSOUT * NK * MROWS * 4;         // cluster staging [s][k][m] fp32 (96 KB)
    static constexpr int BAR_OFF = RING > OUT ? RING : OUT;
    static constexpr int BYTES = BAR_OFF + 512 + 1024;
    static constexpr int TX_BYTES = RAW;                       // TMA bytes per stage
    static constexpr int TMEM_COLS = 4 * NK;                   // 256
    static_assert(SR >= 3, "raw ring too shallow");
    static_assert(RAW % 1024 == 0 && OP % 1024 == 0, "stage alignment");
};

struct Bars3 {
    uint64_t full[8];      // raw stage landed (TMA)
    uint64_t rempty[8];    // raw stage consumed (4 FT warps)
    uint64_t opfull[8];    // operand stage written (4 FT warps)
    uint64_t opempty[8];   // operand stage read by the MMAs (commit)
    uint64_t accfull;
    uint32_t tmem_base;
};

// K-major, no swizzle: element (row, k) of a slab at (row/8)*256 + (k/4)*128
// + (row%8)*16 + (k%4)*4; LBO = 128 (next 4 depth entries), SBO = 256 (next 8 rows).
__device__ __forceinline__ uint64_t desc_k(uint32_t addr) {
    return (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)(128 >> 4) << 16) | ((uint64_t)(256 >> 4) << 32) |
           (1ull << 46);
}
// kind::tf32 instruction descriptor: D f32, A/B tf32 (2), both K-major, N = NK, M = 128.
template <int NK>
__host__ __device__ constexpr uint32_t idesc_tf32() {
    return (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(NK >> 3) << 17) | ((uint32_t)(MROWS >> 4) << 24);
}
template <int NK>
__device__ __forceinline__ void umma_tf32(uint32_t d, uint64_t a, uint64_t b, uint32_t acc) {
    asm volatile(
        "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n"
        :: "r"(d), "l"(a), "l"(b), "r"(idesc_tf32<NK>()), "r"(acc));
}
// lo part of the 3xTF32 split (hi = the word itself: the tensor core reads its top 19 bits)
__device__ __forceinline__ float tf32_lo(float x) { return x - __uint_as_float(__float_as_uint(x) & 0xFFFFE000u); }
__device__ __forceinline__ float lds32(uint32_t a) {
    float v;
    asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ void sts4f(uint32_t a, float x, float y, float z, float w) {
    asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" :: "r"(a), "f"(x), "f"(y), "f"(z), "f"(w) : "memory");
}
__device__ __forceinline__ uint32_t koff(int row, int k4) { return (uint32_t)((row >> 3) * 256 + k4 * 128 + (row & 7) * 16); }

template <int F, int NK>
__global__ void __launch_bounds__(NTHREADS, 1)
bfc_tc3_kernel(const __grid_constant__ Args args, const __grid_constant__ CUtensorMap tmX,
               const __grid_constant__ CUtensorMap tmY) {
    using namespace tc2;
    using L = Lay3<F, NK>;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw_s = su(smem_raw);
    uint8_t* smem = smem_raw + (((raw_s + 1023u) & ~1023u) - raw_s);
    const uint32_t sbase = su(smem);
    Bars3* bars = reinterpret_cast<Bars3*>(smem + L::BAR_OFF);
    const Geometry& g = args.g;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

    const int rank = (int)(blockIdx.x % g.csplit);
    const CtaCoord cc = decode_cta(g, blockIdx.x / g.csplit);
    const int fh_base = cc.fh;
    const int c_base = cc.cb * L::BC;
    const int k_base = cc.kb * NK;
    const int seg = cc.band * g.seg_cols + cc.col;
    float* bucket = seg == 0 ? args.dW : args.ws + (long long)(seg - 1) * g.dw_elems;
    int hs, he, w_first, units;
    group_rows(g, cc.band, cc.fh, &hs, &he);
    seg_units(g, cc.col, &w_first, &units);
    const long long depth = (long long)(he > hs ? he - hs : 0) * units * g.N;
    int c_lo, c_hi;
    split_chunks((int)((depth + KT - 1) / KT), rank, g.csplit, &c_lo, &c_hi);
    const bool empty_range = c_hi <= c_lo;
    const int fw0 = cc.ft * NSOUT;

    if (threadIdx.x == 0) {
        for (int s = 0; s < L::SR; ++s) {
            mbar_init(&bars->full[s], 1);
            mbar_init(&bars->rempty[s], 4);   // the four warps of an FT group
        }
        for (int s = 0; s < L::SO; ++s) {
            mbar_init(&bars->opfull[s], 4);
            mbar_init(&bars->opempty[s], 1);
        }
        mbar_init(&bars->accfull, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 0 && lane == 0) {
        asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(&tmX)) : "memory");
        asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(&tmY)) : "memory");
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                     :: "r"(su(&bars->tmem_base)), "r"((uint32_t)L::TMEM_COLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_before();
    __syncthreads();
    tc_after();
    if (threadIdx.x == 0) pdl_trigger();
    const uint32_t tmem = bars->tmem_base;

    if (warp == 0 || warp == PW2) {
        // ============================ TMA producers (even / odd stages) =======
        const int pp = warp == 0 ? 0 : 1;
        long long d = (long long)(c_lo + pp) * KT;
        int n = 0, h = hs, u = 0;
        if (d < depth) depth_nhu((int)d, g.N, units, hs, &n, &h, &u);
        ImgTracker itk;
        itk.init(g, n);
        int xdt[F], xdr[F];
#pragma unroll
        for (int f = 0; f < F; ++f) {
            const int fh = fh_base + f;
            xdt[f] = (g.T > 1 || g.D > 1) ? fh / g.Rh - g.pad : 0;
            xdr[f] = fh < g.R ? fh % g.Rh - g.pad : -(1 << 20);   // a slot past the last filter row: zero fill
        }
        int s = pp;
        uint32_t ph = 0;
        for (int ch = c_lo + pp; ch < c_hi; ch += 2) {
            mbar_wait(&bars->rempty[s], ph ^ 1);
            uint64_t* fb = &bars->full[s];
            const uint32_t st = sbase + (uint32_t)(s * L::RAW);
            const bool in = d < depth;
            const ImgCoord ic = itk.at(g, in);
            const int hh = in ? h : hs;
            const int w0 = w_first + (in ? u : 0) * 2;
            if (elect_one()) {
                mbar_expect_tx(fb, (uint32_t)L::TX_BYTES);
#pragma unroll
                for (int f = 0; f < F; ++f)   // X columns x0..x3 of fh slot f: box {BC, 8, 1, 1, 4}
                    tma5(st + L::OFF_X + f * L::XSLOT, &tmX, fb, c_base, ic.a + xdt[f], ic.b, hh + xdr[f],
                         w0 + fw0 - g.pad);
                tma5(st + L::OFF_Y, &tmY, fb, k_base, ic.a, ic.b, hh, w0);   // dY w0, w1: box {64, 8, 1, 1, 2}
            }
            __syncwarp();
            d += 2 * KT;
            n += 2 * KT;
            bool wrapped = false;
            while (n >= g.N) {
                n -= g.N;
                wrapped = true;
                if (++u == units) { u = 0; ++h; }
            }
            itk.advance(2 * KT, wrapped, n);
            s += 2;
            if (s >= L::SR) { s -= L::SR; ph ^= 1; }
        }
    } else if (warp == 1) {
        // ============================ MMA issuer ==============================
        int s = 0;
        uint32_t ph = 0;
        for (int ch = c_lo; ch < c_hi; ++ch) {
            mbar_wait(&bars->opfull[s], ph);
            tc_after();
            const uint32_t st = sbase + (uint32_t)(L::OP_OFF + s * L::OP);
            const uint32_t acc = ch > c_lo ? 1u : 0u;
            if (elect_one()) {
#pragma unroll
                for (int x = 0; x < 4; ++x) {
                    const uint64_t ah = desc_k(st + L::OFF_A + x * L::ASLAB);
                    const uint64_t al = desc_k(st + L::OFF_A + (4 + x) * L::ASLAB);
                    const uint64_t bh = desc_k(st + L::OFF_B + x * L::BSLAB);
                    const uint64_t bl = desc_k(st + L::OFF_B + (4 + x) * L::BSLAB);
                    umma_tf32<NK>(tmem + x * NK, ah, bh, acc);   // fixed order: hi.hi, hi.lo, lo.hi
                    umma_tf32<NK>(tmem + x * NK, ah, bl, 1u);
                    umma_tf32<NK>(tmem + x * NK, al, bh, 1u);
                }
                umma_commit<1>(&bars->opempty[s]);
            }
            __syncwarp();
            if (++s == L::SO) { s = 0; ph ^= 1; }
        }
        if (elect_one()) umma_commit<1>(&bars->accfull);
        __syncwarp();
    } else {
        // ================================= FT =================================
        // Group G = (warp - 2) / 4 takes stages G, G + 2, ... (safe by
        // construction as in bfc_tc2.cuh: slot s is refilled only after the
        // MMAs of this group's previous stage in it).  Warp q of the group:
        // IT of A rows m = 32q + lane (one channel per lane: the raw row of
        // 128 / F channels is read 128 B per warp access), FT of dY items
        // (k = t % 64, depth half t / 64) for t = 32q + lane.
        const int tw = warp - 2, G = tw >> 2, q = tw & 3;
        const int m = q * 32 + lane;
        const int f = m / L::BC, cm = m % L::BC;
        const uint32_t xrow = (uint32_t)(L::OFF_X + f * L::XSLOT + cm * 4);
        const int t = q * 32 + lane;
        int s = G, so = G;                     // raw slot, operand slot
        uint32_t ph = 0, pho = 0;
        for (int ch = c_lo + G; ch < c_hi; ch += 2) {
            mbar_wait(&bars->full[s], ph);
            mbar_wait(&bars->opempty[so], pho ^ 1);   // the MMAs of this slot's previous stage are done
            const uint32_t st = sbase + (uint32_t)(s * L::RAW);
            const uint32_t ot = sbase + (uint32_t)(L::OP_OFF + so * L::OP);
#pragma unroll
            for (int k4 = 0; k4 < 2; ++k4) {          // depth entries 4 k4 .. 4 k4 + 3
                float hi[4][4], lo[4][4];
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const int img = 4 * k4 + j;
                    float x[4];
#pragma unroll
                    for (int c = 0; c < 4; ++c) x[c] = lds32(st + xrow + (uint32_t)((c * KT + img) * L::BC * 4));
                    hi[0][j] = x[1] + x[2];
                    hi[1][j] = x[2] - x[1];
                    hi[2][j] = x[0] - x[2];
                    hi[3][j] = x[3] - x[1];
#pragma unroll
                    for (int a = 0; a < 4; ++a) lo[a][j] = tf32_lo(hi[a][j]);
                }
                const uint32_t o = koff(m, k4);
#pragma unroll
                for (int a = 0; a < 4; ++a) {
                    sts4f(ot + L::OFF_A + a * L::ASLAB + o, hi[a][0], hi[a][1], hi[a][2], hi[a][3]);
                    sts4f(ot + L::OFF_A + (4 + a) * L::ASLAB + o, lo[a][0], lo[a][1], lo[a][2], lo[a][3]);
                }
            }
#pragma unroll
            for (int it2 = 0; it2 < NK / 64; ++it2) {   // dY items (k, depth half): NK x 2 over 128 threads
                const int ti = t + it2 * 128, kk = ti % NK, dh = ti / NK;
                float w[4][4];   // [xi][depth j]
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const int img = 4 * dh + j;
                    const float w0 = lds32(st + L::OFF_Y + (uint32_t)(((0 * KT + img) * NK + kk) * 4));
                    const float w1 = lds32(st + L::OFF_Y + (uint32_t)(((1 * KT + img) * NK + kk) * 4));
                    w[0][j] = w0 + w1;
                    w[1][j] = w0 - w1;
                    w[2][j] = w0;
                    w[3][j] = w1;
                }
                const uint32_t o = koff(kk, dh);
#pragma unroll
                for (int a = 0; a < 4; ++a) {
                    sts4f(ot + L::OFF_B + a * L::BSLAB + o, w[a][0], w[a][1], w[a][2], w[a][3]);
                    sts4f(ot + L::OFF_B + (4 + a) * L::BSLAB + o, tf32_lo(w[a][0]), tf32_lo(w[a][1]),
                          tf32_lo(w[a][2]), tf32_lo(w[a][3]));
                }
            }
            fence_async();     // generic-proxy stores -> visible to the tensor core (async proxy)
            __syncwarp();
            if (lane == 0) {
                mbar_arrive(&bars->rempty[s]);   // raw reads retired (the loads fed the stores above)
                mbar_arrive(&bars->opfull[so]);
            }
            s += 2;
            if (s >= L::SR) { s -= L::SR; ph ^= 1; }
            so += 2;
            if (so >= L::SO) { so -= L::SO; pho ^= 1; }
        }
        // ============================ epilogue (as bfc_tc2.cuh) ===============
        mbar_wait(&bars->accfull, 0);
        tc_after();
        const int qq = warp & 3;                     // TMEM lane quarter of this warp
        const int half = (warp - 2) >> 2;            // k half
        const int mm = qq * 32 + lane;
        const int fh = fh_base + mm / L::BC;
        const int c = c_base + mm % L::BC;
        const bool row_ok = fh < g.R && c < g.C;
        float* Out = reinterpret_cast<float*>(smem);  // staging [s][k][m] (overlays the idle ring)
        const uint32_t lane_base = tmem + ((uint32_t)(qq * 32) << 16);
#pragma unroll 1
        for (int k0 = half * (NK / 2); k0 < (half + 1) * (NK / 2); k0 += 8) {
            float v[4][8];
            if (!empty_range) {
#pragma unroll
                for (int x = 0; x < 4; ++x) tmem_ld8(lane_base + (uint32_t)(x * NK + k0), v[x]);
                tmem_wait_ld();
            } else {
#pragma unroll
                for (int x = 0; x < 4; ++x)
#pragma unroll
                    for (int i = 0; i < 8; ++i) v[x][i] = 0.f;
            }
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                const float sp = 0.5f * (v[0][i] + v[1][i]);
                const float y0 = sp + v[2][i], y1 = 0.5f * (v[0][i] - v[1][i]), y2 = sp + v[3][i];
                if (g.csplit > 1) {
                    Out[(0 * NK + k0 + i) * MROWS + mm] = y0;
                    Out[(1 * NK + k0 + i) * MROWS + mm] = y1;
                    Out[(2 * NK + k0 + i) * MROWS + mm] = y2;
                } else {
                    const int k = k_base + k0 + i;
                    if (row_ok && k < g.K) {
                        float* o = bucket + (((long long)k * g.R + fh) * g.S + fw0) * g.C + c;
                        o[0] = y0;
                        o[g.C] = y1;
                        o[2 * g.C] = y2;
                    }
                }
            }
        }
    }
    tc_before();
    __syncthreads();
    if (g.csplit > 1) {
        // deterministic cluster reduction: rank r sums rows (s, k) of its slice
        // over ranks 0..cs-1 in order (dsmem_sum4) and writes them
        constexpr int ROWS = NSOUT * NK, M4 = MROWS / 4;
        cluster_sync_all();
        const int r_lo = ROWS * rank / g.csplit, r_hi = ROWS * (rank + 1) / g.csplit;
        for (int p = r_lo * M4 + (int)threadIdx.x; p < r_hi * M4; p += NTHREADS) {
            const int row = p / M4, m4 = p % M4;
            const int sidx = row / NK, kl = row % NK;
            const float4 acc = dsmem_sum4(sbase + (uint32_t)((row * MROWS + m4 * 4) * 4), g.csplit);
            const int m0 = m4 * 4;
            const int fh = fh_base + m0 / L::BC, c = c_base + m0 % L::BC, k = k_base + kl;
            if (fh < g.R && c < g.C && k < g.K)
                *reinterpret_cast<float4*>(bucket + (((long long)k * g.R + fh) * g.S + fw0 + sidx) * g.C + c) = acc;
        }
        cluster_sync_all();
    }
    if (warp == 1) {
        tc_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(tmem), "r"((uint32_t)L::TMEM_COLS));
    }
}

}  // namespace tc3
}  // namespace winrs
