// Second-generation FP16 / BF16 tensor-core WinRS BFC kernel for sm_100a
// (tcgen05 + TMEM + TMA + mbarrier), kernel Omega_4(3,2) (Figure 6,
// P@28451; the F_W = 3 member of the ported FP16 set, P@28616).
//
// What it computes (§3 eq. (6), P@31000-32161): for a CTA tile
// (segment z, filter-row group, c-block, k-block) and every unit u of r0 = 2
// dY columns of every clipped dY row h of the segment and every image n,
//     v[xi][m][k] += Xhat[xi](n, h + fh(m) - pad, u)[c(m)] * What[xi](n, h, u)[k]
// with What = G w (FT of the dY unit, P@30202 Alg. 3) and Xhat = D^T x (IT of
// the alpha = 4 X window, P@30341), then dW_z[k][fh][s][c] = (A^T v)[s] (OT,
// P@31000).  The transforms (R20):
//     FT  What = (w0 + w1, w0 - w1, w0, w1)
//     IT  Xhat = (x1 + x2, x2 - x1, x0 - x2, x3 - x1)
//     OT  y0 = (v0 + v1)/2 + v2,  y1 = (v0 - v1)/2,  y2 = (v0 + v1)/2 + v3
// (interpolation points 1, -1, 0, inf: the Cook-Toom F(3,2) of
// tools/gen_winograd.py with the eq. (7) row scaling moved from G and D^T into
// A, so every FT / IT output is ONE add or subtract of two inputs).
//
// B200 design (each choice measured on B200):
//   * The EWM is a 4-batched GEMM with M = 128 TMEM lanes = X rows (fh slot,
//     c) and N = NK = 64 / 128 k columns (all 512 TMEM columns at NK = 128).
//   * The IT runs INSIDE the tensor core: by linearity
//         v0 = x1 W0 + x2 W0,  v1 = x2 W1 - x1 W1,
//         v2 = x0 W2 - x2 W2,  v3 = x3 W3 - x1 W3,
//     8 MMAs per 16-deep stage whose A operands are the raw X columns x_t,
//     landed by TMA directly in the UMMA operand layout (MN-major, 128-byte
//     swizzle), the minus signs being the instruction descriptor's negate-A
//     bit.  Measured (WINRS_TC2_NO_MMA / _NO_STS ablations): the tensor core's
//     shared-memory reads do not compete with TMA / LDS / STS traffic, while
//     thread-side operand stores cost a third of every stage, so trading the
//     IT's 16 KB of loads + 16 KB of stores per stage for 4 extra MMAs is a
//     net win.  The products are exact and accumulate in FP32: the IT adds no
//     rounding at all.
//   * The FT stays on threads (What[0,1] = w0 +- w1 in packed 16-bit adds:
//     one correctly rounded add, the FP16 value P@38729's "computed in FP32,
//     then converted" produces); What[2,3] are the raw dY columns (TMA).
//   * For C <= 64 two filter rows share the M = 128 tile (F = 2: rows
//     [0,64) are fh0's X windows, [64,128) fh0+1's) so K = C = 64 layers do
//     not waste half of every MMA.
//   * One ring of S stages (KC = 16 depth entries each); a stage holds the TMA
//     data and the FT operands of the same 16 depth entries, so it has exactly
//     one owner at a time: TMA -> FT threads -> MMA -> (commit) TMA.  Every
//     FT warp processes every stage in order and only the MMA commit frees a
//     stage, so a warp can never be a full ring ahead of the MMAs and no
//     phase-parity wait can alias (safe by construction; round 1's
//     dynamically handed-out units needed a timing argument).
//
// Warp roles (352 threads, one CTA per SM):
//   warps 0,10 TMA producers (even / odd stages; one elected lane per box)
//   warp 1     TMEM allocator + MMA issuer
//   warps 2-9  FT (256 threads: at most one (k octet, depth) item per stage),
//              then the epilogue (tcgen05.ld -> OT -> bucket, or -> shared
//              staging tile -> DSMEM cluster reduction).
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include "dsmem.cuh"
#include "winrs_internal.h"

namespace winrs {
namespace tc2 {

constexpr int KC = 16;                 // depth entries per stage = UMMA K
constexpr int MROWS = 128;             // UMMA M = TMEM lanes
constexpr int NTX = 8;                 // transformer warps
constexpr int NTHREADS = 64 + 32 * NTX + 32;
constexpr int PW2 = 2 + NTX;           // second TMA producer warp (odd stages; warp 0: even stages)
// TA kernels: NTX_TA / 4 groups of four FT warps taking alternate stages
constexpr int NTX_TA = 8;     // (16 measured: no gain, VGG conv1_2 650 -> 679 us)
template <bool TA> __host__ __device__ constexpr int tc2_threads() { return 64 + 32 * (TA ? NTX_TA : NTX) + 32; }
constexpr int NSOUT = 3;               // n0: outputs per unit (S = 3)
#ifndef WINRS_TC2_PF
#define WINRS_TC2_PF 0     // TA producers: L2 prefetch (cp.async.bulk.prefetch.tensor) of the stage PF stages
                           // ahead of the one being loaded (0: off).  Measured: PF = 8 / 16 / 32
                           // all ~20 % SLOWER (ResNet-50 L4 33.8 -> 40 us, VGG conv1_2 656 -> 830 us): the
                           // prefetch boxes cost TMA-engine time like loads; kept as a build option only.
#endif
#ifndef WINRS_TC2_TA_S
#define WINRS_TC2_TA_S 8   // TA shared-memory ring depth (6 / 8 / 9; at 9 the TMEM A ring keeps 8 slots with its
                           // own release barrier and the FT groups an extra opfull guard: measured slower,
                           // DESIGN.md §6.4b)
#endif
#ifndef WINRS_TC2_TA_DEAD_S
#define WINRS_TC2_TA_DEAD_S 0   // TA, F = 2: ring depth of the CTAs whose second fh slot is dead (the {2, -}
                                // group of R = 3): one X atom, 17 KB stages; 0 = same ring as the live groups
#endif
#ifndef WINRS_TC2_STX4
#define WINRS_TC2_STX4 1   // TA: one tcgen05.st .x4 per 16-row half (0: four .x1 stores)
#endif
#ifndef WINRS_TC2_ITM
#define WINRS_TC2_ITM 0    // 1: IT inside the tensor core (8 MMAs per stage on the raw X columns, by linearity);
                           // 0: IT on the FT warps, in place over the raw X slabs (4 MMAs per stage: the
                           //    alpha = 4 Winograd EWM).  A/B on B200 in DESIGN.md §6.4.
#endif

template <int F, int NK, int CG = 1, bool TA = false>
struct Lay {
    static constexpr int BC = MROWS / F;                 // channels c per fh slot
    static constexpr int NKL = NK / CG;                  // k rows of the What operand held by this CTA
    // One stage = 16 depth entries (images n of one (h, u)), three regions of
    // 64-channel swizzle atoms [atom][col][n (16 rows of 128 B)]:
    //   X   [2 atoms][4 cols x_t]   16 KB   A operand of column t: +t*2 KB, atoms 8 KB apart
    //                                        (atom = c half for F = 1, fh slot for F = 2)
    //   Y   [NK/64 atoms][w0, w1]   8/4 KB  What[2], What[3]: +0 / +2 KB, atoms 4 KB apart
    //   FT  [NK/64 atoms][W0, W1]   8/4 KB  What[0], What[1] (stored by the FT threads)
    static constexpr int ATOM = KC * 128;                // 2 KB: 64 channels x 16 depth rows
    static constexpr int X_LBO = 4 * ATOM;               // 8 KB
    static constexpr int Y_LBO = 2 * ATOM;               // 4 KB
    // TA (Xhat in TMEM; X is read only by ldmatrix.trans): per X atom two
    // boxes of 8 images x 4 cols (rows col * 8 + n, 4 KB), the upper-image box
    // two 128-byte rows further (the TMA swizzle follows the absolute address
    // bits [7:9]: probed, tools/microbench/tma_offset.cu), so that the 8 rows
    // of every ldmatrix phase -- depth entries {4p, 4p+1} or {4p+2, 4p+3},
    // p = 0..3, of one column -- fall in 8 distinct 16-byte bank groups.
    static constexpr int XT_HI = 4096 + 256;             // upper 8 images
    static constexpr int XT_GRP = 2 * 4096 + 256;        // between the two X atoms (66 rows)
    static constexpr int X_GRP = TA ? XT_GRP : X_LBO;    // producer: X atom a at a * X_GRP
    static constexpr int OFF_Y = TA ? 17 * 1024 : 2 * X_LBO;   // 16 KB (TA: 17 KB, 1 KB aligned)
    static constexpr int OFF_F = OFF_Y + (NKL / 64) * Y_LBO;
    static constexpr int STAGE = OFF_F + (NKL / 64) * Y_LBO;   // 32 / 24 KB (cta pair: 24 KB)
    static constexpr int LIMIT = 227 * 1024 - 1024 - 512;
    static constexpr int SCAP = TA ? (WINRS_TC2_TA_S < 9 ? WINRS_TC2_TA_S : 9) : 8;
    static constexpr int S = LIMIT / STAGE > SCAP ? SCAP : LIMIT / STAGE;
    // TA, F = 2, dead second fh slot: X atom 0 only (two 4 KB boxes, 8.25 KB), so What / FT move
    // up and a stage is 17 KB; S_D of them (the TMEM A ring stays 8 slots: its own release barrier)
    static constexpr bool DRING = TA && F == 2 && WINRS_TC2_TA_DEAD_S > 0;
    static constexpr int OFF_Y_D = 9 * 1024;
    static constexpr int OFF_F_D = OFF_Y_D + (NKL / 64) * Y_LBO;
    static constexpr int STAGE_D = OFF_F_D + (NKL / 64) * Y_LBO;
    static constexpr int S_D = DRING ? WINRS_TC2_TA_DEAD_S : S;
    static constexpr int RING_D = DRING ? S_D * STAGE_D : 0;
    static constexpr int RING = S * STAGE > RING_D ? S * STAGE : RING_D;
    static constexpr int OUT = NSOUT * NK * MROWS * 4;   // staging tile [s][k][m] fp32 (cluster split)
    static constexpr int BAR_OFF = RING > OUT ? RING : OUT;
    static constexpr int BYTES = BAR_OFF + 512 + 1024;   // + alignment slack
    static constexpr int TX_BYTES = 2 * X_LBO + (NKL / 64) * Y_LBO;   // TMA bytes per stage
    static constexpr int TMEM_COLS = 4 * NK;
    static_assert(STAGE % 1024 == 0, "stages must keep the 1 KB swizzle-atom alignment");
    static_assert(S >= 4, "ring too shallow");
    static_assert(!DRING || (S_D % 2 == 0 && S_D <= 12 && STAGE_D % 1024 == 0 && RING_D <= LIMIT),
                  "dead-slot ring: even depth (two FT groups), <= 12 barrier slots, fits");
    static_assert(MROWS == F * BC && BC % 64 == 0, "fh slots of whole 64-channel atoms");
    static_assert(NKL % 64 == 0, "whole 64-channel k atoms per CTA");
};

struct Args {
    Geometry g;
    float* dW;
    float* ws;
    int nb;            // images per TMA box (divides N and KC, >= 8)
    // stream-K xi-split pairs (bfc_tc2x.cuh SK): number of pairs, per-tile
    // chain flags (library-owned, zero-initialised) and this launch's epoch tag
    int sk_pairs = 0;
    unsigned int* sk_flags = nullptr;
    unsigned int sk_epoch = 0;
};

struct Bars {
    uint64_t full[12];      // TMA data landed
    uint64_t opfull[12];    // FT operands stored (one warp per stage)
    uint64_t empty[12];     // MMAs of the stage done (commit)
    uint64_t accfull;
    uint32_t tmem_base;
    uint32_t spare;
    uint64_t aempty[8];     // TA with a 9-slot ring: MMAs that read TMEM A slot a done (commit)
};
static_assert(sizeof(Bars) <= 512, "barrier block");

// ----------------------------------------------------------------------------- PTX helpers
__device__ __forceinline__ uint32_t su(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t n) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(su(b)), "r"(n));
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(su(b)) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
    asm volatile(
        "{\n.reg .pred P;\nW_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1, %2;\n"
        "@!P bra W_%=;\n}\n" :: "r"(su(b)), "r"(parity), "r"(1000000) : "memory");
}
__device__ __forceinline__ void tma4(uint32_t dst, const CUtensorMap* m, uint64_t* bar, int c0, int c1, int c2, int c3) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];"
        :: "r"(dst), "l"(reinterpret_cast<uint64_t>(m)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(su(bar)) : "memory");
}
// One lane of a converged warp (elect.sync).  Issuing tcgen05.mma / TMA from
// an elected lane of a converged warp lets the compiler keep the operands in
// uniform registers; inside `if (lane == 0)` every operand goes through an
// R2UR waterfall loop (~50-70 cycles per instruction, measured: the MMA issue
// and the TMA issue each took ~500 cycles per stage that way).
__device__ __forceinline__ bool elect_one() {
    uint32_t pred;
    asm volatile("{\n.reg .pred p;\nelect.sync _|p, 0xffffffff;\nselp.u32 %0, 1, 0, p;\n}\n" : "=r"(pred));
    return pred != 0;
}
// L2 prefetch of a box (no shared-memory destination, no barrier).
__device__ __forceinline__ void tma5_pf(const CUtensorMap* m, int c0, int c1, int c2, int c3, int c4) {
    asm volatile("cp.async.bulk.prefetch.tensor.5d.L2.global.tile [%0, {%1, %2, %3, %4, %5}];"
                 :: "l"(reinterpret_cast<uint64_t>(m)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4) : "memory");
}
__device__ __forceinline__ void tma5(uint32_t dst, const CUtensorMap* m, uint64_t* bar, int c0, int c1, int c2, int c3,
                                     int c4) {
    asm volatile(
        "cp.async.bulk.tensor.5d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
        :: "r"(dst), "l"(reinterpret_cast<uint64_t>(m)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4), "r"(su(bar))
        : "memory");
}
// Image index img of the 2-D decomposition -> (inner, outer) TMA coordinates:
// 2-D plans: (img, 0) of maps {ch, N, 1, H, W}; N-D plans (PAPER.md P@17805,
// Level-2 dimension reduction): (depth slice img % Do, batch img / Do) of maps
// {ch, D or Do, Nb, H, W}.  Past the end: outer = Nb (zero fill).  Tracked
// incrementally next to the producer's (n, u, h): a per-stage division on an
// SM sub-partition shared with other warps cost ~30 % of the kernel (measured).
struct ImgCoord {
    int a, b;
};
struct ImgTracker {
    int a, b, inner;
    __device__ __forceinline__ void init(const Geometry& g, int img) {
        inner = (g.T > 1 || g.D > 1) ? g.Do : g.N;
        a = img % inner;
        b = img / inner;
    }
    // After the producer's n += by and its wrap loop: image n (n < by when
    // wrapped, since n < N before the step); a < inner + by, so the loop runs
    // at most by / 16 times (inner >= 16).
    __device__ __forceinline__ void advance(int by, bool wrapped, int n) {
        if (wrapped) { a = n; b = 0; } else { a += by; }
        while (a >= inner) { a -= inner; ++b; }
    }
    __device__ __forceinline__ ImgCoord at(const Geometry& g, bool in) const {
        ImgCoord c;
        c.a = in ? a : 0;
        c.b = in ? b : ((g.T > 1 || g.D > 1) ? g.Nb : 1);
        return c;
    }
};
__device__ __forceinline__ void fence_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void tc_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
// Programmatic dependent launch: once every CTA of this grid has started, the
// bucket reduction queued behind it (reduce.cu, launched with programmatic
// stream serialisation) may be scheduled; it waits in griddepcontrol.wait
// until this grid has completed and its writes are visible.
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

// UMMA shared-memory descriptor, MN-major, 128-byte swizzle: atoms of 64 MN
// elements x 8 K rows (1 KB); LBO = MN-atom stride, SBO = K-atom stride
// (probed on B200, tools/microbench/umma_mn.cu), version bit 46, layout 2.
__device__ __forceinline__ uint64_t desc_sw128(uint32_t addr, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46) | (2ull << 61);
}
// kind::f16 instruction descriptor: D f32, A/B f16 (0) or bf16 (1), both
// MN-major (bits 15, 16), N >> 3 at bit 17, M >> 4 at bit 24.
// Bit 13: negate A (the IT's minus signs).
// cta_group::2: M = 256 over a CTA pair (each CTA's 128 A rows and NK / 2 B
// rows; each CTA's TMEM holds its 128 rows x NK accumulator columns).
template <int NK, bool BF, bool NEG = false, int CG = 1>
__host__ __device__ constexpr uint32_t idesc() {
    return (1u << 4) | ((BF ? 1u : 0u) << 7) | ((BF ? 1u : 0u) << 10) | ((NEG ? 1u : 0u) << 13) | (1u << 15) |
           (1u << 16) | ((uint32_t)(NK >> 3) << 17) | ((uint32_t)((MROWS * CG) >> 4) << 24);
}
template <int NK, bool BF, bool NEG = false, int CG = 1>
__device__ __forceinline__ void umma(uint32_t d, uint64_t a, uint64_t b, uint32_t acc) {
    if constexpr (CG == 1)
        asm volatile(
            "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
            "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n"
            :: "r"(d), "l"(a), "l"(b), "r"(idesc<NK, BF, NEG, CG>()), "r"(acc));
    else
        asm volatile(
            "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
            "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n}\n"
            :: "r"(d), "l"(a), "l"(b), "r"(idesc<NK, BF, NEG, CG>()), "r"(acc));
}
// A operand from TMEM (the TA kernels): A K-major in 128 lanes x 8 columns
// (lane = row m, column j = depth entries 2j, 2j + 1), B MN-major SW128.
template <int NK, bool BF>
__host__ __device__ constexpr uint32_t idesc_ta() {
    return (1u << 4) | ((BF ? 1u : 0u) << 7) | ((BF ? 1u : 0u) << 10) | (1u << 16) | ((uint32_t)(NK >> 3) << 17) |
           ((uint32_t)(MROWS >> 4) << 24);
}
template <int NK, bool BF, bool NEGB = false>
__device__ __forceinline__ void umma_ta(uint32_t d, uint32_t a_tmem, uint64_t b, uint32_t acc) {
    // bit 14: negate B
    asm volatile(
        "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}\n"
        :: "r"(d), "r"(a_tmem), "l"(b), "r"(idesc_ta<NK, BF>() | (NEGB ? (1u << 14) : 0u)), "r"(acc));
}
// ldmatrix.x4.trans: thread t receives, of matrix i (row addresses from
// threads 8i..8i+7), the 16-bit elements (row 2(t%4), column t/4) and (row
// 2(t%4) + 1, column t/4) packed -- rows = depth entries, columns = channels.
__device__ __forceinline__ void ldsm_x4_t(uint32_t addr, uint32_t (&r)[4]) {
    asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "r"(addr));
}
// tcgen05.st 16x256b (probed on B200, tools/microbench/tmem_a.cu): thread t
// writes r0, r1 to lane t/4, columns 2(t%4), 2(t%4) + 1 and r2, r3 to lane
// t/4 + 8, same columns.
__device__ __forceinline__ void tmem_st16x256(uint32_t taddr, const uint32_t (&r)[4]) {
    asm volatile("tcgen05.st.sync.aligned.16x256b.x1.b32 [%0], {%1, %2, %3, %4};"
                 :: "r"(taddr), "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]) : "memory");
}
// The same shape repeated over 4 consecutive 8-column chunks (.x4): registers
// 4i..4i+3 go to columns 8i..8i+7 (one instruction for the four xi slabs of a
// ring slot instead of four).
__device__ __forceinline__ void tmem_st16x256_x4(uint32_t taddr, const uint32_t (&r)[4][4]) {
    asm volatile("tcgen05.st.sync.aligned.16x256b.x4.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, "
                 "%13, %14, %15, %16};"
                 :: "r"(taddr), "r"(r[0][0]), "r"(r[0][1]), "r"(r[0][2]), "r"(r[0][3]), "r"(r[1][0]), "r"(r[1][1]),
                    "r"(r[1][2]), "r"(r[1][3]), "r"(r[2][0]), "r"(r[2][1]), "r"(r[2][2]), "r"(r[2][3]), "r"(r[3][0]),
                    "r"(r[3][1]), "r"(r[3][2]), "r"(r[3][3])
                 : "memory");
}
__device__ __forceinline__ void tmem_st16x256_x2(uint32_t taddr, const uint32_t (&r)[2][4]) {
    asm volatile("tcgen05.st.sync.aligned.16x256b.x2.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};"
                 :: "r"(taddr), "r"(r[0][0]), "r"(r[0][1]), "r"(r[0][2]), "r"(r[0][3]), "r"(r[1][0]), "r"(r[1][1]),
                    "r"(r[1][2]), "r"(r[1][3])
                 : "memory");
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

// Commit: arrives on `bar` once every MMA issued so far completed; for a CTA
// pair on the barrier at the same offset in both CTAs (mask = the pair).
template <int CG = 1>
__device__ __forceinline__ void umma_commit(uint64_t* bar, uint16_t mask = 3) {
    if constexpr (CG == 1)
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(su(bar)) : "memory");
    else
        asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                     :: "r"(su(bar)), "h"(mask) : "memory");
}
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
// Arrive on the mbarrier at local shared offset `bar` of cluster CTA `rank`.
__device__ __forceinline__ void mbar_arrive_cluster(uint64_t* bar, uint32_t rank) {
    uint32_t remote;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(su(bar)), "r"(rank));
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" :: "r"(remote) : "memory");
}
__device__ __forceinline__ void tmem_ld8(uint32_t taddr, float* v) {
    uint32_t r[8];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                 : "r"(taddr));
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] = __uint_as_float(r[i]);
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// Byte offset of the 16-byte chunk (8 channels, octet o) at depth d of an
// MN-major SW128 operand whose 64-channel atoms are `lbo` bytes apart (KC =
// 16: two 1 KB K-atoms per atom; the chunk index is XORed with the row).
__device__ __forceinline__ uint32_t opoff(int o, int d, int lbo) {
    return (uint32_t)((o >> 3) * lbo + (d >> 3) * 1024 + (d & 7) * 128 + (((o & 7) ^ (d & 7)) << 4));
}

// Packed 16-bit add / subtract of four pairs (one rounding per element).
template <bool BF> struct P16;
template <> struct P16<false> {
    __device__ static __forceinline__ uint32_t add(uint32_t a, uint32_t b) {
        uint32_t r; asm("add.rn.f16x2 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b)); return r;
    }
    __device__ static __forceinline__ uint32_t sub(uint32_t a, uint32_t b) {
        uint32_t r; asm("sub.rn.f16x2 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b)); return r;
    }
};
template <> struct P16<true> {
    __device__ static __forceinline__ uint32_t add(uint32_t a, uint32_t b) {
        uint32_t r; asm("add.rn.bf16x2 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b)); return r;
    }
    __device__ static __forceinline__ uint32_t sub(uint32_t a, uint32_t b) {
        uint32_t r; asm("sub.rn.bf16x2 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b)); return r;
    }
};
template <bool BF>
__device__ __forceinline__ uint4 vadd(const uint4& a, const uint4& b) {
    return make_uint4(P16<BF>::add(a.x, b.x), P16<BF>::add(a.y, b.y), P16<BF>::add(a.z, b.z), P16<BF>::add(a.w, b.w));
}
template <bool BF>
__device__ __forceinline__ uint4 vsub(const uint4& a, const uint4& b) {
    return make_uint4(P16<BF>::sub(a.x, b.x), P16<BF>::sub(a.y, b.y), P16<BF>::sub(a.z, b.z), P16<BF>::sub(a.w, b.w));
}
__device__ __forceinline__ uint4 lds16(uint32_t a) {
    uint4 v;
    asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
    return v;
}
__device__ __forceinline__ void sts16(uint32_t a, const uint4& v) {
    asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" :: "r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}

#ifdef WINRS_TC2_TRACE
// Debug-build timeline (clock64) of CTA `g_tc2_trace_cta`, per stage:
// [0] producer past `empty`, [1] TMAs issued, [2] transformer warp 2 past `full`,
// [3] its `opfull` arrival, [4] MMA warp past `opfull`, [5] MMAs + commit issued.
__device__ long long g_tc2_trace[512][8];
__device__ int g_tc2_trace_cta;
#define TC2_TRACE(ch, ev) do { if (blockIdx.x == (unsigned)g_tc2_trace_cta && (ch) < 512) g_tc2_trace[ch][ev] = clock64(); } while (0)
#else
#define TC2_TRACE(ch, ev) do { } while (0)
#endif

#ifdef WINRS_TC2_JITTER
// Debug build: pseudo-random sleeps in every role, every stage, so the ring
// protocol is exercised under arbitrary relative warp timing (stress test:
// results must stay bitwise identical to an undisturbed run).
__device__ __forceinline__ void jitter(int ch, int who) {
    uint32_t x = (uint32_t)ch * 2654435761u ^ (uint32_t)who * 40503u ^ (uint32_t)blockIdx.x * 97u;
    x ^= x >> 13; x *= 0x5bd1e995u; x ^= x >> 15;
    if ((x & 3) == 0) __nanosleep(64 + (x >> 20) % 2048);
}
#define TC2_JITTER(ch, who) jitter((ch), (who))
#else
#define TC2_JITTER(ch, who) do { } while (0)
#endif

// Depth entry d of a CTA -> (n, h, u): n fastest (d = ((h - hs) * units + u) * N + n).
__device__ __forceinline__ void depth_nhu(int d, int N, int units, int hs, int* n, int* h, int* u) {
    *n = d % N;
    const int t = d / N;
    *u = t % units;
    *h = hs + t / units;
}

// ---- stream-K schedule (SK): the pairs (bfc_tc2x.cuh) take equal contiguous ranges of the
// concatenated depth chunks of all tiles (tiles = segments x fh groups x tile
// coordinates in decode_cta order; a segment's tiles of one fh group form a
// contiguous block of equal depth; Z > 1 segments write their own buckets).  A tile split over several pairs is combined in dW in a fixed
// order -- the pair holding its first chunks first (plain store), then the
// higher pairs in increasing index (read-add-write) -- through one chain flag
// per tile; a pair only ever waits for a lower pair (see the piece loop).
struct SkTile {
    long long t;       // tile index
    long long g0;      // global chunk index of its first chunk
    int depth;         // its chunks
};
// Blocks of equal-depth tiles: block bi = (band * seg_cols + col) * fhg + fh group
// holds the kblocks x cblocks x ftiles tiles of one segment and filter-row group
// (decode_cta order).  With N % 16 == 0 (every tc2-family plan) a tile's chunks
// are rows(band, group) x units(col) x N / 16, so the prefix over blocks factors
// by band, column and group: sk_total / sk_find walk bands, then columns, then
// groups (O(bands + seg_cols + fhg) instead of a walk over every block).
__device__ __forceinline__ int sk_rows(const Geometry& g, int band, int f) {
    int hs, he;
    group_rows(g, band, f * g.fhs, &hs, &he);
    return he > hs ? he - hs : 0;
}
__device__ __forceinline__ int sk_units(const Geometry& g, int col) {
    int wf, units;
    seg_units(g, col, &wf, &units);
    return units;
}
__device__ __forceinline__ long long sk_total(const Geometry& g) {
    const long long per = (long long)g.kblocks * g.cblocks * g.ftiles * (g.N / KC);
    long long rows = 0, units = 0;
    for (int b = 0; b < g.bands; ++b)
        for (int f = 0; f < g.fhg; ++f) rows += sk_rows(g, b, f);
    for (int c = 0; c < g.seg_cols; ++c) units += sk_units(g, c);
    return per * rows * units;
}
// The tile holding global chunk gi.
__device__ __forceinline__ SkTile sk_find(const Geometry& g, long long gi) {
    const long long per = (long long)g.kblocks * g.cblocks * g.ftiles;
    const long long n16 = g.N / KC;
    long long utot = 0;
    for (int c = 0; c < g.seg_cols; ++c) utot += sk_units(g, c);
    long long acc = 0;
    SkTile r{0, 0, 0};
    for (int b = 0; b < g.bands; ++b) {
        long long rb = 0;
        for (int f = 0; f < g.fhg; ++f) rb += sk_rows(g, b, f);
        const long long bsz = per * n16 * rb * utot;
        if (gi >= acc + bsz) { acc += bsz; continue; }
        for (int c = 0; c < g.seg_cols; ++c) {
            const long long uc = sk_units(g, c);
            const long long csz = per * n16 * rb * uc;
            if (gi >= acc + csz) { acc += csz; continue; }
            for (int f = 0; f < g.fhg; ++f) {
                const long long d = (long long)sk_rows(g, b, f) * uc * n16;
                if (d > 0 && gi < acc + per * d) {
                    const long long i = (gi - acc) / d;
                    r.t = ((long long)(b * g.seg_cols + c) * g.fhg + f) * per + i;
                    r.g0 = acc + i * d;
                    r.depth = (int)d;
                    return r;
                }
                acc += per * d;
            }
            return r;
        }
        return r;
    }
    return r;
}
constexpr int SK_MAX_TILES = 1 << 16;   // flag slots; then the pair-ticket and finished-pair counters
constexpr int SK_TICKET = SK_MAX_TILES;
__device__ __forceinline__ long long sk_start(long long tot, int p, int P) { return tot * p / P; }
// The pair whose range holds global chunk gi: the largest p with sk_start(p) <= gi.
__device__ __forceinline__ int sk_pair_of(long long tot, long long gi, int P) {
    return (int)(((gi + 1) * P - 1) / tot);
}
__device__ __forceinline__ unsigned int ld_acquire(const unsigned int* p) {
    unsigned int v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(unsigned int* p, unsigned int v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}

// TA = true: the transformed X operand (Xhat) goes to TMEM (tcgen05.st) and
// the MMAs read A from there: the IT's shared-memory write-back and the MMAs'
// A reads leave the shared-memory port.  TMEM: 4 NK
// accumulator columns + S ring slots x 4 xi x 8 columns (NK = 64: 256 + 256).
template <int F, int NK, bool BF, int CG = 1, bool TA = false>
__global__ void __launch_bounds__(tc2_threads<TA>(), 1)
bfc_tc2_kernel(const __grid_constant__ Args args, const __grid_constant__ CUtensorMap tmX,
               const __grid_constant__ CUtensorMap tmY) {
    using L = Lay<F, NK, CG, TA>;
    constexpr int NTXK = TA ? NTX_TA : NTX;          // FT warps
    constexpr int NTHK = tc2_threads<TA>();
    constexpr int PW2K = 2 + NTXK;                   // second producer warp
    constexpr int NG = NTXK / 4;                     // TA: FT groups of four warps
    static_assert(!TA || (CG == 1 && NK == 64 && L::S <= 9), "TA: single CTA, NK = 64, <= 9-slot ring");
    constexpr bool ASEP = TA && L::S != 8;          // TMEM A ring (8 slots) decoupled from the SMEM ring
    constexpr uint32_t TMEM_ALLOC = TA ? 512u : (uint32_t)L::TMEM_COLS;
    constexpr uint32_t A_COL = 4 * NK;          // TA: first A ring column
    extern __shared__ uint8_t smem_raw[];
    // 1 KB-aligned base (SW128 atoms, TMA swizzle pattern)
    const uint32_t raw_s = su(smem_raw);
    uint8_t* smem = smem_raw + (((raw_s + 1023u) & ~1023u) - raw_s);
    const uint32_t sbase = su(smem);
    Bars* bars = reinterpret_cast<Bars*>(smem + L::BAR_OFF);
    const Geometry& g = args.g;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 64) TC2_TRACE(511, 0);

    // Cluster = CG x csplit CTAs: a CTA pair (cta_group::2, CG = 2: ranks 2j,
    // 2j + 1; the even one issues the MMAs) per depth-split rank j.
    const int crank = CG * g.csplit > 1 ? (int)cluster_rank() : 0;
    const int e = CG == 2 ? (crank & 1) : 0;                 // half of the pair
    const int rank = CG == 2 ? (crank >> 1) : (int)(blockIdx.x % g.csplit);   // depth-split rank
    const uint32_t leader = (uint32_t)(crank & ~(CG - 1));
    const uint16_t pair_mask = (uint16_t)(3u << leader);
    const CtaCoord cc = decode_cta(g, blockIdx.x / (CG * g.csplit));
    // this CTA's 128 A rows: F = 1: channels c_base.. of filter row fh_base;
    // F = 2: fh slots fh_base, fh_base + 1 of channels c_base..c_base + 63.
    // A pair covers 256 channels (F = 1) or 4 filter rows (F = 2).
    const int fh_base = cc.fh + (F == 2 ? 2 * e : 0);
    // TA, F = 2: a CTA whose second fh slot lies past the last filter row runs the deeper
    // ring of 17 KB stages (Lay::DRING; its TMEM A ring keeps 8 slots and its own release)
    const bool dring = L::DRING && fh_base + 1 >= g.R;
    const int RS = dring ? L::S_D : L::S;
    const uint32_t RSTAGE = dring ? (uint32_t)L::STAGE_D : (uint32_t)L::STAGE;
    const uint32_t OFFY = dring ? (uint32_t)L::OFF_Y_D : (uint32_t)L::OFF_Y;
    const uint32_t OFFF = dring ? (uint32_t)L::OFF_F_D : (uint32_t)L::OFF_F;
    const bool asep = ASEP || dring;
    const int c_base = F == 2 ? cc.cb * 64 : cc.cb * (128 * CG) + e * 128;
    const int k_base = cc.kb * NK + e * L::NKL;              // this CTA's What rows
    const int seg = cc.band * g.seg_cols + cc.col;
    float* bucket = seg == 0 ? args.dW : args.ws + (long long)(seg - 1) * g.dw_elems;
    int hs, he, w_first, units;
    group_rows(g, cc.band, cc.fh, &hs, &he);
    seg_units(g, cc.col, &w_first, &units);
    const long long depth = (long long)(he > hs ? he - hs : 0) * units * g.N;
    int c_lo, c_hi;
    split_chunks((int)((depth + KC - 1) / KC), rank, g.csplit, &c_lo, &c_hi);
    const bool empty_range = c_hi <= c_lo;
    const int fw0 = cc.ft * NSOUT;       // first output column of this fw-tile (S = 3 * ftiles)

    if (threadIdx.x == 0) {
        for (int s = 0; s < RS; ++s) {
            mbar_init(&bars->full[s], 1);
            mbar_init(&bars->opfull[s], 1);
            mbar_init(&bars->empty[s], 1);
        }
        mbar_init(&bars->accfull, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (CG == 2 && threadIdx.x == 0 && e == 0)   // the leader's opfull gathers both CTAs' FT warps
        for (int s = 0; s < RS; ++s) mbar_init(&bars->opfull[s], 2);
    if (TA && threadIdx.x == 0) {                // TA: the four lane-quarter warps of a group
        for (int s = 0; s < RS; ++s) mbar_init(&bars->opfull[s], 4);
        for (int a = 0; a < 8; ++a) mbar_init(&bars->aempty[a], 1);
    }
    if (warp == 0 && lane == 0) {
        asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(&tmX)) : "memory");
        asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(&tmY)) : "memory");
    }
    if (warp == 1) {
        if constexpr (CG == 2) {
            asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;"
                         :: "r"(su(&bars->tmem_base)), "r"(L::TMEM_COLS));
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
        } else {
            asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                         :: "r"(su(&bars->tmem_base)), "r"(TMEM_ALLOC));
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
        }
    }
    tc_before();
    __syncthreads();
    if (CG == 2) cluster_sync_all();   // peer barriers initialised before any remote arrive / multicast commit
    tc_after();
    if (threadIdx.x == 0) pdl_trigger();
    const uint32_t tmem = bars->tmem_base;
    if (threadIdx.x == 64) TC2_TRACE(511, 1);

    if (warp == 0 || warp == PW2K) {
        // ============================ TMA producers ===========================
        // Two converged warps (warp 0: even stages, warp PW2: odd stages; the
        // per-stage issue path is ~120 dependent instructions, which alone
        // bounded the small-tile kernels: ncu source counters), one elected
        // lane issues the stage's boxes: X atoms 0 and 1 (c halves, or fh
        // slots for F = 2) and the dY k atoms, each [64 ch][16 images][1 row]
        // [cols], i.e. one 128-byte swizzled row per (col, image) = the UMMA
        // operand layout.  (n, u, h) advance incrementally (per-stage integer
        // divisions cost ~700 cycles on an SM sub-partition shared with other
        // warps: WINRS_TC2_TRACE timeline.)
        const int pp = warp == 0 ? 0 : 1;
        long long d = (long long)(c_lo + pp) * KC;
        int n = 0, h = hs, u = 0;
        if (d < depth) depth_nhu((int)d, g.N, units, hs, &n, &h, &u);
        ImgTracker itk;
        itk.init(g, n);
        // per X atom: depth-tap shift and height-tap row offset of its filter row
        // (constant per CTA: no per-stage division)
        int xdt[2], xdr[2];
#pragma unroll
        for (int a = 0; a < 2; ++a) {
            const int fh = F == 2 ? fh_base + a : fh_base;
            xdt[a] = (g.T > 1 || g.D > 1) ? fh / g.Rh - g.pad : 0;
            xdr[a] = fh < g.R ? fh % g.Rh - g.pad : -(1 << 20);   // a slot past the last filter row: zero fill
        }
        // TA, F = 2: the second fh slot lies past the last filter row (e.g. the
        // {2, -} group of R = 3): its X boxes and IT are skipped; the MMAs still
        // run M = 128, and the dead rows' accumulators are never written out.
        const bool dead1 = F == 2 && fh_base + 1 >= g.R;
        // L2 prefetch walker (TA): stages c_lo + pp + S, + S + 2, ... are
        // prefetched while stage ch - PF + S .. ch is being loaded, so their
        // TMA loads later hit L2 instead of waiting the HBM round trip.
        constexpr int PF = TA ? WINRS_TC2_PF : 0;
        int pch = c_lo + pp + RS;
        long long pd = (long long)pch * KC;
        int pn = 0, ph_ = hs, pu = 0;
        ImgTracker pitk;
        if (PF > 0) {
            if (pd < depth) depth_nhu((int)pd, g.N, units, hs, &pn, &ph_, &pu);
            pitk.init(g, pn);
        }
        int s = pp;
        uint32_t ph = 0;
        for (int ch = c_lo + pp; ch < c_hi; ch += 2) {
            if constexpr (PF > 0) {
                while (pch < c_hi && pch <= ch + PF) {
                    const ImgCoord pc = pitk.at(g, true);
                    const int pw0 = w_first + pu * 2;
                    if (elect_one()) {
#pragma unroll
                        for (int a = 0; a < 2; ++a) {
                            if (a == 1 && dead1) continue;
                            const int c0 = F == 2 ? c_base : c_base + a * 64;
                            tma5_pf(&tmX, c0, pc.a + xdt[a], pc.b, ph_ + xdr[a], pw0 + fw0 - g.pad);
                            tma5_pf(&tmX, c0, pc.a + 8 + xdt[a], pc.b, ph_ + xdr[a], pw0 + fw0 - g.pad);
                        }
#pragma unroll
                        for (int ka = 0; ka < L::NKL / 64; ++ka) tma5_pf(&tmY, k_base + ka * 64, pc.a, pc.b, ph_, pw0);
                    }
                    __syncwarp();
                    pch += 2;
                    pn += 2 * KC;
                    bool pw = false;
                    while (pn >= g.N) {
                        pn -= g.N;
                        pw = true;
                        if (++pu == units) { pu = 0; ++ph_; }
                    }
                    pitk.advance(2 * KC, pw, pn);
                }
            }
            mbar_wait(&bars->empty[s], ph ^ 1);
            TC2_JITTER(ch, 0);
            TC2_TRACE(ch - c_lo, 0);
            uint64_t* fb = &bars->full[s];
            const uint32_t st = sbase + (uint32_t)(s * RSTAGE);
            const bool in = d < depth;               // past the end: outer image coordinate out of range (zero fill)
            const ImgCoord ic = itk.at(g, in);
            const int hh = in ? h : hs;
            const int w0 = w_first + (in ? u : 0) * 2;
            if (elect_one()) {
#ifdef WINRS_TC2_NO_TMA   // debug ablation: stages carry no data (barrier protocol kept)
                mbar_arrive(fb);
#else
                mbar_expect_tx(fb, (uint32_t)L::TX_BYTES - (TA && dead1 ? 8192u : 0u));
#pragma unroll
                for (int a = 0; a < 2; ++a) {
                    // X window columns x0..x3 of atom a; an fh slot past the last
                    // filter row reads rows far outside (zero fill)
                    const int c0 = F == 2 ? c_base : c_base + a * 64;
                    if constexpr (TA) {   // two 8-image boxes (tmX box {64, 8, 1, 1, 4})
                        if (a == 1 && dead1) continue;   // no X rows for an fh slot past the last filter row
                        tma5(st + a * L::X_GRP, &tmX, fb, c0, ic.a + xdt[a], ic.b, hh + xdr[a], w0 + fw0 - g.pad);
                        tma5(st + a * L::X_GRP + L::XT_HI, &tmX, fb, c0, ic.a + 8 + xdt[a], ic.b, hh + xdr[a],
                             w0 + fw0 - g.pad);
                    } else {
                        tma5(st + a * L::X_LBO, &tmX, fb, c0, ic.a + xdt[a], ic.b, hh + xdr[a], w0 + fw0 - g.pad);
                    }
                }
#pragma unroll
                for (int ka = 0; ka < L::NKL / 64; ++ka)   // dY unit columns w0, w0 + 1 of k atom ka
                    tma5(st + OFFY + ka * L::Y_LBO, &tmY, fb, k_base + ka * 64, ic.a, ic.b, hh, w0);
#endif
            }
            __syncwarp();
            TC2_TRACE(ch - c_lo, 1);
            d += 2 * KC;
            n += 2 * KC;
            bool wrapped = false;
            while (n >= g.N) {
                n -= g.N;
                wrapped = true;
                if (++u == units) { u = 0; ++h; }
            }
            itk.advance(2 * KC, wrapped, n);
            s += 2;
            if (s >= RS) { s -= RS; ph ^= 1; }
        }
    } else if (warp == 1) {
        // ============================ MMA issuer ==============================
        // Converged warp; descriptors are computed uniformly, one elected lane
        // issues the MMAs and the commit (a pair: the leader only, for both).
        if (CG == 2 && e != 0) goto mma_done;
        {
        int s = 0;
        uint32_t ph = 0;
        for (int ch = c_lo; ch < c_hi; ++ch) {
            mbar_wait(&bars->opfull[s], ph);
            TC2_JITTER(ch, 1);
            TC2_TRACE(ch - c_lo, 4);
            tc_after();
            const uint32_t st = sbase + (uint32_t)(s * RSTAGE);
            const uint32_t acc = ch > c_lo ? 1u : 0u;
            // A: raw X column x_t (M = 128: two atoms X_LBO apart); B: What[xi]
            const uint64_t x0 = desc_sw128(st, L::X_LBO, 1024);
            const uint64_t x1 = x0 + (L::ATOM >> 4), x2 = x0 + (2 * L::ATOM >> 4), x3 = x0 + (3 * L::ATOM >> 4);
            const uint64_t w0d = desc_sw128(st + OFFF, L::Y_LBO, 1024), w1d = w0d + (L::ATOM >> 4);
            const uint64_t w2d = desc_sw128(st + OFFY, L::Y_LBO, 1024), w3d = w2d + (L::ATOM >> 4);
            if (elect_one()) {
#ifndef WINRS_TC2_NO_MMA   // debug ablation: no tensor-core work (barrier protocol kept)
              if (TA) {               // Xhat[xi] from the TMEM ring slot x What[xi]
                const int aslot = asep ? (ch - c_lo) % 8 : s;
                const uint32_t a = tmem + A_COL + (uint32_t)(aslot * 32);
                umma_ta<NK, BF>(tmem + 0 * NK, a + 0, w0d, acc);
                umma_ta<NK, BF>(tmem + 1 * NK, a + 8, w1d, acc);
                umma_ta<NK, BF>(tmem + 2 * NK, a + 16, w2d, acc);
                umma_ta<NK, BF>(tmem + 3 * NK, a + 24, w3d, acc);
              } else if (!WINRS_TC2_ITM) {   // Xhat[xi] (IT done in place by the FT warps) x What[xi]
                umma<NK, BF, false, CG>(tmem + 0 * NK, x0, w0d, acc);
                umma<NK, BF, false, CG>(tmem + 1 * NK, x1, w1d, acc);
                umma<NK, BF, false, CG>(tmem + 2 * NK, x2, w2d, acc);
                umma<NK, BF, false, CG>(tmem + 3 * NK, x3, w3d, acc);
              } else {
                umma<NK, BF, false, CG>(tmem + 0 * NK, x1, w0d, acc);          // v0 = (x1 + x2) W0
                umma<NK, BF, false, CG>(tmem + 0 * NK, x2, w0d, 1u);
                umma<NK, BF, false, CG>(tmem + 1 * NK, x2, w1d, acc);          // v1 = (x2 - x1) W1
                umma<NK, BF, true, CG>(tmem + 1 * NK, x1, w1d, 1u);
                umma<NK, BF, false, CG>(tmem + 2 * NK, x0, w2d, acc);          // v2 = (x0 - x2) W2
                umma<NK, BF, true, CG>(tmem + 2 * NK, x2, w2d, 1u);
                umma<NK, BF, false, CG>(tmem + 3 * NK, x3, w3d, acc);          // v3 = (x3 - x1) W3
                umma<NK, BF, true, CG>(tmem + 3 * NK, x1, w3d, 1u);
              }
#else
                (void)x0; (void)x1; (void)x2; (void)x3; (void)w0d; (void)w1d; (void)w2d; (void)w3d; (void)acc;
#endif
                umma_commit<CG>(&bars->empty[s], pair_mask);
                if (asep) umma_commit<1>(&bars->aempty[(ch - c_lo) % 8]);
            }
            __syncwarp();
            TC2_TRACE(ch - c_lo, 5);
            if (++s == RS) { s = 0; ph ^= 1; }
        }
        if (elect_one()) umma_commit<CG>(&bars->accfull, pair_mask);   // arrives once all issued MMAs completed
        __syncwarp();
        }
    mma_done:;
    } else {
        // ================================= FT =================================
        // What[0] = w0 + w1, What[1] = w0 - w1 for the stage's NK k x 16 depth
        // entries.  FT warp w owns ring slot w (w < S): it takes the whole
        // stages ch = c_lo + w, c_lo + w + S, ... (all FT items of a stage: IPT
        // per lane), so S stages are in flight on the FT side at once: warps
        // splitting every stage in lockstep put the whole LDS -> STS -> proxy
        // fence round trip (~400-700 cycles, WINRS_TC2_TRACE) on each stage's
        // critical path.  One warp per slot keeps the ring safe by construction:
        // slot w is refilled only after the MMAs of this warp's previous stage
        // in it, so its parity wait can never see a phase two rounds ahead.
        constexpr int KO = L::NKL / 8;              // k octets of this CTA's What rows
        constexpr int IPT = KO * KC / 32;           // items per lane: 8 (NK 128) / 4 (NK 64 or a pair)
        static_assert(TA || L::S <= NTXK, "one FT warp per ring slot");
        const int tw = warp - 2;
        if constexpr (TA) {
            // Two groups of four warps take alternate stages (group G: slots
            // s = G, G + 2, ...); warp q = warp % 4 of a group owns TMEM lanes
            // 32q..32q+31 = A rows (fh slot / channel half q / 2, channels
            // 32 (q % 2) ..), the only lanes it may write.  Per 16-row half:
            // four ldmatrix.x4.trans (x0..x3) give each thread two channels x
            // four depth entries of every column, already in the 16x256b
            // fragment order (matrix i: channel octet o0 + i/2, depth rows
            // permuted so that lane t/4's columns 2(t%4), 2(t%4)+1 hold depth
            // entries 4(t%4)..4(t%4)+3, i.e. column j = entries 2j, 2j+1); the
            // IT runs on the packed registers and 4 stores fill the slot's
            // xi = 0..3 A columns.  Ring safety as below: slot s is refilled
            // only after the MMAs of this group's previous stage in it.
            static_assert(ASEP || L::S % NG == 0, "TA: each FT group owns every NG-th ring slot");
            const int G = tw >> 2, q = warp & 3;
            const int i4 = lane >> 3, rho = lane & 7;
            const int img = 4 * (rho >> 1) + (rho & 1) + 2 * (i4 & 1);
            uint32_t xoff[2];
#pragma unroll
            for (int hf = 0; hf < 2; ++hf) {
                const int oct = 4 * (q & 1) + 2 * hf + (i4 >> 1);
                // row of (image img, column 0); columns are 8 rows (1 KB) apart
                const uint32_t row = (uint32_t)((q >> 1) * L::X_GRP + (img >> 3) * L::XT_HI + (img & 7) * 128);
                xoff[hf] = row + (uint32_t)((oct ^ ((row >> 7) & 7)) << 4);   // stages are 1 KB aligned
            }
            const uint32_t trow = tmem + ((uint32_t)(q * 32) << 16) + A_COL;
            // lanes of an fh slot past the last filter row: no X, no IT (their A
            // rows stay stale; the rows they feed are never written out)
            const bool xdead = F == 2 && fh_base + (q >> 1) >= g.R;
            const int it = q * 32 + lane;           // FT item: depth it / KO, k octet it % KO (KO * KC = 128)
            const uint32_t foff = opoff(it % KO, it / KO, L::Y_LBO);
            int s = G;
            uint32_t ph = 0;
            for (int ch = c_lo + G; ch < c_hi; ch += NG) {
                // odd ring depth (ASEP, S = 9): a group meets each slot every other
                // round, so first wait for the other group's stage in this slot to be
                // through (its opfull): the full wait below then never sees a phase
                // two rounds old (parity aliasing)
                if (ASEP && ch - c_lo >= L::S)
                    mbar_wait(&bars->opfull[s], (uint32_t)(((ch - c_lo - L::S) / L::S) & 1));
                mbar_wait(&bars->full[s], ph);
                tc_after();
                TC2_JITTER(ch, warp);
                if (tw == 0 && lane == 0) TC2_TRACE(ch - c_lo, 2);
                const uint32_t st = sbase + (uint32_t)(s * RSTAGE);
                const int aslot = asep ? (ch - c_lo) % 8 : s;
                if (asep && ch - c_lo >= 8)   // the MMAs of stage ch - 8 read this A slot
                    mbar_wait(&bars->aempty[aslot], (uint32_t)(((ch - c_lo) / 8 - 1) & 1));
#pragma unroll
                for (int hf = 0; hf < 2 && !xdead; ++hf) {
                    uint32_t x[4][4];
#pragma unroll
                    for (int c = 0; c < 4; ++c) ldsm_x4_t(st + xoff[hf] + c * 1024, x[c]);
                    uint32_t o[4][4];
#pragma unroll
                    for (int r = 0; r < 4; ++r) {
                        o[0][r] = P16<BF>::add(x[1][r], x[2][r]);
                        o[1][r] = P16<BF>::sub(x[2][r], x[1][r]);
                        o[2][r] = P16<BF>::sub(x[0][r], x[2][r]);
                        o[3][r] = P16<BF>::sub(x[3][r], x[1][r]);
                    }
                    const uint32_t ta = trow + ((uint32_t)(hf * 16) << 16) + (uint32_t)(aslot * 32);
#ifndef WINRS_TC2_NO_STTM   // debug ablation: no TMEM stores of the A operand (the MMAs read stale A)
#if WINRS_TC2_STX4
                    tmem_st16x256_x4(ta, o);   // the slot's four xi slabs are 4 consecutive 8-column chunks
#else
#pragma unroll
                    for (int xi = 0; xi < 4; ++xi) tmem_st16x256(ta + xi * 8, o[xi]);
#endif
#else
                    asm volatile("" :: "r"(o[0][0] ^ o[1][1] ^ o[2][2] ^ o[3][3] ^ ta));
#endif
                }
                const uint4 w0 = lds16(st + OFFY + foff), w1 = lds16(st + OFFY + L::ATOM + foff);
                sts16(st + OFFF + foff, vadd<BF>(w0, w1));
                sts16(st + OFFF + L::ATOM + foff, vsub<BF>(w0, w1));
                tmem_wait_st();
                fence_async();
                tc_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&bars->opfull[s]);
                if (tw == 0 && lane == 0) TC2_TRACE(ch - c_lo, 3);
                s += NG;
                if (s >= RS) { s -= RS; ph ^= 1; }
            }
        } else {
        uint32_t ph = 0;
        for (int ch = c_lo + tw; tw < L::S && ch < c_hi; ch += L::S) {
            const int s = tw;
            mbar_wait(&bars->full[s], ph);
            ph ^= 1;
            TC2_JITTER(ch, warp);
            if (tw == 0 && lane == 0) TC2_TRACE(ch - c_lo, 2);
            const uint32_t st = sbase + (uint32_t)(s * L::STAGE);
            if (!WINRS_TC2_ITM) {
                // IT in place: item (row octet o, depth d) reads x0..x3 of its 8 rows
                // and overwrites them with Xhat = (x1 + x2, x2 - x1, x0 - x2, x3 - x1)
                // (no other item touches those bytes); 256 items, 8 per lane, in
                // two batches of 4 to bound the live registers.
#pragma unroll
                for (int bt = 0; bt < 2; ++bt) {
                    uint4 xv[4][4];
                    uint32_t xo[4];
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        const int t = (bt * 4 + i) * 32 + lane;     // depth t / 16, row octet t % 16
                        const int o = t & 15;
                        xo[i] = st + (uint32_t)((o >> 3) * L::X_LBO) + opoff(o & 7, t >> 4, 0);
#pragma unroll
                        for (int c = 0; c < 4; ++c) xv[i][c] = lds16(xo[i] + c * L::ATOM);
                    }
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        sts16(xo[i], vadd<BF>(xv[i][1], xv[i][2]));
                        sts16(xo[i] + L::ATOM, vsub<BF>(xv[i][2], xv[i][1]));
                        sts16(xo[i] + 2 * L::ATOM, vsub<BF>(xv[i][0], xv[i][2]));
                        sts16(xo[i] + 3 * L::ATOM, vsub<BF>(xv[i][3], xv[i][1]));
                    }
                }
            }
            uint4 w0[IPT], w1[IPT];
            uint32_t off[IPT];
#pragma unroll
            for (int i = 0; i < IPT; ++i) {
                const int t = i * 32 + lane;        // item: depth t / KO, k octet t % KO
                off[i] = opoff(t % KO, t / KO, L::Y_LBO);
                w0[i] = lds16(st + L::OFF_Y + off[i]);
                w1[i] = lds16(st + L::OFF_Y + L::ATOM + off[i]);
            }
#pragma unroll
            for (int i = 0; i < IPT; ++i) {
#ifndef WINRS_TC2_NO_STS   // debug ablation: no operand stores
                sts16(st + L::OFF_F + off[i], vadd<BF>(w0[i], w1[i]));
                sts16(st + L::OFF_F + L::ATOM + off[i], vsub<BF>(w0[i], w1[i]));
#endif
            }
            fence_async();     // generic-proxy stores -> visible to the tensor core (async proxy)
            __syncwarp();
            if (lane == 0) {
                if (CG == 2) mbar_arrive_cluster(&bars->opfull[s], leader);
                else mbar_arrive(&bars->opfull[s]);
            }
            if (tw == 0 && lane == 0) TC2_TRACE(ch - c_lo, 3);
        }
        }
        // ============================ epilogue ================================
        mbar_wait(&bars->accfull, 0);
        tc_after();
        if (threadIdx.x == 64) TC2_TRACE(511, 2);
        const int q = warp & 3;                      // TMEM lane quarter of this warp
        constexpr int NPART = NTXK / 4;              // k column parts (one per group of four warps)
        const int half = (warp - 2) >> 2;            // this warp's k part
        const int m = q * 32 + lane;
        const int fh = fh_base + m / L::BC;
        const int c = c_base + m % L::BC;
        const bool row_ok = fh < g.R && c < g.C;
        float* Out = reinterpret_cast<float*>(smem);  // staging [s][k][m] (overlays the idle ring)
        const uint32_t lane_base = tmem + ((uint32_t)(q * 32) << 16);
#pragma unroll 1
        for (int k0 = half * (NK / NPART); k0 < (half + 1) * (NK / NPART); k0 += 8) {
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
                    Out[(0 * NK + k0 + i) * MROWS + m] = y0;
                    Out[(1 * NK + k0 + i) * MROWS + m] = y1;
                    Out[(2 * NK + k0 + i) * MROWS + m] = y2;
                } else {
                    const int k = cc.kb * NK + k0 + i;
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
    if (threadIdx.x == 64) TC2_TRACE(511, 3);
    if (g.csplit > 1) {
        // ---- deterministic cluster reduction: rank r sums rows (s, k) of its
        // slice over ranks 0..cs-1 in order (dsmem_sum4) and writes them.
        constexpr int ROWS = NSOUT * NK, M4 = MROWS / 4;
        cluster_sync_all();
        if (threadIdx.x == 64) TC2_TRACE(511, 4);
        const int r_lo = ROWS * rank / g.csplit, r_hi = ROWS * (rank + 1) / g.csplit;
        const uint32_t out_s = sbase;
        for (int p = r_lo * M4 + (int)threadIdx.x; p < r_hi * M4; p += NTHK) {
            const int row = p / M4, m4 = p % M4;
            const int sidx = row / NK, kl = row % NK;
            const float4 acc = dsmem_sum4(out_s + (uint32_t)((row * MROWS + m4 * 4) * 4), g.csplit, CG, e);
            const int m = m4 * 4;
            const int fh = fh_base + m / L::BC, c = c_base + m % L::BC, k = cc.kb * NK + kl;
            if (fh < g.R && c < g.C && k < g.K)
                *reinterpret_cast<float4*>(bucket + (((long long)k * g.R + fh) * g.S + fw0 + sidx) * g.C + c) = acc;
        }
        if (threadIdx.x == 64) TC2_TRACE(511, 5);
        cluster_sync_all();
    }
    if (threadIdx.x == 64) TC2_TRACE(511, 6);
    if (CG == 2 && g.csplit <= 1) cluster_sync_all();   // the pair's MMAs wrote both TMEMs
    if (warp == 1) {
        tc_after();
        if constexpr (CG == 2)
            asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" :: "r"(tmem), "r"(L::TMEM_COLS));
        else
            asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(tmem), "r"(TMEM_ALLOC));
    }
}


// ============================================================================
// Swapped CTA pair ("v2s"): the same computation with the operand roles
// exchanged.  M = 256 What rows (k: 128 per CTA), N = 128 Xhat columns
// (c: 64 per CTA), cta_group::2.  In a pair the B operand is shared, so each
// SM now fetches and transforms only HALF of the X side -- the expensive side
// (4 window columns and the 4-output IT per channel against 2 columns and 2
// computed outputs for What): per SM and 16-deep stage 16 KB of TMA fill, 16 KB
// of IT and 16 KB of FT traffic instead of 24 + 32 + 16 KB for one CTA
// (§6.4: the shared-memory port bounds the stage).  For K >= 256 tiles
// (ResNet-50 L3 / L4, VGG-16 conv3-5).
struct LaySw {
    static constexpr int ATOM = KC * 128;                // 2 KB: 64 channels x 16 depth rows
    static constexpr int OFF_X = 0;                      // X columns x0..x3 of this CTA's 64 c: [col][n]
    static constexpr int OFF_Y = 4 * ATOM;               // raw dY columns: [k atom 0/1][w0, w1][n]
    static constexpr int Y_LBO = 2 * ATOM;               // 4 KB between the two k atoms
    static constexpr int OFF_F = OFF_Y + 2 * Y_LBO;      // What[0], What[1]: same shape
    static constexpr int STAGE = OFF_F + 2 * Y_LBO;      // 24 KB
    static constexpr int S = 8;
    static constexpr int RING = S * STAGE;               // 192 KB
    static constexpr int OUT_LD = 128 + 4;               // staging row stride (floats): float4 stores of 8
                                                         // lanes on consecutive k rows hit distinct banks
    static constexpr int OUT = NSOUT * 128 * OUT_LD * 4;  // staging [s][k 128][c 128 (+4)] fp32, 198 KB
    static constexpr int BAR_OFF = RING > OUT ? RING : OUT;
    static constexpr int BYTES = BAR_OFF + 512 + 1024;
    static constexpr int TX_BYTES = OFF_F;               // 16 KB per stage
    static constexpr int TMEM_COLS = 512;                // 4 xi x N = 128
    static_assert(BYTES <= 227 * 1024, "smem");
};

template <bool BF>
__global__ void __launch_bounds__(NTHREADS, 1)
bfc_tc2s_kernel(const __grid_constant__ Args args, const __grid_constant__ CUtensorMap tmX,
                const __grid_constant__ CUtensorMap tmY) {
    using L = LaySw;
    constexpr int NN = 128;                              // UMMA N (c per pair)
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw_s = su(smem_raw);
    uint8_t* smem = smem_raw + (((raw_s + 1023u) & ~1023u) - raw_s);
    const uint32_t sbase = su(smem);
    Bars* bars = reinterpret_cast<Bars*>(smem + L::BAR_OFF);
    const Geometry& g = args.g;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 64) TC2_TRACE(511, 0);

    const int crank = (int)cluster_rank();
    const int e = crank & 1;
    const int rank = crank >> 1;                         // depth-split rank
    const uint32_t leader = (uint32_t)(crank & ~1);
    const uint16_t pair_mask = (uint16_t)(3u << leader);
    const CtaCoord cc = decode_cta(g, blockIdx.x / (2 * g.csplit));
    const int k_base = cc.kb * 256 + e * 128;            // this CTA's What rows (TMEM lanes)
    const int c_base = cc.cb * 128 + e * 64;             // this CTA's half of the Xhat columns
    const int fh = cc.fh;
    const int seg = cc.band * g.seg_cols + cc.col;
    float* bucket = seg == 0 ? args.dW : args.ws + (long long)(seg - 1) * g.dw_elems;
    int hs, he, w_first, units;
    group_rows(g, cc.band, cc.fh, &hs, &he);
    seg_units(g, cc.col, &w_first, &units);
    const long long depth = (long long)(he > hs ? he - hs : 0) * units * g.N;
    int c_lo, c_hi;
    split_chunks((int)((depth + KC - 1) / KC), rank, g.csplit, &c_lo, &c_hi);
    const bool empty_range = c_hi <= c_lo;
    const int fw0 = cc.ft * NSOUT;

    if (threadIdx.x == 0) {
        for (int s = 0; s < L::S; ++s) {
            mbar_init(&bars->full[s], 1);
            mbar_init(&bars->opfull[s], e == 0 ? 2 : 1);   // the leader gathers both CTAs' FT warps
            mbar_init(&bars->empty[s], 1);
        }
        mbar_init(&bars->accfull, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 0 && lane == 0) {
        asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(&tmX)) : "memory");
        asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(&tmY)) : "memory");
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;"
                     :: "r"(su(&bars->tmem_base)), "r"(L::TMEM_COLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
    }
    tc_before();
    __syncthreads();
    cluster_sync_all();
    tc_after();
    if (threadIdx.x == 0) pdl_trigger();
    const uint32_t tmem = bars->tmem_base;
    if (threadIdx.x == 64) TC2_TRACE(511, 1);

    if (warp == 0 || warp == PW2) {
        // ---- TMA (warp 0: even stages, warp PW2: odd stages): X columns x0..x3
        // of this CTA's 64 channels; dY w0, w1 of its 128 k
        const int pp = warp == 0 ? 0 : 1;
        long long d = (long long)(c_lo + pp) * KC;
        int n = 0, h = hs, u = 0;
        if (d < depth) depth_nhu((int)d, g.N, units, hs, &n, &h, &u);
        ImgTracker itk;
        itk.init(g, n);
        const int xdt = (g.T > 1 || g.D > 1) ? fh / g.Rh - g.pad : 0;   // per CTA, not per stage
        const int xdr = fh < g.R ? fh % g.Rh - g.pad : -(1 << 20);
        int s = pp;
        uint32_t ph = 0;
        for (int ch = c_lo + pp; ch < c_hi; ch += 2) {
            mbar_wait(&bars->empty[s], ph ^ 1);
            TC2_JITTER(ch, 0);
            TC2_TRACE(ch - c_lo, 0);
            uint64_t* fb = &bars->full[s];
            const uint32_t st = sbase + (uint32_t)(s * L::STAGE);
            const bool in = d < depth;
            const ImgCoord ic = itk.at(g, in);
            const int hh = in ? h : hs;
            const int w0 = w_first + (in ? u : 0) * 2;
            if (elect_one()) {
                mbar_expect_tx(fb, (uint32_t)L::TX_BYTES);
                tma5(st + L::OFF_X, &tmX, fb, c_base, ic.a + xdt, ic.b, hh + xdr, w0 + fw0 - g.pad);
                tma5(st + L::OFF_Y, &tmY, fb, k_base, ic.a, ic.b, hh, w0);
                tma5(st + L::OFF_Y + L::Y_LBO, &tmY, fb, k_base + 64, ic.a, ic.b, hh, w0);
            }
            __syncwarp();
            TC2_TRACE(ch - c_lo, 1);
            d += 2 * KC;
            n += 2 * KC;
            bool wrapped = false;
            while (n >= g.N) {
                n -= g.N;
                wrapped = true;
                if (++u == units) { u = 0; ++h; }
            }
            itk.advance(2 * KC, wrapped, n);
            s += 2;
            if (s >= L::S) { s -= L::S; ph ^= 1; }
        }
    } else if (warp == 1) {
        // ---- MMA (the pair's leader): D[xi] (256 k x 128 c) += What[xi] . Xhat[xi]
        if (e == 0) {
            int s = 0;
            uint32_t ph = 0;
            for (int ch = c_lo; ch < c_hi; ++ch) {
                mbar_wait(&bars->opfull[s], ph);
                TC2_JITTER(ch, 1);
                TC2_TRACE(ch - c_lo, 4);
                tc_after();
                const uint32_t st = sbase + (uint32_t)(s * L::STAGE);
                const uint32_t acc = ch > c_lo ? 1u : 0u;
                const uint64_t a0 = desc_sw128(st + L::OFF_F, L::Y_LBO, 1024), a1 = a0 + (L::ATOM >> 4);
                const uint64_t a2 = desc_sw128(st + L::OFF_Y, L::Y_LBO, 1024), a3 = a2 + (L::ATOM >> 4);
                const uint64_t b0 = desc_sw128(st + L::OFF_X, 8 * 1024, 1024);
                if (elect_one()) {
#ifndef WINRS_TC2_NO_MMA
                    umma<NN, BF, false, 2>(tmem + 0 * NN, a0, b0, acc);
                    umma<NN, BF, false, 2>(tmem + 1 * NN, a1, b0 + (L::ATOM >> 4), acc);
                    umma<NN, BF, false, 2>(tmem + 2 * NN, a2, b0 + (2 * L::ATOM >> 4), acc);
                    umma<NN, BF, false, 2>(tmem + 3 * NN, a3, b0 + (3 * L::ATOM >> 4), acc);
#else
                    (void)a0; (void)a1; (void)a2; (void)a3; (void)b0; (void)acc;
#endif
                    umma_commit<2>(&bars->empty[s], pair_mask);
                }
                __syncwarp();
                TC2_TRACE(ch - c_lo, 5);
                if (++s == L::S) { s = 0; ph ^= 1; }
            }
            if (elect_one()) umma_commit<2>(&bars->accfull, pair_mask);
            __syncwarp();
        }
    } else {
        // ---- FT warp w owns ring slot w: IT in place over its 64 c (4 items/lane),
        // FT What[0,1] = w0 +- w1 over its 128 k (8 items/lane)
        const int tw = warp - 2;
        uint32_t ph = 0;
        for (int ch = c_lo + tw; ch < c_hi; ch += L::S) {
            const int s = tw;
            mbar_wait(&bars->full[s], ph);
            ph ^= 1;
            TC2_JITTER(ch, warp);
            if (lane == 0) TC2_TRACE(ch - c_lo, 2);
            const uint32_t st = sbase + (uint32_t)(s * L::STAGE);
            {
                uint4 xv[4][4];
                uint32_t xo[4];
#pragma unroll
                for (int i = 0; i < 4; ++i) {
                    const int t = i * 32 + lane;                // depth t / 8, c octet t % 8
                    xo[i] = st + L::OFF_X + opoff(t & 7, t >> 3, 0);
#pragma unroll
                    for (int c = 0; c < 4; ++c) xv[i][c] = lds16(xo[i] + c * L::ATOM);
                }
#pragma unroll
                for (int i = 0; i < 4; ++i) {
                    sts16(xo[i], vadd<BF>(xv[i][1], xv[i][2]));
                    sts16(xo[i] + L::ATOM, vsub<BF>(xv[i][2], xv[i][1]));
                    sts16(xo[i] + 2 * L::ATOM, vsub<BF>(xv[i][0], xv[i][2]));
                    sts16(xo[i] + 3 * L::ATOM, vsub<BF>(xv[i][3], xv[i][1]));
                }
            }
            {
                uint4 w0[8], w1[8];
                uint32_t off[8];
#pragma unroll
                for (int i = 0; i < 8; ++i) {
                    const int t = i * 32 + lane;                // depth t / 16, k octet t % 16
                    off[i] = opoff(t & 15, t >> 4, L::Y_LBO);
                    w0[i] = lds16(st + L::OFF_Y + off[i]);
                    w1[i] = lds16(st + L::OFF_Y + L::ATOM + off[i]);
                }
#pragma unroll
                for (int i = 0; i < 8; ++i) {
                    sts16(st + L::OFF_F + off[i], vadd<BF>(w0[i], w1[i]));
                    sts16(st + L::OFF_F + L::ATOM + off[i], vsub<BF>(w0[i], w1[i]));
                }
            }
            fence_async();
            __syncwarp();
            if (lane == 0) mbar_arrive_cluster(&bars->opfull[s], leader);
            if (lane == 0) TC2_TRACE(ch - c_lo, 3);
        }
        // ---- epilogue: TMEM lane = k, columns = xi * 128 + c (c of the whole pair)
        mbar_wait(&bars->accfull, 0);
        tc_after();
        if (threadIdx.x == 64) TC2_TRACE(511, 2);
        const int q = warp & 3;
        const int half = (warp - 2) >> 2;                // c half of the 128 columns
        const int kl = q * 32 + lane;                    // local k row
        const int k = k_base + kl;
        float* Out = reinterpret_cast<float*>(smem);      // staging [s][kl][c 128 (+4)]
        const uint32_t lane_base = tmem + ((uint32_t)(q * 32) << 16);
#pragma unroll 1
        for (int cl0 = half * 64; cl0 < half * 64 + 64; cl0 += 8) {
            float v[4][8];
            if (!empty_range) {
#pragma unroll
                for (int x = 0; x < 4; ++x) tmem_ld8(lane_base + (uint32_t)(x * NN + cl0), v[x]);
                tmem_wait_ld();
            } else {
#pragma unroll
                for (int x = 0; x < 4; ++x)
#pragma unroll
                    for (int i = 0; i < 8; ++i) v[x][i] = 0.f;
            }
            float y[3][8];
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                const float sp = 0.5f * (v[0][i] + v[1][i]);
                y[0][i] = sp + v[2][i];
                y[1][i] = 0.5f * (v[0][i] - v[1][i]);
                y[2][i] = sp + v[3][i];
            }
            // pair column cl -> channel: CTA e' holds c_pair [e' * 64, e' * 64 + 64)
            const int cg = cc.cb * 128 + cl0;
#pragma unroll
            for (int j = 0; j < 3; ++j) {
                if (g.csplit > 1) {
                    float4* o = reinterpret_cast<float4*>(Out + (j * 128 + kl) * L::OUT_LD + cl0);
                    o[0] = make_float4(y[j][0], y[j][1], y[j][2], y[j][3]);
                    o[1] = make_float4(y[j][4], y[j][5], y[j][6], y[j][7]);
                } else if (k < g.K && cg < g.C && fh < g.R) {   // C % 8 == 0: octets all in or all out
                    float4* o = reinterpret_cast<float4*>(bucket + (((long long)k * g.R + fh) * g.S + fw0 + j) * g.C + cg);
                    o[0] = make_float4(y[j][0], y[j][1], y[j][2], y[j][3]);
                    o[1] = make_float4(y[j][4], y[j][5], y[j][6], y[j][7]);
                }
            }
        }
    }
    tc_before();
    __syncthreads();
    if (threadIdx.x == 64) TC2_TRACE(511, 3);
    if (g.csplit > 1) {
        // ---- depth-split reduction over the ranks with the same pair half e
        constexpr int ROWS = NSOUT * 128, C4 = 128 / 4;
        cluster_sync_all();
        if (threadIdx.x == 64) TC2_TRACE(511, 4);
        const int r_lo = ROWS * rank / g.csplit, r_hi = ROWS * (rank + 1) / g.csplit;
        for (int p = r_lo * C4 + (int)threadIdx.x; p < r_hi * C4; p += NTHREADS) {
            const int row = p / C4, c4 = p % C4;
            const int j = row / 128, kl = row % 128;
            const float4 acc = dsmem_sum4(sbase + (uint32_t)((row * L::OUT_LD + c4 * 4) * 4), g.csplit, 2, e);
            const int k = k_base + kl, c = cc.cb * 128 + c4 * 4;
            if (k < g.K && c < g.C && fh < g.R)
                *reinterpret_cast<float4*>(bucket + (((long long)k * g.R + fh) * g.S + fw0 + j) * g.C + c) = acc;
        }
        if (threadIdx.x == 64) TC2_TRACE(511, 5);
        cluster_sync_all();
    } else {
        cluster_sync_all();
    }
    if (threadIdx.x == 64) TC2_TRACE(511, 6);
    if (warp == 1) {
        tc_after();
        asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" :: "r"(tmem), "r"(L::TMEM_COLS));
    }
}

}  // namespace tc2
}  // namespace winrs
