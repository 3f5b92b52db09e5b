// xi-split FP16 / BF16 tensor-core WinRS BFC kernel for sm_100a ("v2x"),
// kernel Omega_4(3,2) (Figure 6, P@28451; F_W = 3 of the FP16 set,
// P@28616).  Same computation as bfc_tc2.cuh (§3 eq. (6),
// P@31000-32161; transforms of DESIGN.md R20):
//     FT  What = (w0 + w1, w0 - w1, w0, w1)
//     IT  Xhat = (x1 + x2, x2 - x1, x0 - x2, x3 - x1)
//     OT  y0 = (v0 + v1)/2 + v2,  y1 = (v0 - v1)/2,  y2 = (v0 + v1)/2 + v3
// but the four Winograd points xi of one tile are split over a CTA pair:
//     half e = 0: xi = 0, 1 (X columns x1, x2; What[0], What[1] = w0 +- w1)
//     half e = 1: xi = 2, 3 (X columns x0..x3; the raw dY columns w0, w1)
// Each CTA keeps only two accumulators in TMEM, so the tile can be NK = 128
// k wide with the transformed X operand still in TMEM (TA):
// 2 x 128 accumulator columns + an 8-slot ring of 2 x 8 A columns, and the
// A-from-TMEM MMAs run at N = 128 (~92 cycles, §6.5) instead of N = 64 (~84,
// bound by the 4 KB TMEM read of A, §6.4b).  The e = 0 half applies its FT by
// linearity in the tensor core (WINRS_TC2X_LIN, default): v0 += Xhat0 w0 +
// Xhat0 w1, v1 += Xhat1 w0 - Xhat1 w1 (negate-B bit) -- four MMAs on the raw
// w0, w1 and no FT stores / proxy fence on its critical path; e = 1 issues two.
// The pair moves 8 + 8 + 8 KB (e = 0: X fill, ldmatrix, dY fill) and
// 16 + 16 + 8 KB (e = 1) per stage through the shared-memory port (DESIGN.md
// §6.10).  On the stream-K schedule (SK = true, §6.11) one wave of pairs takes
// equal ranges of all tiles' depth chunks.
//
// The OT is linear in v, so each half applies its share of A^T to its own
// accumulators (e=0: y0 = y2 = (v0+v1)/2, y1 = (v0-v1)/2; e=1: y0 = v2,
// y1 = 0, y2 = v3) and the pair's partial tiles are summed with the cluster
// depth-split ranks in one deterministic DSMEM reduction (fixed cluster-rank
// order): cluster = 2 x csplit CTAs, rank = 2 * depth rank + e.
//
// Warp roles (352 threads, one CTA per SM), as in the TA kernel:
//   warps 0,10 TMA producers (even / odd stages)
//   warp 1     TMEM allocator + MMA issuer
//   warps 2-9  two groups of four FT warps taking alternate stages (warp q of
//              a group owns TMEM lanes 32q..32q+31), then the epilogue.
#pragma once
#include "bfc_tc2.cuh"

#ifndef WINRS_TC2X_BAL
#define WINRS_TC2X_BAL 2   // balanced split (e = 0: xi 0, 2 from x0..x2; e = 1: xi 1, 3 from x1..x3; three MMAs
                           // each, 21 KB stages, 10-deep rings on both halves): 0 never, 1 always, 2 for the F = 2
                           // tiles only (measured: VGG conv2_1 294 vs 310 us; slower on the F = 1 layers)
#endif
#ifndef WINRS_TC2X_S0
#define WINRS_TC2X_S0 12   // ring depth of the e = 0 half (17 KB stages without the FT region); e = 1: 8 x 25 KB
#endif
#ifndef WINRS_TC2X_LIN
#define WINRS_TC2X_LIN 1   // e = 0 half: What[0,1] = w0 +- w1 applied by the tensor core (four MMAs on the raw
                           // w0, w1 by linearity, negate-B for -w1) instead of the FT warps' stores (0: FT stores)
#endif

namespace winrs {
namespace tc2 {

template <int F>
struct LayX {
    static constexpr bool BAL = WINRS_TC2X_BAL == 1 || (WINRS_TC2X_BAL == 2 && F == 2);
    static constexpr int NK = 128;                       // k per tile (both halves)
    static constexpr int BC = MROWS / F;                 // channels per fh slot
    static constexpr int ATOM = KC * 128;                // 2 KB: 64 channels x 16 depth rows
    static constexpr int Y_LBO = 2 * ATOM;               // 4 KB: [k atom][w0, w1]
    // X (ldmatrix.trans only): per 64-channel atom two 8-image boxes, the upper
    // one two 128-byte rows further (conflict-free ldmatrix phases, §6.4a).
    //   e = 1: 4 columns x0..x3 per box (4 KB), e = 0: 2 columns x1, x2 (2 KB)
    static constexpr int X4_HI = 4096 + 256, X4_GRP = 2 * 4096 + 256;
    static constexpr int X2_HI = 2048 + 256, X2_GRP = 2 * X2_HI;
    static constexpr int OFF_Y0 = 9 * 1024;              // e = 0: X 9 KB, dY 8 KB, FT 8 KB
    static constexpr int OFF_F0 = OFF_Y0 + 2 * Y_LBO;
    static constexpr int OFF_Y1 = 17 * 1024;             // e = 1: X 17 KB, dY 8 KB
    static constexpr int STAGE = 25 * 1024;
    static constexpr int S = 8;
    static constexpr int RING = S * STAGE;               // 200 KB
    // e = 0 with the FT by linearity needs no FT region: 17 KB stages, a deeper ring
    static constexpr int STAGE0 = WINRS_TC2X_LIN ? 17 * 1024 : STAGE;
    static constexpr int S0 = WINRS_TC2X_LIN ? WINRS_TC2X_S0 : S;
    static constexpr int SMAX = BAL ? 10 : (S0 > S ? S0 : S);
    static constexpr int RING0 = S0 * STAGE0;
    static constexpr int OUT = NSOUT * NK * MROWS * 4;   // staging [s][k][m] fp32, 192 KB
    static constexpr int X3_HI = 3072 + 256, X3_GRP = 2 * X3_HI;   // balanced split: 3 columns per half
    static constexpr int OFF_Y3 = 13 * 1024, STAGE3 = 21 * 1024, S3 = 10, RING3 = S3 * STAGE3;
    static constexpr int TX3 = 4 * 3072 + 2 * Y_LBO;
    static constexpr int RINGM = BAL ? RING3 : (RING > RING0 ? RING : RING0);
    static constexpr int BAR_OFF = RINGM > OUT ? RINGM : OUT;
    static constexpr int BYTES = BAR_OFF + 512 + 1024;
    static_assert(SMAX <= 12 && 2 * NK + SMAX * 16 <= 512 && BYTES <= 227 * 1024, "ring / TMEM / smem budget");
    static constexpr int TX0 = 4 * 2048 + 2 * Y_LBO;     // TMA bytes per stage: 16 KB (e = 0)
    static constexpr int TX1 = 4 * 4096 + 2 * Y_LBO;     //                      24 KB (e = 1)
    static constexpr uint32_t A_COL = 2 * NK;            // first A ring column (after 2 x 128 accumulators)
    static_assert(OFF_F0 + 2 * Y_LBO == STAGE && OFF_Y1 + 2 * Y_LBO == STAGE, "stage layout");
    static_assert(2 * X2_GRP <= OFF_Y0 && 2 * X4_GRP - 256 <= OFF_Y1, "X regions");
    static_assert(A_COL + S * 16 <= 512, "TMEM");
    static_assert(BYTES <= 227 * 1024, "smem");
};

// The stream-K schedule helpers (SkTile, sk_find, ...) are in bfc_tc2.cuh.

template <int F, bool BF, bool SK = false>
__global__ void __launch_bounds__(tc2_threads<true>(), 1)
bfc_tc2x_kernel(const __grid_constant__ Args args, const __grid_constant__ CUtensorMap tmX4,
                const __grid_constant__ CUtensorMap tmX2, const __grid_constant__ CUtensorMap tmY) {
    using L = LayX<F>;
    constexpr int NK = L::NK;
    constexpr int NTHK = tc2_threads<true>();
    constexpr int PW2K = 2 + NTX_TA;                     // second producer warp
    constexpr int NG = NTX_TA / 4;                       // FT groups
    static_assert(L::S % NG == 0 && L::S0 % NG == 0 && L::S3 % NG == 0, "each FT group owns every NG-th ring slot");
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw_s = su(smem_raw);
    uint8_t* smem = smem_raw + (((raw_s + 1023u) & ~1023u) - raw_s);
    const uint32_t sbase = su(smem);
    Bars* bars = reinterpret_cast<Bars*>(smem + L::BAR_OFF);
    const Geometry& g = args.g;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 64) TC2_TRACE(511, 0);

    const int crank = (int)cluster_rank();               // cluster = 2 x csplit CTAs (SK: one pair)
    const int nranks = 2 * g.csplit;
    const int e = crank & 1;                             // xi half
    const int rank = crank >> 1;                         // depth-split rank
    // per-half stage layout
    const int x_hi = L::BAL ? L::X3_HI : (e ? L::X4_HI : L::X2_HI);
    const int x_grp = L::BAL ? L::X3_GRP : (e ? L::X4_GRP : L::X2_GRP);
    const int off_y = L::BAL ? L::OFF_Y3 : (e ? L::OFF_Y1 : L::OFF_Y0);
    const int RS = L::BAL ? L::S3 : (e ? L::S : L::S0);          // this half's ring depth and stage size
    const uint32_t RSTAGE = L::BAL ? (uint32_t)L::STAGE3 : (e ? (uint32_t)L::STAGE : (uint32_t)L::STAGE0);

    if (threadIdx.x == 0) {
        for (int s = 0; s < L::SMAX; ++s) {
            mbar_init(&bars->full[s], 1);
            mbar_init(&bars->opfull[s], 4);              // the four lane-quarter warps of a group
            mbar_init(&bars->empty[s], 1);
        }
        mbar_init(&bars->accfull, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 0 && lane == 0) {
        asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(e ? &tmX4 : &tmX2)) : "memory");
        asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(&tmY)) : "memory");
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                     :: "r"(su(&bars->tmem_base)), "r"(512));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_before();
    __syncthreads();
    tc_after();
    if (threadIdx.x == 0) pdl_trigger();
    const uint32_t tmem = bars->tmem_base;
    if (threadIdx.x == 64) TC2_TRACE(511, 1);

    // ---- the pieces this CTA works on: one (tile, depth-rank range) without
    // SK; with SK the tiles (or tile parts) of this pair's chunk range
    const int P = SK ? args.sk_pairs : 1;
    // SK pair index = a ticket taken in dispatch order (rank 0 of the cluster takes
    // it, rank 1 reads it over DSMEM): every lower pair is already running when a
    // pair starts, so waiting only on lower pairs is safe whatever the residency.
    int pair = 0;
    if constexpr (SK) {
        uint32_t* slot = reinterpret_cast<uint32_t*>(&bars->accfull) + 3;   // spare word after tmem_base
        if (crank == 0 && threadIdx.x == 0)   // arrival order; the last pair to finish resets the counters
            *slot = atomicAdd(args.sk_flags + SK_TICKET, 1u) % (unsigned)P;
        cluster_sync_all();
        uint32_t remote, v;
        asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(su(slot)), "r"(0));
        asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(remote) : "memory");
        pair = (int)v;
        cluster_sync_all();   // rank 0's slot is not reused before rank 1 read it
    }
    const long long tot = SK ? sk_total(g) : 1;
    // SK: the pair walks its range BACKWARDS (the head of its last tile first), and
    // a tile's parts are combined in increasing pair order: the pair holding the
    // tile's first chunks stores (that part is its first piece, done early), each
    // higher pair adds when its turn comes (its part of the tile is its last
    // piece).  A pair only ever waits for LOWER pairs, which are dispatched no
    // later than it, so the chain needs no co-residency guarantee.
    const long long gbeg = SK ? sk_start(tot, pair, P) : 0;
    long long gcur = SK ? sk_start(tot, pair + 1, P) : 1;   // exclusive end of the part still to do
    for (int piece = 0;; ++piece) {
        long long tile;
        int c_lo, c_hi, order = 0;
        if constexpr (SK) {
            if (gcur <= gbeg) break;
            const SkTile st = sk_find(g, gcur - 1);
            tile = st.t;
            c_lo = (int)(max(st.g0, gbeg) - st.g0);
            c_hi = (int)(gcur - st.g0);
            order = pair - sk_pair_of(tot, st.g0, P);   // 0: the pair holding the tile's first chunks
            gcur -= c_hi - c_lo;
            if (piece > 0) {   // the previous piece drained: every barrier is quiescent
                if (threadIdx.x == 0) {
                    for (int s = 0; s < L::SMAX; ++s) {
                        asm volatile("mbarrier.inval.shared::cta.b64 [%0];" :: "r"(su(&bars->full[s])) : "memory");
                        asm volatile("mbarrier.inval.shared::cta.b64 [%0];" :: "r"(su(&bars->opfull[s])) : "memory");
                        asm volatile("mbarrier.inval.shared::cta.b64 [%0];" :: "r"(su(&bars->empty[s])) : "memory");
                        mbar_init(&bars->full[s], 1);
                        mbar_init(&bars->opfull[s], 4);
                        mbar_init(&bars->empty[s], 1);
                    }
                    asm volatile("mbarrier.inval.shared::cta.b64 [%0];" :: "r"(su(&bars->accfull)) : "memory");
                    mbar_init(&bars->accfull, 1);
                    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
                }
                tc_before();
                __syncthreads();
                tc_after();
            }
        } else {
            if (piece > 0) break;
            tile = blockIdx.x / nranks;
        }
        if (SK && threadIdx.x == 64 && piece < 3) TC2_TRACE(490 + piece * 6, 0);
        const CtaCoord cc = decode_cta(g, tile);
        const int fh_base = cc.fh;
        const int c_base = F == 2 ? cc.cb * 64 : cc.cb * 128;
        const int k_base = cc.kb * NK;
        const int seg = cc.band * g.seg_cols + cc.col;
        float* bucket = seg == 0 ? args.dW : args.ws + (long long)(seg - 1) * g.dw_elems;
        int hs, he, w_first, units;
        group_rows(g, cc.band, cc.fh, &hs, &he);
        seg_units(g, cc.col, &w_first, &units);
        const long long depth = (long long)(he > hs ? he - hs : 0) * units * g.N;
        if constexpr (!SK) split_chunks((int)((depth + KC - 1) / KC), rank, g.csplit, &c_lo, &c_hi);
        const bool empty_range = c_hi <= c_lo;
        const int fw0 = cc.ft * NSOUT;
        if (warp == 0 || warp == PW2K) {
            // ============================ TMA producers ===========================
            const int pp = warp == 0 ? 0 : 1;
            const CUtensorMap* mx = e ? &tmX4 : &tmX2;
            const int xcol = L::BAL ? e : (e ? 0 : 1);   // first X window column loaded
            const uint32_t tx = L::BAL ? (uint32_t)L::TX3 : (e ? (uint32_t)L::TX1 : (uint32_t)L::TX0);
            long long d = (long long)(c_lo + pp) * KC;
            int n = 0, h = hs, u = 0;
            if (d < depth) depth_nhu((int)d, g.N, units, hs, &n, &h, &u);
            ImgTracker itk;
            itk.init(g, n);
            int xdt[2], xdr[2];
    #pragma unroll
            for (int a = 0; a < 2; ++a) {
                const int fh = F == 2 ? fh_base + a : fh_base;
                xdt[a] = (g.T > 1 || g.D > 1) ? fh / g.Rh - g.pad : 0;
                xdr[a] = fh < g.R ? fh % g.Rh - g.pad : -(1 << 20);   // a slot past the last filter row: zero fill
            }
            int s = pp;
            uint32_t ph = 0;
            for (int ch = c_lo + pp; ch < c_hi; ch += 2) {
                mbar_wait(&bars->empty[s], ph ^ 1);
                TC2_JITTER(ch, 0);
                TC2_TRACE(ch - c_lo, 0);
                uint64_t* fb = &bars->full[s];
                const uint32_t st = sbase + (uint32_t)s * RSTAGE;
                const bool in = d < depth;
                const ImgCoord ic = itk.at(g, in);
                const int hh = in ? h : hs;
                const int w0 = w_first + (in ? u : 0) * 2;
                if (elect_one()) {
                    mbar_expect_tx(fb, tx);
    #pragma unroll
                    for (int a = 0; a < 2; ++a) {
                        const int c0 = F == 2 ? c_base : c_base + a * 64;
                        const int wx = w0 + fw0 - g.pad + xcol;
                        tma5(st + a * x_grp, mx, fb, c0, ic.a + xdt[a], ic.b, hh + xdr[a], wx);
                        tma5(st + a * x_grp + x_hi, mx, fb, c0, ic.a + 8 + xdt[a], ic.b, hh + xdr[a], wx);
                    }
    #pragma unroll
                    for (int ka = 0; ka < 2; ++ka)
                        tma5(st + off_y + ka * L::Y_LBO, &tmY, fb, k_base + ka * 64, ic.a, ic.b, hh, w0);
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
            // B: e = 0 What[0], What[1] (FT region); e = 1 the raw w0, w1.
            const int off_b = L::BAL ? L::OFF_Y3 : (e ? L::OFF_Y1 : (WINRS_TC2X_LIN ? L::OFF_Y0 : L::OFF_F0));
            int s = 0;
            uint32_t ph = 0;
            for (int ch = c_lo; ch < c_hi; ++ch) {
                mbar_wait(&bars->opfull[s], ph);
                TC2_JITTER(ch, 1);
                TC2_TRACE(ch - c_lo, 4);
                tc_after();
                const uint32_t st = sbase + (uint32_t)s * RSTAGE;
                const uint32_t acc = ch > c_lo ? 1u : 0u;
                const uint64_t b0 = desc_sw128(st + off_b, L::Y_LBO, 1024), b1 = b0 + (L::ATOM >> 4);
                if (elect_one()) {
                    const uint32_t a = tmem + L::A_COL + (uint32_t)(s * 16);
                    if (L::BAL && e == 0) {   // v0 += Xhat0 (w0 + w1), v2 += Xhat2 w0
                        umma_ta<NK, BF>(tmem + 0, a + 0, b0, acc);
                        umma_ta<NK, BF>(tmem + 0, a + 0, b1, 1u);
                        umma_ta<NK, BF>(tmem + NK, a + 8, b0, acc);
                    } else if (L::BAL) {       // v1 += Xhat1 (w0 - w1), v3 += Xhat3 w1
                        umma_ta<NK, BF>(tmem + 0, a + 0, b0, acc);
                        umma_ta<NK, BF, true>(tmem + 0, a + 0, b1, 1u);
                        umma_ta<NK, BF>(tmem + NK, a + 8, b1, acc);
                    } else if (WINRS_TC2X_LIN && e == 0) {   // v0 += Xhat0 (w0 + w1), v1 += Xhat1 (w0 - w1)
                        umma_ta<NK, BF>(tmem + 0, a + 0, b0, acc);
                        umma_ta<NK, BF>(tmem + 0, a + 0, b1, 1u);
                        umma_ta<NK, BF>(tmem + NK, a + 8, b0, acc);
                        umma_ta<NK, BF, true>(tmem + NK, a + 8, b1, 1u);
                    } else {
                        umma_ta<NK, BF>(tmem + 0, a + 0, b0, acc);
                        umma_ta<NK, BF>(tmem + NK, a + 8, b1, acc);
                    }
                    umma_commit<1>(&bars->empty[s]);
                }
                __syncwarp();
                TC2_TRACE(ch - c_lo, 5);
                if (++s == RS) { s = 0; ph ^= 1; }
            }
            if (elect_one()) umma_commit<1>(&bars->accfull);
            __syncwarp();
        } else {
            // ================================= FT =================================
            // Group G takes stages G, G + NG, ...; warp q owns TMEM lanes 32q..
            // (A rows: fh slot / channel half q / 2, channels 32 (q % 2) ..).  Per
            // 16-row half, ldmatrix.x4.trans of the needed columns gives each
            // thread two channels x four depth entries in the tcgen05.st 16x256b
            // fragment order (bfc_tc2.cuh TA), the IT runs on the packed
            // registers and two stores fill the slot's two xi A columns.
            const int tw = warp - 2;
            const int G = tw >> 2, q = warp & 3;
            const int i4 = lane >> 3, rho = lane & 7;
            const int img = 4 * (rho >> 1) + (rho & 1) + 2 * (i4 & 1);
            uint32_t xoff[2];
    #pragma unroll
            for (int hf = 0; hf < 2; ++hf) {
                const int oct = 4 * (q & 1) + 2 * hf + (i4 >> 1);
                const uint32_t row = (uint32_t)((q >> 1) * x_grp + (img >> 3) * x_hi + (img & 7) * 128);
                xoff[hf] = row + (uint32_t)((oct ^ ((row >> 7) & 7)) << 4);   // stages are 1 KB aligned
            }
            const uint32_t trow = tmem + ((uint32_t)(q * 32) << 16) + L::A_COL;
            // FT items (e = 0): 16 k octets x 16 depth entries = 256 per stage, 2 per lane
            const int it0 = q * 32 + lane;
            const uint32_t foff0 = opoff(it0 % 16, it0 / 16, L::Y_LBO);
            const uint32_t foff1 = opoff((it0 + 128) % 16, (it0 + 128) / 16, L::Y_LBO);
            int s = G;
            uint32_t ph = 0;
            for (int ch = c_lo + G; ch < c_hi; ch += NG) {
                mbar_wait(&bars->full[s], ph);
                tc_after();
                TC2_JITTER(ch, warp);
                if (tw == 0 && lane == 0) TC2_TRACE(ch - c_lo, 2);
                const uint32_t st = sbase + (uint32_t)s * RSTAGE;
    #pragma unroll
                for (int hf = 0; hf < 2; ++hf) {
                    uint32_t o[2][4];
                    if (L::BAL) {   // box columns p0..p2 = x0..x2 (e = 0) / x1..x3 (e = 1)
                        uint32_t x[3][4];
#pragma unroll
                        for (int c = 0; c < 3; ++c) ldsm_x4_t(st + xoff[hf] + c * 1024, x[c]);
#pragma unroll
                        for (int r = 0; r < 4; ++r) {
                            if (e == 0) {
                                o[0][r] = P16<BF>::add(x[1][r], x[2][r]);   // Xhat0 = x1 + x2
                                o[1][r] = P16<BF>::sub(x[0][r], x[2][r]);   // Xhat2 = x0 - x2
                            } else {
                                o[0][r] = P16<BF>::sub(x[1][r], x[0][r]);   // Xhat1 = x2 - x1
                                o[1][r] = P16<BF>::sub(x[2][r], x[0][r]);   // Xhat3 = x3 - x1
                            }
                        }
                    } else if (e == 0) {
                        uint32_t x1[4], x2[4];
                        ldsm_x4_t(st + xoff[hf], x1);
                        ldsm_x4_t(st + xoff[hf] + 1024, x2);
    #pragma unroll
                        for (int r = 0; r < 4; ++r) {
                            o[0][r] = P16<BF>::add(x1[r], x2[r]);
                            o[1][r] = P16<BF>::sub(x2[r], x1[r]);
                        }
                    } else {
                        uint32_t x[4][4];
    #pragma unroll
                        for (int c = 0; c < 4; ++c) ldsm_x4_t(st + xoff[hf] + c * 1024, x[c]);
    #pragma unroll
                        for (int r = 0; r < 4; ++r) {
                            o[0][r] = P16<BF>::sub(x[0][r], x[2][r]);
                            o[1][r] = P16<BF>::sub(x[3][r], x[1][r]);
                        }
                    }
                    const uint32_t ta = trow + ((uint32_t)(hf * 16) << 16) + (uint32_t)(s * 16);
                    tmem_st16x256_x2(ta, o);
                }
                if (e == 0 && !WINRS_TC2X_LIN) {   // What[0] = w0 + w1, What[1] = w0 - w1 (128 k x 16 depth)
                    const uint32_t y = st + L::OFF_Y0, f = st + L::OFF_F0;
                    const uint4 a0 = lds16(y + foff0), a1 = lds16(y + L::ATOM + foff0);
                    const uint4 b0 = lds16(y + foff1), b1 = lds16(y + L::ATOM + foff1);
                    sts16(f + foff0, vadd<BF>(a0, a1));
                    sts16(f + L::ATOM + foff0, vsub<BF>(a0, a1));
                    sts16(f + foff1, vadd<BF>(b0, b1));
                    sts16(f + L::ATOM + foff1, vsub<BF>(b0, b1));
                }
                tmem_wait_st();
                fence_async();
                tc_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&bars->opfull[s]);
                if (tw == 0 && lane == 0) TC2_TRACE(ch - c_lo, 3);
                s += NG;
                if (s >= RS) { s -= RS; ph ^= 1; }
            }
            // ============================ epilogue ================================
            // This half's share of the OT into the staging tile [s][k][m]; e = 1
            // has no y1 term (its rows are skipped by the reduction).
            mbar_wait(&bars->accfull, 0);
            tc_after();
            if (threadIdx.x == 64) TC2_TRACE(511, 2);
            const int m = q * 32 + lane;
            float* Out = reinterpret_cast<float*>(smem);      // overlays the idle ring
            const uint32_t lane_base = tmem + ((uint32_t)(q * 32) << 16);
    #pragma unroll 1
            for (int k0 = G * (NK / NG); k0 < (G + 1) * (NK / NG); k0 += 8) {
                float va[8], vb[8];
                if (!empty_range) {
                    tmem_ld8(lane_base + (uint32_t)k0, va);
                    tmem_ld8(lane_base + (uint32_t)(NK + k0), vb);
                    tmem_wait_ld();
                } else {
    #pragma unroll
                    for (int i = 0; i < 8; ++i) va[i] = vb[i] = 0.f;
                }
    #pragma unroll
                for (int i = 0; i < 8; ++i) {
                    if (L::BAL) {   // e = 0: (v0 / 2 + v2, v0 / 2, v0 / 2); e = 1: (v1 / 2, -v1 / 2, v1 / 2 + v3)
                        const float h = 0.5f * va[i];
                        Out[(0 * NK + k0 + i) * MROWS + m] = e == 0 ? h + vb[i] : h;
                        Out[(1 * NK + k0 + i) * MROWS + m] = e == 0 ? h : -h;
                        Out[(2 * NK + k0 + i) * MROWS + m] = e == 0 ? h : h + vb[i];
                    } else if (e == 0) {
                        const float sp = 0.5f * (va[i] + vb[i]);
                        Out[(0 * NK + k0 + i) * MROWS + m] = sp;
                        Out[(1 * NK + k0 + i) * MROWS + m] = 0.5f * (va[i] - vb[i]);
                        Out[(2 * NK + k0 + i) * MROWS + m] = sp;
                    } else {
                        Out[(0 * NK + k0 + i) * MROWS + m] = va[i];
                        Out[(2 * NK + k0 + i) * MROWS + m] = vb[i];
                    }
                }
            }
        }
        tc_before();
        __syncthreads();
        if (threadIdx.x == 64) TC2_TRACE(511, 3);
        // ---- deterministic cluster reduction over the 2 x csplit ranks: cluster
        // rank r sums rows (s, k) of its slice over ranks 0..nranks-1 in order
        // (the y1 rows over the e = 0 ranks only) and writes them to the bucket.
        {
            constexpr int ROWS = NSOUT * NK, M4 = MROWS / 4;
            cluster_sync_all();
            if (threadIdx.x == 64) TC2_TRACE(511, 4);
            unsigned int* flag = SK ? args.sk_flags + tile : nullptr;
            const int r_lo = ROWS * crank / nranks, r_hi = ROWS * (crank + 1) / nranks;
            if constexpr (SK) {
                // 1. the pair's sum of this CTA's row slice, written back in place (only
                //    this CTA reads its own slice rows); 2. wait for this tile's chain
                //    turn; 3. read-add-write (or store, order 0) from shared memory.
                for (int p = r_lo * M4 + (int)threadIdx.x; p < r_hi * M4; p += NTHK) {
                    const int row = p / M4, m4 = p % M4;
                    const uint32_t addr = sbase + (uint32_t)((row * MROWS + m4 * 4) * 4);
                    const float4 acc = (!L::BAL && row / NK == 1) ? dsmem_sum4(addr, 1, 2, 0) : dsmem_sum4(addr, 2);
                    *reinterpret_cast<float4*>(smem + (size_t)(row * MROWS + m4 * 4) * 4) = acc;
                }
                if (threadIdx.x == 64 && piece < 3) TC2_TRACE(490 + piece * 6 + 1, 0);
                if (order > 0 && threadIdx.x == 0) {
                    const unsigned int want = (args.sk_epoch << 8) | (unsigned int)order;
                    const long long t0 = clock64();
                    while (ld_acquire(flag) != want) {
                        __nanosleep(64);
                        if (clock64() - t0 > 40000000000LL) __trap();   // ~20 s: a broken chain fails loudly, never hangs
                    }
                }
                __syncthreads();
                if (threadIdx.x == 64 && piece < 3) TC2_TRACE(490 + piece * 6 + 2, 0);
#pragma unroll 4
                for (int p = r_lo * M4 + (int)threadIdx.x; p < r_hi * M4; p += NTHK) {
                    const int row = p / M4, m4 = p % M4;
                    const int sidx = row / NK, kl = row % NK;
                    float4 acc = *reinterpret_cast<const float4*>(smem + (size_t)(row * MROWS + m4 * 4) * 4);
                    const int mm = m4 * 4;
                    const int fh = fh_base + mm / L::BC, c = c_base + mm % L::BC, k = k_base + kl;
                    if (fh < g.R && c < g.C && k < g.K) {
                        float4* o = reinterpret_cast<float4*>(bucket + (((long long)k * g.R + fh) * g.S + fw0 + sidx) * g.C + c);
                        if (order > 0) {   // the tile's earlier parts first, this part added last (fixed order)
                            const float4 prev = __ldcg(o);
                            acc = make_float4(prev.x + acc.x, prev.y + acc.y, prev.z + acc.z, prev.w + acc.w);
                        }
                        *o = acc;
                    }
                }
            } else {
                for (int p = r_lo * M4 + (int)threadIdx.x; p < r_hi * M4; p += NTHK) {
                    const int row = p / M4, m4 = p % M4;
                    const int sidx = row / NK, kl = row % NK;
                    const uint32_t addr = sbase + (uint32_t)((row * MROWS + m4 * 4) * 4);
                    const float4 acc = (!L::BAL && sidx == 1) ? dsmem_sum4(addr, g.csplit, 2, 0) : dsmem_sum4(addr, nranks);
                    const int mm = m4 * 4;
                    const int fh = fh_base + mm / L::BC, c = c_base + mm % L::BC, k = k_base + kl;
                    if (fh < g.R && c < g.C && k < g.K)
                        *reinterpret_cast<float4*>(bucket + (((long long)k * g.R + fh) * g.S + fw0 + sidx) * g.C + c) = acc;
                }
            }
            if (threadIdx.x == 64) TC2_TRACE(511, 5);
            if (SK) __threadfence();
            cluster_sync_all();
            if (SK && crank == 0 && threadIdx.x == 0) st_release(flag, (args.sk_epoch << 8) | (unsigned int)(order + 1));
            if (SK && threadIdx.x == 64 && piece < 3) {
                TC2_TRACE(490 + piece * 6 + 3, 0);
                TC2_TRACE(490 + piece * 6 + 4, 0);
#ifdef WINRS_TC2_TRACE
                if (blockIdx.x == (unsigned)g_tc2_trace_cta) { g_tc2_trace[490 + piece * 6 + 5][0] = order; g_tc2_trace[490 + piece * 6 + 5][1] = c_hi - c_lo; }
#endif
            }
        }
    }
    if (threadIdx.x == 64) TC2_TRACE(511, 6);
    if (SK && crank == 0 && threadIdx.x == 0) {   // every ticket is taken: the last pair out resets both counters
        if (atomicAdd(args.sk_flags + SK_TICKET + 1, 1u) == (unsigned)P - 1u) {
            atomicExch(args.sk_flags + SK_TICKET, 0u);
            atomicExch(args.sk_flags + SK_TICKET + 1, 0u);
        }
    }
    if (warp == 1) {
        tc_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(tmem), "r"(512));
    }
}

}  // namespace tc2
}  // namespace winrs
