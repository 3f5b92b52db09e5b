// Host planner: the three-step configuration adaptation of PAPER.md §4
// (P@20113-28371), integer-only and deterministic, restricted to the kernel
// instantiations present in the registry.
//
//   1. Fastest kernel pair (§4.1 P@20377, criteria (1)-(3), Figure 5): n0 and
//      n1 divide F_W; k0*r0 + k1*r1 covers O_W (the last unit may carry
//      zero-masked columns, R6); minimal Winograd-domain EWM work
//      sum k_i*alpha_i*(S/n_i)/tau_i (R7).
//   2. Baseline segment count Z^ (§4.2 Algorithm 1; the unspecified functions
//      are read as in DESIGN.md R8).
//   3. Segment shape S^_H x S^_W and the final segment count (§4.3 Algorithm 2,
//      eq. (5); readings R9, R10).
//
// Debug overrides (tests only): WINRS_FORCE_Z=<z>, WINRS_FORCE_TILE=<bn>x<bm>, WINRS_FORCE_CSPLIT=<1|2|4|8>,
// WINRS_FORCE_PAIR=a0,n0,r0,a1,n1,r1, WINRS_TC_GEN=1|2 (tensor-core kernel generation), WINRS_FORCE_CG=1|2.  Policy: WINRS_WS_CAP=<fraction> replaces the
// 4% workspace cap (R11).
#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>
#include "planner.h"

namespace winrs {

static long long cdiv(long long a, long long b) { return (a + b - 1) / b; }

struct PairChoice {
    const KernelEntry* proto = nullptr;   // any entry of the pair (tile chosen later)
    int k0 = 0, k1 = 0, masked = 0;
    double cost = 0;
};

// "Throughput coefficients" tau (P@20823): relative efficiency of a kernel on
// B200.  Default 1 (pure alpha-count model, R7).
static double tau(int /*alpha*/, int /*n*/, int /*r*/) { return 1.0; }

static bool same_pair(const KernelEntry& a, const KernelEntry& b) {
    return a.dtype == b.dtype && a.a0 == b.a0 && a.n0 == b.n0 && a.r0 == b.r0 && a.a1 == b.a1 &&
           a.n1 == b.n1 && a.r1 == b.r1;
}

static bool parse_force_pair(int out[6]) {
    const char* s = getenv("WINRS_FORCE_PAIR");
    if (!s || !*s) return false;
    return sscanf(s, "%d,%d,%d,%d,%d,%d", &out[0], &out[1], &out[2], &out[3], &out[4], &out[5]) == 6;
}

// The paper's ordering of pair candidates: least cost, then fewest masked
// columns, more bulk units, larger alpha0, smaller alpha1.
static bool pair_better(const PairChoice& cur, bool have, double c, int masked, int k0, const KernelEntry& e) {
    if (!have) return true;
    if (c != cur.cost) return c < cur.cost;
    if (masked != cur.masked) return masked < cur.masked;
    if (k0 != cur.k0) return k0 > cur.k0;
    if (e.a0 != cur.proto->a0) return e.a0 > cur.proto->a0;
    return e.a1 < cur.proto->a1;
}

// Step 1: kernel-pair selection.  `best` receives the paper's choice; `all`
// (optional) every valid pair with its own best (k0, k1) split.
static bool choose_pair(const Problem& p, const KernelEntry* es, int ne, PairChoice* best,
                        std::vector<PairChoice>* all = nullptr) {
    int forced[6];
    const bool force = parse_force_pair(forced);
    bool found = false;
    for (int i = 0; i < ne; ++i) {
        const KernelEntry& e = es[i];
        if (e.dtype != p.dtype) continue;
        bool dup = false;   // evaluate each pair once (tile variants share it)
        for (int j = 0; j < i; ++j)
            if (same_pair(es[j], e)) { dup = true; break; }
        if (dup) continue;
        if (force && !(e.a0 == forced[0] && e.n0 == forced[1] && e.r0 == forced[2] && e.a1 == forced[3] &&
                       e.n1 == forced[4] && e.r1 == forced[5]))
            continue;
        if (p.S % e.n0 != 0) continue;                       // criterion (1)
        if (e.a1 && (p.S % e.n1 != 0 || e.n0 % e.n1 != 0)) continue;
        PairChoice local;
        bool lfound = false;
        auto consider = [&](int k0, int k1, int masked) {
            const double c = k0 * (double)e.a0 * (p.S / e.n0) / tau(e.a0, e.n0, e.r0) +
                             (e.a1 ? k1 * (double)e.a1 * (p.S / e.n1) / tau(e.a1, e.n1, e.r1) : 0.0);
            if (pair_better(local, lfound, c, masked, k0, e)) {
                local.proto = &e;
                local.k0 = k0; local.k1 = k1; local.masked = masked; local.cost = c;
                lfound = true;
            }
        };
        if (e.a1 == 0) {
            const int k0 = (int)cdiv(p.Wo, e.r0);             // criterion (2) with masking
            consider(k0, 0, k0 * e.r0 - p.Wo);
        } else {
            for (int k0 = p.Wo / e.r0; k0 >= 1; --k0) {
                const int rem = p.Wo - k0 * e.r0;
                if (rem <= 0) continue;
                const int k1 = (int)cdiv(rem, e.r1);
                const int masked = k1 * e.r1 - rem;
                consider(k0, k1, masked);
            }
        }
        if (!lfound) continue;
        if (all) all->push_back(local);
        if (pair_better(*best, found, local.cost, local.masked, local.k0, e)) {
            *best = local;
            found = true;
        }
    }
    return found;
}

// Step 2: Algorithm 1 (R8).
static int alg1(const Problem& p, const KernelEntry& e, int num_sms, int* zmax_out) {
    const long long b2 = cdiv(p.K, e.bn) * cdiv(p.C, e.bm) * (long long)p.R * (p.S / e.n0);
    const long long b0 = cdiv(p.K, 64) * cdiv((long long)p.N * cdiv(p.Ho, 2) * cdiv(p.Wo, 2), 32);
    const long long b1 = cdiv(p.C, 64) * cdiv((long long)p.N * cdiv(p.H, 2) * cdiv(p.W, 2), 32);
    double zh = (double)(b0 + b1) / (1.45 * (double)b2);                          // line 1
    const long long bhat2 = (long long)e.occ * num_sms;                             // line 2
    const double esz = p.dtype == 0 ? 4.0 : 2.0;
    const double data = esz * ((double)p.N * p.H * p.W * p.C + (double)p.N * p.Ho * p.Wo * p.K);
    const double dw_bytes = 4.0 * (double)p.K * p.R * p.S * p.C;
    double cap = 0.04;                                   // R11: workspace <= 4% of X+dY bytes
    if (const char* c = getenv("WINRS_WS_CAP")) {       // policy knob (fraction of X+dY bytes)
        const double v = atof(c);
        if (v > 0) cap = v;
    }
    const int zmax = 1 + (int)std::floor(cap * data / dw_bytes);
    *zmax_out = zmax;
    if (zh < 2.0 && b2 >= bhat2) return 1;                                          // line 3
    const long long z1 = cdiv(2LL * e.occ * num_sms, b2);                          // line 4
    const double direct = 2.0 * p.N * p.C * p.K * (double)p.Ho * p.Wo * p.R * p.S;
    const long long z2 = std::max(1LL, (long long)std::floor(direct / 1073741824.0));   // line 5
    const long long z3 = std::max(1LL, (long long)p.N * p.Ho * p.Wo / 512);
    long long z = std::min(std::min((long long)std::ceil(zh), z1), std::min(z2, z3));   // line 6
    if (z < 1) z = 1;
    long long P = 1;                                                                // line 7
    while (P < z) P <<= 1;
    if (P > 8) P = 8;
    z = P * cdiv(z, P);
    if (z > zmax) z = zmax;
    return (int)std::max(1LL, z);
}

// Step 3: Algorithm 2 on the Omega_a0 region (width k0*r0, W_max = k0 units).
static void alg2(const Problem& p, int r0, int k0, int z, int* z_used, int* seg_h, int* seg_w) {
    const int Ho = p.Ho;
    const int Hmax = p.pad > 0 ? std::max(1, Ho / p.pad) : Ho;
    const int Wmax = k0;
    z = std::min<long long>(z, (long long)Hmax * Wmax);                            // line 1
    if (z < 1) z = 1;
    *z_used = z;
    int sh, sw;
    if (z == 1) {                                                                   // line 2
        sh = Ho; sw = k0 * r0;
    } else if (z >= Wmax) {                                                         // line 3
        // S^_H ~ Ho*W_max/Z^; the band count floor(Ho/S^_H) is rounded to the
        // nearest integer of Z^/W_max instead of truncated (R9).
        const long long nb = std::max(1LL, ((long long)z + Wmax / 2) / Wmax);
        sh = (int)(Ho / nb); sw = r0;
    } else if (Wmax % z == 0) {                                                     // line 4
        sh = Ho; sw = r0 * (Wmax / z);
    } else {                                                                        // lines 5-7
        const int lo = (int)cdiv(Wmax, z), hi = (int)((long long)Hmax * Wmax / z);
        int x = 0;
        for (int c = lo; c <= hi && c <= Wmax; ++c)
            if (Wmax % c == 0) { x = c; break; }
        if (x) { sh = (int)((long long)Ho * Wmax / ((long long)z * x)); sw = x * r0; }
        else { sh = Ho; sw = k0 * r0; }
    }
    *seg_h = std::min(std::max(sh, 1), Ho);
    *seg_w = std::max(sw, r0);
}

static void fill_geometry(const Problem& p, const KernelEntry& e, const PairChoice& pc, int seg_h, int seg_w,
                          Geometry* g) {
    memset(g, 0, sizeof(*g));
    g->N = p.N; g->C = p.C; g->H = p.H; g->W = p.W; g->K = p.K; g->R = p.R; g->S = p.S; g->pad = p.pad;
    g->Ho = p.Ho; g->Wo = p.Wo;
    g->ldy = p.K;
    g->a0 = e.a0; g->n0 = e.n0; g->r0 = e.r0; g->k0 = pc.k0;
    g->seg_h = seg_h;
    g->bands = std::max(1, p.Ho / seg_h);
    g->seg_w = seg_w;
    g->seg_cols = (int)cdiv((long long)pc.k0 * e.r0, seg_w);
    g->a1 = e.a1; g->n1 = e.n1; g->r1 = e.r1; g->k1 = pc.k1;
    g->res_col0 = pc.k0 * e.r0;
    g->tile_k = e.bn; g->tile_c = e.bm;
    g->kblocks = (int)cdiv(p.K, e.bn);
    g->cblocks = (int)cdiv(p.C, e.bm);
    g->ftiles = p.S / e.n0;
    g->fhs = e.fhs > 0 ? e.fhs : 1;
    g->cg = e.cg > 0 ? e.cg : 1;
    g->fhg = (int)cdiv(p.R, g->fhs);
    g->Z = g->bands * g->seg_cols;
    g->csplit = 1;
    g->chunk = p.dtype == 0 ? 8 : 16;
    g->dw_elems = (long long)p.K * p.R * p.S * p.C;
    g->Rh = p.Rh > 0 ? p.Rh : p.R;
    g->T = p.T;
    g->D = p.D;
    g->Do = p.Do;
    g->Nb = p.Nb > 0 ? p.Nb : p.N;
}

// Fewest chunks any tile of the Omega_a0 phase walks (its segment's clipped
// rows x units x N / chunk).
static long long min_tile_chunks(const Geometry& g) {
    long long best = -1;
    for (int band = 0; band < g.bands; ++band)
        for (int fh = 0; fh < g.R; fh += g.fhs) {
            int hs, he;
            group_rows(g, band, fh, &hs, &he);
            for (int col = 0; col < g.seg_cols; ++col) {
                int wf, units;
                seg_units(g, col, &wf, &units);
                const long long d = (long long)(he - hs) * units * g.N;
                const long long c = (d + g.chunk - 1) / g.chunk;
                if (c > 0 && (best < 0 || c < best)) best = c;
            }
        }
    return best < 0 ? 0 : best;
}

// B200 time model used to pick the CTA tile, the segment count Z and the
// cluster split, fitted by tools/fit_model.py to a
// tools/sweep.py calibration run on B200 (profiles/r01/planner_fit.md).  It
// simulates the block scheduler: a CTA (cluster) costs
//   D[cs > 1] + max over ranks (F + chunks0 * T0 + jobs * (J + chunks1 * T1)),
// T_a = a * chunk * BN * BM * 2 / rate (its Winograd-domain EWM flops at the
// tile's sustained per-SM rate), and clusters are list-scheduled in launch
// order onto the free slots (cs = 4 / 8 clusters: the measured resident
// cluster counts).  Z > 1 adds the bucket reduction launch.
struct TimeModel {
    double fixed_s;    // F: per-CTA prologue, pipeline fill, OT, epilogue
    double rate_sm;    // EWM FLOP/s of one CTA (one CTA per SM)
};
struct SharedModel {
    double job_s;       // J: per residual job (OT + job boundary)
    double cluster_s;   // D: per-cluster DSMEM reduction / barriers
    double reduce_s;    // fixed cost of the bucket-reduce launch
    double reduce_bw;   // its bytes/s over (2Z) * |dW| fp32
    double slots4, slots8;   // resident 4- / 8-CTA clusters on 148 SMs
};

static TimeModel time_model(const KernelEntry& e) {
    const int dtype = e.dtype, bn = e.bn, bm = e.bm;
    if (e.fhs > 0 && e.ta == 3)   // stream-K xi-split pairs, all 74 pairs busy (tools/ab_sk.sh); F = 2 tiles
        return {0.0, e.fhs == 2 ? 11.0e12 : 11.46e12};   // carry the dead fh slot (VGG conv2_1: 312 vs TA 329 us)
    if (e.fhs > 0 && e.ta == 2)   // bfc_tc2x.cuh xi-split pair (128 k x 128 rows, Xhat in TMEM): rate of the
        // pair over its tile (tools/ab_xs.sh: VGG conv4_2 cs = 1, 3136 stages per pair in 508 us); the
        // F = 2 tiles carry the dead fh slot of R = 3 through every MMA (VGG conv2_1: 343 vs TA 331 us)
        return {4.0e-6, e.fhs == 2 ? 12.4e12 : 13.2e12};
    if (e.fhs > 0 && e.cg == 2 && bn == 256)   // swapped CTA pair (256 k x 128 c): X side shared
        return {4.5e-6, 12.6e12};              // (re-fitted with two producer warps: tools/sweep_tc2.py)
    if (e.fhs > 0 && e.cg == 2)   // bfc_tc2.cuh CTA pair: rate of the pair over its 256-row tile
        return {4.5e-6, 11.0e12};
    if (e.fhs > 0 && e.tf32)   // bfc_tc3.cuh: FP32 inputs, 12 tf32 MMAs per 8-deep stage (3xTF32)
        return {4.0e-6, bn >= 128 ? 1.45e12 : 1.05e12};   // tools/tc3_check.py --time: NK = 128 ~1.4x per flop
    if (e.fhs > 0 && e.ta)   // bfc_tc2.cuh TA (Xhat in TMEM, NK = 64, two TMA producer warps):
        return {4.0e-6, 5.6e12};   // tools/ta_ab.py: VGG L1 988 -> 644 us, R50 L1 57.3 -> 44.0 us
    if (e.fhs > 0) {
        // bfc_tc2.cuh, rate over the whole 128-row UMMA tile (fhs filter rows).
        // Measured on B200 (tools/trace_tc2.py, WINRS_TC2_TRACE): a 16-deep stage
        // takes ~820 cycles at NK = 128 and ~600 at NK = 64 -- the shared-memory
        // port (~128 B/clk: 8 MMAs' operand reads + TMA fill + FT traffic,
        // DESIGN.md §6.4); fixed = setup + pipeline fill + epilogue.
        if (bn >= 128) return {4.5e-6, 5.5e12};
        return {4.0e-6, 3.4e12};
    }
    if (dtype != 0 && !e.cc16) {
        if (bm >= 128) return {11.02e-6, 3.095e12};
        if (bm >= 64) return {6.19e-6, 1.545e12};
        return {3.80e-6, 0.812e12};
    }
    if (bn * bm >= 4096) return {7.12e-6, 3.49e11};
    if (bn * bm >= 2048) return {5.61e-6, 2.59e11};
    return {4.02e-6, 1.95e11};
}
static SharedModel shared_model(int dtype) {
    if (dtype != 0) return {2.02e-6, 2.13e-6, 8.3e-6, 7.86e12, 33.1, 14.0};   // reduce_s: 10.8 us before the PDL launch (ablations/ab_pdl.txt: -2..4 us)
    return {0.0, 2.01e-6, 20.8e-6, 2.0e13, 34.8, 15.6};
}

// Resident cluster slots for a cluster size on num_sms SMs.
static long long cluster_slots(int cs, int occ, int num_sms, const SharedModel& sm) {
    const double f = (double)num_sms / 148.0;
    long long s;
    if (cs > 8) return std::max(1LL, (long long)(occ * 8 * f));   // 16-CTA clusters: one per GPC
    if (cs == 1) s = (long long)occ * num_sms;
    else if (cs == 2) s = (long long)occ * num_sms / 2;
    else if (cs == 4) s = (long long)(occ * sm.slots4 * f);
    else if (cs == 8) s = (long long)(occ * sm.slots8 * f);
    else s = (long long)(occ * 0.9 * num_sms / cs);   // 3, 6: clusters within a GPC, some SMs stranded
    return std::max(1LL, s);
}

static double model_time(const Geometry& g, const KernelEntry& e, int num_sms) {
    const TimeModel m = time_model(e);
    if (e.ta == 3) {
        // stream-K pairs (bfc_tc2x.cuh SK): every co-resident pair takes an equal share
        // of the concatenated tile depths; each tile part ends with the pair's OT /
        // DSMEM reduction and a read-add-write of dW in the chain order.
        long long chunks = 0;
        for (int band = 0; band < g.bands; ++band)
            for (int col = 0; col < g.seg_cols; ++col)
                for (int fh = 0; fh < g.R; fh += g.fhs) {
                    int hs, he, wf, units;
                    group_rows(g, band, fh, &hs, &he);
                    seg_units(g, col, &wf, &units);
                    chunks += (long long)g.kblocks * g.cblocks * g.ftiles *
                              (((long long)(he - hs) * units * g.N + g.chunk - 1) / g.chunk);
                }
        // Fitted on B200 (tools/ab_sk.sh, profiles/r02/ablations/ab_sk3.txt): ~183 ns per
        // chunk per pair with every pair busy, ~9 us per tile part a pair walks (ring
        // fill, OT, DSMEM pair reduction) and ~6.5 us per step of a tile's chain.
        const double pairs = std::max(1.0, std::min((double)chunks, std::floor(num_sms / 2.0)));
        const double part_s = 9.0e-6, step_s = 6.5e-6;
        const double per_chunk = (double)g.chunk * e.bn * e.bm * e.fhs * 2.0 * g.a0 / m.rate_sm;
        const double tiles = (double)num_tiles(g);
        const double parts = 1.0 + std::ceil(tiles / pairs), chain = 1.0 + std::ceil(pairs / tiles);
        // (long chains -- few tiles -- also leave the middle parts waiting: +3 us per step past 4)
        double t = m.fixed_s + std::ceil(chunks / pairs) * per_chunk + parts * part_s + chain * step_s +
                   std::max(0.0, chain - 4.0) * 3.0e-6;
        if (g.Z > 1) {   // the segments' buckets are summed by the reduction launch
            const SharedModel sh = shared_model(e.dtype);
            t += sh.reduce_s + 2.0 * g.Z * (double)g.dw_elems * 4.0 / sh.reduce_bw;
        }
        return t;
    }
    SharedModel sh = shared_model(e.cc16 ? 0 : e.dtype);
    const int fhs = e.fhs > 0 ? e.fhs : 1;
    const double per_chunk = (double)g.chunk * e.bn * e.bm * fhs * 2.0 / m.rate_sm;
    if (e.fhs > 0)   // rank skew + DSMEM reduction of the n0 x 128 x 128 (per SM) FP32 output tile (~20 B/clk/SM)
        sh.cluster_s = 1.5e-6 + (double)g.n0 * (e.bn > 128 ? 128 : e.bn) * 128 * 4 / 30e9;
    const double t0 = g.a0 * per_chunk, t1 = (g.a1 ? g.a1 : 1) * per_chunk;
    const long long mult = (long long)g.kblocks * g.cblocks * g.ftiles;
    const int jobs_res = g.a1 ? g.n0 / g.n1 : 0;
    const long long slots = cluster_slots(g.csplit * g.cg, e.occ, num_sms, sh) ;
    // min-heap of slot free times (list scheduling in launch order: band, col, fh outer; kb fastest)
    std::vector<double> heap((size_t)slots, 0.0);
    auto push_root = [&](double v) {   // replace the minimum (root) by v and sift down
        size_t k = 0;
        const size_t n = heap.size();
        for (;;) {
            size_t l = 2 * k + 1, r = l + 1, s = k;
            double sv = v;
            if (l < n && heap[l] < sv) { s = l; sv = heap[l]; }
            if (r < n && heap[r] < sv) { s = r; sv = heap[r]; }
            if (s == k) break;
            heap[k] = heap[s];
            k = s;
        }
        heap[k] = v;
    };
    for (int band = 0; band < g.bands; ++band)
        for (int col = 0; col < g.seg_cols; ++col)
            for (int fh = 0; fh < g.R; fh += g.fhs) {
                int hs, he, wf, units;
                group_rows(g, band, fh, &hs, &he);
                seg_units(g, col, &wf, &units);
                const long long rows = he - hs;
                const long long cm = (rows * units * g.N + g.chunk - 1) / g.chunk;
                const bool res = has_residual(g, col);
                const long long cr = res ? (rows * g.k1 * g.N + g.chunk - 1) / g.chunk : 0;
                double t = 0;
                for (int r = 0; r < g.csplit; ++r) {
                    const long long a = cm * (r + 1) / g.csplit - cm * r / g.csplit;
                    const long long b = cr * (r + 1) / g.csplit - cr * r / g.csplit;
                    const double tr = m.fixed_s + a * t0 + (res ? jobs_res * (sh.job_s + b * t1) : 0.0);
                    t = std::max(t, tr);
                }
                if (g.csplit > 1 || e.ta == 2) t += sh.cluster_s;   // xi-split: always a pair reduction
                for (long long q = 0; q < mult; ++q) push_root(heap[0] + t);
            }
    double mk = 0;
    for (double v : heap) mk = std::max(mk, v);
    if (g.Z > 1) mk += sh.reduce_s + 2.0 * g.Z * (double)g.dw_elems * 4.0 / sh.reduce_bw;
    return mk;
}

// Cluster depth splits a kernel may run.  The round-1 FP16 kernel (bfc_f16.cuh)
// keeps its round-1 set {1, 2, 4}: with 3, 6 or 8 ranks it fails
// intermittently at large depth (VGG-16 conv2_2, N = 128: an unspecified launch
// failure within 12-24 calls; not reproducible under compute-sanitizer,
// DESIGN.md §10).  The tc2 and FP32 kernels take {1, 2, 3, 4, 6, 8}.
static bool cs_allowed(const KernelEntry& e, int cs) {
    if (cs == 1) return true;
    if (!e.csplit_ok) return false;
    if ((cs == 5 || cs == 7) && e.fhs <= 0) return false;   // 5 / 7 ranks: tc2 / tc3 kernels only
    if (e.cg == 2 && cs > 4) return false;                  // CTA pairs: clusters of 2 x cs <= 8 CTAs
    if (e.ta == 3) return false;                            // stream-K pairs: no cluster depth split
    if (e.dtype != 0 && e.fhs <= 0 && !e.cc16) return cs == 2 || cs == 4;
    return true;
}

static int forced_csplit() {
    if (const char* f = getenv("WINRS_FORCE_CSPLIT")) {
        const int v = atoi(f);
        if (v >= 1 && v <= 8) return v;
    }
    return 0;
}

// Winograd-domain EWM flops the kernels issue (clipped rows, masked columns
// counted as work): 2*K*C*N * sum_{fh, band} rows_valid * (units*alpha*S/n).
static double ewm_flops(const Geometry& g) {
    double tot = 0;
    for (int band = 0; band < g.bands; ++band)
        for (int fh = 0; fh < g.R; ++fh) {
            int hs, he;
            band_rows(g, band, fh, &hs, &he);
            const double rows = he - hs;
            double per_row = (double)g.k0 * g.a0 * (g.S / g.n0);
            if (g.a1 && g.k1) per_row += (double)g.k1 * g.a1 * (g.S / g.n1);
            tot += rows * per_row;
        }
    return 2.0 * g.K * g.C * (double)g.N * tot;
}

// Steps 2-3 for one CTA tile.  Algorithm 1 gives Z^ (reported as z_hat);
// on B200 the planner then evaluates every segment count Z <= Z_max (the
// workspace cap, R11) through Algorithm 2 and every cluster split, and keeps
// the (Z, cs) of least model time (R19).  WINRS_PLANNER=paper keeps
// Algorithm 1's Z^ (only cs is searched).
static double plan_with_tile(const Problem& p, const KernelEntry& e, const PairChoice& pc, int num_sms,
                             PlanResult* out) {
    int zmax = 1;
    const int z_alg1 = alg1(p, e, num_sms, &zmax);
    int z_lo = 1, z_hi = zmax;
    const char* mode = getenv("WINRS_PLANNER");
    if (mode && strcmp(mode, "paper") == 0) z_lo = z_hi = std::min(z_alg1, zmax);
    if (const char* fz = getenv("WINRS_FORCE_Z")) {
        const int v = atoi(fz);
        if (v >= 1) { z_lo = z_hi = v; zmax = 1 << 30; }
    }

    int zhat_used = 1, sh0 = p.Ho, sw0 = pc.k0 * e.r0;
    alg2(p, e.r0, pc.k0, std::min(z_alg1, zmax), &zhat_used, &sh0, &sw0);
    const int fcs = forced_csplit();
    const long long zlimit = (long long)std::max(1, p.pad > 0 ? p.Ho / p.pad : p.Ho) * pc.k0;   // alg2 line 1
    if (z_hi > zlimit) z_hi = (int)std::max<long long>(z_lo, zlimit);
    double best_t = 1e30;
    bool have = false;
    int last_bands = -1, last_cols = -1, last_sh = -1, last_sw = -1;
    for (int z = z_lo; z <= z_hi; ++z) {
        int z_used = 1, seg_h = p.Ho, seg_w = pc.k0 * e.r0;
        alg2(p, e.r0, pc.k0, z, &z_used, &seg_h, &seg_w);
        Geometry g;
        fill_geometry(p, e, pc, seg_h, seg_w, &g);
        if (g.Z > zmax && z > 1) continue;   // workspace cap (R11)
        if (z > z_lo && num_tiles(g) > 32LL * e.occ * num_sms) break;   // > 32 waves: per-CTA cost dominates
        if (g.bands == last_bands && g.seg_cols == last_cols && seg_h == last_sh && seg_w == last_sw) continue;
        last_bands = g.bands; last_cols = g.seg_cols; last_sh = seg_h; last_sw = seg_w;
        const long long mc = min_tile_chunks(g);
        for (int cs : {1, 2, 3, 4, 5, 6, 7, 8}) {
            if (cs == 7 && fcs != cs) continue;   // 7 ranks: measured slower everywhere (tools/sweep_tc2.py --cs57)
            if (!cs_allowed(e, cs)) continue;   // never launch a cluster the kernel cannot reduce (even if forced)
            if (e.cg == 2 && cs > 4) continue;   // 16-CTA clusters (pairs x 8): ~half the clusters co-resident (measured 2x slower)
            if (fcs ? cs != fcs : (cs > 1 && mc < cs)) continue;
            g.csplit = cs;
            const double t = model_time(g, e, num_sms);
            if (!have || t < best_t * (1.0 - 1e-9)) {
                best_t = t;
                have = true;
                out->geom = g;
            }
        }
    }
    if (!have) {   // forced values that the loop filtered: plan Z^ with cs = 1 (or forced)
        int z_used = 1, seg_h = p.Ho, seg_w = pc.k0 * e.r0;
        alg2(p, e.r0, pc.k0, z_lo, &z_used, &seg_h, &seg_w);
        fill_geometry(p, e, pc, seg_h, seg_w, &out->geom);
        out->geom.csplit = fcs && cs_allowed(e, fcs) ? fcs : 1;
        best_t = model_time(out->geom, e, num_sms);
    }
    out->entry = &e;
    out->z_hat = zhat_used;
    out->masked = pc.masked;
    return best_t;
}

static int parse_force_tile(int* bn, int* bm) {
    const char* s = getenv("WINRS_FORCE_TILE");
    if (!s || !*s) return 0;
    return sscanf(s, "%dx%d", bn, bm) == 2;
}

winrs_status_t make_plan(const Problem& p, int num_sms, PlanResult* out) {
    int ne = 0;
    const KernelEntry* es = kernel_entries(&ne);
    PairChoice pc;
    std::vector<PairChoice> pairs;
    if (!choose_pair(p, es, ne, &pc, &pairs)) return WINRS_ERR_UNSUPPORTED;
    // Step 1 with measured throughput (B200, R19): the paper's cost divides by
    // kernel-specific throughput coefficients tau (P@20823); here every valid
    // pair x compiled CTA tile is planned (Z, segments, cluster split) and
    // scored by the B200 time model, whose per-tile rates play tau's role.
    // WINRS_PLANNER=paper keeps the pure alpha-count pair choice.
    const char* mode = getenv("WINRS_PLANNER");
    if (mode && strcmp(mode, "paper") == 0) pairs.assign(1, pc);
    int fbn = 0, fbm = 0;
    const bool force_tile = parse_force_tile(&fbn, &fbm);
    PlanResult best;
    bool have = false;
    double best_t = 1e30;
    for (const PairChoice& cand : pairs) {
        std::vector<const KernelEntry*> tiles;
        for (int i = 0; i < ne; ++i)
            if (same_pair(es[i], *cand.proto)) tiles.push_back(&es[i]);
        std::sort(tiles.begin(), tiles.end(), [](const KernelEntry* a, const KernelEntry* b) {
            if (a->bn * a->bm != b->bn * b->bm) return a->bn * a->bm > b->bn * b->bm;
            return a->bn > b->bn;
        });
        for (const KernelEntry* e : tiles) {
            if (force_tile && (e->bn != fbn || e->bm != fbm)) continue;
            const bool nd = p.T > 1 || p.D > 1;
            // tcgen05 kernels: one 16-image (tc2) / 8-image (tc3, FP32) TMA box per stage
            if (e->fhs > 0 && (nd ? p.Do : p.N) % (e->tf32 ? 8 : 16) != 0) continue;
            if (e->fhs > 0 && p.N % (e->tf32 ? 8 : 16) != 0) continue;
            if (const char* v = getenv("WINRS_FP32_TC")) {   // debug: FP32 on the tensor cores only (1) / never (0)
                if (e->dtype == 0 && (atoi(v) != 0) != (e->tf32 != 0)) continue;
            }
            // N-D: the FP32 kernel, or the tc2 kernels (16 depth slices of one image per TMA box)
            if (nd && e->dtype != 0 && !e->cc16 && (e->fhs <= 0 || p.Do % 16 != 0)) continue;
            if (const char* v = getenv("WINRS_TC_GEN")) {   // debug: restrict to one tensor-core generation
                if (e->dtype != 0 && !e->cc16 && ((atoi(v) == 2) != (e->fhs > 0))) continue;
            }
            if (const char* v = getenv("WINRS_FORCE_CG")) {  // debug: tc2 CTA pair (2) or single CTA (1)
                if (e->fhs > 0 && atoi(v) != (e->cg > 0 ? e->cg : 1)) continue;
            }
            if (const char* v = getenv("WINRS_FORCE_TA")) {  // debug: tc2 with Xhat in SMEM (0), in TMEM (1),
                if (e->fhs > 0 && atoi(v) != e->ta) continue;  // or in TMEM with the xi split over a pair (2)
            }
            PlanResult r;
            const double t = plan_with_tile(p, *e, cand, num_sms, &r);
            if (!have || t < best_t * (1.0 - 1e-9)) { best = r; best_t = t; have = true; }
        }
    }
    if (!have) return WINRS_ERR_UNSUPPORTED;
    best.ewm_flops = ewm_flops(best.geom);
    best.model_s = best_t;
    *out = best;
    return WINRS_OK;
}

}  // namespace winrs
