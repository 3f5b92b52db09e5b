// Internal plan layout and the index math shared by the CUDA kernels and the
// host-side FP64 emulator (winrs_debug_emulate).  Not part of the public ABI.
//
// Geometry (§3 P@15252-17405, Figures 3/4; R6, R9, R10):
//   * dY columns [0, k0*r0) form the Omega_a0 region, split into `bands` row
//     bands (seg_h rows each, the last absorbs the remainder) and `seg_cols`
//     column segments of seg_w columns (the last may be narrower).  Segment
//     z = band*seg_cols + col writes dW bucket z (bucket 0 is dW itself).
//   * dY columns [k0*r0, k0*r0 + k1*r1) are the residual region handled by
//     Omega_a1 units; per band it is processed by the CTAs of the band's LAST
//     column segment as a second phase that adds into the same bucket, so no
//     extra workspace and no second launch is needed.  Columns >= Wo inside
//     the last unit are zero-masked (R6).
//   * CTA = (segment, fh group, fw-tile, c-block, k-block); it computes the
//     B_N x B_M x n0 tile dW_z[kb*B_N.., fh, ft*n0 .. ft*n0+n0, cb*B_M..] for
//     each filter row fh of its group.  A group is `fhs` consecutive filter
//     rows (1 for every kernel except the stacked tcgen05 kernel of
//     bfc_tc2.cuh, which puts 2 rows' X windows into one 128-row UMMA tile
//     when C <= 64).
//   * Height clipping (P@32013-33698, Figure 7): a CTA only visits dY rows h
//     whose X row h+fh-pad lies inside [0, H).
//   * Cluster split (B200 addition): the depth of one tile can
//     be split over `csplit` CTAs of a thread-block cluster; each computes a
//     partial output tile in shared memory and the cluster sums them through
//     distributed shared memory in fixed rank order (deterministic, no
//     workspace).  CTA = (cluster of csplit ranks) x (tile coordinate).
#pragma once
#include <stdint.h>
#include <stddef.h>

#if defined(__CUDACC__)
#define WINRS_HD __host__ __device__ __forceinline__
#else
#define WINRS_HD inline
#endif

namespace winrs {

struct KernelId {
    int alpha, n, r;
};

// Everything a launch needs; passed by value to the kernels (< 4 KB).
struct Geometry {
    int N, C, H, W, K, R, S, pad, Ho, Wo;
    int ldy;                    // dY pixel stride in elements (>= K; K-sharding passes a channel slice)
    // Omega_a0 region
    int a0, n0, r0, k0;
    int seg_h, bands, seg_w, seg_cols;
    // residual region (a1 == 0: none)
    int a1, n1, r1, k1;
    int res_col0;               // = k0 * r0
    // CTA tiling
    int tile_k, tile_c;         // B_N (k), B_M (c)
    int kblocks, cblocks, ftiles;   // ceil(K/B_N), ceil(C/B_M), S/n0
    int fhs, fhg;               // filter rows per CTA (fh group size) and groups ceil(R / fhs)
    int Z;                      // buckets
    int csplit;                 // depth-split ranks per tile (thread-block cluster), >= 1
    int cg;                     // CTAs per UMMA (2: a cta_group::2 pair per depth rank), >= 1
    int chunk;                  // depth entries per main-loop chunk (8 FP32, 16 FP16)
    long long dw_elems;         // K*R*S*C
    // N-D (Level-2 dimension reduction, PAPER.md P@17805): R = T * Rh filter rows
    // (depth tap fh / Rh, height tap fh % Rh); N = Nb * Do images (depth slice
    // img % Do of batch image img / Do).  2-D: T = D = Do = 1, Rh = R, Nb = N.
    int Rh, T, D, Do, Nb;
};

struct CtaCoord {
    int kb, cb, ft, fh, band, col;
};

// bid: tile index (blockIdx.x / csplit).
WINRS_HD CtaCoord decode_cta(const Geometry& g, long long bid) {
    CtaCoord c;
    c.kb = (int)(bid % g.kblocks); bid /= g.kblocks;
    c.cb = (int)(bid % g.cblocks); bid /= g.cblocks;
    c.ft = (int)(bid % g.ftiles);  bid /= g.ftiles;
    c.fh = (int)(bid % g.fhg) * g.fhs; bid /= g.fhg;   // first filter row of the group
    c.col = (int)(bid % g.seg_cols);
    c.band = (int)(bid / g.seg_cols);
    return c;
}

WINRS_HD long long num_tiles(const Geometry& g) {
    return (long long)g.kblocks * g.cblocks * g.ftiles * g.fhg * g.seg_cols * g.bands;
}
WINRS_HD long long num_ctas(const Geometry& g) { return num_tiles(g) * g.csplit * (g.cg > 1 ? g.cg : 1); }

// Chunk range [lo, hi) of cluster rank `rank` out of `nchunks` chunks.
WINRS_HD void split_chunks(int nchunks, int rank, int csplit, int* lo, int* hi) {
    *lo = (int)((long long)nchunks * rank / csplit);
    *hi = (int)((long long)nchunks * (rank + 1) / csplit);
}

// Valid (clipped) dY rows [hs, he) of a band for filter row fh (height tap
// fh % Rh; an N-D plan's depth tap fh / Rh is clipped by the zero fill).
WINRS_HD void band_rows(const Geometry& g, int band, int fh, int* hs, int* he) {
    const int h0 = band * g.seg_h;
    const int h1 = (band == g.bands - 1) ? g.Ho : h0 + g.seg_h;
    const int r = g.Rh > 0 ? fh % g.Rh : fh;
    int a = g.pad - r; if (a < h0) a = h0;
    int b = g.H + g.pad - r; if (b > h1) b = h1;
    *hs = a;
    *he = b > a ? b : a;
}

// dY rows a CTA of an fh group walks: the union of its rows' clipped ranges
// (for a row outside a member's range that member's X row lies in the zero
// padding, so it contributes nothing; the kernel reads it as TMA zero fill).
WINRS_HD void group_rows(const Geometry& g, int band, int fh0, int* hs, int* he) {
    int a = 0, b = 0;
    bool any = false;
    for (int f = 0; f < g.fhs && fh0 + f < g.R; ++f) {
        int x, y;
        band_rows(g, band, fh0 + f, &x, &y);
        if (y <= x) continue;
        if (!any || x < a) a = x;
        if (!any || y > b) b = y;
        any = true;
    }
    if (!any) band_rows(g, band, fh0, &a, &b);
    *hs = a;
    *he = b;
}

// Omega_a0 units of a column segment: first dY column and unit count.
WINRS_HD void seg_units(const Geometry& g, int col, int* w_first, int* units) {
    const int w0 = col * g.seg_w;
    int w1 = w0 + g.seg_w;
    const int lim = g.k0 * g.r0;
    if (w1 > lim) w1 = lim;
    *w_first = w0;
    *units = (w1 - w0) / g.r0;
}

WINRS_HD bool has_residual(const Geometry& g, int col) {
    return g.a1 != 0 && g.k1 > 0 && col == g.seg_cols - 1;
}

}  // namespace winrs
