/*
 * ORACLE — TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct FP64 CPU implementation of the
 * backward-filter convolution (BFC) that WinRS accelerates.  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
 * may load this library.  It shares no code, header, table or helper with the
 * CUDA path (paper_conf_icpp_zhangc0zx0025_b200/csrc); neither includes the
 * other.
 *
 * What it computes (the plain definition; WinRS reaches it exactly up to
 * rounding, so the oracle is the definition and not the Winograd algorithm):
 *
 *   Ho = H + 2*pad - R + 1,  Wo = W + 2*pad - S + 1
 *   dW[k][r][s][c] = sum_{n<N} sum_{h<Ho} sum_{w<Wo}
 *                      Xp(n, h+r-pad, w+s-pad, c) * dY[n][h][w][k]
 *   Xp(n,i,j,c) = X[n][i][j][c] if 0<=i<H and 0<=j<W, else 0
 *
 * Passages followed (PAPER.md is one line; "P@offset" = character offset):
 *   - "BFC convolves X with nabla Y to compute filter gradients nabla W"
 *     P@10786 §2.2; the same statement opens §3 (P@12976-13153).
 *   - Layouts (Table 1, P@14515-15243 §3): X in R^{N x I_H x I_W x I_C} (NHWC),
 *     nabla Y in R^{N x O_H x O_W x O_C} (NHWC), nabla W in
 *     R^{O_C x F_H x F_W x I_C} (KRSC).
 *   - Throughput formula 2*O_C*F_H*F_W*I_C*O_H*O_W*N (P@43462 §6.2) is the
 *     direct-convolution work of exactly this sum.
 *   - Correlation orientation, symmetric padding, stride 1: DESIGN.md readings
 *     R1-R3.
 *
 * Accumulation is FP64 in loop order n, h, w (any order is a valid oracle).
 */
#include <stddef.h>
#include <stdint.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

static int out_dims(int H, int W, int R, int S, int pad, int* Ho, int* Wo) {
    *Ho = H + 2 * pad - R + 1;
    *Wo = W + 2 * pad - S + 1;
    return (*Ho >= 1 && *Wo >= 1) ? 0 : -1;
}

/* Full dW, parallel over output channels k.  Returns 0 on success. */
int oracle_bfc_f64(int N, int C, int H, int W, int K, int R, int S, int pad,
                   const double* X, const double* dY, double* dW, int nthreads) {
    int Ho, Wo;
    if (N <= 0 || C <= 0 || H <= 0 || W <= 0 || K <= 0 || R <= 0 || S <= 0 || pad < 0) return -1;
    if (out_dims(H, W, R, S, pad, &Ho, &Wo)) return -1;
    memset(dW, 0, sizeof(double) * (size_t)K * R * S * C);
#ifdef _OPENMP
    if (nthreads > 0) omp_set_num_threads(nthreads);
#pragma omp parallel for schedule(dynamic, 1)
#endif
    for (int k = 0; k < K; ++k) {
        for (int n = 0; n < N; ++n)
            for (int h = 0; h < Ho; ++h)
                for (int w = 0; w < Wo; ++w) {
                    const double g = dY[(((size_t)n * Ho + h) * Wo + w) * K + k];
                    for (int r = 0; r < R; ++r) {
                        const int i = h + r - pad;
                        if (i < 0 || i >= H) continue;            /* zero padding */
                        for (int s = 0; s < S; ++s) {
                            const int j = w + s - pad;
                            if (j < 0 || j >= W) continue;        /* zero padding */
                            const double* x = X + (((size_t)n * H + i) * W + j) * C;
                            double* d = dW + (((size_t)k * R + r) * S + s) * C;
                            for (int c = 0; c < C; ++c) d[c] += x[c] * g;
                        }
                    }
                }
    }
    return 0;
}

/* FP32 inputs (exactly upcast to FP64 element by element), FP64 result.
 * Used for large layers so the caller does not need an FP64 copy. */
int oracle_bfc_f32in(int N, int C, int H, int W, int K, int R, int S, int pad,
                     const float* X, const float* dY, double* dW, int nthreads) {
    int Ho, Wo;
    if (N <= 0 || C <= 0 || H <= 0 || W <= 0 || K <= 0 || R <= 0 || S <= 0 || pad < 0) return -1;
    if (out_dims(H, W, R, S, pad, &Ho, &Wo)) return -1;
    memset(dW, 0, sizeof(double) * (size_t)K * R * S * C);
#ifdef _OPENMP
    if (nthreads > 0) omp_set_num_threads(nthreads);
#pragma omp parallel for schedule(dynamic, 1)
#endif
    for (int k = 0; k < K; ++k) {
        for (int n = 0; n < N; ++n)
            for (int h = 0; h < Ho; ++h)
                for (int w = 0; w < Wo; ++w) {
                    const double g = (double)dY[(((size_t)n * Ho + h) * Wo + w) * K + k];
                    for (int r = 0; r < R; ++r) {
                        const int i = h + r - pad;
                        if (i < 0 || i >= H) continue;
                        for (int s = 0; s < S; ++s) {
                            const int j = w + s - pad;
                            if (j < 0 || j >= W) continue;
                            const float* x = X + (((size_t)n * H + i) * W + j) * C;
                            double* d = dW + (((size_t)k * R + r) * S + s) * C;
                            for (int c = 0; c < C; ++c) d[c] += (double)x[c] * g;
                        }
                    }
                }
    }
    return 0;
}

/* Selected dW elements only: idx[t] is a flat KRSC index.  Each element is
 * the same sum over n, h, w, computed on its own (used at full sizes where
 * the whole dW would take too long on the host). */
int oracle_bfc_f32in_sampled(int N, int C, int H, int W, int K, int R, int S, int pad,
                             const float* X, const float* dY, const int64_t* idx, int nidx,
                             double* out, int nthreads) {
    int Ho, Wo;
    if (out_dims(H, W, R, S, pad, &Ho, &Wo)) return -1;
#ifdef _OPENMP
    if (nthreads > 0) omp_set_num_threads(nthreads);
#pragma omp parallel for schedule(dynamic, 1)
#endif
    for (int t = 0; t < nidx; ++t) {
        int64_t f = idx[t];
        const int c = (int)(f % C); f /= C;
        const int s = (int)(f % S); f /= S;
        const int r = (int)(f % R); f /= R;
        const int k = (int)f;
        double acc = 0.0;
        for (int n = 0; n < N; ++n)
            for (int h = 0; h < Ho; ++h) {
                const int i = h + r - pad;
                if (i < 0 || i >= H) continue;
                for (int w = 0; w < Wo; ++w) {
                    const int j = w + s - pad;
                    if (j < 0 || j >= W) continue;
                    acc += (double)X[(((size_t)n * H + i) * W + j) * C + c] *
                           (double)dY[(((size_t)n * Ho + h) * Wo + w) * K + k];
                }
            }
        out[t] = acc;
    }
    return 0;
}

int oracle_max_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
