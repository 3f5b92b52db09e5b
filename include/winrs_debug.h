/*
 * winrs_debug.h — test-support entry points of libwinrs.so (not needed to
 * run the method).  Host-only; no device memory is touched.
 */
#ifndef WINRS_DEBUG_H
#define WINRS_DEBUG_H
#include "winrs.h"

#ifdef __cplusplus
extern "C" {
#endif

/* FP64 host emulation of the plan's full decomposition (§3
 * P@15252-17405 and eq. (6) P@29449): the same CTA / segment / row-clipping /
 * unit / residual-phase / bucket structure the kernels execute, with the
 * library's generated transforms evaluated in double, then the bucket sum.
 * X: host NHWC double [N][H][W][C]; dY: host NHWC double [N][Ho][Wo][K];
 * dW: host KRSC double [K][R][S][C] (overwritten).  Slow: small shapes only. */
WINRS_API winrs_status_t winrs_debug_emulate(winrs_plan_t plan, const double* X, const double* dY, double* dW);

/* Apply one generated transform of Omega_alpha(n,r) in double (eq. (1)
 * P@9107): which = 0: FT  out[alpha] = G in[r];  1: IT  out[alpha] = D^T in[alpha];
 * 2: OT  out[n] = A^T in[alpha].  UNSUPPORTED for an unknown kernel. */
WINRS_API winrs_status_t winrs_debug_transform(int alpha, int n, int r, int which, const double* in, double* out);

/* Compiled kernel instantiations (pair + CTA tile), and their names. */
WINRS_API int winrs_debug_kernel_count(void);
WINRS_API const char* winrs_debug_kernel_name(int i);

/* Name of the instantiation a plan uses. */
WINRS_API const char* winrs_debug_plan_kernel(winrs_plan_t plan);

/* The planner's B200 time-model estimate for the plan (microseconds; the
 * quantity it minimised over pair x tile x Z x cluster split, R19).
 * -1 for a null plan. */
WINRS_API double winrs_debug_plan_model_us(winrs_plan_t plan);

#ifdef __cplusplus
}
#endif
#endif /* WINRS_DEBUG_H */
