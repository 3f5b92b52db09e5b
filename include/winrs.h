/*
 * winrs.h — C ABI of the B200-native WinRS fused Winograd backward-filter
 * convolution (BFC).  Implemented by libwinrs.so
 * (paper_conf_icpp_zhangc0zx0025_b200/csrc/).
 *
 * Citations are character offsets into the single-line PAPER.md ("P@offset")
 * plus the section; DESIGN.md lists every reading of the paper taken here.
 *
 * The operation (§2.2 P@10786 "BFC convolves X with nabla Y to
 * compute filter gradients nabla W"; Table 1 P@14515 §3 for shapes/layouts):
 *
 *   Ho = H + 2*pad - R + 1,   Wo = W + 2*pad - S + 1
 *   dW[k][r][s][c] = sum_{n,h,w} Xp[n][h+r-pad][w+s-pad][c] * dY[n][h][w][k]
 *   (Xp = X with zero padding; stride 1, dilation 1, one group)
 *
 * Layouts (Table 1): X is NHWC [N][H][W][C]; dY is NHWC [N][Ho][Wo][K]; dW is
 * KRSC [K][R][S][C] and is ALWAYS float32.  X and dY are both float32
 * (WINRS_F32), both IEEE binary16 (WINRS_F16) or both bfloat16 (WINRS_BF16;
 * the BF16 variant named in the paper's conclusion, P@56336).  These are exactly the
 * physical orders of PyTorch channels_last activations and channels_last
 * 4-D weights.
 *
 * Method (§3 P@15252-17405): a plan fixes the kernel pair
 * Omega_a0(n0,r0) / Omega_a1(n1,r1) (§4.1 P@20377), the segment count and
 * segment shape (§4.2 Alg. 1, §4.3 Alg. 2).  winrs_bfc launches the fused
 * kernels over the segments of dY; each writes one of Z dW "buckets" (bucket 0
 * is dW itself, buckets 1..Z-1 live in the workspace, P@15661), then one
 * reduction kernel sums the buckets into dW in fixed order with FP32 Kahan
 * summation (P@17126, P@39101).
 *
 * Ownership and threading:
 *   - The caller owns X, dY, dW and the workspace.  The library never
 *     allocates or frees device memory and never synchronises a stream.
 *   - A plan is immutable after creation and may be used concurrently from
 *     several host threads / streams as long as each concurrent call has its
 *     own dW and workspace.
 *   - dW is overwritten (beta = 0).  For a fixed plan and device the result
 *     is bitwise deterministic (no floating-point atomics).
 * Errors: status codes only; nothing is thrown across the ABI and the
 * library never calls exit/abort.  Asynchronous device faults surface at the
 * caller's next synchronisation (as with cuBLAS).
 */
#ifndef WINRS_H
#define WINRS_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define WINRS_API __attribute__((visibility("default")))
#else
#define WINRS_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum { WINRS_F32 = 0, WINRS_F16 = 1, WINRS_BF16 = 2 } winrs_dtype_t;

typedef enum {
    WINRS_OK = 0,
    WINRS_ERR_INVALID_ARG = 1,   /* bad dimension, null/unaligned pointer      */
    WINRS_ERR_UNSUPPORTED = 2,   /* no kernel for S/dtype, channel alignment,
                                    N*Ho*Wo >= 2^31, or the device is not
                                    sm_100                                     */
    WINRS_ERR_WORKSPACE = 3,     /* workspace == NULL but workspace_bytes > 0  */
    WINRS_ERR_CUDA = 4,          /* a CUDA launch/runtime error                */
    WINRS_ERR_HOST_ALLOC = 5     /* host allocation of the plan failed         */
} winrs_status_t;

/* Opaque, host-owned plan. */
typedef struct winrs_plan_s* winrs_plan_t;

/* Device properties the planner uses (winrs_plan queries the current device;
 * winrs_plan_for_device takes them explicitly, e.g. for host-only tests). */
typedef struct {
    int num_sms;      /* streaming multiprocessors (148 on B200)            */
    int cc_major;     /* compute capability; the kernels are built for 10.0 */
    int cc_minor;
} winrs_device_t;

/* Read-only description of a plan (all sizes in elements unless noted). */
typedef struct {
    int N, C, H, W, K, R, S, pad;
    int dtype;                     /* winrs_dtype_t                                       */
    int Ho, Wo;
    int alpha0, n0, r0, k0;        /* bulk kernel Omega_alpha0(n0,r0), k0 units per row   */
    int alpha1, n1, r1, k1;        /* residual kernel (alpha1 == 0: none), k1 units       */
    int masked_cols;               /* zero-masked dY columns in the last residual unit    */
    int z_hat;                     /* Alg. 1 estimate after Alg. 2 line 1                 */
    int Z;                         /* number of dW buckets (block groups of Omega_alpha0) */
    int seg_h, seg_w;              /* S^_H (rows per band), S^_W (dY columns per segment) */
    int bands, seg_cols;           /* segment grid: bands x seg_cols Omega_alpha0 segments */
    int tile_k0, tile_c0;          /* CTA tile B_N x B_M of the bulk kernel               */
    int tile_k1, tile_c1;          /* CTA tile of the residual kernel                     */
    long long ctas_main, ctas_resid, ctas_reduce;
    int csplit;                    /* CTAs per tile: thread-block cluster depth split   */
    size_t workspace_bytes;        /* (Z-1) * 4 * K*R*S*C, 0 when Z == 1                  */
    double direct_flops;           /* 2*N*C*K*Ho*Wo*R*S (P@43462) (x D_o*T for N-D)       */
    double ewm_flops;              /* Winograd-domain EWM flops actually issued           */
    int D, T, Do;                  /* N-D plans (winrs_plan3d): depth of X, of the filter  */
                                   /* and of dY; 1, 1, 1 for the 2-D plans                */
} winrs_plan_info_t;

/* Create a plan for the current CUDA device.
 *   dims: N,C,H,W (X), K (dY channels), R,S (dW height/width), pad (>= 0).
 * Returns INVALID_ARG for a dimension <= 0, pad < 0, Ho < 1, Wo < 1 or a null
 * `out`; UNSUPPORTED when S has no divisor n in {2..9} of the kernel set
 * (§5 P@28451: F_W in {n*k : 2 <= k <= 9}), when C % 4 or K % 4 != 0
 * (FP32) / C % 8 or K % 8 != 0 (FP16, BF16), or when the device is not sm_100.
 * On success *out owns a new plan (free with winrs_plan_destroy). */
WINRS_API winrs_status_t winrs_plan(int N, int C, int H, int W, int K, int R, int S, int pad,
                          winrs_dtype_t dtype, winrs_plan_t* out);

/* Same, for explicitly given device properties (no CUDA call is made). */
WINRS_API winrs_status_t winrs_plan_for_device(int N, int C, int H, int W, int K, int R, int S, int pad,
                                     winrs_dtype_t dtype, const winrs_device_t* dev,
                                     winrs_plan_t* out);

/* N-D (3-D) BFC by Level-2 dimension reduction (§3 P@17805-18294: an
 * N-D problem reduces to the 2-D machinery over the extra spatial axis):
 *   X  [N][D][H][W][C] (NDHWC), dY [N][Do][Ho][Wo][K] (NDHWC),
 *   dW [K][T][R][S][C] FP32 (KTRSC), Do = D + 2 pad - T + 1 (one symmetric pad),
 *   dW[k][t][r][s][c] = sum_{n,d,h,w} Xp[n][d+t-pad][h+r-pad][w+s-pad][c] dY[n][d][h][w][k].
 * The T x R filter planes become T*R "filter rows" of the 2-D decomposition and
 * the N x Do dY slices its images; a row's depth offset t reads X slice d+t-pad
 * (zero outside [0, D)).  Run with winrs_bfc.  UNSUPPORTED beyond the 2-D rules
 * when Do % 16 != 0 for FP16 / BF16 (the second-generation tensor-core kernel
 * loads 16 depth slices of one image per TMA box); FP32 runs the FP32 kernel. */
WINRS_API winrs_status_t winrs_plan3d(int N, int C, int D, int H, int W, int K, int T, int R, int S, int pad,
                            winrs_dtype_t dtype, winrs_plan_t* out);
WINRS_API winrs_status_t winrs_plan3d_for_device(int N, int C, int D, int H, int W, int K, int T, int R, int S,
                                       int pad, winrs_dtype_t dtype, const winrs_device_t* dev,
                                       winrs_plan_t* out);

/* Copy the plan description into *info (host memory). */
WINRS_API winrs_status_t winrs_plan_info(winrs_plan_t plan, winrs_plan_info_t* info);

/* Workspace bytes winrs_bfc needs for this plan (0 when Z == 1); 0 for NULL. */
WINRS_API size_t winrs_workspace_bytes(winrs_plan_t plan);

/* Run the BFC asynchronously on `stream` (a cudaStream_t; NULL = legacy
 * default stream).  X, dY: device pointers in the plan's dtype, NHWC;
 * dW: device float32 KRSC, overwritten; workspace: device buffer of at least
 * winrs_workspace_bytes(plan) bytes (may be NULL when that is 0).  All device
 * pointers must be 16-byte aligned; X and dY must not alias dW or workspace.
 * Returns INVALID_ARG (null plan/pointer, misalignment), WORKSPACE, or CUDA. */
WINRS_API winrs_status_t winrs_bfc(winrs_plan_t plan, const void* X, const void* dY, float* dW,
                         void* workspace, void* stream);

/* Same as winrs_bfc for a dY whose pixels are `ldy` elements apart (ldy >= K,
 * ldy % 4 == 0 for FP32, % 8 for FP16): dY points at channel k0 of a wider
 * NHWC tensor, so a rank can compute dW for the channel slice [k0, k0+K) of a
 * K-sharded layer without copying (BASELINE.json's K-sharding alternative,
 * DESIGN.md §8).  dW is the [K][R][S][C] slice (contiguous in KRSC).  Returns
 * INVALID_ARG for a bad ldy. */
WINRS_API winrs_status_t winrs_bfc_strided(winrs_plan_t plan, const void* X, const void* dY, long long ldy,
                                           float* dW, void* workspace, void* stream);

/* Same computation with HOST buffers: copies X and dY host->device into
 * caller-provided device staging buffers, runs winrs_bfc and copies dW back to
 * host_dW, all on `stream`, then synchronises that stream.  Used for the
 * end-to-end measurement.  dev_X/dev_dY/dev_dW are device buffers of the
 * respective sizes. */
WINRS_API winrs_status_t winrs_bfc_host(winrs_plan_t plan, const void* host_X, const void* host_dY,
                              float* host_dW, void* dev_X, void* dev_dY, float* dev_dW,
                              void* workspace, void* stream);

/* Destroy a plan (NULL is a no-op). */
WINRS_API void winrs_plan_destroy(winrs_plan_t plan);

/* Static, human-readable name of a status code. */
WINRS_API const char* winrs_status_string(winrs_status_t s);

/* Library version string (static). */
WINRS_API const char* winrs_version(void);

/* Number of GPU kernel launches one winrs_bfc call of this plan issues. */
WINRS_API int winrs_launch_count(winrs_plan_t plan);

/* ---------------------------------------------------------------------------
 * FC and BDC on the same machinery (§8 P@56407: "with moderate
 * modifications, WinRS can support FC and BDC").  Stride 1, one symmetric pad,
 * NHWC activations, KRSC weights, FP32 outputs:
 *   FC : Y [N][Ho][Wo][K] = sum_{r,s,c} Xp[n][h+r-pad][w+s-pad][c] * Wt[k][r][s][c]
 *   BDC: dX[N][H][W][C]   = sum_{r,s,k} dY[n][i-r+pad][j-s+pad][k] * Wt[k][r][s][c]
 * (dY zero outside [0,Ho) x [0,Wo)).  Each is run as the BFC of a transposed
 * problem (FC: N' = C, C' = N, R' x S' = Ho x Wo, the filter as dY'; BDC: the
 * FC of dY with the spatially flipped filter and pad R-1-pad) between layout
 * kernels; the BFC plan, kernels and reduction are the ones above unchanged.
 * Constraints are the mapped BFC's: FC needs N % 4 (FP32) / % 8 (FP16, BF16),
 * K likewise, and a kernel divisor n of Wo; BDC needs N and C aligned, a
 * divisor n of W, R == S and pad <= R-1.  UNSUPPORTED otherwise. */
typedef enum { WINRS_CONV_FC = 0, WINRS_CONV_BDC = 1 } winrs_conv_kind_t;
typedef struct winrs_conv_plan_s* winrs_conv_plan_t;

/* Plan an FC or BDC of the layer (N,C,H,W,K,R,S,pad) for the current device
 * (or explicitly given properties).  On success *out owns a new plan. */
WINRS_API winrs_status_t winrs_conv_plan(winrs_conv_kind_t kind, int N, int C, int H, int W, int K, int R, int S,
                                         int pad, winrs_dtype_t dtype, winrs_conv_plan_t* out);
WINRS_API winrs_status_t winrs_conv_plan_for_device(winrs_conv_kind_t kind, int N, int C, int H, int W, int K,
                                                    int R, int S, int pad, winrs_dtype_t dtype,
                                                    const winrs_device_t* dev, winrs_conv_plan_t* out);

/* Workspace bytes (always > 0: it holds the transposed operands, the
 * transposed FP32 result and the mapped BFC's bucket workspace). */
WINRS_API size_t winrs_conv_workspace_bytes(winrs_conv_plan_t plan);

/* The mapped BFC plan (owned by the conv plan; for winrs_plan_info). */
WINRS_API winrs_status_t winrs_conv_bfc_plan(winrs_conv_plan_t plan, winrs_plan_t* bfc);

/* GPU launches per winrs_fc / winrs_bdc call (3 layout kernels + the BFC's). */
WINRS_API int winrs_conv_launch_count(winrs_conv_plan_t plan);

/* Run asynchronously on `stream`.  X / dY / Wt device pointers in the plan's
 * dtype; Y / dX device FP32, overwritten; workspace >= winrs_conv_workspace_bytes.
 * All pointers 16-byte aligned, no aliasing.  INVALID_ARG for a null or
 * misaligned pointer or a plan of the other kind, WORKSPACE for a null
 * workspace, CUDA for a launch error. */
WINRS_API winrs_status_t winrs_fc(winrs_conv_plan_t plan, const void* X, const void* Wt, float* Y,
                                  void* workspace, void* stream);
WINRS_API winrs_status_t winrs_bdc(winrs_conv_plan_t plan, const void* dY, const void* Wt, float* dX,
                                   void* workspace, void* stream);

/* Destroy a conv plan and its BFC plan (NULL is a no-op). */
WINRS_API void winrs_conv_plan_destroy(winrs_conv_plan_t plan);

/* ---------------------------------------------------------------------------
 * Data-parallel BFC with the bucket reduction and the cross-rank sum fused
 * into one kernel over peer memory (§3
 * P@17126 "launch a reduction kernel to sum all nabla W buckets", §5.2 P@39101
 * FP32 Kahan summation).  Each rank runs winrs_bfc_allreduce on its batch
 * shard; afterwards every rank's dW holds
 *     dW = sum_{q = 0..world-1, in rank order} ( Kahan_z bucket_z of rank q )
 * in FP32, bit-identical on all ranks and to the unfused path (winrs_bfc on
 * each rank, then an FP32 sum of the ranks' dW in rank order).
 * Buffers are shared between processes with CUDA IPC:
 *   winrs_ipc_alloc  cudaMalloc + zero fill + the 64-byte IPC handle;
 *   winrs_ipc_open   map a peer's handle (not one's own) into this process;
 *   winrs_ipc_close / winrs_ipc_free.
 * Per rank q: stage[q] and dW[q] of |dW| = K*R*S*C floats, flags[q] of
 * winrs_allreduce_flag_bytes() bytes (zero-initialised, owned by rank q).
 * peer_* are HOST arrays of world device pointers as seen by this process
 * (peer_dW[rank] == dW).  epoch: 1, 2, 3, ... -- the same value on every rank
 * for a given call, one larger than the previous call's.  world <= 8.
 * The kernel is a cooperative launch whose barriers spin on the peers' flags;
 * a rank that never arrives makes it trap after ~20 s (WINRS_ERR_CUDA or a
 * sticky CUDA error) instead of hanging.  INVALID_ARG for a bad rank / world /
 * epoch, a null or misaligned pointer, or peer_dW[rank] != dW. */
WINRS_API winrs_status_t winrs_ipc_alloc(size_t bytes, void** ptr, unsigned char* handle);
WINRS_API winrs_status_t winrs_ipc_open(const unsigned char* handle, void** ptr);
WINRS_API winrs_status_t winrs_ipc_close(void* ptr);
WINRS_API winrs_status_t winrs_ipc_free(void* ptr);
WINRS_API size_t winrs_allreduce_flag_bytes(void);
WINRS_API winrs_status_t winrs_bfc_allreduce(winrs_plan_t plan, const void* X, const void* dY, float* dW,
                                             void* workspace, void* const* peer_stage, float* const* peer_dW,
                                             void* const* peer_flags, int rank, int world, unsigned int epoch,
                                             void* stream);

#ifdef __cplusplus
}
#endif
#endif /* WINRS_H */
