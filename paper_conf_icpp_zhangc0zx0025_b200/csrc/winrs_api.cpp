// C ABI of libwinrs (include/winrs.h, include/winrs_debug.h): plan objects,
// argument validation and the launch sequence of PAPER.md §3 (P@15252-17405):
// (2) Kernel Execution — one fused launch over all segments (both kernels of
// the pair), (3) Reduction — the bucket reduction kernel when Z > 1.
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <new>
#include <vector>
#include "../../include/winrs.h"
#include "../../include/winrs_debug.h"
#include "planner.h"
#include "winograd_generated.cuh"

struct winrs_plan_s {
    winrs::PlanResult pr;
    winrs_plan_info_t info;
    int num_sms;
};

using namespace winrs;

// D, T: the N-D depth axes (1, 1 for a 2-D plan); see winrs_plan3d.
static winrs_status_t build_plan(int N, int C, int H, int W, int K, int R, int S, int pad,
                                 winrs_dtype_t dtype, const winrs_device_t* dev, winrs_plan_t* out,
                                 int D = 1, int T = 1) {
    if (!out) return WINRS_ERR_INVALID_ARG;
    *out = nullptr;
    if (N <= 0 || C <= 0 || H <= 0 || W <= 0 || K <= 0 || R <= 0 || S <= 0 || pad < 0 || D <= 0 || T <= 0)
        return WINRS_ERR_INVALID_ARG;
    const int Do = D + 2 * (T > 1 || D > 1 ? pad : 0) - T + 1;
    if (Do < 1) return WINRS_ERR_INVALID_ARG;
    if (dtype != WINRS_F32 && dtype != WINRS_F16 && dtype != WINRS_BF16) return WINRS_ERR_INVALID_ARG;
    const int Ho = H + 2 * pad - R + 1, Wo = W + 2 * pad - S + 1;
    if (Ho < 1 || Wo < 1) return WINRS_ERR_INVALID_ARG;
    if (!dev || dev->num_sms <= 0) return WINRS_ERR_INVALID_ARG;
    if (dev->cc_major != 10 || dev->cc_minor != 0) return WINRS_ERR_UNSUPPORTED;   // sm_100a build
    const int align = dtype == WINRS_F32 ? 4 : 8;                                  // 16-byte vectors
    if (C % align || K % align) return WINRS_ERR_UNSUPPORTED;
    const bool nd = T > 1 || D > 1;
    if ((long long)N * Do * Ho * Wo >= (1LL << 31) || (long long)R * T > (1 << 20))
        return WINRS_ERR_UNSUPPORTED;   // 32-bit depth index
    // N-D -> the 2-D decomposition: N*Do images, T*R filter rows
    Problem p{N * Do, C, H, W, K, R * T, S, pad, Ho, Wo, (int)dtype};
    p.Nb = N; p.Rh = R; p.T = T; p.D = D; p.Do = Do;
    PlanResult pr;
    const winrs_status_t st = make_plan(p, dev->num_sms, &pr);
    if (st != WINRS_OK) return st;
    winrs_plan_s* pl = new (std::nothrow) winrs_plan_s;
    if (!pl) return WINRS_ERR_HOST_ALLOC;
    pl->pr = pr;
    pl->num_sms = dev->num_sms;
    const Geometry& g = pr.geom;
    winrs_plan_info_t& in = pl->info;
    memset(&in, 0, sizeof(in));
    in.N = N; in.C = C; in.H = H; in.W = W; in.K = K; in.R = R; in.S = S; in.pad = pad;
    in.D = D; in.T = T; in.Do = Do;
    in.dtype = dtype; in.Ho = Ho; in.Wo = Wo;
    in.alpha0 = g.a0; in.n0 = g.n0; in.r0 = g.r0; in.k0 = g.k0;
    in.alpha1 = g.a1; in.n1 = g.n1; in.r1 = g.r1; in.k1 = g.k1;
    in.masked_cols = pr.masked;
    in.z_hat = pr.z_hat;
    in.Z = g.Z;
    in.seg_h = g.seg_h; in.seg_w = g.seg_w; in.bands = g.bands; in.seg_cols = g.seg_cols;
    in.tile_k0 = g.tile_k; in.tile_c0 = g.tile_c;
    in.tile_k1 = g.a1 ? g.tile_k : 0; in.tile_c1 = g.a1 ? g.tile_c : 0;
    in.ctas_main = num_ctas(g);
    in.csplit = g.csplit;
    in.ctas_resid = 0;   // the residual phase runs inside the main launch's last-column CTAs
    in.ctas_reduce = g.Z > 1 ? 1 : 0;
    in.workspace_bytes = g.Z > 1 ? (size_t)(g.Z - 1) * 4u * (size_t)g.dw_elems : 0;
    in.direct_flops = 2.0 * N * (double)Do * C * K * Ho * Wo * R * T * S;
    in.ewm_flops = pr.ewm_flops;
    *out = pl;
    return WINRS_OK;
}

extern "C" {

winrs_status_t winrs_plan_for_device(int N, int C, int H, int W, int K, int R, int S, int pad,
                                     winrs_dtype_t dtype, const winrs_device_t* dev, winrs_plan_t* out) {
    return build_plan(N, C, H, W, K, R, S, pad, dtype, dev, out);
}

winrs_status_t winrs_plan(int N, int C, int H, int W, int K, int R, int S, int pad,
                          winrs_dtype_t dtype, winrs_plan_t* out) {
    if (!out) return WINRS_ERR_INVALID_ARG;
    int d = 0;
    if (cudaGetDevice(&d) != cudaSuccess) { cudaGetLastError(); return WINRS_ERR_CUDA; }
    winrs_device_t dev{};
    if (cudaDeviceGetAttribute(&dev.num_sms, cudaDevAttrMultiProcessorCount, d) != cudaSuccess ||
        cudaDeviceGetAttribute(&dev.cc_major, cudaDevAttrComputeCapabilityMajor, d) != cudaSuccess ||
        cudaDeviceGetAttribute(&dev.cc_minor, cudaDevAttrComputeCapabilityMinor, d) != cudaSuccess) {
        cudaGetLastError();
        return WINRS_ERR_CUDA;
    }
    const winrs_status_t st = build_plan(N, C, H, W, K, R, S, pad, dtype, &dev, out);
    // stream-K plans: allocate the device's chain-flag regions now (not inside a
    // later launch that a caller may be capturing into a CUDA graph)
    if (st == WINRS_OK && (*out)->pr.entry->ta == 3 && sk_prepare(d) != cudaSuccess) {
        cudaGetLastError();
        winrs_plan_destroy(*out);
        *out = nullptr;
        return WINRS_ERR_CUDA;
    }
    return st;
}

winrs_status_t winrs_plan3d_for_device(int N, int C, int D, int H, int W, int K, int T, int R, int S, int pad,
                                       winrs_dtype_t dtype, const winrs_device_t* dev, winrs_plan_t* out) {
    return build_plan(N, C, H, W, K, R, S, pad, dtype, dev, out, D, T);
}

winrs_status_t winrs_plan3d(int N, int C, int D, int H, int W, int K, int T, int R, int S, int pad,
                            winrs_dtype_t dtype, winrs_plan_t* out) {
    if (!out) return WINRS_ERR_INVALID_ARG;
    int d = 0;
    if (cudaGetDevice(&d) != cudaSuccess) { cudaGetLastError(); return WINRS_ERR_CUDA; }
    winrs_device_t dev{};
    if (cudaDeviceGetAttribute(&dev.num_sms, cudaDevAttrMultiProcessorCount, d) != cudaSuccess ||
        cudaDeviceGetAttribute(&dev.cc_major, cudaDevAttrComputeCapabilityMajor, d) != cudaSuccess ||
        cudaDeviceGetAttribute(&dev.cc_minor, cudaDevAttrComputeCapabilityMinor, d) != cudaSuccess) {
        cudaGetLastError();
        return WINRS_ERR_CUDA;
    }
    return build_plan(N, C, H, W, K, R, S, pad, dtype, &dev, out, D, T);
}

winrs_status_t winrs_plan_info(winrs_plan_t plan, winrs_plan_info_t* info) {
    if (!plan || !info) return WINRS_ERR_INVALID_ARG;
    *info = plan->info;
    return WINRS_OK;
}

size_t winrs_workspace_bytes(winrs_plan_t plan) { return plan ? plan->info.workspace_bytes : 0; }

int winrs_launch_count(winrs_plan_t plan) {
    if (!plan) return 0;
    return 1 + (plan->pr.geom.Z > 1 ? 1 : 0);
}

static bool misaligned(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) != 0; }

winrs_status_t winrs_bfc(winrs_plan_t plan, const void* X, const void* dY, float* dW, void* workspace,
                         void* stream) {
    if (!plan) return WINRS_ERR_INVALID_ARG;
    return winrs_bfc_strided(plan, X, dY, (long long)plan->info.K, dW, workspace, stream);
}

winrs_status_t winrs_bfc_strided(winrs_plan_t plan, const void* X, const void* dY, long long ldy, float* dW,
                                 void* workspace, void* stream) {
    if (!plan || !X || !dY || !dW) return WINRS_ERR_INVALID_ARG;
    if (misaligned(X) || misaligned(dY) || misaligned(dW)) return WINRS_ERR_INVALID_ARG;
    const int align = plan->info.dtype == WINRS_F32 ? 4 : 8;
    if (ldy < plan->info.K || ldy % align != 0 || ldy > (1LL << 30)) return WINRS_ERR_INVALID_ARG;
    Geometry g = plan->pr.geom;
    g.ldy = (int)ldy;
    if (plan->info.workspace_bytes > 0) {
        if (!workspace) return WINRS_ERR_WORKSPACE;
        if (misaligned(workspace)) return WINRS_ERR_INVALID_ARG;
    }
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    cudaError_t e = plan->pr.entry->launch(g, X, dY, dW, static_cast<float*>(workspace), s);
    if (e != cudaSuccess) return WINRS_ERR_CUDA;
    if (g.Z > 1) {
        e = launch_bucket_reduce(dW, static_cast<const float*>(workspace), g.dw_elems, g.Z, plan->num_sms, s);
        if (e != cudaSuccess) return WINRS_ERR_CUDA;
    }
    return WINRS_OK;
}

winrs_status_t winrs_bfc_host(winrs_plan_t plan, const void* host_X, const void* host_dY, float* host_dW,
                              void* dev_X, void* dev_dY, float* dev_dW, void* workspace, void* stream) {
    if (!plan || !host_X || !host_dY || !host_dW || !dev_X || !dev_dY || !dev_dW) return WINRS_ERR_INVALID_ARG;
    const winrs_plan_info_t& in = plan->info;
    const size_t esz = in.dtype == WINRS_F32 ? 4 : 2;
    const size_t bx = esz * (size_t)in.N * in.D * in.H * in.W * in.C;
    const size_t by = esz * (size_t)in.N * in.Do * in.Ho * in.Wo * in.K;
    const size_t bw = 4 * (size_t)in.K * in.T * in.R * in.S * in.C;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    if (cudaMemcpyAsync(dev_X, host_X, bx, cudaMemcpyHostToDevice, s) != cudaSuccess ||
        cudaMemcpyAsync(dev_dY, host_dY, by, cudaMemcpyHostToDevice, s) != cudaSuccess) {
        cudaGetLastError();
        return WINRS_ERR_CUDA;
    }
    const winrs_status_t st = winrs_bfc(plan, dev_X, dev_dY, dev_dW, workspace, stream);
    if (st != WINRS_OK) return st;
    if (cudaMemcpyAsync(host_dW, dev_dW, bw, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
        cudaStreamSynchronize(s) != cudaSuccess) {
        cudaGetLastError();
        return WINRS_ERR_CUDA;
    }
    return WINRS_OK;
}

// ---------------------------------------------------------------------------
// Fused bucket reduction + cross-rank all-reduce over peer memory (allreduce.cu).

winrs_status_t winrs_ipc_alloc(size_t bytes, void** ptr, unsigned char* handle) {
    if (!ptr || !handle || bytes == 0) return WINRS_ERR_INVALID_ARG;
    *ptr = nullptr;
    void* p = nullptr;
    if (cudaMalloc(&p, bytes) != cudaSuccess) { cudaGetLastError(); return WINRS_ERR_CUDA; }
    cudaIpcMemHandle_t h;
    if (cudaMemset(p, 0, bytes) != cudaSuccess || cudaIpcGetMemHandle(&h, p) != cudaSuccess) {
        cudaGetLastError();
        cudaFree(p);
        return WINRS_ERR_CUDA;
    }
    memcpy(handle, &h, sizeof(h));
    *ptr = p;
    return WINRS_OK;
}

winrs_status_t winrs_ipc_open(const unsigned char* handle, void** ptr) {
    if (!ptr || !handle) return WINRS_ERR_INVALID_ARG;
    cudaIpcMemHandle_t h;
    memcpy(&h, handle, sizeof(h));
    if (cudaIpcOpenMemHandle(ptr, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
        cudaGetLastError();
        *ptr = nullptr;
        return WINRS_ERR_CUDA;
    }
    return WINRS_OK;
}

winrs_status_t winrs_ipc_close(void* ptr) {
    if (!ptr) return WINRS_ERR_INVALID_ARG;
    if (cudaIpcCloseMemHandle(ptr) != cudaSuccess) { cudaGetLastError(); return WINRS_ERR_CUDA; }
    return WINRS_OK;
}

winrs_status_t winrs_ipc_free(void* ptr) {
    if (!ptr) return WINRS_ERR_INVALID_ARG;
    if (cudaFree(ptr) != cudaSuccess) { cudaGetLastError(); return WINRS_ERR_CUDA; }
    return WINRS_OK;
}

size_t winrs_allreduce_flag_bytes(void) { return 128; }

winrs_status_t winrs_bfc_allreduce(winrs_plan_t plan, const void* X, const void* dY, float* dW, void* workspace,
                                   void* const* peer_stage, float* const* peer_dW, void* const* peer_flags,
                                   int rank, int world, unsigned int epoch, void* stream) {
    if (!plan || !X || !dY || !dW || !peer_stage || !peer_dW || !peer_flags) return WINRS_ERR_INVALID_ARG;
    if (world < 1 || world > AR_MAX || rank < 0 || rank >= world || epoch == 0) return WINRS_ERR_INVALID_ARG;
    if (peer_dW[rank] != dW) return WINRS_ERR_INVALID_ARG;
    PeerArgs pa = {};
    for (int q = 0; q < world; ++q) {
        if (!peer_stage[q] || !peer_dW[q] || !peer_flags[q] || misaligned(peer_stage[q]) || misaligned(peer_dW[q]) ||
            misaligned(peer_flags[q]))
            return WINRS_ERR_INVALID_ARG;
        pa.stage[q] = static_cast<float*>(peer_stage[q]);
        pa.dW[q] = peer_dW[q];
        pa.flags[q] = static_cast<unsigned int*>(peer_flags[q]);
    }
    if (misaligned(X) || misaligned(dY) || misaligned(dW)) return WINRS_ERR_INVALID_ARG;
    Geometry g = plan->pr.geom;
    g.ldy = plan->info.K;
    if (plan->info.workspace_bytes > 0) {
        if (!workspace) return WINRS_ERR_WORKSPACE;
        if (misaligned(workspace)) return WINRS_ERR_INVALID_ARG;
    }
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    cudaError_t e = plan->pr.entry->launch(g, X, dY, dW, static_cast<float*>(workspace), s);
    if (e != cudaSuccess) return WINRS_ERR_CUDA;
    // this rank's arrival counter lives after the 2 x AR_MAX flag words of its own block
    unsigned int* counter = pa.flags[rank] + 2 * AR_MAX;
    e = launch_fused_reduce_allreduce(dW, static_cast<const float*>(workspace), g.dw_elems, g.Z, pa, counter, rank,
                                      world, epoch, plan->num_sms, s);
    return e == cudaSuccess ? WINRS_OK : WINRS_ERR_CUDA;
}

void winrs_plan_destroy(winrs_plan_t plan) { delete plan; }

const char* winrs_status_string(winrs_status_t s) {
    switch (s) {
        case WINRS_OK: return "WINRS_OK";
        case WINRS_ERR_INVALID_ARG: return "WINRS_ERR_INVALID_ARG";
        case WINRS_ERR_UNSUPPORTED: return "WINRS_ERR_UNSUPPORTED";
        case WINRS_ERR_WORKSPACE: return "WINRS_ERR_WORKSPACE";
        case WINRS_ERR_CUDA: return "WINRS_ERR_CUDA";
        case WINRS_ERR_HOST_ALLOC: return "WINRS_ERR_HOST_ALLOC";
    }
    return "WINRS_ERR_UNKNOWN";
}

const char* winrs_version(void) { return "winrs-b200 0.1.0 (sm_100a)"; }

}  // extern "C"

// ----------------------------------------------------------------------------
// Host FP64 emulator of the plan's decomposition (include/winrs_debug.h).
// Walks exactly the CTA/segment/unit/row structure the kernels walk (same
// index helpers from winrs_internal.h, same generated transforms instantiated
// for double), so host-only tests can check the decomposition — pair split,
// masked tail, clipping, segments, buckets, residual phase, reduction —
// against the oracle before any GPU is involved.

namespace {

template <int A, int NN, int RR>
void emu_phase(const Geometry& g, const double* X, const double* dY, double* bucket, const CtaCoord& cc,
               int hs, int he, int w_first, int units, int fw0, bool accumulate, int rank) {
    using WT = Wino<A, NN, RR>;
    const int BN = g.tile_k, BM = g.tile_c;
    const int k0 = cc.kb * BN, c0 = cc.cb * BM;
    std::vector<double> v((size_t)A * BN * BM, 0.0), gt((size_t)A * BN), xt((size_t)A * BM);
    const long long depth = (long long)(he > hs ? he - hs : 0) * units * g.N;
    int c_lo, c_hi;
    split_chunks((int)((depth + g.chunk - 1) / g.chunk), rank, g.csplit, &c_lo, &c_hi);
    const long long d_hi = std::min<long long>(depth, (long long)c_hi * g.chunk);
    for (long long d = (long long)c_lo * g.chunk; d < d_hi; ++d) {
                const int n = (int)(d % g.N);
                const int u = (int)((d / g.N) % units);
                const int h = hs + (int)(d / g.N / units);
                const int w0 = w_first + u * RR;
                for (int k = 0; k < BN; ++k) {
                    double w[RR], o[A];
                    for (int i = 0; i < RR; ++i) {
                        const int kk = k0 + k, col = w0 + i;
                        w[i] = (kk < g.K && col < g.Wo) ? dY[(((size_t)n * g.Ho + h) * g.Wo + col) * g.ldy + kk] : 0.0;
                    }
                    WT::ft(w, o);
                    for (int x = 0; x < A; ++x) gt[(size_t)x * BN + k] = o[x];
                }
                // N-D: filter row fh = (depth tap fh / Rh, height tap fh % Rh); image n =
                // (batch n / Do, dY depth slice n % Do) reads X slice (n % Do) + t - pad
                const int rh = g.Rh > 0 ? g.Rh : g.R;
                const int xrow = h + cc.fh % rh - g.pad;
                const bool nd = g.T > 1 || g.D > 1;
                const int Do = g.Do > 0 ? g.Do : 1;
                const int xd = (n % Do) + (nd ? cc.fh / rh - g.pad : 0);
                const bool dok = xd >= 0 && xd < (g.D > 0 ? g.D : 1);
                const long long ximg = (long long)(n / Do) * (g.D > 0 ? g.D : 1) + xd;
                for (int c = 0; c < BM; ++c) {
                    double xv[A], o[A];
                    for (int t = 0; t < A; ++t) {
                        const int col = w0 + fw0 - g.pad + t, ccn = c0 + c;
                        xv[t] = (dok && col >= 0 && col < g.W && ccn < g.C && xrow >= 0 && xrow < g.H)
                                    ? X[(((size_t)ximg * g.H + xrow) * g.W + col) * g.C + ccn] : 0.0;
                    }
                    WT::it(xv, o);
                    for (int x = 0; x < A; ++x) xt[(size_t)x * BM + c] = o[x];
                }
                for (int x = 0; x < A; ++x)
                    for (int k = 0; k < BN; ++k)
                        for (int c = 0; c < BM; ++c)
                            v[((size_t)x * BN + k) * BM + c] += gt[(size_t)x * BN + k] * xt[(size_t)x * BM + c];
    }
    for (int k = 0; k < BN; ++k)
        for (int c = 0; c < BM; ++c) {
            const int kg = k0 + k, cg = c0 + c;
            if (kg >= g.K || cg >= g.C) continue;
            double vv[A], y[NN];
            for (int x = 0; x < A; ++x) vv[x] = v[((size_t)x * BN + k) * BM + c];
            WT::ot(vv, y);
            for (int j = 0; j < NN; ++j) {
                double& dst = bucket[(((size_t)kg * g.R + cc.fh) * g.S + fw0 + j) * g.C + cg];
                dst = accumulate ? dst + y[j] : y[j];
            }
        }
}

typedef void (*EmuFn)(const Geometry&, const double*, const double*, double*, const CtaCoord&, int, int, int,
                      int, int, bool, int);

EmuFn emu_fn(int a, int n, int r) {
#define WINRS_EMU_CASE(A, N, R) if (a == A && n == N && r == R) return &emu_phase<A, N, R>;
    WINRS_EMU_CASE(2, 2, 1) WINRS_EMU_CASE(4, 2, 3) WINRS_EMU_CASE(4, 3, 2)
    WINRS_EMU_CASE(8, 3, 6) WINRS_EMU_CASE(8, 4, 5) WINRS_EMU_CASE(8, 5, 4) WINRS_EMU_CASE(8, 6, 3)
    WINRS_EMU_CASE(8, 7, 2) WINRS_EMU_CASE(16, 5, 12) WINRS_EMU_CASE(16, 6, 11) WINRS_EMU_CASE(16, 7, 10)
    WINRS_EMU_CASE(16, 8, 9) WINRS_EMU_CASE(16, 9, 8)
#undef WINRS_EMU_CASE
    return nullptr;
}

}  // namespace

extern "C" {

winrs_status_t winrs_debug_emulate(winrs_plan_t plan, const double* X, const double* dY, double* dW) {
    if (!plan || !X || !dY || !dW) return WINRS_ERR_INVALID_ARG;
    const Geometry& g = plan->pr.geom;
    EmuFn f0 = emu_fn(g.a0, g.n0, g.r0);
    EmuFn f1 = g.a1 ? emu_fn(g.a1, g.n1, g.r1) : nullptr;
    if (!f0 || (g.a1 && !f1)) return WINRS_ERR_UNSUPPORTED;
    std::vector<double> buckets((size_t)g.Z * g.dw_elems, 0.0);
    std::vector<double> part((size_t)g.dw_elems);
    const long long nt = num_tiles(g);
    for (long long b = 0; b < nt; ++b) {
        const CtaCoord cc = decode_cta(g, b);
        const int seg = cc.band * g.seg_cols + cc.col;
        double* bucket = buckets.data() + (size_t)seg * g.dw_elems;
        int hs, he, wf, units;
        group_rows(g, cc.band, cc.fh, &hs, &he);   // fh group: the union of its rows' ranges
        seg_units(g, cc.col, &wf, &units);
        const int fw0 = cc.ft * g.n0;
        // cluster ranks each compute a partial tile; the tile is their sum
        for (int f = 0; f < g.fhs && cc.fh + f < g.R; ++f) {
            CtaCoord cf = cc;
            cf.fh = cc.fh + f;
            for (int rank = 0; rank < g.csplit; ++rank) {
                std::fill(part.begin(), part.end(), 0.0);
                f0(g, X, dY, part.data(), cf, hs, he, wf, units, fw0, false, rank);
                if (f1 && has_residual(g, cc.col))
                    for (int j = 0; j < g.n0 / g.n1; ++j)
                        f1(g, X, dY, part.data(), cf, hs, he, g.res_col0, g.k1, fw0 + j * g.n1, true, rank);
                for (long long i = 0; i < g.dw_elems; ++i) bucket[i] += part[i];
            }
        }
    }
    for (long long i = 0; i < g.dw_elems; ++i) {
        double s = 0.0;
        for (int z = 0; z < g.Z; ++z) s += buckets[(size_t)z * g.dw_elems + i];
        dW[i] = s;
    }
    return WINRS_OK;
}

winrs_status_t winrs_debug_transform(int alpha, int n, int r, int which, const double* in, double* out) {
    // which: 0 = ft (in[r] -> out[alpha]), 1 = it (in[alpha] -> out[alpha]), 2 = ot (in[alpha] -> out[n])
    if (!in || !out) return WINRS_ERR_INVALID_ARG;
#define WINRS_T_CASE(A, N, R)                                        \
    if (alpha == A && n == N && r == R) {                            \
        if (which == 0) { Wino<A, N, R>::ft(in, out); return WINRS_OK; }  \
        if (which == 1) { Wino<A, N, R>::it(in, out); return WINRS_OK; }  \
        if (which == 2) { Wino<A, N, R>::ot(in, out); return WINRS_OK; }  \
        return WINRS_ERR_INVALID_ARG;                                \
    }
    WINRS_T_CASE(2, 2, 1) WINRS_T_CASE(4, 2, 3) WINRS_T_CASE(4, 3, 2)
    WINRS_T_CASE(8, 3, 6) WINRS_T_CASE(8, 4, 5) WINRS_T_CASE(8, 5, 4) WINRS_T_CASE(8, 6, 3)
    WINRS_T_CASE(8, 7, 2) WINRS_T_CASE(16, 5, 12) WINRS_T_CASE(16, 6, 11) WINRS_T_CASE(16, 7, 10)
    WINRS_T_CASE(16, 8, 9) WINRS_T_CASE(16, 9, 8)
#undef WINRS_T_CASE
    return WINRS_ERR_UNSUPPORTED;
}

int winrs_debug_kernel_count(void) {
    int n = 0;
    kernel_entries(&n);
    return n;
}

const char* winrs_debug_kernel_name(int i) {
    int n = 0;
    const KernelEntry* e = kernel_entries(&n);
    return (i >= 0 && i < n) ? e[i].name : nullptr;
}

const char* winrs_debug_plan_kernel(winrs_plan_t plan) { return plan ? plan->pr.entry->name : nullptr; }

double winrs_debug_plan_model_us(winrs_plan_t plan) { return plan ? plan->pr.model_s * 1e6 : -1.0; }

}  // extern "C"
