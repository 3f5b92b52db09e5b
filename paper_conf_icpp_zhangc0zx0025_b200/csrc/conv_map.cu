// FC and BDC on the BFC machinery (§8 P@56407: "with moderate
// modifications, WinRS can support FC and BDC").
//
// A stride-1 convolution is a correlation of two spatial signals with a sum
// over one batch-like and one channel-like axis; the three convolutions of a
// layer differ only in which of the axes is summed.  The forward convolution
//     Y[n][h][w][k] = sum_{c,r,s} Xp[n][h+r-p][w+s-p][c] Wt[k][r][s][c]
// is exactly the BFC  dW'[k'][r'][s'][c'] = sum_{n',h',w'} Xp'[n'][h'+r'-p][w'+s'-p][c'] dY'[n'][h'][w'][k']
// with  n' = c (FC input channel), (h', w') = (r, s) (FC filter tap),
// (r', s') = (h, w) (FC output pixel), c' = n (FC image), k' = k:
//     X'  [C][H][W][N]   = X  [N][H][W][C]   with the outer and inner axes swapped,
//     dY' [C][R][S][K]   = Wt [K][R][S][C]   swapped,
//     dW' [K][Ho][Wo][N] = Y  [N][Ho][Wo][K] swapped back,
// and the BFC problem (N' = C, C' = N, H' = H, W' = W, K' = K, R' = Ho, S' = Wo,
// pad' = p) has Ho' = H + 2p - Ho + 1 = R and Wo' = S.  The backward-data
// convolution  dX[n][i][j][c] = sum_{k,r,s} dY[n][i-r+p][j-s+p][k] Wt[k][r][s][c]
// is the FC of dY with the spatially flipped filter Wt~[c][r][s][k] =
// Wt[k][R-1-r][S-1-s][c] and pad R-1-p, so its BFC operand dY'[k][r][s][c] is
// Wt with the (r, s) block reversed — no channel swap.  Everything between the
// layout kernels below is the planned BFC (kernel pair, segments, buckets,
// reduction) unchanged.  DESIGN.md §6.7.
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <new>
#include "../../include/winrs.h"

namespace winrs {
namespace convmap {

constexpr int TB = 32;   // transpose tile (a, b)

// out[b][m][a] = in[a][m][b]  (in: [A][M][B], out: [B][M][A]); grid (ceil(B/32),
// ceil(A/32), min(M, 65535)) with a grid-stride loop over m.  32x32 tile in
// shared memory: reads coalesced along b, writes along a.
template <typename T>
__global__ void __launch_bounds__(TB * 8) swap_outer_inner(const T* __restrict__ in, T* __restrict__ out, int A,
                                                           long long M, int B) {
    __shared__ T tile[TB][TB + 1];
    const int b0 = blockIdx.x * TB, a0 = blockIdx.y * TB;
    for (long long m = blockIdx.z; m < M; m += gridDim.z) {
        for (int i = threadIdx.y; i < TB; i += 8) {
            const int a = a0 + i, b = b0 + threadIdx.x;
            if (a < A && b < B) tile[i][threadIdx.x] = in[((long long)a * M + m) * B + b];
        }
        __syncthreads();
        for (int i = threadIdx.y; i < TB; i += 8) {
            const int b = b0 + i, a = a0 + threadIdx.x;
            if (a < A && b < B) out[((long long)b * M + m) * A + a] = tile[threadIdx.x][i];
        }
        __syncthreads();
    }
}

// out[a][M-1-m][b] = in[a][m][b]: the (r, s) block reversed (BDC filter flip).
template <typename T>
__global__ void flip_middle(const T* __restrict__ in, T* __restrict__ out, int A, int M, int B) {
    const long long total = (long long)A * M * B;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total;
         i += (long long)gridDim.x * blockDim.x) {
        const int b = (int)(i % B);
        const long long am = i / B;
        const int m = (int)(am % M);
        const long long a = am / M;
        out[(a * M + (M - 1 - m)) * B + b] = in[i];
    }
}

template <typename T>
cudaError_t swap(const void* in, void* out, int A, long long M, int B, cudaStream_t s) {
    if ((long long)A * M * B == 0) return cudaSuccess;
    const dim3 grid((B + TB - 1) / TB, (A + TB - 1) / TB, (unsigned)(M < 65535 ? M : 65535));
    swap_outer_inner<T><<<grid, dim3(TB, 8), 0, s>>>(static_cast<const T*>(in), static_cast<T*>(out), A, M, B);
    return cudaGetLastError();
}

template <typename T>
cudaError_t flip(const void* in, void* out, int A, int M, int B, cudaStream_t s) {
    const long long total = (long long)A * M * B;
    if (total == 0) return cudaSuccess;
    const long long blocks = (total + 255) / 256;
    flip_middle<T><<<(unsigned)(blocks < 148 * 16 ? blocks : 148 * 16), 256, 0, s>>>(
        static_cast<const T*>(in), static_cast<T*>(out), A, M, B);
    return cudaGetLastError();
}

}  // namespace convmap
}  // namespace winrs

struct winrs_conv_plan_s {
    int kind;                               // winrs_conv_kind_t
    int N, C, H, W, K, R, S, pad, Ho, Wo;   // the caller's convolution
    int dtype;
    winrs_plan_t bfc;                       // the mapped BFC plan
    size_t off_w, off_o, off_ws, total;     // workspace carve-up (X' at 0)
    int launches;
};

namespace {

size_t up256(size_t x) { return (x + 255) & ~(size_t)255; }

winrs_status_t conv_plan(winrs_conv_kind_t kind, int N, int C, int H, int W, int K, int R, int S, int pad,
                         winrs_dtype_t dtype, const winrs_device_t* dev, winrs_conv_plan_t* out) {
    if (!out) return WINRS_ERR_INVALID_ARG;
    *out = nullptr;
    if (kind != WINRS_CONV_FC && kind != WINRS_CONV_BDC) return WINRS_ERR_INVALID_ARG;
    if (N <= 0 || C <= 0 || H <= 0 || W <= 0 || K <= 0 || R <= 0 || S <= 0 || pad < 0) return WINRS_ERR_INVALID_ARG;
    const int Ho = H + 2 * pad - R + 1, Wo = W + 2 * pad - S + 1;
    if (Ho < 1 || Wo < 1) return WINRS_ERR_INVALID_ARG;
    winrs_plan_t bfc = nullptr;
    winrs_status_t st;
    if (kind == WINRS_CONV_FC) {
        // N' = C, C' = N, H' = H, W' = W, K' = K, R' = Ho, S' = Wo, pad' = pad
        st = dev ? winrs_plan_for_device(C, N, H, W, K, Ho, Wo, pad, dtype, dev, &bfc)
                 : winrs_plan(C, N, H, W, K, Ho, Wo, pad, dtype, &bfc);
    } else {
        // one symmetric pad for the flipped filter: R - 1 - pad == S - 1 - pad
        if (R != S || pad > R - 1) return WINRS_ERR_UNSUPPORTED;
        // FC of dY (channels K) with Wt~ (out channels C), pad R-1-pad:
        // N' = K, C' = N, H' = Ho, W' = Wo, K' = C, R' = H, S' = W
        st = dev ? winrs_plan_for_device(K, N, Ho, Wo, C, H, W, R - 1 - pad, dtype, dev, &bfc)
                 : winrs_plan(K, N, Ho, Wo, C, H, W, R - 1 - pad, dtype, &bfc);
    }
    if (st != WINRS_OK) return st;
    winrs_conv_plan_s* p = new (std::nothrow) winrs_conv_plan_s;
    if (!p) {
        winrs_plan_destroy(bfc);
        return WINRS_ERR_HOST_ALLOC;
    }
    p->kind = kind; p->N = N; p->C = C; p->H = H; p->W = W; p->K = K; p->R = R; p->S = S; p->pad = pad;
    p->Ho = Ho; p->Wo = Wo; p->dtype = dtype; p->bfc = bfc;
    const size_t esz = dtype == WINRS_F32 ? 4 : 2;
    const size_t in_elems = kind == WINRS_CONV_FC ? (size_t)N * H * W * C : (size_t)N * Ho * Wo * K;
    const size_t out_elems = kind == WINRS_CONV_FC ? (size_t)N * Ho * Wo * K : (size_t)N * H * W * C;
    p->off_w = up256(esz * in_elems);
    p->off_o = p->off_w + up256(esz * (size_t)K * R * S * C);
    p->off_ws = p->off_o + up256(4 * out_elems);
    p->total = p->off_ws + up256(winrs_workspace_bytes(bfc));
    p->launches = 3 + winrs_launch_count(bfc);
    *out = p;
    return WINRS_OK;
}

bool misaligned(const void* q) { return (reinterpret_cast<uintptr_t>(q) & 15u) != 0; }

template <typename T>
winrs_status_t run(winrs_conv_plan_t p, const void* in, const void* Wt, float* out, void* workspace,
                   cudaStream_t s) {
    using namespace winrs::convmap;
    uint8_t* ws = static_cast<uint8_t*>(workspace);
    void* in_t = ws;
    void* w_t = ws + p->off_w;
    float* o_t = reinterpret_cast<float*>(ws + p->off_o);
    void* bws = winrs_workspace_bytes(p->bfc) ? ws + p->off_ws : nullptr;
    cudaError_t e;
    if (p->kind == WINRS_CONV_FC) {
        e = swap<T>(in, in_t, p->N, (long long)p->H * p->W, p->C, s);                // X  -> [C][H][W][N]
        if (e == cudaSuccess) e = swap<T>(Wt, w_t, p->K, (long long)p->R * p->S, p->C, s);   // Wt -> [C][R][S][K]
    } else {
        e = swap<T>(in, in_t, p->N, (long long)p->Ho * p->Wo, p->K, s);              // dY -> [K][Ho][Wo][N]
        if (e == cudaSuccess) e = flip<T>(Wt, w_t, p->K, p->R * p->S, p->C, s);      // Wt -> Wt (r,s) reversed
    }
    if (e != cudaSuccess) return WINRS_ERR_CUDA;
    const winrs_status_t st = winrs_bfc(p->bfc, in_t, w_t, o_t, bws, s);
    if (st != WINRS_OK) return st;
    // [K'][R'][S'][N] -> [N][R'][S'][K']
    const int Kp = p->kind == WINRS_CONV_FC ? p->K : p->C;
    const long long Mp = p->kind == WINRS_CONV_FC ? (long long)p->Ho * p->Wo : (long long)p->H * p->W;
    e = swap<float>(o_t, out, Kp, Mp, p->N, s);
    return e == cudaSuccess ? WINRS_OK : WINRS_ERR_CUDA;
}

winrs_status_t conv_run(winrs_conv_plan_t p, int kind, const void* in, const void* Wt, float* out, void* workspace,
                        void* stream) {
    if (!p || p->kind != kind || !in || !Wt || !out) return WINRS_ERR_INVALID_ARG;
    if (!workspace) return WINRS_ERR_WORKSPACE;
    if (misaligned(in) || misaligned(Wt) || misaligned(out) || misaligned(workspace)) return WINRS_ERR_INVALID_ARG;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    return p->dtype == WINRS_F32 ? run<float>(p, in, Wt, out, workspace, s)
                                 : run<uint16_t>(p, in, Wt, out, workspace, s);
}

}  // namespace

extern "C" {

winrs_status_t winrs_conv_plan(winrs_conv_kind_t kind, int N, int C, int H, int W, int K, int R, int S, int pad,
                               winrs_dtype_t dtype, winrs_conv_plan_t* out) {
    return conv_plan(kind, N, C, H, W, K, R, S, pad, dtype, nullptr, out);
}

winrs_status_t winrs_conv_plan_for_device(winrs_conv_kind_t kind, int N, int C, int H, int W, int K, int R, int S,
                                          int pad, winrs_dtype_t dtype, const winrs_device_t* dev,
                                          winrs_conv_plan_t* out) {
    if (!dev) return WINRS_ERR_INVALID_ARG;
    return conv_plan(kind, N, C, H, W, K, R, S, pad, dtype, dev, out);
}

size_t winrs_conv_workspace_bytes(winrs_conv_plan_t plan) { return plan ? plan->total : 0; }

winrs_status_t winrs_conv_bfc_plan(winrs_conv_plan_t plan, winrs_plan_t* bfc) {
    if (!plan || !bfc) return WINRS_ERR_INVALID_ARG;
    *bfc = plan->bfc;
    return WINRS_OK;
}

int winrs_conv_launch_count(winrs_conv_plan_t plan) { return plan ? plan->launches : 0; }

winrs_status_t winrs_fc(winrs_conv_plan_t plan, const void* X, const void* Wt, float* Y, void* workspace,
                        void* stream) {
    return conv_run(plan, WINRS_CONV_FC, X, Wt, Y, workspace, stream);
}

winrs_status_t winrs_bdc(winrs_conv_plan_t plan, const void* dY, const void* Wt, float* dX, void* workspace,
                         void* stream) {
    return conv_run(plan, WINRS_CONV_BDC, dY, Wt, dX, workspace, stream);
}

void winrs_conv_plan_destroy(winrs_conv_plan_t plan) {
    if (!plan) return;
    winrs_plan_destroy(plan->bfc);
    delete plan;
}

}  // extern "C"
