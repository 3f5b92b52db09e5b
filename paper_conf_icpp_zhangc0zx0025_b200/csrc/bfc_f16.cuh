// FP16- (or BF16-) in / FP32-accumulate tensor-core fused WinRS BFC kernel for sm_100a
// (tcgen05 + TMEM + TMA + mbarrier, warp-specialised).
//
// PAPER.md §5 (P@28371-39921) ported FP16 kernels run the alpha-batched GEMM
// on Tensor Cores with FT, IT and OT in FP32 (P@38729 "FT, IT, and OT are
// temporarily computed in FP32 precision, and finally converted to FP16").
// This is the B200 design of that kernel:
//
//   warp 0      TMA producer: per chunk of KC = 16 depth entries d = (h, u, n)
//               it loads the raw dY units (box [B_N=128 k][r][1][NB images])
//               and X windows (box [B_M=64 c][alpha][1][NB]) into a 2-stage
//               raw ring; TMA out-of-bounds zero fill implements the width
//               padding (P@33854), the masked tail unit (R6), the
//               channel tails and the depth tail.
//   warp 1      TMEM owner + MMA issuer: per chunk one
//               tcgen05.mma.cta_group::1.kind::f16 (M=128 k, N=64 c, K=16 d)
//               per Winograd point xi, accumulators D[xi] in TMEM columns
//               [xi*64, xi*64+64) (eq. (6): everything stays in the Winograd
//               domain for the whole main loop, P@29449).
//   warps 2..7  transformers: FT G*w (dY) and IT D^T*x (X) in FP32 — packed
//               f32x2 lanes (FFMA2) — then RN conversion to FP16 and 16-byte
//               stores straight into the UMMA K-major (no-swizzle) operand
//               layout of a 2-stage operand ring.  After the last chunk
//               warps 2..5 (one per TMEM lane quarter) are the epilogue:
//               tcgen05.ld -> OT A^T v in FP32 -> bucket (store or add).
// The residual kernel Omega_a1 runs as further jobs of the same CTA (last
// column segment only), adding into the same bucket (R10).
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include "dsmem.cuh"
#include "winograd_generated.cuh"
#include "winrs_internal.h"
#include "winrs_vec.cuh"

namespace winrs {
namespace f16k {

constexpr int BN = 128;          // k rows = UMMA M (TMEM lanes)
constexpr int KC = 16;           // depth entries per chunk = UMMA K
#ifndef WINRS_F16_SOP
#define WINRS_F16_SOP 0          // 0: as many operand stages (<= 4) as leave 3 raw stages
#endif
#ifndef WINRS_F16_NATIVE
#define WINRS_F16_NATIVE 0       // 1: Omega_4(3,2) in 16-bit arithmetic, MN-major SW128 operands (measured 6% slower on B200)
#endif
#ifndef WINRS_F16_PUSH
#define WINRS_F16_PUSH 0         // 1: fused epilogue + one-way DSMEM push reduction for cluster-split single-job tiles (measured: no gain, DSMEM-bandwidth bound either way)
#endif
#ifndef WINRS_F16_UPAIR
#define WINRS_F16_UPAIR 2        // dynamic schedule: a unit covers both depth octets of its row block (2: alpha = 4 kernels only)
#endif
#ifndef WINRS_F16_DIRECT
#define WINRS_F16_DIRECT 1       // single-job tiles: OT straight to the staging tile / bucket (no TMEM stash, no final pass)
#endif
#ifndef WINRS_F16_RR
#define WINRS_F16_RR 2           // 1: static round-robin unit assignment instead of the shared counter; 2: for alpha = 4 only
                                 // (measured on B200: round-robin 6-12% faster for alpha = 4, 15% slower for alpha = 8)
#endif
#ifndef WINRS_F16_DEEPRAW
#define WINRS_F16_DEEPRAW 0      // paired Omega_4(3,2) at B_M = 128: 3 operand + 5 raw stages, 14 transformer warps.
                                 // Off: 14 > 3 * 4 breaks the operand-ring parity bound (intermittent hang
                                 // under cold L2 on B200, tools/hang_repro.py); the static_assert now rejects it.
#endif
#ifndef WINRS_F16_RAWMAX
#define WINRS_F16_RAWMAX 4       // cap on raw (TMA) ring stages
#endif
#ifndef WINRS_F16_DQ
#define WINRS_F16_DQ 8           // depth entries per transformer unit (8: octet; 4 measured slower)
#endif
// transformer warps: one thread per (row pair, depth group of DQ) unit of a
// chunk: FT (BN/2 k pairs x KC/DQ groups) + IT (BM/2 c pairs x KC/DQ groups)
constexpr int DQ_FT = WINRS_F16_DQ;      // depth entries per FT unit
constexpr int DQ_IT = WINRS_F16_DQ;      // depth entries per IT unit
#ifndef WINRS_F16_DYN
#define WINRS_F16_DYN 1          // 1: transformer warps grab work units dynamically (else a fixed role per warp)
#endif
#ifndef WINRS_F16_TXW
#define WINRS_F16_TXW 0          // transformer warps (0: one per unit of a chunk)
#endif
// A chunk's transform work is split into warp-sized units: FT units (32 k
// pairs x one depth group) and IT units (32 c pairs, or BM/2 pairs x several
// groups, x depth groups).
template <int BM, int YB = BN> __host__ __device__ constexpr int ft_warps() { return (YB / 2) * (KC / DQ_FT) / 32; }
template <int BM> __host__ __device__ constexpr int it_warps() { return (BM / 2) * (KC / DQ_IT) / 32; }
template <int BM, int YB = BN> __host__ __device__ constexpr int n_units() { return ft_warps<BM, YB>() + it_warps<BM>(); }
// More warps than units per chunk let several chunks be in flight, which
// hides the shared-memory latency of the transforms; measured best on B200
// (A/B of 8..16 warps over the ResNet-50 / VGG-16 layers): 10 warps for the
// 128x64 / 128x32 tiles, 14 for 128x128.
// ---- native path (Omega_4(3,2), B_M a multiple of 64).  Every output of
// this kernel's FT (G w) and IT (D^T x) is one add or subtract of two inputs
// followed by an exact halving, so computing it in the input's own 16-bit
// arithmetic (one fused rounding, HFMA2) gives the correctly rounded FP16 /
// BF16 operand — what P@38729's "computed in FP32, then converted" produces,
// without the FP32 unpack / repack.  Operands are then stored MN-major (k or
// c contiguous, the raw TMA order) in the 128-byte-swizzled canonical UMMA
// layout, so a thread moves 8 channels per 16-byte load and store.
template <int A0, int N0, int R0, int A1, int BM>
__host__ __device__ constexpr bool native_path() {
    return WINRS_F16_NATIVE && A0 == 4 && N0 == 3 && R0 == 2 && A1 == 0 && BM % 64 == 0 && WINRS_F16_DYN;
}
#ifndef WINRS_NAT_IPT
#define WINRS_NAT_IPT 4
#endif
constexpr int NAT_IPT = WINRS_NAT_IPT;   // (channel octet, depth) items per thread per unit
template <int BM> __host__ __device__ constexpr int nat_ft_units() { return (BN / 8) * KC / (32 * NAT_IPT); }
template <int BM> __host__ __device__ constexpr int nat_it_units() { return (BM / 8) * KC / (32 * NAT_IPT); }
// Paired units (dynamic schedule): one grab covers both depth octets of a
// row block (FT always; IT when a block spans a whole warp of c pairs), so a
// chunk has half as many units and half the barrier hand-offs.
// Measured on B200: 2-9 % faster for the alpha = 4 kernels, much slower for
// alpha = 8 (too few units per chunk to keep the transformer warps busy).
template <int A0, int R0> __host__ __device__ constexpr bool pair_units() {
    return WINRS_F16_DYN && (WINRS_F16_UPAIR == 1 || (WINRS_F16_UPAIR == 2 && A0 == 4 && R0 == 2));
}
template <int BM, bool P> __host__ __device__ constexpr bool it_paired() { return P && BM / 2 >= 32; }
template <int BM, bool P, int YB = BN> __host__ __device__ constexpr int ft_units_p() {
    return P ? ft_warps<BM, YB>() / 2 : ft_warps<BM, YB>();
}
template <int BM, bool P> __host__ __device__ constexpr int it_units_p() { return it_paired<BM, P>() ? it_warps<BM>() / 2 : it_warps<BM>(); }
template <int BM, bool NAT, bool P = false, int YB = BN> __host__ __device__ constexpr int units_per_chunk() {
    return NAT ? nat_ft_units<BM>() + nat_it_units<BM>() : ft_units_p<BM, P, YB>() + it_units_p<BM, P>();
}

// Transformer warps.  The ring waits are parity waits, so a unit of chunk c
// must not start before the raw data of chunk c - S_RAW has landed: with
// units handed out in order, at most TX - 1 other units are in flight, which
// the kernel bounds statically (TX <= (S_RAW - 1) * units_per_chunk + 1).
// With paired / native units (4 per chunk at B_M = 128) that caps TX at 12.
template <int BM, bool FEW = false> __host__ __device__ constexpr int tx_warps() {
    return !WINRS_F16_DYN ? n_units<BM>() : WINRS_F16_TXW > 0 ? WINRS_F16_TXW : BM >= 128 ? (FEW ? 12 : 14) : 10;
}
template <int BM, bool FEW = false> __host__ __device__ constexpr int nthreads() { return 64 + 32 * tx_warps<BM, FEW>(); }
// Deep raw ring for the paired Omega_4(3,2) kernels at B_M = 128: 5 raw
// stages keep the parity bound with 14 transformer warps (17 >= 14).
template <int A0, int R0, int BM> __host__ __device__ constexpr bool deep_raw() {
    return WINRS_F16_DEEPRAW && pair_units<A0, R0>() && BM >= 128;
}
// FEW: 4 units per chunk at B_M = 128 (paired or native units) with the
// 4-stage raw ring -> 12 transformer warps.
template <int A0, int N0, int R0, int A1, int BM> __host__ __device__ constexpr bool few_units() {
    return (pair_units<A0, R0>() && !deep_raw<A0, R0, BM>()) || native_path<A0, N0, R0, A1, BM>();
}
template <int A0, int N0, int R0, int A1, int BM> __host__ __device__ constexpr int kthreads() {
    return nthreads<BM, few_units<A0, N0, R0, A1, BM>()>();
}

struct Args {
    Geometry g;
    float* dW;
    float* ws;
    int nb;          // images per TMA box (divides N and KC)
    int ybn;         // k rows per dY box: B_N, or 64 when K <= 64 (no zero-filled rows to land in SMEM)
};

// ----------------------------------------------------------------------------- PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(bar)), "r"(bytes) : "memory");
}
// Wait for the phase with the given parity.  The suspend-time hint lets the
// waiting warp sleep in hardware until the phase completes instead of
// re-polling, so idle producer / MMA warps do not steal issue slots from the
// transformer warps sharing their SM sub-partition.
#ifndef WINRS_WAIT_HINT
#define WINRS_WAIT_HINT 1000000
#endif
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    const uint32_t a = smem_u32(bar);
#if WINRS_WAIT_HINT > 0
    asm volatile(
        "{\n"
        ".reg .pred P;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1, %2;\n"
        "@!P bra WAIT_%=;\n"
        "}\n" :: "r"(a), "r"(parity), "r"(WINRS_WAIT_HINT) : "memory");
#else
    asm volatile(
        "{\n"
        ".reg .pred P;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n"
        "@!P bra WAIT_%=;\n"
        "}\n" :: "r"(a), "r"(parity) : "memory");
#endif
}
__device__ __forceinline__ void tma_load_4d(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1,
                                            int c2, int c3) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];"
        :: "r"(smem_u32(dst)), "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(c3),
           "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void prefetch_tmap(const CUtensorMap* map) {
    asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(map)) : "memory");
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// UMMA shared-memory descriptor, K-major, no swizzle: core matrices of 8 rows
// x 16 bytes; LBO = byte distance between the two K-halves (8 elements each)
// of a 16-deep slab, SBO = byte distance between 8-row groups.
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46);
}
// kind::f16 instruction descriptor: D f32, A/B f16, both K-major, M = 128, N = BM.
// A/B format field (bits 7-9, 10-12): 0 = F16, 1 = BF16.
// Bits 15 / 16: A / B MN-major (the native path).
template <int BM, bool BF, bool MN = false>
__host__ __device__ constexpr uint32_t idesc() {
    return (1u << 4) | ((BF ? 1u : 0u) << 7) | ((BF ? 1u : 0u) << 10) | ((MN ? 1u : 0u) << 15) | ((MN ? 1u : 0u) << 16) |
           ((uint32_t)(BM >> 3) << 17) | ((uint32_t)(BN >> 4) << 24);
}
// MN-major, 128-byte swizzle (layout type 2): atoms of 64 MN elements x 8 K
// rows (1 KB); LBO = byte stride between MN atoms, SBO = between K atoms
// (probed on B200: tools/microbench/umma_mn.cu).  Atom bases 1 KB aligned.
__device__ __forceinline__ uint64_t umma_desc_sw128(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46) | (2ull << 61);
}

template <int BM, bool BF, bool MN = false>
__device__ __forceinline__ void umma_f16(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t accumulate) {
    asm volatile(
        "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n"
        :: "r"(tmem_d), "l"(adesc), "l"(bdesc), "r"(idesc<BM, BF, MN>()), "r"(accumulate));
}
__device__ __forceinline__ void umma_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                 :: "r"(smem_u32(bar)) : "memory");
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

// 16-bit element traits: FP16 (IEEE binary16) or BF16 inputs / operands.
template <bool BF> struct Elem;
template <> struct Elem<false> {
    __device__ static __forceinline__ float2 unpack(uint32_t w) {
        return __half22float2(*reinterpret_cast<const __half2*>(&w));
    }
    __device__ static __forceinline__ uint32_t pack(float lo, float hi) {   // cvt.rn.f16x2.f32
        __half2 h = __floats2half2_rn(lo, hi);
        return *reinterpret_cast<uint32_t*>(&h);
    }
};
template <> struct Elem<true> {
    __device__ static __forceinline__ float2 unpack(uint32_t w) {
        return __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&w));
    }
    __device__ static __forceinline__ uint32_t pack(float lo, float hi) {   // cvt.rn.bf16x2.f32
        __nv_bfloat162 h = __floats2bfloat162_rn(lo, hi);
        return *reinterpret_cast<uint32_t*>(&h);
    }
};

__device__ __forceinline__ uint32_t pack_h2(float lo, float hi) { return Elem<false>::pack(lo, hi); }
__device__ __forceinline__ F2 ld_h2(const __half* p) {
    const __half2 h = *reinterpret_cast<const __half2*>(p);
    const float2 f = __half22float2(h);
    return F2{f.x, f.y};
}

// ----------------------------------------------------------------------------- shared memory plan
// DR (deep raw ring): 3 operand stages and up to 5 raw stages instead of 4 + 4.
template <int A0, int R0, int BM, int YB = BN, bool DR = false>
struct Smem {
    static constexpr int RAW_Y = KC * R0 * YB * 2;       // bytes per raw stage (dY; YB k rows per box)
    static constexpr int RAW_X = KC * A0 * BM * 2;       // bytes per raw stage (X)
    static constexpr int RAW = RAW_Y + RAW_X;
    static constexpr int OPA = BN * KC * 2;              // one A_xi slab (4 KB)
    static constexpr int OPB = BM * KC * 2;              // one B_xi slab
    static constexpr int OP = A0 * (OPA + OPB);
    static constexpr int LIMIT = 227 * 1024 - 256;
    // operand stages: the deeper the ring, the less the transformers wait for
    // the MMAs of the chunk S_OP back; keep >= 3 raw stages for TMA latency.
    static constexpr int S_OP = WINRS_F16_SOP > 0 ? WINRS_F16_SOP
                              : DR ? 3 : (LIMIT - 4 * OP) / RAW >= 3 ? 4 : (LIMIT - 3 * OP) / RAW >= 3 ? 3 : 2;
    // as many raw (TMA) stages as fit: the raw ring is the latency-hiding depth
    static constexpr int RAWMAX = DR ? 5 : WINRS_F16_RAWMAX;
    static constexpr int S_RAW = (LIMIT - S_OP * OP) / RAW > RAWMAX ? RAWMAX : (LIMIT - S_OP * OP) / RAW;
    static_assert(S_RAW >= 2 && S_RAW <= 8, "raw ring: 2..8 stages");
    static constexpr int raw_off = 0;
    static constexpr int op_off = S_RAW * RAW;
    static constexpr int bar_off = op_off + S_OP * OP;
    static constexpr int bytes = bar_off + 256;
};

// Operand layout (K-major, no swizzle): element (row, kk) of a 16-deep slab at
// byte (row/8)*256 + (kk/8)*128 + (row%8)*16 + (kk%8)*2.
//
// Rows are stored permuted within blocks of 16: logical row r -> physical
// perm16(r) = 16*(r/16) + 8*(r%2) + (r%16)/2.  A transformer thread owns the
// logical row pair (2p, 2p+1); with the permutation the 8 lanes of a
// quarter-warp store 8 distinct physical row%8 values, so the 16-byte operand
// stores are bank-conflict free.  The MMA is row-order agnostic: the
// permutation reappears as a TMEM lane (k) / column (c) permutation that the
// final output pass undoes.
__host__ __device__ __forceinline__ int perm16(int r) { return (r & ~15) | ((r & 1) << 3) | ((r >> 1) & 7); }
__host__ __device__ __forceinline__ int iperm16(int l) { return (l & ~15) | ((l & 7) << 1) | ((l >> 3) & 1); }

__device__ __forceinline__ uint32_t op_row_off(int row, int dgroup) {
    return (uint32_t)((row >> 3) * 256 + dgroup * 128 + (row & 7) * 16);
}

#ifdef WINRS_TRACE
// Debug-build timeline of CTA 0 (globaltimer ns): [role][chunk][event].
__device__ unsigned long long g_trace[4][256][4];
__device__ unsigned long long g_trace_w[256][24][3];   // per-warp (raw ok, op ok, chunk done) times
__device__ unsigned int g_warpslot[24];                 // %warpid of each warp (SM sub-partition = %4)
__device__ __forceinline__ unsigned long long gtime() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
#define TRACE(role, ch, ev) do { if (blockIdx.x == 0 && (ch) < 256) g_trace[role][ch][ev] = gtime(); } while (0)
__device__ unsigned long long g_cta_time[2048][8];      // per-CTA phase times (all CTAs)
#define PTRACE(i) do { if (blockIdx.x == 0) g_trace[0][240 + (i)][0] = gtime(); \
                       if (blockIdx.x < 2048) g_cta_time[blockIdx.x][i] = gtime(); } while (0)
#else
#define PTRACE(i) do { } while (0)
#define TRACE(role, ch, ev) do { } while (0)
#endif

struct Job {
    int phase;          // 0: Omega_a0, 1: Omega_a1
    int units, w_first, fw0;
    bool accumulate;
};

struct Barriers {
    uint64_t raw_full[8], raw_empty[8], op_full[4], op_empty[4], acc_full, acc_empty;
    uint32_t tmem_base;
    int unit_ctr;       // next transform unit (dynamic scheduling)
};

// Depth entry -> (n, h, u) for chunk-box issue.
// 32-bit: depth < N*Ho*Wo < 2^31 (winrs_plan rejects larger problems).
__device__ __forceinline__ void depth_coord(int d, int N, int units, int hs, int* n, int* h, int* u) {
    *n = d % N;
    const int t = d / N;
    *u = t % units;
    *h = hs + t / units;
}

// ---- transformer work for one chunk.  A unit is (row pair 2p/2p+1, 8
// consecutive depth entries = a depth octet for FT, 4 = a quad for IT, whose
// units cost more): FT units cover the B_N/2 k pairs of every A_xi, IT units
// the B_M/2 c pairs of every B_xi.  Each raw load is a half2 of the row pair at one depth (one
// 128-byte wavefront per warp); a thread computes its transforms two depth
// entries at a time in packed f32x2 (lanes = depth d, d+1) separately for
// each row, so each FP16 pack is already a K-adjacent half2 and the 8 results
// of a row form one 16-byte core-matrix row: two STS.128 per xi, conflict
// free through perm16.  FT and IT warps are interleaved so every SM
// sub-partition (warp % 4) gets the same mix.

// `mid()` runs between the transform (raw ring -> registers) and the operand
// stores: the caller releases the raw stage there and waits for the operand
// stage to be free, so the transform math of chunk c+S_OP overlaps the MMAs
// of chunk c instead of waiting for them.
struct NoMid { __device__ __forceinline__ void operator()() const {} };

template <int WT_FN, int A, int NN, int RR, int NIN, int DQ, bool BF, class Mid>
__device__ __forceinline__ void unit_transform(const uint16_t* src, int tap_stride, int depth_stride, uint8_t* dst0,
                                               int slab_bytes, int p, int grp, const Mid& mid) {
    using WT = Wino<A, NN, RR>;
    const int oct = grp;     // depth group index (DQ entries each)
    uint32_t pk[A][2][DQ / 2];   // [xi][row 2p / 2p+1][half2 of depth (2j, 2j+1)]
#pragma unroll
    for (int j = 0; j < DQ / 2; ++j) {
        F2 in0[NIN], in1[NIN], o[A];
        const uint16_t* s0 = src + (oct * DQ + 2 * j) * depth_stride + 2 * p;
#pragma unroll
        for (int i = 0; i < NIN; ++i) {
            const float2 a = Elem<BF>::unpack(*reinterpret_cast<const uint32_t*>(s0 + i * tap_stride));
            const float2 b = Elem<BF>::unpack(*reinterpret_cast<const uint32_t*>(s0 + depth_stride + i * tap_stride));
            in0[i] = F2{a.x, b.x};    // row 2p,   depth 2j, 2j+1
            in1[i] = F2{a.y, b.y};    // row 2p+1, depth 2j, 2j+1
        }
        if (WT_FN == 0) WT::ft(in0, o); else WT::it(in0, o);
#pragma unroll
        for (int x = 0; x < A; ++x) pk[x][0][j] = Elem<BF>::pack(o[x].x, o[x].y);
        if (WT_FN == 0) WT::ft(in1, o); else WT::it(in1, o);
#pragma unroll
        for (int x = 0; x < A; ++x) pk[x][1][j] = Elem<BF>::pack(o[x].x, o[x].y);
    }
    mid();
    // depth group -> K position kk0 = grp*DQ: K half kk0/8, byte offset (kk0%8)*2 in the 16-byte row
    const int kk0 = grp * DQ;
#pragma unroll
    for (int x = 0; x < A; ++x)
#pragma unroll
        for (int e = 0; e < 2; ++e) {
            uint8_t* d = dst0 + x * slab_bytes + op_row_off(perm16(2 * p + e), kk0 >> 3) + (kk0 & 7) * 2;
            if constexpr (DQ == 8)
                *reinterpret_cast<uint4*>(d) = make_uint4(pk[x][e][0], pk[x][e][1], pk[x][e][2], pk[x][e][3]);
            else
                *reinterpret_cast<uint2*>(d) = make_uint2(pk[x][e][0], pk[x][e][1]);
        }
}

// tx warp tw (0 .. tx_warps-1) -> IT warp index (>= 0) or FT warp index
// (-1 - idx).  IT units cost ~1.3x FT units; the IT warps are spread over
// the SM sub-partitions (warp w runs on w % 4).  Measured on B200: the
// per-chunk time is bounded by shared-memory / LSU throughput, so more or
// smaller units do not help.
template <int BM>
__host__ __device__ __forceinline__ bool tx_is_it(int tw) {
    constexpr int T = tx_warps<BM>(), I = it_warps<BM>();
    if (T == 3 * I) return tw % 3 == 2;
    if (T == 2 * I) return ((tw & 1) ^ ((tw >> 2) & 1)) != 0;
    return (tw + 1) * I / T > tw * I / T;
}
template <int BM>
__device__ __forceinline__ int tx_role(int tw) {
    int before = 0;
#pragma unroll 1
    for (int t = 0; t < tw; ++t) before += tx_is_it<BM>(t) ? 1 : 0;
    return tx_is_it<BM>(tw) ? before : -1 - (tw - before);
}

// kv / cv: valid k rows / c columns of this tile (< B_N / B_M in the last
// K- / C-block).  A warp whose whole row block lies past them skips its
// transforms: those operand rows stay zero (the op ring is cleared once at
// kernel start) and their accumulator rows are never written out.
// role >= 0: IT unit `role`; role < 0: FT unit -1 - role.
template <int A, int NN, int RR, int BM, bool BF, class Mid = NoMid, int YB = BN>
__device__ __forceinline__ void transform_role(const uint8_t* raw, uint8_t* op, int role, int lane, int kv, int cv,
                                               const Mid& mid = Mid(), int yb = BN) {
    constexpr int RAW_Y = KC * RR * YB * 2;
    const uint16_t* rawY = reinterpret_cast<const uint16_t*>(raw);            // [KC][RR][BN]
    const uint16_t* rawX = reinterpret_cast<const uint16_t*>(raw + RAW_Y);    // [KC][A][BM]
    constexpr int OPA = BN * KC * 2, OPB = BM * KC * 2;
    if (role < 0) {
        const int f = -1 - role;   // FT warp: 32 k pairs x one octet
        if ((f % (YB / 64)) * 64 >= kv) { mid(); return; }
        unit_transform<0, A, NN, RR, RR, DQ_FT, BF>(rawY, yb, RR * yb, op, OPA, (f % (YB / 64)) * 32 + lane,
                                                f / (YB / 64), mid);
    } else {                       // IT warp: 32 c pairs (or BM/2 pairs x 32/(BM/2) quads) x quads
        constexpr int PW = BM / 2 < 32 ? BM / 2 : 32;
        const int q = (role % ((BM / 2) / PW)) * PW + (lane % PW);
        const int quad = role / ((BM / 2) / PW) * (32 / PW) + lane / PW;
        if ((role % ((BM / 2) / PW)) * PW * 2 >= cv) { mid(); return; }
        unit_transform<1, A, NN, RR, A, DQ_IT, BF>(rawX, BM, A * BM, op + A * OPA, OPB, q, quad, mid);
    }
}
// Dynamic schedule with paired units: unit u -> one or two roles (IT first).
// mid_op (wait for the operand stage) runs before the first stores, mid_raw
// (release the raw stage) after the last raw loads of the unit.
template <int A, int NN, int RR, int BM, bool BF, bool P, int YB, class MidOp, class MidRaw>
__device__ __forceinline__ void transform_unit_paired(const uint8_t* raw, uint8_t* op, int u, int lane, int kv, int cv,
                                                      const MidOp& mid_op, const MidRaw& mid_raw, int yb) {
    const auto both = [&]() { mid_raw(); mid_op(); };
    if (u < it_units_p<BM, P>()) {
        if (it_paired<BM, P>()) {   // block u, octets 0 and 1 (roles octet * nblk + block)
            constexpr int NB = (BM / 2) / 32;
            transform_role<A, NN, RR, BM, BF, decltype(mid_op), YB>(raw, op, u, lane, kv, cv, mid_op, yb);
            transform_role<A, NN, RR, BM, BF, decltype(mid_raw), YB>(raw, op, NB + u, lane, kv, cv, mid_raw, yb);
        } else {
            transform_role<A, NN, RR, BM, BF, decltype(both), YB>(raw, op, u, lane, kv, cv, both, yb);
        }
    } else {
        const int f2 = u - it_units_p<BM, P>();
        if (P) {   // block f2 % nb, octets 2*(f2 / nb) + {0, 1} (roles octet * nb + block)
            constexpr int NB = YB / 64;
            const int blk = f2 % NB, oct = 2 * (f2 / NB);
            transform_role<A, NN, RR, BM, BF, decltype(mid_op), YB>(raw, op, -1 - (oct * NB + blk), lane, kv, cv, mid_op, yb);
            transform_role<A, NN, RR, BM, BF, decltype(mid_raw), YB>(raw, op, -1 - ((oct + 1) * NB + blk), lane, kv, cv, mid_raw, yb);
        } else {
            transform_role<A, NN, RR, BM, BF, decltype(both), YB>(raw, op, -1 - f2, lane, kv, cv, both, yb);
        }
    }
}

// Static schedule: transformer warp tw always runs the same unit.
template <int A, int NN, int RR, int BM, bool BF>
__device__ __forceinline__ void transform_chunk(const uint8_t* raw, uint8_t* op, int tw, int lane, int kv, int cv, int yb) {
    transform_role<A, NN, RR, BM, BF>(raw, op, tx_role<BM>(tw), lane, kv, cv, NoMid(), yb);
}
// Dynamic schedule: unit u of a chunk, the (costlier) IT units first.
template <int A, int NN, int RR, int BM, bool BF, class Mid>
__device__ __forceinline__ void transform_unit(const uint8_t* raw, uint8_t* op, int u, int lane, int kv, int cv,
                                               const Mid& mid) {
    transform_role<A, NN, RR, BM, BF>(raw, op, u < it_warps<BM>() ? u : -1 - (u - it_warps<BM>()), lane, kv, cv, mid);
}

// 16-bit pair arithmetic for the native path.
template <bool BF> struct H2;
template <> struct H2<false> {
    typedef __half2 T;
    __device__ static __forceinline__ T c(float v) { return __float2half2_rn(v); }
};
template <> struct H2<true> {
    typedef __nv_bfloat162 T;
    __device__ static __forceinline__ T c(float v) { return __float2bfloat162_rn(v); }
};
template <bool BF>
__device__ __forceinline__ uint4 h2_scale(uint4 a, typename H2<BF>::T k) {
    typedef typename H2<BF>::T T;
    uint4 r;
    T* ra = reinterpret_cast<T*>(&r);
    const T* aa = reinterpret_cast<const T*>(&a);
#pragma unroll
    for (int i = 0; i < 4; ++i) ra[i] = __hmul2(aa[i], k);
    return r;
}
template <bool BF>   // a * k + b, one rounding per element
__device__ __forceinline__ uint4 h2_fma(uint4 a, typename H2<BF>::T k, uint4 b) {
    typedef typename H2<BF>::T T;
    uint4 r;
    T* ra = reinterpret_cast<T*>(&r);
    const T* aa = reinterpret_cast<const T*>(&a);
    const T* bb = reinterpret_cast<const T*>(&b);
#pragma unroll
    for (int i = 0; i < 4; ++i) ra[i] = __hfma2(aa[i], k, bb[i]);
    return r;
}
template <bool BF>
__device__ __forceinline__ uint4 h2_neg(uint4 a) {
    typedef typename H2<BF>::T T;
    uint4 r;
    T* ra = reinterpret_cast<T*>(&r);
    const T* aa = reinterpret_cast<const T*>(&a);
#pragma unroll
    for (int i = 0; i < 4; ++i) ra[i] = __hneg2(aa[i]);
    return r;
}

// Byte offset of the 16-byte (8-channel) group g at depth d in an MN-major
// SW128 operand slab whose MN extent is `mn` channels (K = KC = 16).
template <int MNEXT>
__device__ __forceinline__ uint32_t nat_off(int g, int d) {
    return (uint32_t)((g >> 3) * 1024 + (d >> 3) * (MNEXT / 64) * 1024 + (d & 7) * 128 + (((g & 7) ^ (d & 7)) << 4));
}

// One native unit: NAT_IPT (channel octet, depth) items per lane.  IT units
// (X, B operand) come first, then FT units (dY, A operand).  A quarter-warp
// covers 8 consecutive octets at one depth: 128 contiguous raw bytes per
// load, 8 distinct swizzled 16-byte chunks per store (conflict free).
template <int BM, bool BF, class Mid>
__device__ __forceinline__ void native_unit(const uint8_t* raw, uint8_t* op, int u, int lane, int kv, int cv,
                                            const Mid& mid) {
    constexpr int A = 4, RR = 2;
    constexpr int RAW_Y = KC * RR * BN * 2;
    constexpr int OPA = BN * KC * 2, OPB = BM * KC * 2;
    typedef typename H2<BF>::T T;
    const T half = H2<BF>::c(0.5f), mhalf = H2<BF>::c(-0.5f);
    if (u < nat_it_units<BM>()) {
        // IT, Omega_4(3,2): o0 = (x2+x1)/2, o1 = (x2-x1)/2, o2 = (x0-x2)/2, o3 = (x3-x1)/2
        constexpr int G = BM / 8;
        uint4 o[NAT_IPT][A];
        int gg[NAT_IPT], dd[NAT_IPT];
#pragma unroll
        for (int i = 0; i < NAT_IPT; ++i) {
            const int idx = (u * NAT_IPT + i) * 32 + lane;
            gg[i] = idx % G;
            dd[i] = idx / G;
            if (gg[i] * 8 < cv) {
                const uint4* x = reinterpret_cast<const uint4*>(raw + RAW_Y + ((dd[i] * A) * BM + gg[i] * 8) * 2);
                const uint4 x0 = x[0], x1 = x[BM / 8], x2 = x[2 * (BM / 8)], x3 = x[3 * (BM / 8)];
                const uint4 x2h = h2_scale<BF>(x2, half), x1h = h2_scale<BF>(x1, half);
                o[i][0] = h2_fma<BF>(x1, half, x2h);
                o[i][1] = h2_fma<BF>(x1, mhalf, x2h);
                o[i][2] = h2_fma<BF>(x0, half, h2_neg<BF>(x2h));
                o[i][3] = h2_fma<BF>(x3, half, h2_neg<BF>(x1h));
            }
        }
        mid();
#pragma unroll
        for (int i = 0; i < NAT_IPT; ++i)
            if (gg[i] * 8 < cv) {
                uint8_t* b = op + A * OPA + nat_off<BM>(gg[i], dd[i]);
#pragma unroll
                for (int x = 0; x < A; ++x) *reinterpret_cast<uint4*>(b + x * OPB) = o[i][x];
            }
    } else {
        // FT, Omega_4(3,2): o0 = (w0+w1)/2, o1 = (w0-w1)/2, o2 = w0, o3 = w1
        constexpr int G = BN / 8;
        const int f = u - nat_it_units<BM>();
        uint4 o[NAT_IPT][2], w0s[NAT_IPT], w1s[NAT_IPT];
        int gg[NAT_IPT], dd[NAT_IPT];
#pragma unroll
        for (int i = 0; i < NAT_IPT; ++i) {
            const int idx = (f * NAT_IPT + i) * 32 + lane;
            gg[i] = idx % G;
            dd[i] = idx / G;
            if (gg[i] * 8 < kv) {
                const uint4* w = reinterpret_cast<const uint4*>(raw + ((dd[i] * RR) * BN + gg[i] * 8) * 2);
                w0s[i] = w[0];
                w1s[i] = w[BN / 8];
                const uint4 e = h2_scale<BF>(w0s[i], half);
                o[i][0] = h2_fma<BF>(w1s[i], half, e);
                o[i][1] = h2_fma<BF>(w1s[i], mhalf, e);
            }
        }
        mid();
#pragma unroll
        for (int i = 0; i < NAT_IPT; ++i)
            if (gg[i] * 8 < kv) {
                uint8_t* b = op + nat_off<BN>(gg[i], dd[i]);
                *reinterpret_cast<uint4*>(b) = o[i][0];
                *reinterpret_cast<uint4*>(b + OPA) = o[i][1];
                *reinterpret_cast<uint4*>(b + 2 * OPA) = w0s[i];
                *reinterpret_cast<uint4*>(b + 3 * OPA) = w1s[i];
            }
    }
}

__device__ __forceinline__ void tmem_st8(uint32_t taddr, const float* v) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};"
                 :: "r"(taddr), "r"(__float_as_uint(v[0])), "r"(__float_as_uint(v[1])), "r"(__float_as_uint(v[2])),
                    "r"(__float_as_uint(v[3])), "r"(__float_as_uint(v[4])), "r"(__float_as_uint(v[5])),
                    "r"(__float_as_uint(v[6])), "r"(__float_as_uint(v[7])) : "memory");
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

// TMEM column where the n0 x BM output tile is staged between jobs (top of
// the 512 columns; the residual job's accumulators live below it).
template <int N0, int BM> __host__ __device__ constexpr int stash_col() { return 512 - N0 * BM; }

// ---- epilogue of one job (warps 2..5, one TMEM lane quarter each):
// accumulators -> OT (FP32) -> output columns [j_off, j_off + NN) of the
// TMEM-staged tile (store for the first job, add for the residual jobs).
// Reading the 8 columns c0.. of every xi before writing the stash columns
// c0.. keeps the in-place overlap with the first job's accumulators safe.
template <int A, int NN, int RR, int N0, int BM>
__device__ __forceinline__ void epilogue(int j_off, bool first, bool empty, uint32_t tmem_base, int warp) {
    using WT = Wino<A, NN, RR>;
    const uint32_t lane_base = tmem_base + ((uint32_t)((warp & 3) * 32) << 16);
#pragma unroll 1
    for (int c0 = 0; c0 < BM; c0 += 8) {
        float v[A][8];
        if (!empty) {
#pragma unroll
            for (int x = 0; x < A; ++x) tmem_ld8(lane_base + (uint32_t)(x * BM + c0), v[x]);
            tmem_wait_ld();
        } else {
#pragma unroll
            for (int x = 0; x < A; ++x)
#pragma unroll
                for (int i = 0; i < 8; ++i) v[x][i] = 0.f;
        }
        float y[NN][8];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            float vv[A], yy[NN];
#pragma unroll
            for (int x = 0; x < A; ++x) vv[x] = v[x][i];
            WT::ot(vv, yy);
#pragma unroll
            for (int j = 0; j < NN; ++j) y[j][i] = yy[j];
        }
        if (!first) {
#pragma unroll
            for (int j = 0; j < NN; ++j) {
                float prev[8];
                tmem_ld8(lane_base + (uint32_t)(stash_col<N0, BM>() + (j_off + j) * BM + c0), prev);
                tmem_wait_ld();
#pragma unroll
                for (int i = 0; i < 8; ++i) y[j][i] += prev[i];
            }
        }
#pragma unroll
        for (int j = 0; j < NN; ++j) tmem_st8(lane_base + (uint32_t)(stash_col<N0, BM>() + (j_off + j) * BM + c0), y[j]);
        tmem_wait_st();
    }
}

template <int BM> __host__ __device__ constexpr int out_ld();
// ---- direct epilogue (single-job tiles): accumulators -> OT (FP32) -> the
// cluster staging tile (csplit > 1) or the bucket, with no TMEM output stash
// and no separate final pass.  Warps 2..5 (one TMEM lane quarter each) take
// 16 physical columns at a time: two 8-column halves are read and
// transformed, then de-interleaved into 16 logical columns (K-major path:
// physical 16b + i holds c = 16b + 2i, 16b + 8 + i holds c = 16b + 2i + 1)
// and written as float4s.  After acc_full no ring access is outstanding
// (every unit stored before its op_full arrival), so the staging tile may
// overlay the rings.
template <int A, int NN, int RR, int BM, bool NAT>
__device__ __forceinline__ void epilogue_direct(const Geometry& g, float* bucket, const CtaCoord& cc, int fw0,
                                                uint32_t tmem_base, int warp, bool empty, float* Out) {
    using WT = Wino<A, NN, RR>;
    const int quarter = warp & 3, lane = threadIdx.x & 31;
    const int L = quarter * 32 + lane;
    const int kl = NAT ? L : iperm16(L);
    const int kg = cc.kb * BN + kl;
    const uint32_t lane_base = tmem_base + ((uint32_t)(quarter * 32) << 16);
#pragma unroll 1
    for (int c0 = 0; c0 < BM; c0 += 16) {
        float y[NN][16];
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            float v[A][8];
            if (!empty) {
#pragma unroll
                for (int x = 0; x < A; ++x) tmem_ld8(lane_base + (uint32_t)(x * BM + c0 + 8 * h), v[x]);
                tmem_wait_ld();
            } else {
#pragma unroll
                for (int x = 0; x < A; ++x)
#pragma unroll
                    for (int i = 0; i < 8; ++i) v[x][i] = 0.f;
            }
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                float vv[A], yy[NN];
#pragma unroll
                for (int x = 0; x < A; ++x) vv[x] = v[x][i];
                WT::ot(vv, yy);
#pragma unroll
                for (int j = 0; j < NN; ++j) y[j][NAT ? 8 * h + i : 2 * i + h] = yy[j];
            }
        }
#pragma unroll
        for (int j = 0; j < NN; ++j) {
            if (g.csplit > 1) {
                float4* o = reinterpret_cast<float4*>(Out + ((long long)j * BN + kl) * out_ld<BM>() + c0);
#pragma unroll
                for (int q = 0; q < 4; ++q) o[q] = make_float4(y[j][4 * q], y[j][4 * q + 1], y[j][4 * q + 2], y[j][4 * q + 3]);
            } else {
                const int cg = cc.cb * BM + c0;
                if (kg < g.K && cg < g.C) {   // C % 8 == 0: 8-column groups are all in or all out
                    float4* d4 = reinterpret_cast<float4*>(bucket + (((long long)kg * g.R + cc.fh) * g.S + fw0 + j) * g.C + cg);
                    const int nq = cg + 16 <= g.C ? 4 : 2;
#pragma unroll
                    for (int q = 0; q < 4; ++q)
                        if (q < nq) d4[q] = make_float4(y[j][4 * q], y[j][4 * q + 1], y[j][4 * q + 2], y[j][4 * q + 3]);
                }
            }
        }
    }
}

// Output staging tile in shared memory for the cluster reduction: [n0][BN][BM+4].
// It overlays the rings (and, when larger, the mbarriers): it is only written
// after the last job, when all of them are idle.
template <int BM> __host__ __device__ constexpr int out_ld() { return BM + 4; }
// The cluster split needs the whole staged output tile in shared memory.
template <int N0, int BM> __host__ __device__ constexpr bool csplit_fits() {
    return (size_t)N0 * BN * out_ld<BM>() * 4 <= 227u * 1024u;
}
template <int A0, int N0, int R0, int BM, int YB = BN> __host__ __device__ constexpr size_t smem_total() {
    const size_t out = csplit_fits<N0, BM>() ? (size_t)N0 * BN * out_ld<BM>() * 4 : 0;
    using SMx = Smem<A0, R0, BM, YB, deep_raw<A0, R0, BM>()>;
    return SMx::bytes > out ? SMx::bytes : out;
}
// The YB = 64 variant (K <= 64: 64-row dY raw stages, only the FT units of
// the first 64-row block, a deeper raw ring) for the alpha = 8 single-kernel
// pairs; the others run the B_N-row layout.
// Both ring-parity bounds must hold (raw ring: in-order hand-out; operand
// ring: TX <= S_OP * units + 1).  Round 1 shipped YB = 64 under a timing
// argument (S_RAW == 2 S_OP) instead of the operand-ring bound; the variant
// is now compiled out unless the proven bound holds (with 10 transformer
// warps and 4 units per chunk it does not, so K <= 64 layers run the B_N
// layout; the default plans for them use the bfc_tc2.cuh kernel anyway).
template <int A0, int R0, int A1, int BM> __host__ __device__ constexpr bool yb64_variant() {
    return WINRS_F16_DYN && A0 == 8 && A1 == 0 && BM >= 64 &&
           tx_warps<BM>() <= (Smem<A0, R0, BM, 64>::S_RAW - 1) * units_per_chunk<BM, false, false, 64>() + 1 &&
           tx_warps<BM>() <= Smem<A0, R0, BM, 64>::S_OP * units_per_chunk<BM, false, false, 64>() + 1;
}

// ---- final pass (warps 2..5): staged tile -> bucket (no cluster split) or ->
// the shared-memory staging tile (cluster split).  Undoes the operand row
// permutation: TMEM lane L holds k = iperm16(L); physical columns
// [16b, 16b+16) hold logical c = 16b + 2i (first 8) and 16b + 2i + 1 (last 8).
template <int N0, int BM, bool NAT = false>
__device__ __forceinline__ void final_out(const Geometry& g, float* bucket, const CtaCoord& cc, int fw0, uint32_t tmem_base,
                                          int warp, float* Out) {
    const int quarter = warp & 3, lane = threadIdx.x & 31;
    const int kl = NAT ? quarter * 32 + lane : iperm16(quarter * 32 + lane);
    const int kg = cc.kb * BN + kl;
    const uint32_t lane_base = tmem_base + ((uint32_t)(quarter * 32) << 16);
#pragma unroll 1
    for (int c0 = 0; c0 < BM; c0 += 16) {
#pragma unroll 1
        for (int j = 0; j < N0; ++j) {
            float ph[16], y[16];
            tmem_ld8(lane_base + (uint32_t)(stash_col<N0, BM>() + j * BM + c0), ph);
            tmem_ld8(lane_base + (uint32_t)(stash_col<N0, BM>() + j * BM + c0 + 8), ph + 8);
            tmem_wait_ld();
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                y[NAT ? i : 2 * i] = ph[i];
                y[NAT ? 8 + i : 2 * i + 1] = ph[8 + i];
            }
            if (g.csplit > 1) {
                float4* o = reinterpret_cast<float4*>(Out + ((long long)j * BN + kl) * out_ld<BM>() + c0);
#pragma unroll
                for (int q = 0; q < 4; ++q) o[q] = make_float4(y[4 * q], y[4 * q + 1], y[4 * q + 2], y[4 * q + 3]);
            } else {
                const int cg = cc.cb * BM + c0;
                if (kg < g.K && cg < g.C) {   // C % 8 == 0: 8-column groups are all in or all out
                    float4* d4 = reinterpret_cast<float4*>(bucket + (((long long)kg * g.R + cc.fh) * g.S + fw0 + j) * g.C + cg);
                    const int nq = cg + 16 <= g.C ? 4 : 2;
#pragma unroll
                    for (int q = 0; q < 4; ++q)
                        if (q < nq) d4[q] = make_float4(y[4 * q], y[4 * q + 1], y[4 * q + 2], y[4 * q + 3]);
                }
            }
        }
    }
}

// ---- cluster reduction (all threads): rank r sums rows [r*rows/cs, ...) of
// the staged tiles of ranks 0..cs-1 in order through DSMEM and writes them.
template <int N0, int BM>
__device__ __forceinline__ void cluster_reduce(const Geometry& g, float* bucket, const CtaCoord& cc, int fw0, int rank,
                                               const float* Out, int nthreads_) {
    constexpr int C4 = BM / 4;
    constexpr int ROWS = N0 * BN;
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    const int r_lo = ROWS * rank / g.csplit, r_hi = ROWS * (rank + 1) / g.csplit;
    const uint32_t out_s = smem_u32(Out);
    for (int p = r_lo * C4 + (int)threadIdx.x; p < r_hi * C4; p += nthreads_) {
        const int row = p / C4, c4 = p % C4;
        const int j = row / BN, kl = row % BN;
        const uint32_t off = (uint32_t)((row * out_ld<BM>() + c4 * 4) * 4);
        const float4 acc = dsmem_sum4(out_s + off, g.csplit);
        const int kg = cc.kb * BN + kl, cg = cc.cb * BM + c4 * 4;
        if (kg < g.K && cg < g.C)
            *reinterpret_cast<float4*>(bucket + (((long long)kg * g.R + cc.fh) * g.S + fw0 + j) * g.C + cg) = acc;
    }
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// ---- fused epilogue + cluster reduction (single-job tiles with a cluster
// depth split).  After barrier B1 (every rank is past its main loop, so every
// rank's rings are free), 12 transformer warps — three per TMEM lane quarter,
// each a third of the column groups — read the accumulators, run the OT
// (FP32) and store each output row straight into the receive buffer of the
// rank that owns that row: rank s owns physical rows [s*ROWS/cs, (s+1)*ROWS/cs)
// (row = j*B_N + TMEM lane) and receives them as [source rank][row][column].
// The stores are one-way DSMEM traffic (no staging tile, no round-trip
// loads).  After barrier B2 each rank sums its rows over the source ranks in
// the fixed order 0..cs-1 (the same order as cluster_reduce: bitwise equal)
// and writes them to the bucket, undoing the operand row / column
// permutation of the K-major path.
template <int BM> __host__ __device__ constexpr int push_warps() { return tx_warps<BM>() >= 12 ? 12 : 8; }
template <int A, int NN, int RR, int N0, int BM, bool NAT>
__device__ __forceinline__ void cluster_push_reduce(const Geometry& g, float* bucket, const CtaCoord& cc, int fw0,
                                                    int rank, uint32_t tmem_base, bool empty, float* Rcv, int nthreads_) {
    using WT = Wino<A, NN, RR>;
    constexpr int ROWS = N0 * BN, LD = out_ld<BM>();
    const int cs = g.csplit, slice = ROWS / cs;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");   // B1
    tc_fence_after();
    constexpr int PUSH_WARPS = push_warps<BM>();
    if (warp >= 2 && warp < 2 + PUSH_WARPS) {
        const int q = warp & 3, part = (warp - 2) >> 2;
        const uint32_t lane_base = tmem_base + ((uint32_t)(q * 32) << 16);
        const uint32_t rcv = smem_u32(Rcv);
#pragma unroll 1
        for (int cg = part; cg < BM / 8; cg += PUSH_WARPS / 4) {
            float v[A][8];
            if (!empty) {
#pragma unroll
                for (int x = 0; x < A; ++x) tmem_ld8(lane_base + (uint32_t)(x * BM + cg * 8), v[x]);
                tmem_wait_ld();
            } else {
#pragma unroll
                for (int x = 0; x < A; ++x)
#pragma unroll
                    for (int i = 0; i < 8; ++i) v[x][i] = 0.f;
            }
            float y[NN][8];
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                float vv[A], yy[NN];
#pragma unroll
                for (int x = 0; x < A; ++x) vv[x] = v[x][i];
                WT::ot(vv, yy);
#pragma unroll
                for (int j = 0; j < NN; ++j) y[j][i] = yy[j];
            }
#pragma unroll
            for (int j = 0; j < NN; ++j) {
                const int prow = j * BN + q * 32 + lane;
                const int owner = prow / slice;
                const uint32_t off = (uint32_t)((((rank * slice) + (prow - owner * slice)) * LD + cg * 8) * 4);
                uint32_t remote;
                asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(rcv + off), "r"(owner));
                asm volatile("st.shared::cluster.v4.f32 [%0], {%1, %2, %3, %4};"
                             :: "r"(remote), "f"(y[j][0]), "f"(y[j][1]), "f"(y[j][2]), "f"(y[j][3]) : "memory");
                asm volatile("st.shared::cluster.v4.f32 [%0], {%1, %2, %3, %4};"
                             :: "r"(remote + 16), "f"(y[j][4]), "f"(y[j][5]), "f"(y[j][6]), "f"(y[j][7]) : "memory");
            }
        }
    }
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");   // B2
    // local sum of my rows: item = (row r of my slice, logical 4-column group m)
    const int r_lo = rank * slice;
    for (int p = (int)threadIdx.x; p < slice * (BM / 4); p += nthreads_) {
        const int r = p / (BM / 4), m = p % (BM / 4);
        const int prow = r_lo + r;
        const int j = prow / BN, L = prow % BN;
        const int kl = NAT ? L : iperm16(L);
        // logical columns 4m..4m+3 -> physical columns (K-major path: block
        // b = 4m/16, t = 4m%16 -> physical 16b + t/2 + {0, 8, 1, 9})
        const int b16 = (4 * m) >> 4, t = (4 * m) & 15;
        const int p0 = NAT ? 4 * m : 16 * b16 + (t >> 1);
        float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
        for (int src = 0; src < cs; ++src) {
            const float* row = Rcv + (size_t)(src * slice + r) * LD;
            float4 e;
            if (NAT) {
                e = *reinterpret_cast<const float4*>(row + p0);
            } else {
                const float2 a = *reinterpret_cast<const float2*>(row + p0);
                const float2 c = *reinterpret_cast<const float2*>(row + p0 + 8);
                e = make_float4(a.x, c.x, a.y, c.y);
            }
            acc.x += e.x; acc.y += e.y; acc.z += e.z; acc.w += e.w;
        }
        const int kg = cc.kb * BN + kl, cgl = cc.cb * BM + 4 * m;
        if (kg < g.K && cgl < g.C)
            *reinterpret_cast<float4*>(bucket + (((long long)kg * g.R + cc.fh) * g.S + fw0 + j) * g.C + cgl) = acc;
    }
}

template <int A0, int N0, int R0, int A1, int N1, int R1, int BM, bool BF, int YB = BN>
__global__ void __launch_bounds__((kthreads<A0, N0, R0, A1, BM>()), 1)
bfc_f16_kernel(const __grid_constant__ Args args, const __grid_constant__ CUtensorMap tmX0,
               const __grid_constant__ CUtensorMap tmY0, const __grid_constant__ CUtensorMap tmX1,
               const __grid_constant__ CUtensorMap tmY1) {
    using SM = Smem<A0, R0, BM, YB, deep_raw<A0, R0, BM>()>;
    static_assert(YB == BN || (YB == 64 && yb64_variant<A0, R0, A1, BM>()), "64-row dY stages: alpha = 8 single-kernel pairs");
    constexpr int S_RAW = SM::S_RAW;
    constexpr int TX_WARPS = tx_warps<BM, few_units<A0, N0, R0, A1, BM>()>();
    constexpr int NTHR = kthreads<A0, N0, R0, A1, BM>();
    static_assert(A1 * BM <= stash_col<N0, BM>(), "residual accumulators overlap the TMEM output stash");
    static_assert(!WINRS_F16_DYN ||
                  TX_WARPS <= (S_RAW - 1) * units_per_chunk<BM, native_path<A0, N0, R0, A1, BM>(), pair_units<A0, R0>(), YB>() + 1,
                  "in-order unit hand-out could run a full raw ring ahead of the TMA (parity-wait aliasing)");
    // Operand ring: a unit of chunk c waits (by parity) for the MMAs of chunk
    // c - S_OP.  While one unit of chunk s is held up, the MMAs stop at s, so
    // units of chunks s+S_OP .. s+2*S_OP-1 block in that wait; a unit of chunk
    // s + 2*S_OP would see the completed phase of chunk s - S_OP and overwrite
    // an operand stage the tensor core has not read.  Reaching it needs more
    // than S_OP * units_per_chunk + 1 warps (in-order hand-out) or a
    // round-robin stride above S_OP * units_per_chunk.  Otherwise the raw ring
    // must gate it: with S_RAW == 2 * S_OP the TMA of chunk s + 2*S_OP waits
    // for chunk s's own raw release, so the held unit would have to stall a
    // whole TMA round trip between its raw release and its operand arrival
    // ("operand-ring parity").  No instantiation relies on
    // that timing gate any more: the bound below is a proof obligation for
    // every compiled kernel.
    constexpr int NU_ = units_per_chunk<BM, native_path<A0, N0, R0, A1, BM>(), pair_units<A0, R0>(), YB>();
    constexpr bool RR_ = WINRS_F16_RR == 1 || (WINRS_F16_RR == 2 && A0 == 4);
    static_assert(!WINRS_F16_DYN || TX_WARPS <= SM::S_OP * NU_ + (RR_ ? 0 : 1),
                  "transformer units could run two operand-ring phases ahead of the MMAs (parity-wait aliasing)");
    constexpr bool kCluster = csplit_fits<N0, BM>();
    constexpr bool NAT = native_path<A0, N0, R0, A1, BM>();
    extern __shared__ __align__(1024) uint8_t smem[];
    const Geometry& g = args.g;
    Barriers* bars = reinterpret_cast<Barriers*>(smem + SM::bar_off);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) PTRACE(0);
#ifdef WINRS_TRACE
    if (threadIdx.x == 0 && blockIdx.x < 2048) {
        unsigned int smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        g_cta_time[blockIdx.x][7] = smid;
    }
#endif

    const int rank = (int)(blockIdx.x % g.csplit);
    const CtaCoord cc = decode_cta(g, blockIdx.x / g.csplit);
    const int seg = cc.band * g.seg_cols + cc.col;
    float* bucket = seg == 0 ? args.dW : args.ws + (long long)(seg - 1) * g.dw_elems;
    int hs, he;
    band_rows(g, cc.band, cc.fh, &hs, &he);
    int w_first, units;
    seg_units(g, cc.col, &w_first, &units);
    const int rows = he - hs;
    const int fw0 = cc.ft * N0;

    // Job list (identical in every role): (phase, units, first dY column,
    // first output column, output column offset in the tile).
    Job jobs[1 + 9];
    int njobs = 0;
    jobs[njobs++] = Job{0, units, w_first, fw0, false};
    if constexpr (A1 != 0) {
        if (has_residual(g, cc.col))
            for (int j = 0; j < N0 / N1; ++j) jobs[njobs++] = Job{1, g.k1, g.res_col0, fw0 + j * N1, true};
    }
    // single-job tile with a cluster split: fused epilogue + push reduction
    const bool fused = kCluster && WINRS_F16_PUSH && WINRS_F16_DYN && njobs == 1 && g.csplit > 1 &&
                       TX_WARPS >= push_warps<BM>();
    // this cluster rank's chunk range of a job
    auto chunk_range = [&](const Job& J, int* lo, int* hi) {
        const long long depth = (long long)(rows > 0 ? rows : 0) * J.units * g.N;
        split_chunks((int)((depth + KC - 1) / KC), rank, g.csplit, lo, hi);
    };

    if (threadIdx.x == 0) {
        constexpr int NU = units_per_chunk<BM, NAT, pair_units<A0, R0>(), YB>();
        for (int s = 0; s < S_RAW; ++s) { mbar_init(&bars->raw_full[s], 1); mbar_init(&bars->raw_empty[s], NU); }
        for (int s = 0; s < SM::S_OP; ++s) { mbar_init(&bars->op_full[s], NU); mbar_init(&bars->op_empty[s], 1); }
        bars->unit_ctr = 0;
        mbar_init(&bars->acc_full, 1);
        mbar_init(&bars->acc_empty, 4);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 0 && lane == 0) {
        prefetch_tmap(&tmX0); prefetch_tmap(&tmY0);
        if (A1 != 0) { prefetch_tmap(&tmX1); prefetch_tmap(&tmY1); }
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;"
                     :: "r"(smem_u32(&bars->tmem_base)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (g.K - cc.kb * BN < BN || g.C - cc.cb * BM < BM) {   // clear the operand ring once (rows past K / C are never transformed)
        uint4* op = reinterpret_cast<uint4*>(smem + SM::op_off);
        for (int i = threadIdx.x; i < SM::S_OP * SM::OP / 16; i += NTHR) op[i] = make_uint4(0, 0, 0, 0);
        fence_proxy_async();   // generic-proxy zeros visible to the tensor core's async proxy
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = bars->tmem_base;
    if (threadIdx.x == 0) PTRACE(1);
#ifdef WINRS_TRACE
    if (blockIdx.x == 0 && lane == 0) {
        unsigned int wid;
        asm volatile("mov.u32 %0, %%warpid;" : "=r"(wid));
        g_warpslot[warp] = wid;
    }
#endif

    if (warp == 0) {
        // ===================== TMA producer (whole warp) =====================
        // Lane 0 arms the stage's mbarrier; lanes 0 .. 2*KC/nb-1 then each issue
        // one box (even lanes dY, odd lanes X) so the boxes of a chunk are in
        // flight together instead of being issued back to back by one thread.
        int s = 0;
        uint32_t ph = 0;
        const int nbox = 2 * (KC / args.nb);
        for (int jb = 0; jb < njobs; ++jb) {
            const Job& J = jobs[jb];
            const int RRj = J.phase == 0 ? R0 : R1;
            const int Aj = J.phase == 0 ? A0 : A1;
            const CUtensorMap* mX = J.phase == 0 ? &tmX0 : &tmX1;
            const CUtensorMap* mY = J.phase == 0 ? &tmY0 : &tmY1;
            const long long depth = (long long)(rows > 0 ? rows : 0) * J.units * g.N;
            int c_lo, c_hi;
            chunk_range(J, &c_lo, &c_hi);
            const uint32_t bytes = (uint32_t)(KC * (RRj * args.ybn + Aj * BM) * 2);
            // This lane's box start d = ch*KC + b and its (n, h, u), advanced
            // incrementally (one division per job, not per chunk: the
            // producer shares its SM sub-partition with transformer warps).
            const int b = (lane >> 1) * args.nb;
            int d = c_lo * KC + b, n = 0, h = hs, u = 0;
            if (d < depth) depth_coord(d, g.N, J.units, hs, &n, &h, &u);
            for (int ch = c_lo; ch < c_hi; ++ch) {
                if (lane == 0) TRACE(0, ch - c_lo + jb * 64, 0);
                mbar_wait(&bars->raw_empty[s], ph ^ 1);
                if (lane == 0) TRACE(0, ch - c_lo + jb * 64, 1);
                uint8_t* raw = smem + SM::raw_off + s * SM::RAW;
#ifdef WINRS_NO_TMA   // debug: the raw ring carries no data (pipeline-only timing)
                if (lane == 0) mbar_arrive(&bars->raw_full[s]);
                (void)bytes; (void)raw; (void)mX; (void)mY;
                if (false) {
#else
                if (lane == 0) mbar_arrive_expect_tx(&bars->raw_full[s], bytes);
                __syncwarp();
                if (lane < nbox) {
#endif
                    const bool in = d < depth;     // past-the-end image => zero fill
                    const int nn = in ? n : g.N, hh = in ? h : hs;
                    const int w0 = J.w_first + (in ? u : 0) * RRj;
                    if ((lane & 1) == 0)
                        tma_load_4d(raw + b * RRj * args.ybn * 2, mY, &bars->raw_full[s], cc.kb * BN, w0, hh, nn);
                    else
                        tma_load_4d(raw + KC * RRj * YB * 2 + b * Aj * BM * 2, mX, &bars->raw_full[s], cc.cb * BM,
                                    w0 + J.fw0 - g.pad, hh + cc.fh - g.pad, nn);
                    if (lane == 0) TRACE(0, ch - c_lo + jb * 64, 2);
                    if (lane == 1) TRACE(0, ch - c_lo + jb * 64, 3);
                }
                d += KC;
                n += KC;
                while (n >= g.N) {
                    n -= g.N;
                    if (++u == J.units) { u = 0; ++h; }
                }
                if (++s == S_RAW) { s = 0; ph ^= 1; }
            }
        }
    } else if (warp == 1) {
        // ===================== MMA issuer =====================
        if (lane == 0) {
            int s = 0;
            uint32_t ph = 0;
            // descriptors differ only in the start-address field (16-byte units,
            // 14 bits: no carry for addresses < 256 KB)
            const uint64_t desc0 = NAT ? umma_desc_sw128(smem_u32(smem + SM::op_off), 1024, 2048)
                                       : umma_desc(smem_u32(smem + SM::op_off), 128, 256);
            // B slabs: SBO (K-atom stride) = (BM / 64) KB instead of 2 KB
            const uint64_t bsbo_fix = NAT ? ((uint64_t)(((BM / 64) * 1024) >> 4) << 32) - ((uint64_t)(2048 >> 4) << 32) : 0;
            for (int jb = 0; jb < njobs; ++jb) {
                const Job& J = jobs[jb];
                const int Aj = J.phase == 0 ? A0 : A1;
                int c_lo, c_hi;
                chunk_range(J, &c_lo, &c_hi);
                if (jb > 0) {
                    mbar_wait(&bars->acc_empty, (uint32_t)((jb - 1) & 1));
                    tc_fence_after();
                }
                for (int ch = c_lo; ch < c_hi; ++ch) {
                    mbar_wait(&bars->op_full[s], ph);
                    TRACE(1, ch - c_lo + jb * 64, 0);
                    tc_fence_after();
                    const uint64_t dstage = desc0 + (uint64_t)((s * SM::OP) >> 4);
                    for (int x = 0; x < Aj; ++x) {
                        const uint64_t ad = dstage + (uint64_t)((x * SM::OPA) >> 4);
                        const uint64_t bd = dstage + (uint64_t)((Aj * SM::OPA + x * SM::OPB) >> 4) + bsbo_fix;
#ifndef WINRS_NO_MMA
                        umma_f16<BM, BF, NAT>(tmem_base + (uint32_t)(x * BM), ad, bd, ch > c_lo ? 1u : 0u);
#else
                        (void)ad; (void)bd;
#endif
                    }
#ifdef WINRS_NO_COMMIT   // debug (with WINRS_NO_MMA only): release the stage without the tensor-core round trip
                    mbar_arrive(&bars->op_empty[s]);
#else
                    umma_commit(&bars->op_empty[s]);
#endif
                    TRACE(1, ch - c_lo + jb * 64, 1);
                    if (++s == SM::S_OP) { s = 0; ph ^= 1; }
                }
                umma_commit(&bars->acc_full);
            }
            PTRACE(2);
        }
    } else if (WINRS_F16_DYN) {
        // ============ transformers (+ epilogue), dynamic unit schedule ============
        // Every chunk of every job is n_units() warp-sized units; warps grab
        // units in global order (job, chunk, unit) from a shared counter, so a
        // warp that ran a cheap unit (FT) or sits on a lightly loaded SM
        // sub-partition takes more: the chunk rate follows the average unit
        // cost instead of the slowest fixed role.  Ring stage / parity follow
        // from the global chunk index, as in the producer and MMA loops.
        constexpr int NU = units_per_chunk<BM, NAT, pair_units<A0, R0>(), YB>();
        const int kv = g.K - cc.kb * BN, cv = g.C - cc.cb * BM;
        int jlo[1 + 9], jhi[1 + 9];
        for (int jb = 0; jb < njobs; ++jb) chunk_range(jobs[jb], &jlo[jb], &jhi[jb]);
        int jb = 0, unit_base = 0, gch_base = 0, epi = 0, rr_iter = 0;
        (void)rr_iter;
        // (the staging tile must not reach the mbarriers / unit counter, which
        // other warps may still touch while the epilogue runs)
        constexpr bool kOutBelowBars = (size_t)N0 * BN * out_ld<BM>() * 4 <= (size_t)SM::bar_off;
        const bool direct = WINRS_F16_DIRECT && njobs == 1 && !fused && (g.csplit <= 1 || kOutBelowBars);
        auto run_epilogue = [&](int e) {
            const Job& J = jobs[e];
            mbar_wait(&bars->acc_full, (uint32_t)(e & 1));
            tc_fence_after();
            const bool empty = jhi[e] <= jlo[e];
            if (direct)
                epilogue_direct<A0, N0, R0, BM, NAT>(g, bucket, cc, fw0, tmem_base, warp, empty, reinterpret_cast<float*>(smem));
            else if (J.phase == 0)
                epilogue<A0, N0, R0, N0, BM>(0, true, empty, tmem_base, warp);
            else if constexpr (A1 != 0)
                epilogue<A1, N1, R1, N0, BM>(J.fw0 - fw0, false, empty, tmem_base, warp);
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&bars->acc_empty);
        };
        for (;;) {
            int gi = 0;
            if constexpr (WINRS_F16_RR == 1 || (WINRS_F16_RR == 2 && A0 == 4)) {
                // round-robin: warp w takes units w, w + T, w + 2T, ... (no atomics)
                gi = (warp - 2) + TX_WARPS * rr_iter++;
            } else {
                if (lane == 0) gi = atomicAdd(&bars->unit_ctr, 1);
                gi = __shfl_sync(0xffffffffu, gi, 0);
            }
            while (jb < njobs && gi >= unit_base + (jhi[jb] - jlo[jb]) * NU) {
                unit_base += (jhi[jb] - jlo[jb]) * NU;
                gch_base += jhi[jb] - jlo[jb];
                ++jb;
            }
            // epilogues of the jobs whose units are all handed out (warps 2..5:
            // one TMEM lane quarter each); the fused push path does its own
            if (warp < 6 && !fused)
                while (epi < jb) run_epilogue(epi++);
            if (jb >= njobs) break;
            const int rel = gi - unit_base;
            const int u = rel % NU, gch = gch_base + rel / NU;
            const int sr = gch % S_RAW, so = gch % SM::S_OP;
            mbar_wait(&bars->raw_full[sr], (uint32_t)((gch / S_RAW) & 1));
#ifdef WINRS_TRACE
            if (lane == 0 && blockIdx.x == 0 && gch < 256) g_trace_w[gch][warp][0] = gtime();
#endif
            const uint8_t* raw = smem + SM::raw_off + sr * SM::RAW;
            uint8_t* op = smem + SM::op_off + so * SM::OP;
            // between transform and stores: every lane's raw reads are done
            // (their values are in registers) -> release the raw stage; then
            // wait for the MMAs of the chunk that last used this operand stage.
            // A skipped unit also waits, so its op_full arrival cannot land in
            // the previous phase of the stage.
            const auto mid_raw = [&]() {
                __syncwarp();
                if (lane == 0) mbar_arrive(&bars->raw_empty[sr]);
            };
            const auto mid_op = [&]() {
                mbar_wait(&bars->op_empty[so], (uint32_t)(((gch / SM::S_OP) & 1) ^ 1));
#ifdef WINRS_TRACE
                if (lane == 0 && blockIdx.x == 0 && gch < 256) g_trace_w[gch][warp][1] = gtime();
#endif
            };
            const auto mid = [&]() { mid_raw(); mid_op(); };
#ifdef WINRS_NO_TX     // debug: transformer units keep only the barrier protocol
            if (true) mid();
            else
#endif
            if constexpr (NAT) native_unit<BM, BF>(raw, op, u, lane, kv, cv, mid);
            else if (jobs[jb].phase == 0) transform_unit_paired<A0, N0, R0, BM, BF, pair_units<A0, R0>(), YB>(raw, op, u, lane, kv, cv, mid_op, mid_raw, args.ybn);
            else if constexpr (A1 != 0) transform_unit_paired<A1, N1, R1, BM, BF, pair_units<A0, R0>(), YB>(raw, op, u, lane, kv, cv, mid_op, mid_raw, args.ybn);
#ifndef WINRS_NO_FENCE
            fence_proxy_async();
#endif
            __syncwarp();
#ifdef WINRS_TRACE
            if (lane == 0 && blockIdx.x == 0 && gch < 256) g_trace_w[gch][warp][2] = gtime();
#endif
            if (lane == 0) mbar_arrive(&bars->op_full[so]);
        }
        if (threadIdx.x == 64) PTRACE(3);
        if (fused) {
            if (warp == 2) {   // the accumulators are final before the CTA-wide sync below
                mbar_wait(&bars->acc_full, 0u);
                tc_fence_after();
            }
        } else if (!direct) {
            __syncwarp();   // converged warp at the named barrier
            asm volatile("barrier.sync 1, %0;" :: "r"(32 * TX_WARPS) : "memory");
            if (warp < 6) {
                final_out<N0, BM, NAT>(g, bucket, cc, fw0, tmem_base, warp, reinterpret_cast<float*>(smem));
                if (threadIdx.x == 64) PTRACE(4);
            }
        }
    } else {
        // ===================== transformers (+ epilogue) =====================
        const int tw = warp - 2;
        const int kv = g.K - cc.kb * BN, cv = g.C - cc.cb * BM;
        int sr = 0, so = 0;
        uint32_t phr = 0, pho = 0;
        for (int jb = 0; jb < njobs; ++jb) {
            const Job& J = jobs[jb];
            int c_lo, c_hi;
            chunk_range(J, &c_lo, &c_hi);
            for (int ch = c_lo; ch < c_hi; ++ch) {
                if (threadIdx.x == 64) TRACE(2, ch - c_lo + jb * 64, 0);
                mbar_wait(&bars->raw_full[sr], phr);
                if (threadIdx.x == 64) TRACE(2, ch - c_lo + jb * 64, 1);
#ifdef WINRS_TRACE
                if (lane == 0 && blockIdx.x == 0 && ch - c_lo + jb * 64 < 256) g_trace_w[ch - c_lo + jb * 64][warp][0] = gtime();
#endif
                mbar_wait(&bars->op_empty[so], pho ^ 1);
                if (threadIdx.x == 64) TRACE(2, ch - c_lo + jb * 64, 2);
#ifdef WINRS_TRACE
                if (lane == 0 && blockIdx.x == 0 && ch - c_lo + jb * 64 < 256) g_trace_w[ch - c_lo + jb * 64][warp][1] = gtime();
#endif
                const uint8_t* raw = smem + SM::raw_off + sr * SM::RAW;
                uint8_t* op = smem + SM::op_off + so * SM::OP;
                if (J.phase == 0) transform_chunk<A0, N0, R0, BM, BF>(raw, op, tw, lane, kv, cv, args.ybn);
                else if constexpr (A1 != 0) transform_chunk<A1, N1, R1, BM, BF>(raw, op, tw, lane, kv, cv, args.ybn);
                if (threadIdx.x == 64) TRACE(3, ch - c_lo + jb * 64, 0);
                if (threadIdx.x == 64 + 32 * 2) TRACE(3, ch - c_lo + jb * 64, 1);   // an IT warp
                fence_proxy_async();
                if (threadIdx.x == 64) TRACE(3, ch - c_lo + jb * 64, 2);
                __syncwarp();
                if (threadIdx.x == 64) TRACE(2, ch - c_lo + jb * 64, 3);
#ifdef WINRS_TRACE
                if (lane == 0 && blockIdx.x == 0 && ch - c_lo + jb * 64 < 256) g_trace_w[ch - c_lo + jb * 64][warp][2] = gtime();
#endif
                if (lane == 0) {
                    mbar_arrive(&bars->op_full[so]);
                    mbar_arrive(&bars->raw_empty[sr]);
                }
                if (++sr == S_RAW) { sr = 0; phr ^= 1; }
                if (++so == SM::S_OP) { so = 0; pho ^= 1; }
            }
            if (warp < 6) {
                mbar_wait(&bars->acc_full, (uint32_t)(jb & 1));
                tc_fence_after();
                const bool empty = c_hi <= c_lo;
                if (J.phase == 0)
                    epilogue<A0, N0, R0, N0, BM>(0, true, empty, tmem_base, warp);
                else if constexpr (A1 != 0)
                    epilogue<A1, N1, R1, N0, BM>(J.fw0 - fw0, false, empty, tmem_base, warp);
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&bars->acc_empty);
            }
        }
        // All transformer warps are past their last raw-ring read before the
        // staging tile (which overlays the rings) is written.  (Already implied
        // by acc_full -> all MMAs -> all op_full arrivals; made explicit.)
        if (threadIdx.x == 64) PTRACE(3);
        __syncwarp();   // converged warp at the named barrier
        asm volatile("barrier.sync 1, %0;" :: "r"(32 * TX_WARPS) : "memory");
        if (warp < 6) {
            // every job's epilogue is done (this warp's own, in program order)
            final_out<N0, BM>(g, bucket, cc, fw0, tmem_base, warp, reinterpret_cast<float*>(smem));
            if (threadIdx.x == 64) PTRACE(4);
        }
    }
    tc_fence_before();
    __syncthreads();
    if (threadIdx.x == 0) PTRACE(5);
    if constexpr (kCluster) {
        if (fused) {
            tc_fence_after();
            int lo, hi;
            chunk_range(jobs[0], &lo, &hi);
            cluster_push_reduce<A0, N0, R0, N0, BM, NAT>(g, bucket, cc, fw0, rank, tmem_base, hi <= lo,
                                                        reinterpret_cast<float*>(smem), NTHR);
            tc_fence_before();
            __syncthreads();
        } else if (g.csplit > 1) {
            cluster_reduce<N0, BM>(g, bucket, cc, fw0, rank, reinterpret_cast<const float*>(smem), NTHR);
        }
    }
    if (threadIdx.x == 0) PTRACE(6);
    if (warp == 1) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(tmem_base));
    }
}

}  // namespace f16k
}  // namespace winrs
