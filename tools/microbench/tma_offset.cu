// Probe (round 2): does a SWIZZLE_128B TMA load into a shared-memory
// destination that is only 256-byte aligned (not 1024) work, and is the
// 16-byte chunk XOR taken from the absolute address bits [7:9] (row phase of
// the destination) or from the row index within the box?
// Build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a tma_offset.cu -o tma_offset.bin
#include <cstdint>
#include <cstdio>
#include <cuda.h>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void k(const __grid_constant__ CUtensorMap m, uint16_t* out, int off) {
    __shared__ __align__(1024) uint8_t sm[4096];
    __shared__ __align__(8) uint64_t bar;
    for (int i = threadIdx.x; i < 4096 / 2; i += blockDim.x) reinterpret_cast<uint16_t*>(sm)[i] = 0xFFFF;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su(&bar)), "r"(8 * 128) : "memory");
        asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                     :: "r"(su(sm) + off), "l"(reinterpret_cast<uint64_t>(&m)), "r"(0), "r"(0), "r"(su(&bar)) : "memory");
    }
    asm volatile("{\n.reg .pred P;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n@!P bra W_%=;\n}\n" :: "r"(su(&bar)) : "memory");
    for (int i = threadIdx.x; i < 4096 / 2; i += blockDim.x) out[i] = reinterpret_cast<uint16_t*>(sm)[i];
}

typedef CUresult (*EncFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                          const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                          CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
    EncFn enc = (EncFn)p;
    uint16_t h[64 * 8];
    for (int r = 0; r < 8; ++r)
        for (int c = 0; c < 64; ++c) h[r * 64 + c] = (uint16_t)(r * 256 + c);   // tag: row << 8 | channel
    uint16_t* g;
    cudaMalloc(&g, sizeof(h));
    cudaMemcpy(g, h, sizeof(h), cudaMemcpyHostToDevice);
    CUtensorMap m;
    const cuuint64_t dims[2] = {64, 8}, strides[1] = {128};
    const cuuint32_t box[2] = {64, 8}, es[2] = {1, 1};
    CUresult r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_UINT16, 2, g, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("encode %d\n", (int)r);
    uint16_t* o;
    cudaMalloc(&o, 4096);
    for (int off : {0, 256, 512, 128}) {
        k<<<1, 128>>>(m, o, off);
        uint16_t s[2048];
        cudaError_t e = cudaMemcpy(s, o, 4096, cudaMemcpyDeviceToHost);
        printf("dst offset %d: %s\n", off, cudaGetErrorString(e));
        if (e != cudaSuccess) { cudaGetLastError(); break; }
        int abs_ok = 0, rel_ok = 0;
        for (int row = 0; row < 8; ++row)
            for (int j = 0; j < 8; ++j) {
                const int a = off + row * 128;
                const int chunk_abs = j ^ (((a >> 7)) & 7), chunk_rel = j ^ (row & 7);
                const uint16_t want = (uint16_t)(row * 256 + j * 8);
                abs_ok += s[(a + chunk_abs * 16) / 2] == want;
                rel_ok += s[(a + chunk_rel * 16) / 2] == want;
            }
        printf("  chunks matching address-based swizzle: %d/64, box-row-based: %d/64\n", abs_ok, rel_ok);
    }
    return 0;
}
