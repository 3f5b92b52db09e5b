// FP16 / BF16 plans of the alpha = 16 widths (Omega_16(9,8),
// Omega_16(7,10) with the eq. (7) scaled transforms): 16-bit inputs on the FP32
// CUDA-core pipeline (R26).
#include "bfc_f32_inst.cuh"
namespace winrs {
const KernelEntry* c16_entries(int* n) {
    static const KernelEntry e[] = {
        WINRS_C16_ENTRY(1, __half, "f16", 16, 9, 8, 0, 0, 0, 64, 32),
        WINRS_C16_ENTRY(1, __half, "f16", 16, 9, 8, 4, 3, 2, 64, 32),
        WINRS_C16_ENTRY(1, __half, "f16", 16, 7, 10, 8, 7, 2, 64, 32),
        WINRS_C16_ENTRY(1, __half, "f16", 16, 7, 10, 0, 0, 0, 64, 32),
        WINRS_C16_ENTRY(2, __nv_bfloat16, "bf16", 16, 9, 8, 0, 0, 0, 64, 32),
        WINRS_C16_ENTRY(2, __nv_bfloat16, "bf16", 16, 9, 8, 4, 3, 2, 64, 32),
        WINRS_C16_ENTRY(2, __nv_bfloat16, "bf16", 16, 7, 10, 8, 7, 2, 64, 32),
        WINRS_C16_ENTRY(2, __nv_bfloat16, "bf16", 16, 7, 10, 0, 0, 0, 64, 32),
    };
    *n = sizeof(e) / sizeof(e[0]);
    return e;
}
}  // namespace winrs
