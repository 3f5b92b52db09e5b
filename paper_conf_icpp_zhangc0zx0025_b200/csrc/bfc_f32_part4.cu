// FP32 instantiations: widths 9, 6 and 8 (Omega_16(9,8), Omega_8(6,3),
// Omega_16(6,11), Omega_16(8,9)).
#include "bfc_f32_inst.cuh"
namespace winrs {
const KernelEntry* f32_entries_part4(int* n) {
    static const KernelEntry e[] = {
        WINRS_F32_ENTRY(16, 9, 8, 0, 0, 0, 64, 32),
        WINRS_F32_ENTRY(16, 9, 8, 0, 0, 0, 32, 32),
        WINRS_F32_ENTRY(16, 9, 8, 4, 3, 2, 64, 32),
        WINRS_F32_ENTRY(8, 6, 3, 0, 0, 0, 64, 64),
        WINRS_F32_ENTRY(8, 6, 3, 4, 3, 2, 64, 64),
        WINRS_F32_ENTRY(16, 6, 11, 0, 0, 0, 64, 32),
        WINRS_F32_ENTRY(16, 8, 9, 0, 0, 0, 64, 32),
        WINRS_F32_ENTRY(16, 8, 9, 8, 4, 5, 64, 32),
    };
    *n = sizeof(e) / sizeof(e[0]);
    return e;
}
}  // namespace winrs
