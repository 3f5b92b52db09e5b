// FP32 instantiations: width 7 (Omega_16(7,10), Omega_8(7,2)).
#include "bfc_f32_inst.cuh"
namespace winrs {
const KernelEntry* f32_entries_part3(int* n) {
    static const KernelEntry e[] = {
        WINRS_F32_ENTRY(16, 7, 10, 8, 7, 2, 64, 32),
        WINRS_F32_ENTRY(16, 7, 10, 8, 7, 2, 32, 32),
        WINRS_F32_ENTRY(16, 7, 10, 0, 0, 0, 64, 32),
        WINRS_F32_ENTRY(16, 7, 10, 0, 0, 0, 32, 32),
        WINRS_F32_ENTRY(8, 7, 2, 0, 0, 0, 64, 64),
        WINRS_F32_ENTRY(8, 7, 2, 0, 0, 0, 32, 32),
    };
    *n = sizeof(e) / sizeof(e[0]);
    return e;
}
}  // namespace winrs
