// FP32 instantiations: 3x3 family (Omega_8(3,6), Omega_4(3,2)).
#include "bfc_f32_inst.cuh"
namespace winrs {
const KernelEntry* f32_entries_part0(int* n) {
    static const KernelEntry e[] = {
        WINRS_F32_ENTRY(8, 3, 6, 4, 3, 2, 64, 64),
        WINRS_F32_ENTRY(8, 3, 6, 4, 3, 2, 32, 32),
        WINRS_F32_ENTRY(8, 3, 6, 4, 3, 2, 64, 32),
        WINRS_F32_ENTRY(8, 3, 6, 0, 0, 0, 64, 64),
        WINRS_F32_ENTRY(8, 3, 6, 0, 0, 0, 32, 32),
        WINRS_F32_ENTRY(4, 3, 2, 0, 0, 0, 64, 64),
        WINRS_F32_ENTRY(4, 3, 2, 0, 0, 0, 32, 32),
    };
    *n = sizeof(e) / sizeof(e[0]);
    return e;
}
}  // namespace winrs
