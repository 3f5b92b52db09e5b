// FP32 instantiations: widths 2 and 4 (Omega_2(2,1), Omega_4(2,3), Omega_8(4,5)).
#include "bfc_f32_inst.cuh"
namespace winrs {
const KernelEntry* f32_entries_part1(int* n) {
    static const KernelEntry e[] = {
        WINRS_F32_ENTRY(4, 2, 3, 0, 0, 0, 64, 64),
        WINRS_F32_ENTRY(4, 2, 3, 0, 0, 0, 32, 32),
        WINRS_F32_ENTRY(4, 2, 3, 2, 2, 1, 64, 64),
        WINRS_F32_ENTRY(2, 2, 1, 0, 0, 0, 64, 64),
        WINRS_F32_ENTRY(8, 4, 5, 4, 2, 3, 64, 64),
        WINRS_F32_ENTRY(8, 4, 5, 4, 2, 3, 32, 32),
        WINRS_F32_ENTRY(8, 4, 5, 0, 0, 0, 64, 64),
        WINRS_F32_ENTRY(8, 4, 5, 0, 0, 0, 32, 32),
    };
    *n = sizeof(e) / sizeof(e[0]);
    return e;
}
}  // namespace winrs
