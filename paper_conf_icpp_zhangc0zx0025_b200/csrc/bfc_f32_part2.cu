// FP32 instantiations: width 5 (Omega_16(5,12), Omega_8(5,4)).
#include "bfc_f32_inst.cuh"
namespace winrs {
const KernelEntry* f32_entries_part2(int* n) {
    static const KernelEntry e[] = {
        WINRS_F32_ENTRY(16, 5, 12, 8, 5, 4, 64, 32),
        WINRS_F32_ENTRY(16, 5, 12, 8, 5, 4, 32, 32),
        WINRS_F32_ENTRY(16, 5, 12, 0, 0, 0, 64, 32),
        WINRS_F32_ENTRY(16, 5, 12, 0, 0, 0, 32, 32),
        WINRS_F32_ENTRY(8, 5, 4, 0, 0, 0, 64, 64),
        WINRS_F32_ENTRY(8, 5, 4, 0, 0, 0, 32, 32),
    };
    *n = sizeof(e) / sizeof(e[0]);
    return e;
}
}  // namespace winrs
