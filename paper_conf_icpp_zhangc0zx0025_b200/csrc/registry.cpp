// Aggregates the kernel instantiations of all translation units.
#include <mutex>
#include <vector>
#include "registry.h"

namespace winrs {
const KernelEntry* f32_entries_part0(int* n);
const KernelEntry* f32_entries_part1(int* n);
const KernelEntry* f32_entries_part2(int* n);
const KernelEntry* f32_entries_part3(int* n);
const KernelEntry* f32_entries_part4(int* n);
const KernelEntry* f16_entries(int* n);
const KernelEntry* tc2_entries(int* n);
const KernelEntry* tc2x_entries(int* n);
const KernelEntry* tc3_entries(int* n);
const KernelEntry* c16_entries(int* n);

const KernelEntry* kernel_entries(int* count) {
    static std::vector<KernelEntry> all;
    static std::once_flag once;
    std::call_once(once, [] {
        const KernelEntry* (*parts[])(int*) = {f32_entries_part0, f32_entries_part1, f32_entries_part2,
                                               f32_entries_part3, f32_entries_part4, f16_entries,
                                               tc2_entries, tc2x_entries, tc3_entries, c16_entries};
        for (auto p : parts) {
            int n = 0;
            const KernelEntry* e = p(&n);
            all.insert(all.end(), e, e + n);
        }
    });
    *count = (int)all.size();
    return all.data();
}

}  // namespace winrs
