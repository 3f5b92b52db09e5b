// FP16 tensor-core kernels (tcgen05) — registered here.
#include "registry.h"
namespace winrs {
const KernelEntry* f16_entries(int* n) {
    *n = 0;
    return nullptr;
}
}  // namespace winrs
