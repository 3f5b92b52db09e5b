// Planner interface (host only).
#pragma once
#include "../../include/winrs.h"
#include "registry.h"
#include "winrs_internal.h"

namespace winrs {

// For an N-D problem N = Nb * Do images and R = T * Rh filter rows (the 2-D
// decomposition the kernels run); Nb, Rh, T, D, Do describe the original axes.
struct Problem {
    int N, C, H, W, K, R, S, pad, Ho, Wo;
    int dtype;
    int Nb = 0, Rh = 0, T = 1, D = 1, Do = 1;
};

struct PlanResult {
    Geometry geom;
    const KernelEntry* entry = nullptr;
    int z_hat = 1;
    int masked = 0;
    double ewm_flops = 0;
    double model_s = 0;   // B200 time-model estimate of the launch(es), seconds
};

winrs_status_t make_plan(const Problem& p, int num_sms, PlanResult* out);

}  // namespace winrs
