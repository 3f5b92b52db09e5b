#!/usr/bin/env python3
"""Run one workload layer's BFC `reps` times (for ncu captures).
Usage: python tools/run_layer.py <layer> [reps]   (env WINRS_* overrides apply)"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_zhangc0zx0025_b200 as W  # noqa: E402
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl  # noqa: E402

l = wl.LAYERS[sys.argv[1]]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
X, dY = wl.make_inputs(l)
to = (lambda a: torch.from_numpy(a).cuda().to(torch.bfloat16)) if l.dtype == "bf16" else (lambda a: torch.from_numpy(a).cuda())
Xg, Gg = to(X), to(dY)
p = W.plan(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
print(p.kernel_name, p.info["Z"], p.info["csplit"], flush=True)
for _ in range(reps):
    W.bfc(p, Xg, Gg)
torch.cuda.synchronize()
