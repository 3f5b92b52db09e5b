#!/usr/bin/env python3
"""Cold-L2 median time of one layer's plan under the current WINRS_* env
(the planner's choice, or forced knobs).  Usage: time_layer.py <layer> [reps]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_zhangc0zx0025_b200 as W  # noqa: E402
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl  # noqa: E402
from sweep_tc2 import time_plan  # noqa: E402

l = wl.LAYERS[sys.argv[1]]
X, dY = wl.make_inputs(l)
to = (lambda a: torch.from_numpy(a).cuda().to(torch.bfloat16)) if l.dtype == "bf16" else (lambda a: torch.from_numpy(a).cuda())
p = W.plan(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
us = time_plan(p, to(X), to(dY), flush, int(sys.argv[2]) if len(sys.argv) > 2 else 20)
env = {k: v for k, v in os.environ.items() if k.startswith("WINRS_")}
print(f"{l.name} {p.kernel_name} cs={p.info['csplit']} Z={p.info['Z']} {us:.2f} us {env}")
