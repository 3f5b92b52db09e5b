#!/usr/bin/env python3
"""Error of the default / forced kernels on one reduced layer against the FP64
oracle, element by element (developer check of the xi-split / stream-K paths'
accuracy relative to TA).  Usage: xs_err_check.py <layer> N"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_zhangc0zx0025_b200 as W  # noqa: E402
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl  # noqa: E402
from oracle import oracle as O  # noqa: E402

l = wl.LAYERS[sys.argv[1]].with_(N=int(sys.argv[2]))
X, dY = wl.make_inputs(l)
ref = O.bfc_c(X, dY, l.R, l.S, l.pad)
for env in ({"WINRS_FORCE_TA": "1"}, {"WINRS_FORCE_TA": "2"}, {"WINRS_FORCE_TA": "3"}, {"WINRS_FORCE_TA": "0"}):
    for k in ("WINRS_FORCE_TA", "WINRS_TC_GEN"):
        os.environ.pop(k, None)
    os.environ.update(env)
    os.environ["WINRS_TC_GEN"] = "2"
    p = W.plan(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
    got = W.as_krsc(W.bfc(p, torch.from_numpy(X).cuda(), torch.from_numpy(dY).cuda())).cpu().numpy().astype(np.float64)
    d = np.abs(got - ref)
    print(f"{env} {p.kernel_name} cs={p.info['csplit']} Z={p.info['Z']}: rel_max {d.max() / np.abs(ref).max():.3e}"
          f" rel_mean {d.mean() / np.abs(ref).mean():.3e}")
