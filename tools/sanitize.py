"""Small runs of every kernel family for compute-sanitizer (memcheck / racecheck / synccheck)."""
import os, sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_zhangc0zx0025_b200 as W
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
from oracle import oracle as O
cases = [
    wl.LAYERS["tiny_f32"],
    wl.LAYERS["r50_c64_56_f32"].with_(N=1, H=14, W=13, C=40, K=36),
    wl.LAYERS["wide_r5_f32"].with_(N=1, H=12, W=14, C=8, K=8),
    wl.LAYERS["r50_c64_56_f16"].with_(N=2, H=14, W=13, C=72, K=136),
    wl.LAYERS["r50_c64_56_f16"].with_(N=3, H=9, W=20, C=8, K=8),
]
envs = [{}, {"WINRS_FORCE_CSPLIT": "2"}, {"WINRS_FORCE_Z": "3"}]
for l in cases:
    for env in envs:
        os.environ.pop("WINRS_FORCE_CSPLIT", None); os.environ.pop("WINRS_FORCE_Z", None)
        os.environ.update(env)
        X, dY = wl.make_inputs(l)
        p = W.plan(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
        dW = W.bfc(p, torch.from_numpy(X).cuda(), torch.from_numpy(dY).cuda())
        torch.cuda.synchronize()
        err = O.rel_max_err(dW.cpu().numpy(), O.bfc_c(X, dY, l.R, l.S, l.pad))
        print(l.name, env, p, "err %.2e" % err, flush=True)
