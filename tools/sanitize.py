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
    # Omega_4(3,2) paired / round-robin units, 128x128 tile, ragged K and C
    wl.LAYERS["r50_c256_14_f16"].with_(N=2, H=14, W=14, C=136, K=200),
    # bfc_tc2.cuh (N % 16 == 0): stacked fh (F = 2), NK 64 / 128, a cta_group::2 pair
    wl.LAYERS["r50_c64_56_f16"].with_(N=16, H=10, W=11),
    wl.LAYERS["r50_c256_14_f16"].with_(N=16, H=7, W=7, C=256, K=128),
    wl.LAYERS["r50_c256_14_f16"].with_(N=16, H=6, W=9, C=200, K=136, dtype="bf16"),
    # bfc_tc3.cuh: FP32 on the tensor cores (N % 8 == 0)
    wl.LAYERS["r50_c64_56_f32"].with_(N=8, H=10, W=11, C=72, K=100),
]
envs = [{}, {"WINRS_FORCE_CSPLIT": "2"}, {"WINRS_FORCE_Z": "3"}, {"WINRS_FORCE_PAIR": "4,3,2,0,0,0", "WINRS_FORCE_CSPLIT": "4"},
        {"WINRS_FORCE_CG": "2", "WINRS_FORCE_CSPLIT": "2"}, {"WINRS_FORCE_CSPLIT": "5"},
        {"WINRS_FORCE_TA": "2", "WINRS_FORCE_CSPLIT": "2"}]
for l in cases:
    for env in envs:
        for k in ("WINRS_FORCE_CSPLIT", "WINRS_FORCE_Z", "WINRS_FORCE_PAIR", "WINRS_FORCE_CG", "WINRS_FORCE_TA"):
            os.environ.pop(k, None)
        if "WINRS_FORCE_PAIR" in env and l.dtype != "f16":
            continue
        if ("WINRS_FORCE_CG" in env or "WINRS_FORCE_TA" in env) and (l.N % 16 or l.dtype == "f32"):
            continue
        os.environ.update(env)
        X, dY = wl.make_inputs(l)
        try:
            p = W.plan(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
        except Exception as e:   # a forced pair that does not apply to this shape
            print(l.name, env, "skipped:", e, flush=True)
            continue
        to = (lambda a: torch.from_numpy(a).cuda().to(torch.bfloat16)) if l.dtype == "bf16" else (lambda a: torch.from_numpy(a).cuda())
        dW = W.as_krsc(W.bfc(p, to(X), to(dY)))
        torch.cuda.synchronize()
        err = O.rel_max_err(dW.cpu().numpy(), O.bfc_c(X, dY, l.R, l.S, l.pad))
        print(l.name, env, p, "err %.2e" % err, flush=True)
