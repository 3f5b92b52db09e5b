#!/usr/bin/env python3
"""Developer check of the second-generation tensor-core kernel (bfc_tc2.cuh)
against the FP64 oracle on reduced layers, with forced tiles / cluster splits /
segment counts.  Prints one line per case.  Usage: python tools/tc2_check.py"""
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icpp_zhangc0zx0025_b200 as W  # noqa: E402
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl  # noqa: E402
from oracle import oracle as O  # noqa: E402

BASE = wl.LAYERS["r50_c64_56_f16"]
CASES = [
    # (name, layer overrides, env)
    ("l1_auto", dict(N=16), {}),
    ("l1_f2nk64", dict(N=16), {"WINRS_FORCE_TILE": "64x64"}),
    ("l1_f1nk64_cs2", dict(N=16), {"WINRS_FORCE_TILE": "64x128", "WINRS_FORCE_CSPLIT": "2"}),
    ("l2_auto", dict(N=16, C=128, K=128, H=28, W=28), {}),
    ("l2_f1nk128_cs1", dict(N=16, C=128, K=128, H=28, W=28), {"WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_CSPLIT": "1"}),
    ("l2_f1nk128_cs4", dict(N=16, C=128, K=128, H=28, W=28), {"WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_CSPLIT": "4"}),
    ("l3_auto", dict(N=16, C=256, K=256, H=14, W=14), {}),
    ("l4_auto", dict(N=16, C=512, K=512, H=7, W=7), {}),
    ("ragged", dict(N=16, C=72, K=200, H=20, W=17), {}),
    ("ragged_f2", dict(N=16, C=40, K=136, H=20, W=17), {"WINRS_FORCE_TILE": "128x64"}),
    ("pad0", dict(N=16, C=64, K=64, H=20, W=20, pad=0), {}),
    ("s6", dict(N=16, C=64, K=64, H=16, W=16, R=3, S=6, pad=2), {"WINRS_FORCE_PAIR": "4,3,2,0,0,0"}),
    ("r5_f2", dict(N=16, C=64, K=128, H=16, W=16, R=5, S=3, pad=2), {"WINRS_FORCE_TILE": "128x64"}),
    ("n32_z5", dict(N=32, C=64, K=64, H=30, W=30), {"WINRS_FORCE_Z": "5"}),
    ("n48_cs8", dict(N=48, C=128, K=64, H=12, W=12), {"WINRS_FORCE_CSPLIT": "8"}),
    ("pair_l3", dict(N=16, C=256, K=256, H=14, W=14), {"WINRS_FORCE_CG": "2", "WINRS_FORCE_CSPLIT": "1"}),
    ("pair_l3_cs4", dict(N=16, C=256, K=256, H=14, W=14), {"WINRS_FORCE_CG": "2", "WINRS_FORCE_CSPLIT": "4"}),
    ("pair_f1_ragged", dict(N=16, C=200, K=136, H=12, W=13), {"WINRS_FORCE_CG": "2", "WINRS_FORCE_TILE": "128x256"}),
    ("pair_f2", dict(N=16, C=64, K=128, H=20, W=20), {"WINRS_FORCE_CG": "2", "WINRS_FORCE_TILE": "128x64"}),
    ("pair_f2_cs2_r5", dict(N=32, C=128, K=128, H=12, W=12, R=5, S=3, pad=2), {"WINRS_FORCE_CG": "2", "WINRS_FORCE_TILE": "128x64", "WINRS_FORCE_CSPLIT": "2"}),
    ("pair_cs8", dict(N=16, C=256, K=128, H=12, W=12), {"WINRS_FORCE_CG": "2", "WINRS_FORCE_CSPLIT": "8"}),
    ("swap_l3", dict(N=16, C=256, K=256, H=14, W=14), {"WINRS_FORCE_TILE": "256x128", "WINRS_FORCE_CSPLIT": "1"}),
    ("swap_l3_cs4", dict(N=16, C=256, K=256, H=14, W=14), {"WINRS_FORCE_TILE": "256x128", "WINRS_FORCE_CSPLIT": "4"}),
    ("swap_ragged", dict(N=16, C=200, K=328, H=12, W=13), {"WINRS_FORCE_TILE": "256x128", "WINRS_FORCE_CSPLIT": "2"}),
    ("swap_l4_z", dict(N=32, C=128, K=256, H=7, W=7), {"WINRS_FORCE_TILE": "256x128", "WINRS_FORCE_CSPLIT": "3"}),
    ("swap_pad0_s6", dict(N=16, C=128, K=256, H=12, W=14, S=6, pad=0), {"WINRS_FORCE_TILE": "256x128", "WINRS_FORCE_PAIR": "4,3,2,0,0,0"}),
]


def main():
    torch.cuda.set_device(0)
    os.environ["WINRS_TC_GEN"] = "2"
    bad = 0
    sel = sys.argv[1:]
    for name, ov, env in CASES:
        if sel and name not in sel:
            continue
        for dt in ("f16", "bf16"):
            for k in ("WINRS_FORCE_TILE", "WINRS_FORCE_CSPLIT", "WINRS_FORCE_Z", "WINRS_FORCE_PAIR", "WINRS_FORCE_CG"):
                os.environ.pop(k, None)
            os.environ.update(env)
            layer = BASE.with_(name=name, dtype=dt, **ov)
            X, dY = wl.make_inputs(layer)
            p = W.plan(layer.N, layer.C, layer.H, layer.W, layer.K, layer.R, layer.S, layer.pad, dt)
            to = (lambda a: torch.from_numpy(a).cuda().to(torch.bfloat16)) if dt == "bf16" else (lambda a: torch.from_numpy(a).cuda())
            t0 = time.time()
            dW = W.as_krsc(W.bfc(p, to(X), to(dY)))
            torch.cuda.synchronize()
            got = dW.cpu().numpy().astype(np.float64)
            ref = O.bfc_c(X, dY, layer.R, layer.S, layer.pad)
            err = O.rel_max_err(got, ref)
            ok = err <= 2e-2 and np.isfinite(got).all()
            bad += not ok
            print(f"{'OK ' if ok else 'BAD'} {name:16s} {dt:5s} err={err:.3e} kernel={p.kernel_name} Z={p.info['Z']} "
                  f"cs={p.info['csplit']} ({time.time() - t0:.2f}s)", flush=True)
    print("FAILURES", bad)
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main())
