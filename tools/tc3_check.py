#!/usr/bin/env python3
"""Developer check of the FP32 tensor-core kernel (bfc_tc3.cuh, 3xTF32)
against the FP64 oracle, plus cold-L2 timings of the ResNet-50 FP32 layers
with and without it.  Usage: python tools/tc3_check.py [--time]"""
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

BASE = wl.LAYERS["r50_c64_56_f32"]
CASES = [
    ("l1", dict(N=8), {}),
    ("l1_f2", dict(N=8), {"WINRS_FORCE_TILE": "64x64"}),
    ("l1_f1_cs2", dict(N=8), {"WINRS_FORCE_TILE": "64x128", "WINRS_FORCE_CSPLIT": "2"}),
    ("l3", dict(N=8, C=256, K=256, H=14, W=14), {}),
    ("ragged", dict(N=8, C=72, K=100, H=20, W=17), {}),
    ("ragged_f2", dict(N=16, C=40, K=136, H=13, W=11), {"WINRS_FORCE_TILE": "64x64", "WINRS_FORCE_CSPLIT": "3"}),
    ("pad0", dict(N=8, C=64, K=64, H=20, W=20, pad=0), {}),
    ("r5", dict(N=8, C=64, K=64, H=16, W=16, R=5, S=3, pad=2), {}),
    ("s6", dict(N=8, C=64, K=64, H=16, W=16, R=3, S=6, pad=2), {"WINRS_FORCE_PAIR": "4,3,2,0,0,0"}),
    ("z5", dict(N=16, C=64, K=64, H=30, W=30), {"WINRS_FORCE_Z": "5"}),
    ("cs8", dict(N=24, C=128, K=64, H=12, W=12), {"WINRS_FORCE_CSPLIT": "8"}),
    ("nk128", dict(N=8, C=128, K=128, H=14, W=14), {"WINRS_FORCE_TILE": "128x128"}),
    ("nk128_f2_ragged", dict(N=16, C=40, K=200, H=13, W=11), {"WINRS_FORCE_TILE": "128x64", "WINRS_FORCE_CSPLIT": "3"}),
    ("nk128_z3_cs4", dict(N=16, C=64, K=128, H=30, W=30), {"WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_Z": "3",
                                                          "WINRS_FORCE_CSPLIT": "4"}),
]
KEYS = ("WINRS_FORCE_TILE", "WINRS_FORCE_CSPLIT", "WINRS_FORCE_Z", "WINRS_FORCE_PAIR", "WINRS_FP32_TC")


def check():
    bad = 0
    for name, ov, env in CASES:
        for dist in ("u01", "signed"):
            for k in KEYS:
                os.environ.pop(k, None)
            os.environ.update(env)
            os.environ["WINRS_FP32_TC"] = "1"
            layer = BASE.with_(name=name, **ov)
            X, dY = wl.make_inputs(layer, dist)
            try:
                p = W.plan(layer.N, layer.C, layer.H, layer.W, layer.K, layer.R, layer.S, layer.pad, "f32")
                dW = W.as_krsc(W.bfc(p, torch.from_numpy(X).cuda(), torch.from_numpy(dY).cuda()))
                torch.cuda.synchronize()
                got = dW.cpu().numpy().astype(np.float64)
                err = O.rel_max_err(got, O.bfc_c(X, dY, layer.R, layer.S, layer.pad))
                ok = err <= 1e-4 and np.isfinite(got).all()
                msg = f"err={err:.3e} kernel={p.kernel_name} Z={p.info['Z']} cs={p.info['csplit']}"
            except Exception as e:
                ok, msg = False, f"EXC {e}"
            bad += not ok
            print(f"{'OK ' if ok else 'BAD'} {name:12s} {dist:6s} {msg}", flush=True)
    print("FAILURES", bad, flush=True)
    return bad


def timing():
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for l in wl.RESNET50_F32 + wl.WIDE_F32[-1:]:
        X, dY = wl.make_inputs(l)
        Xg, Gg = torch.from_numpy(X).cuda(), torch.from_numpy(dY).cuda()
        for tc, tile in (("0", None), ("1", None), ("1", "64x128"), ("1", "128x128"), ("1", "128x64"), ("1", "64x64")):
            for k in KEYS:
                os.environ.pop(k, None)
            os.environ["WINRS_FP32_TC"] = tc
            if tile:
                os.environ["WINRS_FORCE_TILE"] = tile
            try:
                p = W.plan(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, "f32")
            except Exception as e:
                print(l.name, tc, e)
                continue
            ts = []
            for i in range(12):
                flush.fill_(i)
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                W.bfc(p, Xg, Gg)
                b.record()
                torch.cuda.synchronize()
                if i >= 2:
                    ts.append(a.elapsed_time(b))
            ms = float(np.median(ts))
            print(f"{l.name:18s} TC={tc} {p.kernel_name:30s} Z={p.info['Z']:3d} cs={p.info['csplit']} "
                  f"{ms * 1e3:8.1f} us  {p.info['direct_flops'] / ms / 1e9:6.1f} TF  model {p.model_us:.1f}", flush=True)


if __name__ == "__main__":
    torch.cuda.set_device(0)
    b = check()
    if "--time" in sys.argv:
        timing()
    sys.exit(1 if b else 0)
