#!/usr/bin/env python3
"""A/B of the tc2 kernels with Xhat in shared memory (WINRS_FORCE_TA=0) and in
TMEM (=1) on the layers where NK = 64 tiles apply: cold-L2 per-call CUDA-event
times (256 MB flush between calls) and the oracle error at a reduced batch.
Usage: python tools/ta_ab.py [layer ...]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_zhangc0zx0025_b200 as W  # noqa: E402
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl  # noqa: E402
from oracle import oracle as O  # noqa: E402

LAYERS = sys.argv[1:] or ["vgg_64_64_224_f16", "r50_c64_56_f16", "vgg_64_128_112_f16"]


def timed(p, Xg, Gg, flush, reps=10):
    out = []
    for i in range(reps + 3):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        W.bfc(p, Xg, Gg)
        b.record()
        torch.cuda.synchronize()
        if i >= 3:
            out.append(a.elapsed_time(b))
    return float(np.median(out))


def main():
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for name in LAYERS:
        l = wl.LAYERS[name]
        X, dY = wl.make_inputs(l)
        Xg, Gg = torch.from_numpy(X).cuda(), torch.from_numpy(dY).cuda()
        small = l.with_(N=16, name=l.name + "_n16")
        Xs, Gs = wl.make_inputs(small)
        ref = O.bfc_c(Xs, Gs, small.R, small.S, small.pad)
        for ta in ("0", "1"):
            for tile in (None, "64x64", "64x128"):
                os.environ["WINRS_FORCE_TA"] = ta
                os.environ["WINRS_TC_GEN"] = "2"
                if tile:
                    os.environ["WINRS_FORCE_TILE"] = tile
                else:
                    os.environ.pop("WINRS_FORCE_TILE", None)
                try:
                    p = W.plan(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
                    ps = W.plan(small.N, small.C, small.H, small.W, small.K, small.R, small.S, small.pad, small.dtype)
                except Exception as e:
                    print(f"{name} TA={ta} tile={tile}: {e}")
                    continue
                ms = timed(p, Xg, Gg, flush)
                got = W.as_krsc(W.bfc(ps, torch.from_numpy(Xs).cuda(), torch.from_numpy(Gs).cuda()))
                torch.cuda.synchronize()
                err = O.rel_max_err(got.cpu().numpy().astype(np.float64), ref)
                flops = 2.0 * l.N * l.C * l.K * l.Ho * l.Wo * l.R * l.S
                print(f"{name:22s} TA={ta} tile={str(tile):7s} {p.kernel_name:28s} Z={p.info['Z']:3d} "
                      f"cs={p.info['csplit']} {ms * 1e3:8.1f} us {flops / ms / 1e9:7.1f} TF  err(n16,{ps.kernel_name})={err:.2e}",
                      flush=True)
        for k in ("WINRS_FORCE_TA", "WINRS_TC_GEN", "WINRS_FORCE_TILE"):
            os.environ.pop(k, None)


if __name__ == "__main__":
    main()
