#!/usr/bin/env python3
"""Cold-L2 timing sweep of the second-generation tensor-core kernel
(bfc_tc2.cuh) over its tiles x cluster splits x segment counts, for
calibrating the planner's time model.  One JSON line per plan.
Usage: python tools/sweep_tc2.py r50_c64_56_f16,r50_c128_28_f16 [--quick | --xs]"""
import json
import os
import statistics
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icpp_zhangc0zx0025_b200 as W  # noqa: E402
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl  # noqa: E402

# (tile NK x bm, CTAs per UMMA, Xhat in TMEM): single CTA NK x (128 / F), a cta_group::2 pair,
# the swapped pair (256x128), or the TA kernels (NK = 64, Xhat in TMEM)
TILES = [("128x128", 1, 0), ("64x128", 1, 0), ("128x64", 1, 0), ("64x64", 1, 0), ("128x256", 2, 0), ("128x64", 2, 0),
         ("256x128", 2, 0), ("64x128", 1, 1), ("64x64", 1, 1), ("128x128", 2, 2), ("128x64", 2, 2)]
XS_TILES = [("128x128", 2, 2), ("128x64", 2, 2)]   # the xi-split pair (bfc_tc2x.cuh)


def time_plan(p, Xg, Gg, flush, reps=10):
    l_dw = torch.empty((p.info["K"], p.info["R"], p.info["S"], p.info["C"]), device="cuda")
    ws = torch.empty(max(16, p.workspace_bytes), dtype=torch.uint8, device="cuda")
    ts = []
    for i in range(reps + 2):
        flush.fill_(i)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        W.bfc(p, Xg, Gg, l_dw, ws)
        b.record()
        torch.cuda.synchronize()
        if i >= 2:
            ts.append(a.elapsed_time(b))
    return statistics.median(ts) * 1e3


def main():
    names = sys.argv[1].split(",")
    quick = "--quick" in sys.argv
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for name in names:
        l = wl.LAYERS[name]
        X, dY = wl.make_inputs(l)
        to = (lambda a: torch.from_numpy(a).cuda().to(torch.bfloat16)) if l.dtype == "bf16" else (lambda a: torch.from_numpy(a).cuda())
        Xg, Gg = to(X), to(dY)
        data = l.N * (l.H * l.W * l.C + (l.H + 2 * l.pad - l.R + 1) * (l.W + 2 * l.pad - l.S + 1) * l.K) * 2
        cfgs = [("auto", None, None, None), ("gen1", None, None, None), ("gen2", None, None, None)]
        zs = [1, 2, 4, 7, 8, 14, 16, 28, 56]
        if "--cs57" in sys.argv:   # odd cluster depth splits of the TA tiles
            cfgs = cfgs[:1] + [("f", t, cs, z) for t in [("64x128", 1, 1), ("64x64", 1, 1)] for cs in (3, 4, 5, 6, 7)
                               for z in zs]
        elif "--xs" in sys.argv:
            cfgs = cfgs[:1] + [("f", t, cs, z) for t in XS_TILES for cs in (1, 2, 3, 4) for z in zs]
        elif not quick:
            cfgs += [("f", t, cs, z) for t in TILES for cs in (1, 2, 3, 4, 6, 8) for z in zs]
        seen = set()
        for kind, t, cs, z in cfgs:
            for k in ("WINRS_FORCE_Z", "WINRS_FORCE_TILE", "WINRS_FORCE_CSPLIT", "WINRS_TC_GEN", "WINRS_FORCE_CG",
                      "WINRS_FORCE_TA"):
                os.environ.pop(k, None)
            if kind == "gen1":
                os.environ["WINRS_TC_GEN"] = "1"
            elif kind != "auto":
                os.environ["WINRS_TC_GEN"] = "2"
            if kind == "f":
                os.environ.update({"WINRS_FORCE_TILE": t[0], "WINRS_FORCE_CG": str(t[1]), "WINRS_FORCE_CSPLIT": str(cs),
                                   "WINRS_FORCE_Z": str(z), "WINRS_FORCE_TA": str(t[2])})
            try:
                p = W.plan(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
            except Exception:
                continue
            key = (p.kernel_name, p.info["csplit"], p.info["Z"], p.info["seg_h"], p.info["seg_w"])
            if kind == "f" and (p.workspace_bytes > 0.04 * data or p.info["csplit"] != cs or key in seen):
                continue
            seen.add(key)
            us = time_plan(p, Xg, Gg, flush)
            flops = p.info["direct_flops"]
            print(json.dumps({"layer": name, "kind": kind, "tile": t and list(t), "cs": p.info["csplit"], "Z": p.info["Z"],
                              "kernel": p.kernel_name, "ctas": p.info["ctas_main"], "model_us": round(p.model_us, 1),
                              "us": round(us, 2), "tflops": round(flops / us / 1e6, 1)}), flush=True)


if __name__ == "__main__":
    main()
