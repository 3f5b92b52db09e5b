"""Calibration sweep: time every (CTA tile, cluster split) variant of the plan
for each benchmark layer (CUDA events, L2 flushed, median of 5).  Output: one
JSON line per (layer, tile, csplit)."""
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_zhangc0zx0025_b200 as W  # noqa: E402
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl  # noqa: E402

layers = [wl.LAYERS[n] for n in sys.argv[1].split(",")] if len(sys.argv) > 1 and sys.argv[1] != "all" else \
    wl.RESNET50_F32 + wl.RESNET50_F16 + wl.WIDE_F32
# optional second argument: comma-separated forced segment counts Z (default: the planner's)
zs = [int(z) for z in sys.argv[2].split(",")] if len(sys.argv) > 2 else [None]
tiles = {"f32": ["64x64", "32x32", "64x32"], "f16": ["128x128", "128x64", "128x32"]}
pairs = {"f32": [None], "f16": [None, "4,3,2,0,0,0"]}
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for l in layers:
    X, dY = wl.make_inputs(l)
    Xg, Gg = torch.from_numpy(X).cuda(), torch.from_numpy(dY).cuda()
    for pair in pairs[l.dtype]:
      for t in tiles[l.dtype]:
       for z in zs:
        for cs in (1, 2, 4, 8):
            if z is None:
                os.environ.pop("WINRS_FORCE_Z", None)
            else:
                os.environ["WINRS_FORCE_Z"] = str(z)
            os.environ["WINRS_FORCE_TILE"] = t
            os.environ["WINRS_FORCE_CSPLIT"] = str(cs)
            if pair:
                os.environ["WINRS_FORCE_PAIR"] = pair
            else:
                os.environ.pop("WINRS_FORCE_PAIR", None)
            try:
                p = W.plan(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
            except Exception:
                continue
            if p.info["tile_k0"] != int(t.split("x")[0]) or p.info["tile_c0"] != int(t.split("x")[1]):
                continue
            dW = torch.empty((l.K, l.R, l.S, l.C), device="cuda")
            ws = torch.empty(max(16, p.workspace_bytes), dtype=torch.uint8, device="cuda")
            ts = []
            for i in range(7):
                flush.fill_(i)
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                W.bfc(p, Xg, Gg, dW, ws)
                b.record()
                torch.cuda.synchronize()
                if i >= 2:
                    ts.append(a.elapsed_time(b))
            ms = statistics.median(ts)
            print(json.dumps({"layer": l.name, "pair": p.kernel_name, "tile": t, "csplit": p.info["csplit"], "Z": p.info["Z"],
                              "ctas": p.info["ctas_main"], "ws": p.workspace_bytes,
                              "data": l.N * (l.H * l.W * l.C + p.info["Ho"] * p.info["Wo"] * l.K) * (4 if l.dtype == "f32" else 2),
                              "ewm": p.info["ewm_flops"], "us": round(ms * 1e3, 1),
                              "tflops": round(l.direct_flops / ms / 1e9, 1)}), flush=True)
os.environ.pop("WINRS_FORCE_TILE", None)
os.environ.pop("WINRS_FORCE_CSPLIT", None)
os.environ.pop("WINRS_FORCE_Z", None)
