#!/usr/bin/env python3
"""Ring-protocol stress: `calls` cold-L2 calls of each default FP16 plan;
every dW must equal the first bitwise.  Run with the jitter build
(python tools/build.py --variant tc2jit --define WINRS_TC2_JITTER;
WINRS_LIB=libwinrs_tc2jit.so) to randomise the relative timing of the TMA,
FT and MMA warps.  Usage: python tools/stress_tc2.py <calls> [layer,...]"""
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_zhangc0zx0025_b200 as W  # noqa: E402
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl  # noqa: E402

calls = int(sys.argv[1]) if len(sys.argv) > 1 else 1000
names = sys.argv[2].split(",") if len(sys.argv) > 2 else [l.name for l in wl.RESNET50_F16] + ["vgg_512_512_14_f16"]
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
bad_total = 0
for name in names:
    l = wl.LAYERS[name]
    X, dY = wl.make_inputs(l)
    Xg, Gg = torch.from_numpy(X).cuda(), torch.from_numpy(dY).cuda()
    p = W.plan(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
    ws = torch.empty(max(16, p.workspace_bytes), dtype=torch.uint8, device="cuda")
    ref = W.as_krsc(W.bfc(p, Xg, Gg, workspace=ws)).clone()
    out = torch.empty_like(ref)
    diff = torch.zeros((), dtype=torch.int64, device="cuda")
    t0 = time.time()
    for i in range(calls):
        flush.fill_(i & 255)
        W.bfc(p, Xg, Gg, out, ws)
        diff += (out != ref).any()      # every call compared on the device (no host sync)
    torch.cuda.synchronize()
    bad = int(diff.item())
    bad_total += bad
    print(f"{name}: {p.kernel_name} Z={p.info['Z']} cs={p.info['csplit']}: {calls} calls, "
          f"{bad} calls differ, finite={bool(torch.isfinite(ref).all())} ({time.time() - t0:.1f}s)", flush=True)
print("STRESS", "FAIL" if bad_total else "OK", bad_total)
sys.exit(1 if bad_total else 0)
