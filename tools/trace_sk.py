#!/usr/bin/env python3
"""Per-piece timeline of one CTA of the stream-K xi-split kernel (trace build:
python tools/build.py --variant tc2trace --define WINRS_TC2_TRACE).
Usage: WINRS_LIB=libwinrs_tc2trace.so WINRS_FORCE_TA=3 python tools/trace_sk.py <layer> [cta]"""
import ctypes
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_zhangc0zx0025_b200 as W  # noqa: E402
from paper_conf_icpp_zhangc0zx0025_b200 import _lib, workloads as wl  # noqa: E402

l = wl.LAYERS[sys.argv[1]]
cta = int(sys.argv[2]) if len(sys.argv) > 2 else 0
X, dY = wl.make_inputs(l)
Xg, Gg = torch.from_numpy(X).cuda(), torch.from_numpy(dY).cuda()
p = W.plan(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
L = _lib.lib()
tr = L.winrs_tc2x_trace
tr.argtypes = [ctypes.c_int, ctypes.c_void_p]
tr(cta, None)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for i in range(3):
    flush.fill_(i)
    W.bfc(p, Xg, Gg)
torch.cuda.synchronize()
buf = np.zeros((512, 8), dtype=np.int64)
tr(-1, buf.ctypes.data)
t0 = buf[511, 0]
print(p.kernel_name, "cta", cta, "setup", buf[511, 1] - t0, "end", buf[511, 6] - t0)
for pc in range(3):
    b = 490 + pc * 6
    if buf[b, 0] == 0:
        break
    print(f"piece {pc}: order {buf[b + 5, 0]} chunks {buf[b + 5, 1]}  start {buf[b, 0] - t0}  staged+reduced {buf[b + 1, 0] - t0}"
          f"  turn {buf[b + 2, 0] - t0}  released {buf[b + 3, 0] - t0}")
