#!/usr/bin/env python3
"""Per-stage timeline of one CTA of the tc2 kernel (debug build
libwinrs_tc2trace.so: python tools/build.py --variant tc2trace --define WINRS_TC2_TRACE).
Usage: WINRS_LIB=libwinrs_tc2trace.so python tools/trace_tc2.py <layer> [cta]"""
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
tr = L.winrs_tc2x_trace if "_v2x_" in p.kernel_name else L.winrs_tc2_trace   # one buffer per translation unit
tr.argtypes = [ctypes.c_int, ctypes.c_void_p]
tr(cta, None)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for i in range(3):
    flush.fill_(i)
    W.bfc(p, Xg, Gg)
torch.cuda.synchronize()
buf = np.zeros((512, 8), dtype=np.int64)
tr(-1, buf.ctypes.data)
print(p.kernel_name, "Z", p.info["Z"], "cs", p.info["csplit"])
t0 = buf[511, 0]
n = 0
while n < 511 and buf[n, 5] > 0:
    n += 1
k = buf[511]
print("kernel phases (cycles from CTA start): setup", k[1] - k[0], " accfull", k[2] - k[0], " epilogue done", k[3] - k[0],
      " cluster sync", k[4] - k[0], " reduction done", k[5] - k[0], " end", k[6] - k[0])
print("stage  prodOK  tmaIss  txFull  txDone  mmaOK  mmaIss   (cycles rel. to stage-0 producer)")
for i in range(n):
    print(f"{i:4d} " + " ".join(f"{int(buf[i, e] - t0):7d}" for e in range(6)))
d = np.diff(buf[:n, 5]) if n > 1 else np.zeros(0)
print("mean cycles/stage (mma issue):", d.mean() if len(d) else 0,
      " full-wait latency (tx full - tma issue):", np.mean(buf[:n, 2] - buf[:n, 1]))
