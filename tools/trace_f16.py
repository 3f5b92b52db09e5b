"""Debug: CTA-0 timeline of the FP16 kernel (needs libwinrs_trace.so)."""
import ctypes, os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_zhangc0zx0025_b200 import _lib
_lib.LIB_PATH = _lib.LIB_PATH.replace("libwinrs.so", os.environ.get("WINRS_TRACE_LIB", "libwinrs_trace.so"))
import paper_conf_icpp_zhangc0zx0025_b200 as W
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
name = sys.argv[1] if len(sys.argv) > 1 else "r50_c512_7_f16"
l = wl.LAYERS[name]
X, dY = wl.make_inputs(l)
p = W.plan(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
Xg, Gg = torch.from_numpy(X).cuda(), torch.from_numpy(dY).cuda()
for _ in range(3):
    W.bfc(p, Xg, Gg)
torch.cuda.synchronize()
buf = np.zeros((4, 256, 4), dtype=np.uint64)
L = _lib.lib()
L.winrs_trace_read.argtypes = [ctypes.c_void_p]
print("rc", L.winrs_trace_read(buf.ctypes.data))
t0 = min(v for v in buf.ravel() if v > 0)
b = np.where(buf > 0, buf.astype(np.int64) - int(t0), -1)
print(p)
print("chunk | prod: before_wait after_wait | tx: start raw_ok op_ok done | mma: opfull issued | ft_computed it_computed ft_fenced")
for c in list(range(0, 40)) + list(range(64, 90)):
    if b[2, c, 0] < 0 and b[0, c, 0] < 0:
        continue
    print(c, "|", b[0, c, 0], b[0, c, 1], "|", b[2, c, 0], b[2, c, 1], b[2, c, 2], b[2, c, 3], "|", b[1, c, 0], b[1, c, 1], "|", b[3, c, 0], b[3, c, 1], b[3, c, 2])

bw = np.zeros((256, 16), dtype=np.uint64)
L.winrs_trace_read_w.argtypes = [ctypes.c_void_p]
L.winrs_trace_read_w(bw.ctypes.data)
print("per-warp chunk-done times (ns from t0), warps 2..")
for c in range(0, 12):
    row = [int(v) - int(t0) if v > 0 else -1 for v in bw[c]]
    print(c, row[2:14])
