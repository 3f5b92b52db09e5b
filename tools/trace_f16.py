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
t0 = int(buf[0, 240, 0]) if buf[0, 240, 0] > 0 else min(v for v in buf.ravel() if v > 0)
b = np.where(buf > 0, buf.astype(np.int64) - int(t0), -1)
print(p)
print("chunk | prod: before_wait after_wait | tx: start raw_ok op_ok done | mma: opfull issued | ft_computed it_computed ft_fenced")
for c in list(range(0, 40)) + list(range(64, 90)):
    if b[2, c, 0] < 0 and b[0, c, 0] < 0:
        continue
    print(c, "|", b[0, c, 0], b[0, c, 1], b[0, c, 2], b[0, c, 3], "|", b[2, c, 0], b[2, c, 1], b[2, c, 2], b[2, c, 3], "|", b[1, c, 0], b[1, c, 1], "|", b[3, c, 0], b[3, c, 1], b[3, c, 2])

names = ["entry", "setup done", "last MMA commit", "tx jobs+epilogues done", "final_out done", "post-sync", "cluster reduce done"]
print("phases (ns from t0):", {n: int(buf[0, 240 + i, 0]) - int(t0) for i, n in enumerate(names) if buf[0, 240 + i, 0] > 0})
bw = np.zeros((256, 24, 3), dtype=np.uint64)
L.winrs_trace_read_w.argtypes = [ctypes.c_void_p]
L.winrs_trace_read_w(bw.ctypes.data)
slots = np.zeros(24, dtype=np.uint32)
L.winrs_trace_read_slots.argtypes = [ctypes.c_void_p]
L.winrs_trace_read_slots(slots.ctypes.data)
print("warp -> %warpid:", list(slots))
print("per-warp (raw_ok, op_ok, done) ns from t0, tx warps")
for c in range(0, 16):
    row = []
    for w in range(2, 24):
        if bw[c, w, 2] == 0:
            continue
        row.append("w%d:%d/%d/%d" % (w, int(bw[c, w, 0]) - int(t0), int(bw[c, w, 1]) - int(t0), int(bw[c, w, 2]) - int(t0)))
    print(c, " ".join(row))

ct = np.zeros((2048, 8), dtype=np.uint64)
L.winrs_trace_read_cta.argtypes = [ctypes.c_void_p]
L.winrs_trace_read_cta(ct.ctypes.data)
n = int(p.info["ctas_main"]) if "ctas_main" in p.info else 0
n = n or int((ct[:, 0] > 0).sum())
c = ct[:n].astype(np.int64)
T0 = c[:, 0].min()
cs = p.info.get("csplit", 1)
print("per-CTA (us from first entry): entry, setup, lastMMA, txdone, finalout, end | smid")
for i in range(n):
    print(i, " ".join("%.1f" % ((c[i, j] - T0) / 1e3) if c[i, j] > 0 else "-" for j in (0, 1, 2, 3, 4, 6)), "| sm", int(ct[i, 7]))
ent, lm, end = (c[:, 0] - T0) / 1e3, (c[:, 2] - T0) / 1e3, (c[:, 6] - T0) / 1e3
print("entry spread %.1f us; main-loop (setup->lastMMA) min %.1f max %.1f mean %.1f; end max %.1f" % (
    ent.max(), ((c[:, 2] - c[:, 1]) / 1e3).min(), ((c[:, 2] - c[:, 1]) / 1e3).max(), ((c[:, 2] - c[:, 1]) / 1e3).mean(), end.max()))
