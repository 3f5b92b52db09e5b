"""Fit the planner's B200 time model (csrc/planner.cpp) to a
calibration sweep (tools/sweep.py output).  The model simulates the block
scheduler: every CTA costs F + chunks * T_chunk(alpha) (+ per residual job J),
clusters are list-scheduled onto the SM slots in launch order, and Z > 1 adds
the bucket reduction (fixed + bytes / bw).

Usage: python tools/fit_model.py sweep.jsonl [f32|f16]
Plans are rebuilt on the CPU (WINRS_FORCE_* env), so no GPU is needed.
"""
import ctypes
import json
import math
import os
import subprocess
import sys

import numpy as np
from scipy.optimize import minimize

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_zhangc0zx0025_b200 as W  # noqa: E402
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl  # noqa: E402


def pair_of(kname):
    """'f16tc_O8(3,6)+O4(3,2)_128x64' -> '8,3,6,4,3,2'."""
    import re
    v = re.findall(r"O(\d+)\((\d+),(\d+)\)", kname)
    return ",".join(",".join(x) for x in v)


def geometry(layer, tile, cs, z, pair=None):
    if pair:
        os.environ["WINRS_FORCE_PAIR"] = pair
    os.environ["WINRS_FORCE_TILE"] = tile
    os.environ["WINRS_FORCE_CSPLIT"] = str(cs)
    os.environ["WINRS_FORCE_Z"] = str(z)
    l = layer
    p = W.plan_for_device(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype, num_sms=148)
    for k in ("WINRS_FORCE_TILE", "WINRS_FORCE_CSPLIT", "WINRS_FORCE_Z", "WINRS_FORCE_PAIR"):
        os.environ.pop(k, None)
    return dict(p.info)


def cta_work(i, chunk):
    """Per tile (in launch order, kb/cb/ft collapsed to a multiplicity) and rank:
    (main chunks, residual chunks per job, jobs)."""
    Ho, pad, H = i["Ho"], i["pad"], i["H"]
    out = []
    for band in range(i["bands"]):
        for col in range(i["seg_cols"]):
            for fh in range(i["R"]):
                h0 = band * i["seg_h"]
                h1 = Ho if band == i["bands"] - 1 else h0 + i["seg_h"]
                hs, he = max(pad - fh, h0), min(H + pad - fh, h1)
                rows = max(0, he - hs)
                w0 = col * i["seg_w"]
                w1 = min(w0 + i["seg_w"], i["k0"] * i["r0"])
                units = (w1 - w0) // i["r0"]
                dm = rows * units * i["N"]
                resid = i["alpha1"] and i["k1"] > 0 and col == i["seg_cols"] - 1
                dr = rows * i["k1"] * i["N"] if resid else 0
                jobs = i["n0"] // i["n1"] if resid else 0
                cm, cr = -(-dm // chunk), -(-dr // chunk)
                ranks = []
                for r in range(i["csplit"]):
                    lo, hi = cm * r // i["csplit"], cm * (r + 1) // i["csplit"]
                    rlo, rhi = cr * r // i["csplit"], cr * (r + 1) // i["csplit"]
                    ranks.append((hi - lo, rhi - rlo, jobs))
                out.append(ranks)
    return out


_ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
_SO = os.path.join(_ROOT, "build", "listsched.so")
if not os.path.exists(_SO):
    os.makedirs(os.path.dirname(_SO), exist_ok=True)
    subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", os.path.join(_ROOT, "tools", "listsched.c"), "-o", _SO])
_ls = ctypes.CDLL(_SO)
_ls.makespan.restype = ctypes.c_double
_ls.makespan.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
_heap = np.zeros(4096)
_cache = {}


def _arrays(i, chunk):
    key = id(i)
    if key not in _cache:
        w = cta_work(i, chunk)
        _cache[key] = tuple(np.array([[x[k] for x in ranks] for ranks in w], dtype=np.float64) for k in range(3))
    return _cache[key]


def model(i, params, dtype):
    F, rate, J, rfix, bw, s4, s8, D = params
    chunk = 8 if dtype == "f32" else 16
    bn, bm, cs = i["tile_k0"], i["tile_c0"], i["csplit"]
    mult = -(-i["K"] // bn) * -(-i["C"] // bm) * (i["S"] // i["n0"])
    t0 = i["alpha0"] * chunk * bn * bm * 2 / rate
    t1 = (i["alpha1"] or 1) * chunk * bn * bm * 2 / rate
    slots = {1: 148, 2: 74, 4: max(1, int(s4)), 8: max(1, int(s8))}[cs]
    CM, CR, JB = _arrays(i, chunk)
    t = (D if cs > 1 else 0.0) + np.max(F + CM * t0 + JB * (J + CR * t1), axis=1)
    t = np.ascontiguousarray(t)
    mk = _ls.makespan(len(t), t.ctypes.data, mult, slots, _heap.ctypes.data)
    if i["Z"] > 1:
        dw = i["K"] * i["R"] * i["S"] * i["C"] * 4
        mk += rfix + (2 * i["Z"]) * dw / bw
    return mk


def main():
    rows = [json.loads(l) for l in open(sys.argv[1])]
    dtype = sys.argv[2] if len(sys.argv) > 2 else "f32"
    rows = [r for r in rows if wl.LAYERS[r["layer"]].dtype == dtype]
    geo = {}
    for r in rows:
        key = (r["layer"], r["pair"], r["tile"], r["csplit"], r["Z"])
        if key not in geo:
            geo[key] = geometry(wl.LAYERS[r["layer"]], r["tile"], r["csplit"], r["Z"], pair_of(r["pair"]))
    tiles = sorted({r["tile"] for r in rows})
    nt = len(tiles)
    # joint fit: per-tile (F, rate), shared (J, rfix, bw, s4, s8, D)
    def unpack(lp):
        p = np.exp(lp)
        return {t: np.array([p[2 * k], p[2 * k + 1], *p[2 * nt:]]) for k, t in enumerate(tiles)}

    def loss(lp):
        ps = unpack(lp)
        err = [math.log(model(geo[(r["layer"], r["pair"], r["tile"], r["csplit"], r["Z"])], ps[r["tile"]], dtype) /
                        (r["us"] * 1e-6)) for r in rows]
        return float(np.mean(np.square(err)))

    x0 = []
    for t in tiles:
        x0 += [8e-6, 2e11 if dtype == "f32" else 1.2e12]
    x0 = np.log(x0 + [2e-6, 4e-6, 4e12, 33, 16, 2e-6])
    best = None
    for it in range(2):   # restarts
        res = minimize(loss, x0 if best is None else best.x, method="Nelder-Mead",
                       options={"maxiter": 8000, "xatol": 1e-5, "fatol": 1e-10, "adaptive": True})
        if best is None or res.fun < best.fun:
            best = res
    fitted = unpack(best.x)
    for t in tiles:
        p = fitted[t]
        print(f"{t}: F={p[0]*1e6:.2f}us rate={p[1]:.4g}")
    p = fitted[tiles[0]]
    print(f"shared: J={p[2]*1e6:.2f}us rfix={p[3]*1e6:.2f}us bw={p[4]/1e12:.2f}TB/s s4={p[5]:.1f} s8={p[6]:.1f} "
          f"D={p[7]*1e6:.2f}us  rms log err={math.sqrt(best.fun):.3f}")
    # regret of the model's argmin per layer
    by = {}
    for r in rows:
        by.setdefault(r["layer"], []).append(r)
    tot = 0
    for L, rs in by.items():
        best = min(rs, key=lambda r: r["us"])
        pick = min(rs, key=lambda r: model(geo[(r["layer"], r["pair"], r["tile"], r["csplit"], r["Z"])], fitted[r["tile"]], dtype))
        tot += pick["us"] / best["us"]
        print(f"  {L}: best {best['pair']} {best['tile']} cs{best['csplit']} Z{best['Z']} {best['us']}us; "
              f"model picks {pick['pair']} {pick['tile']} cs{pick['csplit']} Z{pick['Z']} {pick['us']}us")
    print("mean regret", tot / len(by))


if __name__ == "__main__":
    main()
