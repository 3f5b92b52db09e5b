"""Fit the planner's B200 time model (csrc/planner.cpp) to a
calibration sweep (tools/sweep.py output).  The model simulates the block
scheduler: every CTA costs F + chunks * T_chunk(alpha) (+ per residual job J),
clusters are list-scheduled onto the SM slots in launch order, and Z > 1 adds
the bucket reduction (fixed + bytes / bw).

Usage: python tools/fit_model.py sweep.jsonl [f32|f16]
Plans are rebuilt on the CPU (WINRS_FORCE_* env), so no GPU is needed.
"""
import heapq
import json
import math
import os
import sys

import numpy as np
from scipy.optimize import minimize

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_zhangc0zx0025_b200 as W  # noqa: E402
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl  # noqa: E402


def geometry(layer, tile, cs, z):
    os.environ["WINRS_FORCE_TILE"] = tile
    os.environ["WINRS_FORCE_CSPLIT"] = str(cs)
    os.environ["WINRS_FORCE_Z"] = str(z)
    l = layer
    p = W.plan_for_device(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype, num_sms=148)
    for k in ("WINRS_FORCE_TILE", "WINRS_FORCE_CSPLIT", "WINRS_FORCE_Z"):
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


def model(i, params, dtype):
    F, rate, J, rfix, bw = params
    chunk = 8 if dtype == "f32" else 16
    bn, bm, cs = i["tile_k0"], i["tile_c0"], i["csplit"]
    mult = -(-i["K"] // bn) * -(-i["C"] // bm) * (i["S"] // i["n0"])
    tch = lambda a: a * chunk * bn * bm * 2 / rate
    frac = 1.0 if cs <= 2 else (132 / 148 if cs == 4 else 128 / 148)
    slots = max(1, int(148 * frac) // cs)
    heap = [0.0] * slots
    for ranks in cta_work(i, chunk):
        t = max(F + cm * tch(i["alpha0"]) + jobs * (J + cr * tch(i["alpha1"] or 1)) for cm, cr, jobs in ranks)
        for _ in range(mult):
            s = heapq.heappop(heap)
            heapq.heappush(heap, s + t)
    mk = max(heap)
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
        key = (r["layer"], r["tile"], r["csplit"], r["Z"])
        if key not in geo:
            geo[key] = geometry(wl.LAYERS[r["layer"]], r["tile"], r["csplit"], r["Z"])
    tiles = sorted({r["tile"] for r in rows})
    fitted = {}
    for tile in tiles:
        R = [r for r in rows if r["tile"] == tile]
        y = np.array([r["us"] * 1e-6 for r in R])

        def loss(lp):
            p = np.exp(lp)
            pred = np.array([model(geo[(r["layer"], r["tile"], r["csplit"], r["Z"])], p, dtype) for r in R])
            return float(np.mean(np.log(pred / y) ** 2))

        x0 = np.log([8e-6, 2e11 if dtype == "f32" else 1.2e12, 2e-6, 4e-6, 4e12])
        res = minimize(loss, x0, method="Nelder-Mead", options={"maxiter": 3000, "xatol": 1e-4, "fatol": 1e-8})
        p = np.exp(res.x)
        fitted[tile] = p
        print(f"{tile}: F={p[0]*1e6:.2f}us rate={p[1]:.3g} J={p[2]*1e6:.2f}us rfix={p[3]*1e6:.2f}us "
              f"bw={p[4]/1e12:.2f}TB/s  rms log err={math.sqrt(res.fun):.3f}")
    # regret of the model's argmin per layer
    by = {}
    for r in rows:
        by.setdefault(r["layer"], []).append(r)
    tot = 0
    for L, rs in by.items():
        best = min(rs, key=lambda r: r["us"])
        pick = min(rs, key=lambda r: model(geo[(r["layer"], r["tile"], r["csplit"], r["Z"])], fitted[r["tile"]], dtype))
        tot += pick["us"] / best["us"]
        print(f"  {L}: best {best['tile']} cs{best['csplit']} Z{best['Z']} {best['us']}us; "
              f"model picks {pick['tile']} cs{pick['csplit']} Z{pick['Z']} {pick['us']}us")
    print("mean regret", tot / len(by))


if __name__ == "__main__":
    main()
