"""Host-side check of the stream-K schedule of the xi-split pairs (DESIGN.md
§6.11; device code: bfc_tc2.cuh sk_total / sk_find / sk_pair_of, bfc_tc2x.cuh
piece loop), replicated in Python over the tile geometry of real plans:

* the pairs' backward walks cover every chunk of every tile exactly once;
* each tile's parts get chain orders 0, 1, 2, ... in increasing pair index;
* the part with order 0 is the FIRST piece its pair processes, or the tile
  starts inside that pair's range (so it never waits);
* a pair only ever waits for a lower pair (deadlock freedom without
  co-residency, given pair indices are tickets in arrival order).
"""
import pytest

import paper_conf_icpp_zhangc0zx0025_b200 as W
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl

KC = 16


def _tiles(info):
    """Chunks per tile in decode_cta order, from the plan's geometry."""
    p = info
    per = p["kblocks"] * p["cblocks"] * p["ftiles"]
    out = []
    for band in range(p["bands"]):
        for col in range(p["seg_cols"]):
            for f in range(p["fhg"]):
                d = p["_rows"][(band, f)] * p["_units"][col] * p["N"] // KC
                out += [d] * per
    return out


def _schedule(depths, P):
    tot = sum(depths)
    start = [0]
    for d in depths:
        start.append(start[-1] + d)
    r = [tot * p // P for p in range(P + 1)]

    def pair_of(gi):
        return ((gi + 1) * P - 1) // tot

    def find(gi):
        lo, hi = 0, len(depths)
        while hi - lo > 1:
            mid = (lo + hi) // 2
            if start[mid] <= gi:
                lo = mid
            else:
                hi = mid
        return lo

    pieces = []
    for p in range(P):
        gcur, gbeg, k = r[p + 1], r[p], 0
        while gcur > gbeg:
            t = find(gcur - 1)
            g0 = start[t]
            c_lo, c_hi = max(g0, gbeg) - g0, gcur - g0
            pieces.append(dict(pair=p, tile=t, lo=c_lo, hi=c_hi, order=p - pair_of(g0), k=k))
            gcur -= c_hi - c_lo
            k += 1
    return pieces


def _geometry(l, env, monkeypatch):
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    p = W.plan_for_device(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
    i = dict(p.info)
    assert "_v2k_" in p.kernel_name, p.kernel_name
    # rows per (band, fh group) and units per column segment, as group_rows / seg_units compute them
    Ho, Wo = i["Ho"], i["Wo"]
    seg_h, seg_w = i["seg_h"], i["seg_w"]
    fhs = 2 if p.kernel_name.endswith("2fh") else 1
    i["fhg"] = -(-l.R // fhs)
    i["kblocks"] = -(-l.K // 128)
    i["cblocks"] = -(-l.C // (128 // fhs))
    i["ftiles"] = l.S // 3
    i["N"] = l.N
    rows = {}
    for band in range(i["bands"]):
        h0 = band * seg_h
        h1 = Ho if band == i["bands"] - 1 else h0 + seg_h
        for f in range(i["fhg"]):
            hs, he, any_ = 0, 0, False
            for r in range(f * fhs, min(l.R, f * fhs + fhs)):
                a = max(l.pad - r, h0)
                b = min(l.H + l.pad - r, h1)
                if b <= a:
                    continue
                hs = a if not any_ or a < hs else hs
                he = b if not any_ or b > he else he
                any_ = True
            rows[(band, f)] = he - hs if any_ else 0
    units = {}
    lim = i["k0"] * 2
    for col in range(i["seg_cols"]):
        w0 = col * seg_w
        units[col] = (min(w0 + seg_w, lim) - w0) // 2
    i["_rows"], i["_units"] = rows, units
    return i


CASES = [
    ("vgg_512_512_28_f16", {}),
    ("vgg_512_512_14_f16", {}),
    ("vgg_256_512_28_f16", {}),
    ("vgg_256_256_56_f16", {}),
    ("vgg_64_128_112_f16", {}),
    ("r50_c512_7_f16", {"WINRS_FORCE_TA": "3"}),
    ("r50_c128_28_f16", {"WINRS_FORCE_TA": "3", "WINRS_TC_GEN": "2"}),
]


@pytest.mark.parametrize("name,env", CASES, ids=[c[0] for c in CASES])
@pytest.mark.parametrize("P", [74, 37, 3])
def test_stream_k_schedule_invariants(name, env, P, monkeypatch):
    info = _geometry(wl.LAYERS[name], env, monkeypatch)
    depths = _tiles(info)
    pieces = _schedule(depths, P)
    # every chunk of every tile exactly once
    cover = {}
    for pc in pieces:
        cover.setdefault(pc["tile"], []).append((pc["lo"], pc["hi"], pc["pair"], pc["order"], pc["k"]))
    assert set(cover) == {t for t, d in enumerate(depths) if d > 0}
    for t, parts in cover.items():
        parts.sort()
        assert parts[0][0] == 0 and parts[-1][1] == depths[t]
        for a, b in zip(parts, parts[1:]):
            assert a[1] == b[0]
        pairs = [pp for _, _, pp, _, _ in parts]
        orders = [o for _, _, _, o, _ in parts]
        assert pairs == sorted(pairs) and orders == list(range(len(parts)))   # chain in increasing pair index
        for lo, hi, pp, o, k in parts:
            if o == 0:
                assert lo == 0                                                # the tile's first chunks store
                if len(parts) > 1:
                    assert k == 0   # a tile cut between pairs: its first part is its pair's first piece (done early)
            else:
                assert pairs[o - 1] < pp                                      # waits only for a lower pair
