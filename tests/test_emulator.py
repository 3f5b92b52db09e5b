"""The plan's full decomposition (segments, row clipping, unit split, masked
tail, residual phase, buckets; §3 P@15252-17405, eq. (6) P@29449)
evaluated in FP64 on the host by winrs_debug_emulate equals the FP64 oracle —
the method reaches the plain definition exactly up to rounding."""
import numpy as np
import pytest

import paper_conf_icpp_zhangc0zx0025_b200 as W
from oracle import oracle as O

CASES = [
    # N, C, H, W, K, R, S, pad, env
    (1, 4, 8, 8, 4, 3, 3, 1, {}),                                    # tiny BASELINE config
    (2, 8, 16, 16, 8, 3, 3, 1, {"WINRS_FORCE_Z": "6"}),              # Figure 3-like: many segments
    (2, 8, 7, 7, 8, 3, 3, 1, {}),                                    # Wo = 7: masked column
    (2, 8, 9, 33, 4, 3, 3, 1, {"WINRS_FORCE_Z": "3"}),
    (1, 4, 12, 12, 8, 2, 2, 1, {}),                                  # Omega_4(2,3)
    (1, 4, 12, 11, 4, 4, 4, 2, {"WINRS_FORCE_Z": "2"}),              # Omega_8(4,5) + Omega_4(2,3), n1 | n0
    (1, 4, 12, 14, 4, 5, 5, 2, {}),                                  # Omega_16(5,12) + Omega_8(5,4)
    (1, 4, 10, 12, 4, 7, 7, 3, {}),                                  # Omega_16(7,10) + Omega_8(7,2)
    (1, 4, 9, 10, 4, 9, 9, 4, {}),                                   # Omega_16(9,8)
    (1, 4, 9, 9, 4, 6, 6, 2, {}),                                    # width 6
    (1, 4, 9, 9, 4, 8, 8, 3, {}),                                    # width 8
    (2, 4, 6, 6, 4, 3, 3, 0, {}),                                    # no padding
    (1, 4, 5, 9, 4, 3, 3, 2, {"WINRS_FORCE_Z": "4"}),                # pad > needed, clipped rows
    (3, 36, 6, 6, 40, 3, 3, 1, {"WINRS_FORCE_TILE": "32x32"}),       # channel tails over 2 tiles
    (2, 8, 10, 10, 8, 3, 3, 1, {"WINRS_FORCE_PAIR": "4,3,2,0,0,0"}),
    (2, 8, 10, 10, 8, 3, 3, 1, {"WINRS_FORCE_PAIR": "8,3,6,0,0,0", "WINRS_FORCE_Z": "4"}),
    (3, 8, 12, 12, 8, 3, 3, 1, {"WINRS_FORCE_CSPLIT": "4"}),                  # cluster depth split
    (2, 4, 9, 12, 8, 4, 4, 2, {"WINRS_FORCE_CSPLIT": "8", "WINRS_FORCE_Z": "2"}),
    (2, 4, 7, 7, 4, 3, 3, 1, {"WINRS_FORCE_CSPLIT": "8"}),                  # more ranks than chunks
]


@pytest.mark.parametrize("case", CASES)
def test_emulated_plan_equals_oracle(case, monkeypatch):
    N, C, H, Wd, K, R, S, pad, env = case
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    p = W.plan_for_device(N, C, H, Wd, K, R, S, pad, "f32")
    Ho, Wo = p.info["Ho"], p.info["Wo"]
    g = np.random.default_rng(sum(case[:8]))
    X = g.uniform(-1, 1, (N, H, Wd, C))
    dY = g.uniform(-1, 1, (N, Ho, Wo, K))
    ref = O.bfc_c(X, dY, R, S, pad)
    got = W.emulate(p, X, dY)
    assert O.rel_max_err(got, ref) < 1e-12, (p, O.rel_max_err(got, ref))


@pytest.mark.parametrize("S", [2, 3, 4, 5, 7, 8, 9])
def test_emulated_f16_plans_equal_oracle(S, monkeypatch):
    """FP16 plans (tile 128 x B_M, 16-deep chunks, cluster split) emulated in FP64."""
    monkeypatch.setenv("WINRS_FORCE_CSPLIT", "2")
    N, C, H, Wd, K, pad = 2, 16, 9, 13, 24, S // 2
    p = W.plan_for_device(N, C, H, Wd, K, S, S, pad, "f16")
    g = np.random.default_rng(S)
    X = g.uniform(-1, 1, (N, H, Wd, C))
    dY = g.uniform(-1, 1, (N, p.info["Ho"], p.info["Wo"], K))
    assert O.rel_max_err(W.emulate(p, X, dY), O.bfc_c(X, dY, S, S, pad)) < 1e-12


XS_CS = [
    ({"WINRS_FORCE_TA": "2", "WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_CSPLIT": "1"}, 144, 40),
    ({"WINRS_FORCE_TA": "2", "WINRS_FORCE_TILE": "128x64", "WINRS_FORCE_CSPLIT": "3"}, 40, 136),
    ({"WINRS_FORCE_TA": "1", "WINRS_FORCE_TILE": "64x128", "WINRS_FORCE_CSPLIT": "5"}, 136, 72),
    ({"WINRS_FORCE_TA": "1", "WINRS_FORCE_TILE": "64x64", "WINRS_FORCE_CSPLIT": "7"}, 40, 72),
]


@pytest.mark.parametrize("env,C,K", XS_CS, ids=lambda v: str(v))
def test_emulated_xs_and_odd_cluster_plans(env, C, K, monkeypatch):
    """The xi-split pair's tiles (128 k x 128 / 64 rows, cg = 2) and 5- / 7-rank
    cluster splits decompose the same BFC: the FP64 emulation of the plan's
    tiles, segments and depth ranks equals the oracle."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    N, H, Wd, R, S, pad = 16, 9, 11, 3, 3, 1
    p = W.plan_for_device(N, C, H, Wd, K, R, S, pad, "f16")
    assert p.info["csplit"] == int(env["WINRS_FORCE_CSPLIT"]), p
    assert ("_v2x_" in p.kernel_name) == (env["WINRS_FORCE_TA"] == "2"), p.kernel_name
    g = np.random.default_rng(C + K)
    X = g.uniform(-1, 1, (N, H, Wd, C))
    dY = g.uniform(-1, 1, (N, p.info["Ho"], p.info["Wo"], K))
    assert O.rel_max_err(W.emulate(p, X, dY), O.bfc_c(X, dY, R, S, pad)) < 1e-12
