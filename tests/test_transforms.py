"""Pins for the generated 1D Winograd transforms F(n, r) (tools/gen_winograd.py,
csrc/winograd_generated.cuh).  PAPER.md eq. (1) P@9107; pinned constants
P@11532 (§2.2); +/- row pairing P@38072 (§5.2); eq. (7) scaling P@39150;
kernel set Figure 6 / P@28451; acceleration figures P@8201, P@49854."""
import json
import os
from fractions import Fraction as Fr

import numpy as np
import pytest

import sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))
import gen_winograd as G  # noqa: E402

JSON = os.path.join(ROOT, "paper_conf_icpp_zhangc0zx0025_b200", "csrc", "winograd_matrices.json")


def _load():
    with open(JSON) as f:
        js = json.load(f)
    return {tuple(map(int, k.split(","))): {m: [[Fr(v) for v in row] for row in js[k][m]] for m in ("A", "G", "DT")}
            for k in js}


MATS = _load()


def test_thirteen_kernels():
    """Figure 6: 13 kernels, alpha in {2,4,8,16}, supporting F_W = n*k, 2<=k<=9 (P@28451)."""
    assert len(MATS) == 13
    assert {a for a, n, r in MATS} == {2, 4, 8, 16}
    assert all(a == n + r - 1 for a, n, r in MATS)
    assert {n for _, n, _ in MATS} == set(range(2, 10))


@pytest.mark.parametrize("key", sorted(MATS))
def test_cook_toom_identity_exact(key):
    """A^T[(G w) (.) (D^T x)] == correlation(x, w)[0:n], in exact rationals, for
    random integer vectors (bilinear, so also checked on all basis pairs)."""
    a, n, r = key
    M = MATS[key]
    rng = np.random.default_rng(a * 100 + n)
    for _ in range(5):
        x = [Fr(int(v)) for v in rng.integers(-9, 10, size=a)]
        w = [Fr(int(v)) for v in rng.integers(-9, 10, size=r)]
        gw = [sum(M["G"][xi][i] * w[i] for i in range(r)) for xi in range(a)]
        dx = [sum(M["DT"][xi][t] * x[t] for t in range(a)) for xi in range(a)]
        y = [sum(M["A"][xi][j] * gw[xi] * dx[xi] for xi in range(a)) for j in range(n)]
        corr = [sum(x[j + i] * w[i] for i in range(r)) for j in range(n)]
        assert y == corr
    assert G.check_identity(a, n, r, M["A"], M["G"], M["DT"])


def test_paper_pinned_constants():
    """P@11532: with the paper's normalisation (fractions in G), D in R^{4x4}
    has only +/-1 non-zeros and D in R^{16x16} involves 164597/576 and 1/16;
    P@39150: the alpha=16 entries span ~1e-8 .. 1e5 — pins the point sets."""
    _, _, DT4 = G.matrices(4, 3, 2, scaling="fracG")
    assert {abs(v) for row in DT4 for v in row} == {Fr(0), Fr(1)}
    A16, G16, DT16 = G.matrices(16, 9, 8, points_key="16paper", scaling="fracG")
    ent = {abs(v) for row in DT16 for v in row}
    assert Fr(164597, 576) in ent and Fr(1, 16) in ent
    mags = [abs(float(v)) for M in (A16, G16, DT16) for row in M for v in row if v != 0]
    assert min(mags) < 1e-7 and max(mags) > 1e4
    # the alpha = 8 point set {0, +/-1, +/-2, +/-1/2} reproduces the standard F(3,6) D^T
    _, _, DT8 = G.matrices(8, 3, 6, scaling="fracG")
    assert {abs(v) for row in DT8 for v in row} == {Fr(0), Fr(1, 4), Fr(1, 2), Fr(1), Fr(2), Fr(5, 4),
                                                   Fr(5, 2), Fr(4), Fr(17, 4), Fr(5), Fr(21, 4)}


@pytest.mark.parametrize("key", sorted(MATS))
def test_pm_row_pairing(key):
    """P@38072: rows 2k, 2k+1 of A, G, D^T are equal at even and opposite at odd
    positions (or the reverse) for every +/-p point pair."""
    a, n, r = key
    M = MATS[key]
    npairs = (a - 2) // 2
    for m in ("A", "G", "DT"):
        for k in range(npairs):
            assert G.row_pairing(M[m], (2 * k, 2 * k + 1)) != 0, (m, k)


@pytest.mark.parametrize("key", sorted(MATS))
def test_eq7_scaling_is_identity(key):
    """eq. (7): the row-scaled matrices equal diag-scalings of the unscaled ones
    with a*g*d = 1 per row, and G, D^T rows have unit L1 norm."""
    a, n, r = key
    A0, G0, D0 = G.matrices(a, n, r, scaling="none")
    A1, G1, D1 = MATS[key]["A"], MATS[key]["G"], MATS[key]["DT"]
    for xi in range(a):
        assert sum(abs(v) for v in G1[xi]) == 1 and sum(abs(v) for v in D1[xi]) == 1
        g = next(G1[xi][i] / G0[xi][i] for i in range(r) if G0[xi][i] != 0)
        d = next(D1[xi][i] / D0[xi][i] for i in range(a) if D0[xi][i] != 0)
        aa = next(A1[xi][j] / A0[xi][j] for j in range(n) if A0[xi][j] != 0) if any(A0[xi]) else 1 / (g * d)
        assert aa * g * d == 1
        assert all(G1[xi][i] == g * G0[xi][i] for i in range(r))
        assert all(D1[xi][i] == d * D0[xi][i] for i in range(a))


def test_acceleration_figures():
    """n*r/alpha: 3x3 -> Omega_8(3,6) = 2.25, 5x5 -> Omega_16(5,12) = 3.75 (P@49854);
    min 1.5 and max 4.5 over the alpha >= 4 kernels (P@8201)."""
    gold = os.path.join(ROOT, "tests", "golden", "acceleration.txt")
    for line in open(gold):
        if line.startswith("#") or not line.strip():
            continue
        a, n, r, num, den = map(int, line.split())
        assert Fr(n * r, a) == Fr(num, den)
    acc = [Fr(n * r, a) for a, n, r in MATS if a >= 4]
    assert min(acc) == Fr(3, 2) and max(acc) == Fr(9, 2)


needs_lib = pytest.mark.skipif(
    not os.path.exists(os.path.join(ROOT, "paper_conf_icpp_zhangc0zx0025_b200", "libwinrs.so")),
    reason="libwinrs.so not built")


@needs_lib
@pytest.mark.parametrize("key", sorted(MATS))
def test_generated_code_matches_matrices(key):
    """The straight-line C++ the kernels compile (evaluated in double through
    winrs_debug_transform) applies exactly these matrices."""
    import paper_conf_icpp_zhangc0zx0025_b200 as W
    a, n, r = key
    M = {m: np.array([[float(v) for v in row] for row in MATS[key][m]]) for m in ("A", "G", "DT")}
    rng = np.random.default_rng(7)
    for _ in range(4):
        w, x, v = rng.standard_normal(r), rng.standard_normal(a), rng.standard_normal(a)
        assert np.allclose(W.transform(a, n, r, "ft", w), M["G"] @ w, rtol=1e-14, atol=1e-14)
        assert np.allclose(W.transform(a, n, r, "it", x), M["DT"] @ x, rtol=1e-14, atol=1e-14)
        assert np.allclose(W.transform(a, n, r, "ot", v), M["A"].T @ v, rtol=1e-13, atol=1e-13)
        # and the whole F(n, r) equals the direct correlation
        y = W.transform(a, n, r, "ot", W.transform(a, n, r, "ft", w) * W.transform(a, n, r, "it", x))
        assert np.allclose(y, [x[j:j + r] @ w for j in range(n)], rtol=1e-11, atol=1e-11)
