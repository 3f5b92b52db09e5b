#!/usr/bin/env python3
"""Offline generator of the 1D Winograd F(n, r) transforms used by the WinRS
kernels (exact rational arithmetic -> straight-line C++ for the CUDA path).

PAPER.md passages followed:
  * eq. (1), §2.1 P@9107: F(n, r) computes Y = A^T[(G W) ⊙ (D^T X)], X of
    length alpha = n + r - 1, W of length r, Y of length n; A in R^{alpha x n},
    G in R^{alpha x r}, D in R^{alpha x alpha}.
  * §2.2 P@11532 "In D in R^{4x4}, non-zero elements are simply ±1; D in
    R^{16x16} involves 164597/576 and 1/16" -> interpolation points (pinned in
    tests/test_transforms.py).
  * §5.2 P@38072 "Transform Simplification": interpolation points in
    {0, ±1, ±2, ±1/2, ±3, ±1/3, ...}; rows 2k and 2k+1 of A, G and D^T are equal
    at even and opposite at odd positions -> halves the multiplies.  The
    generated code exploits exactly that pairing.
  * §5.2 P@39150 eq. (7): row scaling matrices A_s, G_s, D_s ("unit L1 norm per
    row of G and D"), A_s compensating in the OT.
  * Figure 6 / §5 P@28451: the 13 kernels Omega_alpha(n, r).

Construction (Cook-Toom for correlation).  With finite points p_0..p_{a-2}
and the point at infinity, let V_k be the alpha x k evaluation matrix (row j =
[1, p_j, ..., p_j^{k-1}], the infinity row = e_{k-1}).  Linear convolution is
c = V_a^{-1}[(V_n a) ⊙ (V_r w)]; its transpose in the data argument is the
correlation y[j] = sum_i x[j+i] w[i]:

    y = V_n^T [ (V_r w) ⊙ (V_a^{-T} x) ]   =>  A = V_n,  G = V_r,  D^T = V_a^{-T}

and any row scaling diag(a) A, diag(g) G, diag(d) D^T with a*g*d = 1 keeps it
exact (eq. (7)).  Default scaling here (R12): every row of G and of
D^T has unit L1 norm, A absorbs the product — the paper's eq. (7) normalisation.

Run:  python tools/gen_winograd.py   (writes the .cuh and the .json below)
"""
from __future__ import annotations

import json
import os
import sys
from fractions import Fraction as Fr

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT_CUH = os.path.join(ROOT, "paper_conf_icpp_zhangc0zx0025_b200", "csrc", "winograd_generated.cuh")
OUT_JSON = os.path.join(ROOT, "paper_conf_icpp_zhangc0zx0025_b200", "csrc", "winograd_matrices.json")

# (alpha, n, r) of the 13 kernels (Figure 6; Omega_2(2,1) per DESIGN.md R5).
KERNELS = [
    (2, 2, 1),
    (4, 2, 3), (4, 3, 2),
    (8, 3, 6), (8, 4, 5), (8, 5, 4), (8, 6, 3), (8, 7, 2),
    (16, 5, 12), (16, 6, 11), (16, 7, 10), (16, 8, 9), (16, 9, 8),
]

H = Fr(1, 2)
T = Fr(1, 3)
# Finite points in +/- pairs (pair first so rows 2k, 2k+1 are +p, -p), then 0.
POINTS = {
    2: [Fr(0)],
    4: [Fr(1), Fr(-1), Fr(0)],
    8: [Fr(1), Fr(-1), Fr(2), Fr(-2), H, -H, Fr(0)],
    # The paper's alpha = 16 set (D contains 164597/576 and 1/16, P@11532).
    "16paper": [Fr(1), Fr(-1), Fr(2), Fr(-2), H, -H, Fr(3), Fr(-3), T, -T, Fr(4), Fr(-4),
                Fr(1, 4), Fr(-1, 4), Fr(0)],
    # Better-conditioned alpha = 16 set (R12): +/-3/2, +/-2/3 replace +/-4, +/-1/4.
    16: [Fr(1), Fr(-1), Fr(2), Fr(-2), H, -H, Fr(3), Fr(-3), T, -T, Fr(3, 2), Fr(-3, 2),
         Fr(2, 3), Fr(-2, 3), Fr(0)],
}


def vander(points, k):
    """alpha x k evaluation matrix: finite rows [1, p, ..., p^{k-1}], then the
    infinity row e_{k-1}."""
    rows = [[p ** i for i in range(k)] for p in points]
    rows.append([Fr(0)] * (k - 1) + [Fr(1)])
    return rows


def inv(M):
    n = len(M)
    A = [list(row) + [Fr(int(i == j)) for j in range(n)] for i, row in enumerate(M)]
    for col in range(n):
        piv = next(r for r in range(col, n) if A[r][col] != 0)
        A[col], A[piv] = A[piv], A[col]
        pv = A[col][col]
        A[col] = [v / pv for v in A[col]]
        for r in range(n):
            if r != col and A[r][col] != 0:
                f = A[r][col]
                A[r] = [a - f * b for a, b in zip(A[r], A[col])]
    return [row[n:] for row in A]


def transpose(M):
    return [list(c) for c in zip(*M)]


def matrices(alpha, n, r, points_key=None, scaling="l1"):
    """Exact (A, G, DT): A is alpha x n, G alpha x r, DT alpha x alpha."""
    pts = POINTS[points_key if points_key is not None else alpha]
    assert len(pts) == alpha - 1 and n + r - 1 == alpha
    A = vander(pts, n)
    G = vander(pts, r)
    DT = transpose(inv(vander(pts, alpha)))
    if scaling == "l1":
        for xi in range(alpha):
            g = sum(abs(v) for v in G[xi])
            d = sum(abs(v) for v in DT[xi])
            G[xi] = [v / g for v in G[xi]]
            DT[xi] = [v / d for v in DT[xi]]
            A[xi] = [v * g * d for v in A[xi]]
    elif scaling == "fracG":
        # The paper's normalisation ("fractions in G"): D^T row j times
        # f_j = prod_{l != j} (p_j - p_l), G row j divided by f_j.
        for j, pj in enumerate(pts):
            f = Fr(1)
            for l, pl in enumerate(pts):
                if l != j:
                    f *= pj - pl
            G[j] = [v / f for v in G[j]]
            DT[j] = [v * f for v in DT[j]]
    elif scaling != "none":
        raise ValueError(scaling)
    return A, G, DT


def check_identity(alpha, n, r, A, G, DT):
    """Exact Cook-Toom identity on the basis vectors (bilinear => complete)."""
    for a in range(alpha):
        for b in range(r):
            gw = [G[xi][b] for xi in range(alpha)]
            dx = [DT[xi][a] for xi in range(alpha)]
            y = [sum(A[xi][j] * gw[xi] * dx[xi] for xi in range(alpha)) for j in range(n)]
            exp = [Fr(int(a == j + b)) for j in range(n)]
            if y != exp:
                return False
    return True


# ----------------------------------------------------------------------------- codegen

def lit(v: Fr) -> str:
    return f"wc<T>({v.numerator}, {v.denominator})"


def _nmul(terms):
    return sum(1 for c, _ in terms if c not in (0, 1, -1))


def lin(terms):
    """sum_i c_i x_i as nested explicit FMA calls (wmul / wfma / wadd / wsub /
    wneg, see winrs_vec.cuh), 'wzero<T>()' if empty.  A common |coefficient| m
    is factored out, m * (sum (c/m) x), when that saves multiplies (the eq. (7)
    row scaling makes many row entries equal)."""
    terms = [(c, v) for c, v in terms if c != 0]
    best, best_n = None, _nmul(terms)
    for m in sorted({abs(c) for c, _ in terms if abs(c) != 1}):
        scaled = [(c / m, v) for c, v in terms]
        if 1 + _nmul(scaled) < best_n:
            best, best_n = m, 1 + _nmul(scaled)
    if best is not None:
        return f"wmul({lit(best)}, {lin_plain([(c / best, v) for c, v in terms])})"
    return lin_plain(terms)


def lin_plain(terms):
    terms = [(c, v) for c, v in terms if c != 0]
    if not terms:
        return "wzero<T>()"
    # start with a +/-1 term when there is one (saves a multiply)
    terms.sort(key=lambda t: 0 if abs(t[0]) == 1 else 1)
    c, v = terms[0]
    if c == 1:
        acc = v
    elif c == -1:
        acc = f"wneg({v})"
    else:
        acc = f"wmul({lit(c)}, {v})"
    for c, v in terms[1:]:
        if c == 1:
            acc = f"wadd({acc}, {v})"
        elif c == -1:
            acc = f"wsub({acc}, {v})"
        else:
            acc = f"wfma({lit(c)}, {v}, {acc})"
    return acc


def _cost(terms):
    """Non-trivial multiplies of lin(terms) after common-factor extraction."""
    return lin(terms).count("wc<T>")


def row_pairing(M, rows):
    """For rows 2k, 2k+1: +1 if M[2k+1][i] == (-1)^i M[2k][i], -1 if
    M[2k+1][i] == -(-1)^i M[2k][i], 0 otherwise."""
    a, b = M[rows[0]], M[rows[1]]
    if all(b[i] == (a[i] if i % 2 == 0 else -a[i]) for i in range(len(a))):
        return 1
    if all(b[i] == (-a[i] if i % 2 == 0 else a[i]) for i in range(len(a))):
        return -1
    return 0


def emit_apply(name, M, in_len, out_len, in_var="x", out_var="o"):
    """o = M x with the +/- row pairing (P@38072)."""
    lines = [f"  template <class T> __host__ __device__ __forceinline__ static void {name}"
             f"(const T* __restrict__ {in_var}, T* __restrict__ {out_var}) {{"]
    xi = 0
    nmul = 0
    while xi < out_len:
        pair = xi + 1 < out_len and row_pairing(M, (xi, xi + 1)) != 0 and xi + 1 < out_len - 0
        if pair and xi + 1 < out_len:
            sgn = row_pairing(M, (xi, xi + 1))
            ev = [(M[xi][i], f"{in_var}[{i}]") for i in range(in_len) if i % 2 == 0]
            od = [(M[xi][i], f"{in_var}[{i}]") for i in range(in_len) if i % 2 == 1]
            nmul += _cost(ev) + _cost(od)
            lines.append(f"    {{ const T e = {lin(ev)}; const T d = {lin(od)};")
            if sgn > 0:
                lines.append(f"      {out_var}[{xi}] = wadd(e, d); {out_var}[{xi + 1}] = wsub(e, d); }}")
            else:
                lines.append(f"      {out_var}[{xi}] = wadd(e, d); {out_var}[{xi + 1}] = wsub(d, e); }}")
            xi += 2
        else:
            row = [(M[xi][i], f"{in_var}[{i}]") for i in range(in_len)]
            nmul += _cost(row)
            lines.append(f"    {out_var}[{xi}] = {lin(row)};")
            xi += 1
    lines.append("  }")
    return lines, nmul


def emit_ot(A, alpha, n):
    """y = A^T v; rows (2k, 2k+1) of A paired: y[j] += A[2k][j] * (v[2k] +/- v[2k+1])."""
    lines = ["  template <class T> __host__ __device__ __forceinline__ static void ot"
             "(const T* __restrict__ v, T* __restrict__ y) {"]
    terms = [[] for _ in range(n)]
    xi = 0
    nmul = 0
    while xi < alpha:
        if xi + 1 < alpha and row_pairing(A, (xi, xi + 1)) != 0:
            sgn = row_pairing(A, (xi, xi + 1))
            s, d = f"s{xi}", f"d{xi}"
            lines.append(f"    const T {s} = wadd(v[{xi}], v[{xi + 1}]); const T {d} = wsub(v[{xi}], v[{xi + 1}]);")
            for j in range(n):
                # even j: A[2k+1][j] = sgn*A[2k][j]; odd j: A[2k+1][j] = -sgn*A[2k][j]
                same = (j % 2 == 0) == (sgn > 0)
                terms[j].append((A[xi][j], s if same else d))
            xi += 2
        else:
            for j in range(n):
                terms[j].append((A[xi][j], f"v[{xi}]"))
            xi += 1
    for j in range(n):
        nmul += _cost(terms[j])
        lines.append(f"    y[{j}] = {lin(terms[j])};")
    lines.append("  }")
    return lines, nmul


def generate():
    out = ["// GENERATED by tools/gen_winograd.py — do not edit.",
           "// 1D Winograd F(n,r) transforms for the WinRS kernels Omega_alpha(n,r), alpha = n + r - 1.",
           "// PAPER.md eq. (1) P@9107: Y = A^T[(G W) (.) (D^T X)];  +/- row pairing P@38072;",
           "// eq. (7) row scaling P@39150 (unit L1 rows of G and D^T, A compensating).",
           "// ft: o[alpha] = G w[r]   it: o[alpha] = D^T x[alpha]   ot: y[n] = A^T v[alpha]",
           "#pragma once",
           "#include \"winrs_vec.cuh\"",
           "",
           "namespace winrs {",
           "",
           "template <int ALPHA, int N, int R> struct Wino;",
           ""]
    js = {}
    for (alpha, n, r) in KERNELS:
        A, G, DT = matrices(alpha, n, r)
        assert check_identity(alpha, n, r, A, G, DT), (alpha, n, r)
        ft, m1 = emit_apply("ft", G, r, alpha, "w", "o")
        it, m2 = emit_apply("it", DT, alpha, alpha, "x", "o")
        ot, m3 = emit_ot(A, alpha, n)
        out.append(f"// Omega_{alpha}({n},{r}): non-trivial multiplies ft {m1}, it {m2}, ot {m3}")
        out.append(f"template <> struct Wino<{alpha}, {n}, {r}> {{")
        out.append(f"  static constexpr int alpha = {alpha}, n = {n}, r = {r};")
        out.extend(ft)
        out.extend(it)
        out.extend(ot)
        out.append("};")
        out.append("")
        js[f"{alpha},{n},{r}"] = {
            "A": [[str(v) for v in row] for row in A],
            "G": [[str(v) for v in row] for row in G],
            "DT": [[str(v) for v in row] for row in DT],
            "points": [str(p) for p in POINTS[alpha]] + ["inf"],
        }
    out.append("}  // namespace winrs")
    return "\n".join(out) + "\n", js


def main():
    src, js = generate()
    with open(OUT_CUH, "w") as f:
        f.write(src)
    with open(OUT_JSON, "w") as f:
        json.dump(js, f, indent=1)
    print(f"wrote {OUT_CUH} and {OUT_JSON}", file=sys.stderr)


if __name__ == "__main__":
    main()
