"""ORACLE — TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct CPU implementations of the backward-filter
convolution (BFC) that WinRS accelerates.  Only ``tests/``,
``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this module.  It imports nothing from the
CUDA package ``paper_conf_icpp_zhangc0zx0025_b200`` and the package imports
nothing from here.

Definition (§2.2 P@10786 "BFC convolves X with nabla Y to compute
filter gradients nabla W"; Table 1 P@14515 §3 for the NHWC / NHWC / KRSC
layouts; readings R1-R3 for correlation orientation, symmetric pad,
stride 1)::

    Ho = H + 2 pad - R + 1,  Wo = W + 2 pad - S + 1
    dW[k, r, s, c] = sum_{n, h, w} Xp[n, h + r - pad, w + s - pad, c] * dY[n, h, w, k]

Three independent formulations, all FP64:

* ``bfc_c``            — C loop nest (oracle/bfc_oracle.c, OpenMP over k).
* ``bfc_numpy``        — zero-pad X, then one tensordot per (r, s): the
                          definition with a library contraction as the step.
* ``bfc_bruteforce``   — pure-Python loops, tiny shapes only.

Plus ``bfc_c_sampled`` (selected dW elements, for full-size parity), and the
N-D (3-D) definition of PAPER.md §3's Level-2 dimension reduction (P@17805:
an N-D BFC reduces to 2-D BFCs over the extra spatial axis)::

    Do = D + 2 pad - T + 1
    dW[k, t, r, s, c] = sum_{n, d, h, w} Xp[n, d+t-pad, h+r-pad, w+s-pad, c] * dY[n, d, h, w, k]

``bfc3d_numpy`` (one tensordot per filter tap) and ``bfc3d_bruteforce``; layouts
NDHWC / NDHWC / KTRSC (Table 1 extended by the depth axis, R23).

The forward and backward-data convolutions of PAPER.md §8 P@56407 ("with
moderate modifications, WinRS can support FC and BDC"), plain definitions,
stride 1, one symmetric pad (NHWC activations, KRSC weights)::

    FC : Y[n, h, w, k]  = sum_{r, s, c} Xp[n, h + r - pad, w + s - pad, c] * Wt[k, r, s, c]
    BDC: dX[n, i, j, c] = sum_{r, s, k} dYq[n, i - r + pad, j - s + pad, k] * Wt[k, r, s, c]

(dYq = dY, zero outside [0, Ho) x [0, Wo)) — ``fc_numpy``, ``bdc_numpy``.

Pins (tests/test_oracle.py): brute force == C == numpy (2-D and 3-D); torch
conv3d_weight in FP64; the D = 1 reduction of the 3-D definition; impulse; all-ones
closed form; adjoint identity against an independent forward convolution;
linearity; dY = 0; the Ho = Wo = 1 GEMM special case; torch.nn.grad
conv2d_weight in FP64.  No function here is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "bfc_oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (FP64, -O2, OpenMP, no fast-math)."""
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-Wall",
                               "-o", _LIB_PATH, _SRC])
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        i, p = ctypes.c_int, ctypes.c_void_p
        lib.oracle_bfc_f64.argtypes = [i] * 8 + [p, p, p, i]
        lib.oracle_bfc_f32in.argtypes = [i] * 8 + [p, p, p, i]
        lib.oracle_bfc_f32in_sampled.argtypes = [i] * 8 + [p, p, p, i, p, i]
        for f in (lib.oracle_bfc_f64, lib.oracle_bfc_f32in, lib.oracle_bfc_f32in_sampled):
            f.restype = ctypes.c_int
        lib.oracle_max_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def out_dims(H, W, R, S, pad):
    return H + 2 * pad - R + 1, W + 2 * pad - S + 1


def max_threads() -> int:
    return int(_load().oracle_max_threads())


def bfc_c(X: np.ndarray, dY: np.ndarray, R: int, S: int, pad: int, threads: int = 0) -> np.ndarray:
    """C FP64 loop nest.  X: [N,H,W,C], dY: [N,Ho,Wo,K] (float64, or float32/
    float16 which are upcast exactly).  Returns dW [K,R,S,C] float64."""
    lib = _load()
    N, H, W, C = X.shape
    _, Ho, Wo, K = dY.shape
    assert (Ho, Wo) == out_dims(H, W, R, S, pad), "dY shape does not match Ho, Wo"
    dW = np.empty((K, R, S, C), dtype=np.float64)
    if X.dtype == np.float64 and dY.dtype == np.float64:
        Xc, dYc = np.ascontiguousarray(X), np.ascontiguousarray(dY)
        fn = lib.oracle_bfc_f64
    else:
        # float16 -> float32 is exact; float32 is passed as is and upcast in C.
        Xc = np.ascontiguousarray(X.astype(np.float32, copy=False))
        dYc = np.ascontiguousarray(dY.astype(np.float32, copy=False))
        fn = lib.oracle_bfc_f32in
    rc = fn(N, C, H, W, K, R, S, pad, Xc.ctypes.data, dYc.ctypes.data, dW.ctypes.data, int(threads))
    if rc != 0:
        raise ValueError("oracle: invalid shape")
    return dW


def bfc_c_sampled(X: np.ndarray, dY: np.ndarray, R: int, S: int, pad: int,
                  flat_idx: np.ndarray, threads: int = 0) -> np.ndarray:
    """dW.flat[flat_idx] (KRSC flat indices), each element summed on its own."""
    lib = _load()
    N, H, W, C = X.shape
    _, Ho, Wo, K = dY.shape
    assert (Ho, Wo) == out_dims(H, W, R, S, pad)
    Xc = np.ascontiguousarray(X.astype(np.float32, copy=False))
    dYc = np.ascontiguousarray(dY.astype(np.float32, copy=False))
    idx = np.ascontiguousarray(flat_idx.astype(np.int64))
    out = np.empty(idx.shape[0], dtype=np.float64)
    rc = lib.oracle_bfc_f32in_sampled(N, C, H, W, K, R, S, pad, Xc.ctypes.data, dYc.ctypes.data,
                                      idx.ctypes.data, int(idx.shape[0]), out.ctypes.data, int(threads))
    if rc != 0:
        raise ValueError("oracle: invalid shape")
    return out


def bfc_numpy(X: np.ndarray, dY: np.ndarray, R: int, S: int, pad: int) -> np.ndarray:
    """Zero-pad X, then for every filter tap (r, s) contract the shifted X
    window with dY over (n, h, w): dW[:, r, s, :] = sum dY[n,h,w,k] Xp[n,h+r,w+s,c]."""
    X = X.astype(np.float64)
    dY = dY.astype(np.float64)
    N, H, W, C = X.shape
    _, Ho, Wo, K = dY.shape
    assert (Ho, Wo) == out_dims(H, W, R, S, pad)
    Xp = np.zeros((N, H + 2 * pad, W + 2 * pad, C), dtype=np.float64)
    Xp[:, pad:pad + H, pad:pad + W, :] = X
    dW = np.empty((K, R, S, C), dtype=np.float64)
    for r in range(R):
        for s in range(S):
            win = Xp[:, r:r + Ho, s:s + Wo, :]
            dW[:, r, s, :] = np.tensordot(dY, win, axes=([0, 1, 2], [0, 1, 2]))
    return dW


def bfc_bruteforce(X, dY, R: int, S: int, pad: int) -> np.ndarray:
    """Pure-Python loops over every index of the definition (tiny shapes)."""
    N, H, W, C = X.shape
    _, Ho, Wo, K = dY.shape
    assert (Ho, Wo) == out_dims(H, W, R, S, pad)
    Xl = np.asarray(X, dtype=np.float64).tolist()
    Gl = np.asarray(dY, dtype=np.float64).tolist()
    out = [[[[0.0] * C for _ in range(S)] for _ in range(R)] for _ in range(K)]
    for k in range(K):
        for r in range(R):
            for s in range(S):
                for c in range(C):
                    acc = 0.0
                    for n in range(N):
                        for h in range(Ho):
                            i = h + r - pad
                            if not 0 <= i < H:
                                continue
                            for w in range(Wo):
                                j = w + s - pad
                                if not 0 <= j < W:
                                    continue
                                acc += Xl[n][i][j][c] * Gl[n][h][w][k]
                    out[k][r][s][c] = acc
    return np.array(out, dtype=np.float64)


def out_dims3(D, H, W, T, R, S, pad):
    return D + 2 * pad - T + 1, H + 2 * pad - R + 1, W + 2 * pad - S + 1


def bfc3d_numpy(X: np.ndarray, dY: np.ndarray, T: int, R: int, S: int, pad: int) -> np.ndarray:
    """3-D BFC, the plain definition: zero-pad X on the three spatial axes, then
    for every filter tap (t, r, s) contract the shifted window with dY over
    (n, d, h, w).  X: [N,D,H,W,C], dY: [N,Do,Ho,Wo,K] -> dW [K,T,R,S,C] (FP64)."""
    X = X.astype(np.float64)
    dY = dY.astype(np.float64)
    N, D, H, W, C = X.shape
    _, Do, Ho, Wo, K = dY.shape
    assert (Do, Ho, Wo) == out_dims3(D, H, W, T, R, S, pad)
    Xp = np.zeros((N, D + 2 * pad, H + 2 * pad, W + 2 * pad, C), dtype=np.float64)
    Xp[:, pad:pad + D, pad:pad + H, pad:pad + W, :] = X
    dW = np.empty((K, T, R, S, C), dtype=np.float64)
    for t in range(T):
        for r in range(R):
            for s in range(S):
                win = Xp[:, t:t + Do, r:r + Ho, s:s + Wo, :]
                dW[:, t, r, s, :] = np.tensordot(dY, win, axes=([0, 1, 2, 3], [0, 1, 2, 3]))
    return dW


def bfc3d_bruteforce(X, dY, T: int, R: int, S: int, pad: int) -> np.ndarray:
    """Pure-Python loops over every index of the 3-D definition (tiny shapes)."""
    N, D, H, W, C = X.shape
    _, Do, Ho, Wo, K = dY.shape
    assert (Do, Ho, Wo) == out_dims3(D, H, W, T, R, S, pad)
    Xl = np.asarray(X, dtype=np.float64).tolist()
    Gl = np.asarray(dY, dtype=np.float64).tolist()
    out = np.zeros((K, T, R, S, C), dtype=np.float64)
    for k in range(K):
        for t in range(T):
            for r in range(R):
                for s in range(S):
                    for c in range(C):
                        acc = 0.0
                        for n in range(N):
                            for d in range(Do):
                                a = d + t - pad
                                if not 0 <= a < D:
                                    continue
                                for h in range(Ho):
                                    i = h + r - pad
                                    if not 0 <= i < H:
                                        continue
                                    for w in range(Wo):
                                        j = w + s - pad
                                        if 0 <= j < W:
                                            acc += Xl[n][a][i][j][c] * Gl[n][d][h][w][k]
                        out[k, t, r, s, c] = acc
    return out


def fc_numpy(X: np.ndarray, Wt: np.ndarray, pad: int) -> np.ndarray:
    """Forward convolution (correlation), FP64: one tensordot per filter tap."""
    X = X.astype(np.float64)
    Wt = Wt.astype(np.float64)
    N, H, W, C = X.shape
    K, R, S, C2 = Wt.shape
    assert C2 == C
    Ho, Wo = out_dims(H, W, R, S, pad)
    Xp = np.zeros((N, H + 2 * pad, W + 2 * pad, C), dtype=np.float64)
    Xp[:, pad:pad + H, pad:pad + W, :] = X
    Y = np.zeros((N, Ho, Wo, K), dtype=np.float64)
    for r in range(R):
        for s in range(S):
            Y += np.tensordot(Xp[:, r:r + Ho, s:s + Wo, :], Wt[:, r, s, :], axes=([3], [1]))
    return Y


def bdc_numpy(dY: np.ndarray, Wt: np.ndarray, pad: int, H: int, W: int) -> np.ndarray:
    """Backward-data convolution (the adjoint of fc_numpy in X), FP64:
    dX[n, i, j, c] = sum_{r, s, k} dY[n, i - r + pad, j - s + pad, k] Wt[k, r, s, c]."""
    dY = dY.astype(np.float64)
    Wt = Wt.astype(np.float64)
    N, Ho, Wo, K = dY.shape
    K2, R, S, C = Wt.shape
    assert K2 == K and (Ho, Wo) == out_dims(H, W, R, S, pad)
    dX = np.zeros((N, H, W, C), dtype=np.float64)
    for r in range(R):
        for s in range(S):
            # output rows i with 0 <= i - r + pad < Ho
            i0, i1 = max(0, r - pad), min(H, Ho + r - pad)
            j0, j1 = max(0, s - pad), min(W, Wo + s - pad)
            if i1 <= i0 or j1 <= j0:
                continue
            src = dY[:, i0 - r + pad:i1 - r + pad, j0 - s + pad:j1 - s + pad, :]
            dX[:, i0:i1, j0:j1, :] += np.tensordot(src, Wt[:, r, s, :], axes=([3], [0]))
    return dX


def rel_max_err(got: np.ndarray, ref: np.ndarray) -> float:
    """max_i |got_i - ref_i| / max_i |ref_i| in FP64 (the BASELINE gate)."""
    got = np.asarray(got, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    den = float(np.max(np.abs(ref))) if ref.size else 0.0
    num = float(np.max(np.abs(got - ref))) if ref.size else 0.0
    return num / den if den > 0 else num


def mare(got: np.ndarray, ref: np.ndarray) -> float:
    """Mean absolute relative error (the paper's Table 4 metric, P@50685)."""
    got = np.asarray(got, dtype=np.float64).ravel()
    ref = np.asarray(ref, dtype=np.float64).ravel()
    m = ref != 0
    return float(np.mean(np.abs(got[m] - ref[m]) / np.abs(ref[m]))) if m.any() else 0.0
