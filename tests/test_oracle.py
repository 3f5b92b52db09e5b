"""Pins for the FP64 oracle (oracle/): each test checks it against something
other than itself — brute force, a closed form, an invariant, a textbook
special case or a library routine — so that a dropped term, a wrong sign or
index, or a transposed operand fails at least one of them.

Definition pinned: PAPER.md §2.2 P@10786 (BFC convolves X with nabla Y to give
nabla W), Table 1 P@14515 (NHWC / NHWC / KRSC layouts), R1-R3.
"""
import numpy as np
import pytest
import torch

from oracle import oracle as O


def _rand(shape, seed, lo=-1.0, hi=1.0):
    g = np.random.Generator(np.random.PCG64(seed))
    return g.uniform(lo, hi, size=shape)


SMALL_SHAPES = [
    # N, C, H, W, K, R, S, pad
    (1, 4, 8, 8, 4, 3, 3, 1),      # the tiny BASELINE config
    (2, 3, 5, 7, 2, 2, 3, 0),      # R != S, H != W, no padding
    (2, 2, 6, 5, 3, 3, 2, 2),      # pad larger than needed (Ho > H)
    (1, 2, 4, 4, 2, 4, 4, 1),      # filter as large as the map
    (3, 1, 3, 9, 1, 1, 5, 2),      # R = 1
]


@pytest.mark.parametrize("shape", SMALL_SHAPES)
def test_c_numpy_bruteforce_agree(shape):
    N, C, H, W, K, R, S, pad = shape
    Ho, Wo = O.out_dims(H, W, R, S, pad)
    X = _rand((N, H, W, C), 1)
    dY = _rand((N, Ho, Wo, K), 2)
    bf = O.bfc_bruteforce(X, dY, R, S, pad)
    c = O.bfc_c(X, dY, R, S, pad)
    nb = O.bfc_numpy(X, dY, R, S, pad)
    assert np.allclose(c, bf, rtol=1e-13, atol=1e-13)
    assert np.allclose(nb, bf, rtol=1e-13, atol=1e-13)


@pytest.mark.parametrize("shape", SMALL_SHAPES)
def test_torch_conv2d_weight_fp64(shape):
    """Library routine: torch.nn.grad.conv2d_weight (NCHW / KCRS) in FP64."""
    N, C, H, W, K, R, S, pad = shape
    Ho, Wo = O.out_dims(H, W, R, S, pad)
    X = _rand((N, H, W, C), 3)
    dY = _rand((N, Ho, Wo, K), 4)
    ref = torch.nn.grad.conv2d_weight(torch.from_numpy(X).permute(0, 3, 1, 2), (K, C, R, S),
                                      torch.from_numpy(dY).permute(0, 3, 1, 2), padding=pad)
    ref = ref.permute(0, 2, 3, 1).numpy()          # KCRS -> KRSC
    assert np.allclose(O.bfc_c(X, dY, R, S, pad), ref, rtol=1e-12, atol=1e-12)


def test_impulse_pins_layout_and_padding():
    """dY = e_{n0,h0,w0,k0}  =>  dW[k0,r,s,c] = Xpad[n0, h0+r-pad, w0+s-pad, c]
    and dW[k != k0] = 0: pins NHWC/KRSC, correlation (not convolution) and the
    pad convention.  Checked at a corner (window partly in the padding) and an
    interior point."""
    N, C, H, W, K, R, S, pad = 2, 3, 6, 7, 3, 3, 4, 2
    Ho, Wo = O.out_dims(H, W, R, S, pad)
    X = _rand((N, H, W, C), 5)
    for (n0, h0, w0, k0) in [(0, 0, 0, 0), (1, 3, 4, 2), (1, Ho - 1, Wo - 1, 1)]:
        dY = np.zeros((N, Ho, Wo, K))
        dY[n0, h0, w0, k0] = 1.0
        dW = O.bfc_c(X, dY, R, S, pad)
        for k in range(K):
            for r in range(R):
                for s in range(S):
                    i, j = h0 + r - pad, w0 + s - pad
                    exp = X[n0, i, j, :] if (k == k0 and 0 <= i < H and 0 <= j < W) else np.zeros(C)
                    assert np.array_equal(dW[k, r, s, :], exp), (n0, h0, w0, k0, k, r, s)


@pytest.mark.parametrize("shape", SMALL_SHAPES + [(4, 2, 16, 16, 2, 5, 3, 2)])
def test_all_ones_closed_form(shape):
    """X = 1, dY = 1  =>  dW[k,r,s,c] = N * cnt(r, H, Ho) * cnt(s, W, Wo), where
    cnt(r, H, Ho) = |[max(0, pad-r), min(Ho, H+pad-r))| is the number of output
    rows whose input row h+r-pad is inside the map.  Exact."""
    N, C, H, W, K, R, S, pad = shape
    Ho, Wo = O.out_dims(H, W, R, S, pad)
    dW = O.bfc_c(np.ones((N, H, W, C)), np.ones((N, Ho, Wo, K)), R, S, pad)

    def cnt(r, H_, Ho_):
        return max(0, min(Ho_, H_ + pad - r) - max(0, pad - r))

    for r in range(R):
        for s in range(S):
            assert np.all(dW[:, r, s, :] == N * cnt(r, H, Ho) * cnt(s, W, Wo))


@pytest.mark.parametrize("shape", SMALL_SHAPES)
def test_adjoint_identity(shape):
    """BFC is the adjoint of the forward convolution in the weight argument:
    <dW, V> = <dY, conv_fwd(X, V)> for any V.  conv_fwd is torch's conv2d
    (cross-correlation) in FP64, independent of the oracle."""
    N, C, H, W, K, R, S, pad = shape
    Ho, Wo = O.out_dims(H, W, R, S, pad)
    X = _rand((N, H, W, C), 6)
    dY = _rand((N, Ho, Wo, K), 7)
    V = _rand((K, R, S, C), 8)
    dW = O.bfc_c(X, dY, R, S, pad)
    Y = torch.nn.functional.conv2d(torch.from_numpy(X).permute(0, 3, 1, 2),
                                   torch.from_numpy(V).permute(0, 3, 1, 2), padding=pad)
    Y = Y.permute(0, 2, 3, 1).numpy()
    lhs = float(np.sum(dW * V))
    rhs = float(np.sum(dY * Y))
    assert abs(lhs - rhs) <= 1e-12 * max(1.0, abs(rhs))


def test_linearity_and_zero():
    N, C, H, W, K, R, S, pad = 2, 3, 7, 6, 4, 3, 3, 1
    Ho, Wo = O.out_dims(H, W, R, S, pad)
    X1, X2 = _rand((N, H, W, C), 9), _rand((N, H, W, C), 10)
    G1, G2 = _rand((N, Ho, Wo, K), 11), _rand((N, Ho, Wo, K), 12)
    a, b = 0.75, -1.5
    f = lambda X, G: O.bfc_c(X, G, R, S, pad)
    assert np.allclose(f(X1, a * G1 + b * G2), a * f(X1, G1) + b * f(X1, G2), rtol=1e-12, atol=1e-12)
    assert np.allclose(f(a * X1 + b * X2, G1), a * f(X1, G1) + b * f(X2, G1), rtol=1e-12, atol=1e-12)
    assert np.all(f(X1, np.zeros_like(G1)) == 0.0)
    assert np.all(f(np.zeros_like(X1), G1) == 0.0)


def test_single_output_position_is_a_gemm():
    """pad = 0, R = H, S = W  =>  Ho = Wo = 1 and
    dW[k, r, s, c] = sum_n dY[n,0,0,k] X[n,r,s,c]: the textbook GEMM dY^T X."""
    N, C, H, W, K = 5, 3, 4, 9, 6
    X = _rand((N, H, W, C), 13)
    dY = _rand((N, 1, 1, K), 14)
    dW = O.bfc_c(X, dY, H, W, 0)
    gemm = (dY.reshape(N, K).T @ X.reshape(N, H * W * C)).reshape(K, H, W, C)
    assert np.allclose(dW, gemm, rtol=1e-13, atol=1e-13)


def test_sampled_and_f32_input_paths():
    N, C, H, W, K, R, S, pad = 3, 8, 10, 9, 4, 3, 5, 2
    Ho, Wo = O.out_dims(H, W, R, S, pad)
    g = np.random.Generator(np.random.PCG64(15))
    X = g.random((N, H, W, C), dtype=np.float32)
    dY = g.random((N, Ho, Wo, K), dtype=np.float32)
    full64 = O.bfc_c(X.astype(np.float64), dY.astype(np.float64), R, S, pad)
    full32 = O.bfc_c(X, dY, R, S, pad)                   # exact upcast inside C
    assert np.array_equal(full64, full32)
    idx = np.arange(0, K * R * S * C, 7)
    samp = O.bfc_c_sampled(X, dY, R, S, pad, idx)
    assert np.allclose(samp, full64.ravel()[idx], rtol=1e-13, atol=0)
    # float16 inputs are upcast exactly as well
    Xh, Gh = X.astype(np.float16), dY.astype(np.float16)
    assert np.array_equal(O.bfc_c(Xh, Gh, R, S, pad),
                          O.bfc_c(Xh.astype(np.float64), Gh.astype(np.float64), R, S, pad))


def test_error_metrics():
    ref = np.array([1.0, -2.0, 4.0])
    got = np.array([1.0, -2.5, 4.0])
    assert O.rel_max_err(got, ref) == pytest.approx(0.125)
    assert O.mare(got, ref) == pytest.approx(0.25 / 3)


def test_rejects_bad_shapes():
    with pytest.raises(AssertionError):
        O.bfc_c(np.zeros((1, 4, 4, 1)), np.zeros((1, 3, 3, 1)), 3, 3, 1)   # dY should be 4x4


# ============================================================== N-D (3-D) definition
SHAPES3 = [
    # N, C, D, H, W, K, T, R, S, pad
    (1, 2, 3, 4, 5, 2, 3, 3, 3, 1),
    (2, 3, 4, 3, 4, 2, 2, 1, 3, 0),
    (1, 2, 2, 5, 4, 3, 3, 2, 2, 2),
]


@pytest.mark.parametrize("shape", SHAPES3)
def test_3d_numpy_bruteforce_torch_agree(shape):
    """3-D definition: brute force == numpy == torch.nn.grad.conv3d_weight (FP64,
    a library routine; NCDHW / KCTRS permuted to NDHWC / KTRSC)."""
    N, C, D, H, W, K, T, R, S, pad = shape
    Do, Ho, Wo = O.out_dims3(D, H, W, T, R, S, pad)
    X = _rand((N, D, H, W, C), 11)
    dY = _rand((N, Do, Ho, Wo, K), 12)
    bf = O.bfc3d_bruteforce(X, dY, T, R, S, pad)
    nb = O.bfc3d_numpy(X, dY, T, R, S, pad)
    ref = torch.nn.grad.conv3d_weight(torch.from_numpy(X).permute(0, 4, 1, 2, 3), (K, C, T, R, S),
                                      torch.from_numpy(dY).permute(0, 4, 1, 2, 3), padding=pad)
    ref = ref.permute(0, 2, 3, 4, 1).numpy()
    assert np.allclose(nb, bf, rtol=1e-13, atol=1e-13)
    assert np.allclose(nb, ref, rtol=1e-12, atol=1e-12)


def test_3d_reduces_to_2d_when_depth_is_one():
    """Level-2 dimension reduction, special case D = 1, T = 3, pad = 1: Do = 1,
    the depth taps t = 0, 2 only see padding (zero), and the middle tap is the
    2-D BFC of the single slice."""
    N, C, H, W, K, R, S, pad = 2, 3, 6, 5, 4, 3, 3, 1
    X = _rand((N, 1, H, W, C), 13)
    Do, Ho, Wo = O.out_dims3(1, H, W, 3, R, S, pad)
    assert Do == 1
    dY = _rand((N, 1, Ho, Wo, K), 14)
    got = O.bfc3d_numpy(X, dY, 3, R, S, pad)
    assert np.all(got[:, 0] == 0) and np.all(got[:, 2] == 0)
    assert np.allclose(got[:, 1], O.bfc_c(X[:, 0], dY[:, 0], R, S, pad), rtol=1e-13, atol=1e-13)


def test_3d_impulse():
    """dY = e_{n0,d0,h0,w0,k0} => dW[k0,t,r,s,c] = Xpad[n0, d0+t-pad, h0+r-pad, w0+s-pad, c]."""
    N, C, D, H, W, K, T, R, S, pad = 2, 3, 4, 5, 5, 2, 3, 3, 3, 1
    Do, Ho, Wo = O.out_dims3(D, H, W, T, R, S, pad)
    X = _rand((N, D, H, W, C), 15)
    dY = np.zeros((N, Do, Ho, Wo, K))
    n0, d0, h0, w0, k0 = 1, 0, 2, 4, 1
    dY[n0, d0, h0, w0, k0] = 1.0
    got = O.bfc3d_numpy(X, dY, T, R, S, pad)
    Xp = np.zeros((N, D + 2 * pad, H + 2 * pad, W + 2 * pad, C))
    Xp[:, pad:pad + D, pad:pad + H, pad:pad + W] = X
    assert np.array_equal(got[k0], Xp[n0, d0:d0 + T, h0:h0 + R, w0:w0 + S, :])
    assert np.all(got[1 - k0] == 0)


# ============================================================== FC and BDC definitions
CONV_SHAPES = [
    # N, C, H, W, K, R, S, pad
    (2, 3, 6, 7, 4, 3, 3, 1),
    (1, 2, 5, 5, 3, 2, 3, 0),
    (2, 4, 4, 6, 2, 3, 2, 2),
]


@pytest.mark.parametrize("shape", CONV_SHAPES)
def test_fc_bdc_against_torch(shape):
    """Library routines in FP64: torch conv2d (correlation) for FC and
    torch.nn.grad.conv2d_input for BDC (NCHW / KCRS permuted to NHWC / KRSC)."""
    N, C, H, W, K, R, S, pad = shape
    Ho, Wo = O.out_dims(H, W, R, S, pad)
    X = _rand((N, H, W, C), 21)
    Wt = _rand((K, R, S, C), 22)
    dY = _rand((N, Ho, Wo, K), 23)
    tX, tW = torch.from_numpy(X).permute(0, 3, 1, 2), torch.from_numpy(Wt).permute(0, 3, 1, 2)
    Y = torch.nn.functional.conv2d(tX, tW, padding=pad).permute(0, 2, 3, 1).numpy()
    dX = torch.nn.grad.conv2d_input((N, C, H, W), tW, torch.from_numpy(dY).permute(0, 3, 1, 2),
                                    padding=pad).permute(0, 2, 3, 1).numpy()
    assert np.allclose(O.fc_numpy(X, Wt, pad), Y, rtol=1e-12, atol=1e-12)
    assert np.allclose(O.bdc_numpy(dY, Wt, pad, H, W), dX, rtol=1e-12, atol=1e-12)


def test_fc_bfc_bdc_adjoint_triangle():
    """<FC(X, Wt), dY> = <X, BDC(dY, Wt)> = <Wt, BFC(X, dY)>: the three
    convolutions of one layer are mutual adjoints."""
    N, C, H, W, K, R, S, pad = 2, 3, 7, 6, 4, 3, 3, 1
    Ho, Wo = O.out_dims(H, W, R, S, pad)
    X, Wt, dY = _rand((N, H, W, C), 24), _rand((K, R, S, C), 25), _rand((N, Ho, Wo, K), 26)
    a = float(np.sum(O.fc_numpy(X, Wt, pad) * dY))
    b = float(np.sum(X * O.bdc_numpy(dY, Wt, pad, H, W)))
    c = float(np.sum(Wt * O.bfc_c(X, dY, R, S, pad)))
    assert abs(a - b) <= 1e-10 * abs(a) and abs(a - c) <= 1e-10 * abs(a)
