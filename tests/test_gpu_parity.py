"""GPU parity: the CUDA path (through the C ABI, via the ctypes binding)
against the FP64 CPU oracle on the same seeded inputs.

Gate (BASELINE.json north_star): max|err| <= 1e-4 * max|ref| for FP32 inputs,
<= 2e-2 * max|ref| for FP16 inputs (FP32 accumulation).  Inputs follow the
paper's accuracy protocol (P@50685): U[0,1], dY x 1e-2 for FP16.
"""
import os

import numpy as np
import pytest
import torch

import paper_conf_icpp_zhangc0zx0025_b200 as W
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
from oracle import oracle as O
from conftest import record_err

pytestmark = pytest.mark.gpu

TOL = {"f32": 1e-4, "f16": 2e-2, "bf16": 2e-2}


def _dev(a, dtype):
    t = torch.from_numpy(a).cuda()
    return t.to(torch.bfloat16) if dtype == "bf16" else t


def _run(layer, X, dY, env=None, monkeypatch=None):
    if env:
        for k, v in env.items():
            monkeypatch.setenv(k, v)
    p = W.plan(layer.N, layer.C, layer.H, layer.W, layer.K, layer.R, layer.S, layer.pad, layer.dtype)
    Xg = _dev(X, layer.dtype)
    Gg = _dev(dY, layer.dtype)
    dW = W.as_krsc(W.bfc(p, Xg, Gg))
    torch.cuda.synchronize()
    return p, dW.cpu().numpy().astype(np.float64)


def _full_check(layer, dist="u01", env=None, monkeypatch=None, tol=None):
    X, dY = wl.make_inputs(layer, dist)
    p, got = _run(layer, X, dY, env, monkeypatch)
    ref = O.bfc_c(X, dY, layer.R, layer.S, layer.pad)
    err = O.rel_max_err(got, ref)
    record_err(f"{layer.name}[{layer.dtype},{dist}]" + (f" {env}" if env else ""), err, p.kernel_name)
    assert err <= (tol or TOL[layer.dtype]), (layer, p, err)
    return p, err


# ---- configs[0]: tiny, full oracle
def test_tiny_f32():
    _full_check(wl.LAYERS["tiny_f32"])


# ---- reduced-size versions of every FP32 config: full oracle, several tiles + ragged tails
REDUCED = [
    wl.LAYERS["r50_c64_56_f32"].with_(N=2, name="r50_l1_n2"),
    wl.LAYERS["r50_c128_28_f32"].with_(N=2, C=72, K=100, name="r50_l2_ragged"),
    wl.LAYERS["r50_c256_14_f32"].with_(N=4, name="r50_l3_n4"),
    wl.LAYERS["r50_c512_7_f32"].with_(N=2, C=136, K=200, name="r50_l4_ragged"),
] + [l.with_(N=2, C=40, K=36, name=l.name + "_small") for l in wl.WIDE_F32]


@pytest.mark.parametrize("layer", REDUCED, ids=lambda l: l.name)
def test_reduced_f32(layer):
    _full_check(layer)


@pytest.mark.parametrize("layer", [l for l in REDUCED if l.R <= 4 or l.name.startswith("r50")], ids=lambda l: l.name)
def test_reduced_f32_signed(layer):
    """Signed U[-1,1) inputs, gated for alpha <= 8 plans (R17)."""
    _full_check(layer, dist="signed")


FORCED = [
    {"WINRS_FORCE_Z": "1"}, {"WINRS_FORCE_Z": "5"}, {"WINRS_FORCE_Z": "12"},
    {"WINRS_FORCE_TILE": "64x64"}, {"WINRS_FORCE_TILE": "32x32", "WINRS_FORCE_Z": "3"},
    {"WINRS_FORCE_PAIR": "8,3,6,0,0,0"}, {"WINRS_FORCE_PAIR": "4,3,2,0,0,0", "WINRS_FORCE_Z": "7"},
    {"WINRS_FORCE_CSPLIT": "1"}, {"WINRS_FORCE_CSPLIT": "2"}, {"WINRS_FORCE_CSPLIT": "8", "WINRS_FORCE_Z": "3"},
    {"WINRS_FORCE_CSPLIT": "4", "WINRS_FORCE_TILE": "32x32"},
]


@pytest.mark.parametrize("env", FORCED, ids=lambda e: ",".join(f"{k[12:]}={v}" for k, v in e.items()))
def test_forced_plans(env, monkeypatch):
    layer = wl.LAYERS["r50_c64_56_f32"].with_(N=2, H=30, W=29, C=68, K=44, name="forced")
    _full_check(layer, env=env, monkeypatch=monkeypatch)


def test_determinism():
    layer = wl.LAYERS["r50_c64_56_f32"].with_(N=3, name="det")
    X, dY = wl.make_inputs(layer)
    _, a = _run(layer, X, dY)
    _, b = _run(layer, X, dY)
    assert np.array_equal(a, b)


def test_zero_and_linearity():
    layer = wl.LAYERS["r50_c128_28_f32"].with_(N=2, name="lin")
    X, dY = wl.make_inputs(layer)
    _, z = _run(layer, X, np.zeros_like(dY))
    assert np.all(z == 0)
    _, a = _run(layer, X, dY)
    _, b = _run(layer, X, (2 * dY).astype(np.float32))
    assert np.allclose(b, 2 * a, rtol=1e-6, atol=0)


# ---- full BASELINE sizes: sampled outputs against the oracle element by element
FULL_F32 = wl.RESNET50_F32 + wl.WIDE_F32


@pytest.mark.parametrize("layer", FULL_F32, ids=lambda l: l.name)
def test_full_size_sampled(layer):
    X, dY = wl.make_inputs(layer)
    p, got = _run(layer, X, dY)
    idx = wl.sample_indices(layer, 384)
    ref = O.bfc_c_sampled(X, dY, layer.R, layer.S, layer.pad, idx)
    err = O.rel_max_err(got.ravel()[idx], ref)
    record_err(f"{layer.name} full size, {len(idx)} sampled outputs", err, p.kernel_name)
    assert err <= TOL[layer.dtype], (layer.name, p, err)
    assert np.isfinite(got).all()


def test_abi_errors():
    import ctypes
    from paper_conf_icpp_zhangc0zx0025_b200 import _lib
    p = W.plan(8, 64, 56, 56, 64, 3, 3, 1, "f32")
    X = torch.zeros(8, 56, 56, 64, device="cuda")
    dY = torch.zeros(8, 56, 56, 64, device="cuda")
    dW = torch.zeros(64, 3, 3, 64, device="cuda")
    L = _lib.lib()
    assert L.winrs_bfc(p.handle, X.data_ptr() + 4, dY.data_ptr(), dW.data_ptr(), None, None) == 1
    assert L.winrs_bfc(None, X.data_ptr(), dY.data_ptr(), dW.data_ptr(), None, None) == 1
    if p.workspace_bytes:
        assert L.winrs_bfc(p.handle, X.data_ptr(), dY.data_ptr(), dW.data_ptr(), None, None) == 3


# ============================================================== FP16 tensor-core path
REDUCED_F16 = [
    wl.LAYERS["r50_c64_56_f16"].with_(N=2, name="r50f16_l1_n2"),
    wl.LAYERS["r50_c128_28_f16"].with_(N=2, C=72, K=200, name="r50f16_l2_ragged"),
    wl.LAYERS["r50_c256_14_f16"].with_(N=4, name="r50f16_l3_n4"),
    wl.LAYERS["r50_c512_7_f16"].with_(N=3, C=136, K=264, name="r50f16_l4_ragged_n3"),
    wl.LAYERS["vgg_64_64_224_f16"].with_(N=1, H=60, W=61, name="vgg_l1_crop"),
    wl.LAYERS["r50_c64_56_f16"].with_(N=5, H=9, W=20, C=8, K=8, name="f16_tiny_channels_n5"),
]


@pytest.mark.parametrize("layer", REDUCED_F16, ids=lambda l: l.name)
def test_reduced_f16(layer):
    _full_check(layer)


@pytest.mark.parametrize("layer", REDUCED_F16[:3], ids=lambda l: l.name)
def test_reduced_f16_signed(layer):
    _full_check(layer, dist="signed")


FORCED_F16 = [
    {"WINRS_FORCE_Z": "1"}, {"WINRS_FORCE_Z": "7"},
    {"WINRS_FORCE_PAIR": "8,3,6,0,0,0"}, {"WINRS_FORCE_PAIR": "8,3,6,4,3,2", "WINRS_FORCE_Z": "3"},
    {"WINRS_FORCE_CSPLIT": "1"}, {"WINRS_FORCE_CSPLIT": "2"}, {"WINRS_FORCE_CSPLIT": "8"},
    {"WINRS_FORCE_CSPLIT": "4", "WINRS_FORCE_TILE": "128x32", "WINRS_FORCE_Z": "2"},
    {"WINRS_FORCE_CSPLIT": "4", "WINRS_FORCE_PAIR": "8,3,6,0,0,0"},
]


# K <= 64: 64-row dY raw stages (the alpha = 8 YB = 64 kernel variant) with
# ragged K and C, the B_N = 128 kernels with 64-row boxes (128x32 tile,
# Omega_4(3,2)), cluster split and buckets.
K64_F16 = [
    ({"K": 64, "C": 64}, {"WINRS_FORCE_PAIR": "8,3,6,0,0,0", "WINRS_FORCE_TILE": "128x64"}),
    ({"K": 40, "C": 72}, {"WINRS_FORCE_PAIR": "8,3,6,0,0,0", "WINRS_FORCE_TILE": "128x64", "WINRS_FORCE_CSPLIT": "4"}),
    ({"K": 8, "C": 136}, {"WINRS_FORCE_PAIR": "8,3,6,0,0,0", "WINRS_FORCE_TILE": "128x64", "WINRS_FORCE_Z": "3"}),
    ({"K": 56, "C": 64}, {"WINRS_FORCE_PAIR": "8,3,6,0,0,0", "WINRS_FORCE_TILE": "128x32"}),
    ({"K": 64, "C": 128}, {"WINRS_FORCE_PAIR": "8,3,6,4,3,2", "WINRS_FORCE_TILE": "128x64", "WINRS_FORCE_CSPLIT": "2"}),
]


@pytest.mark.parametrize("shape,env", K64_F16, ids=lambda v: ",".join(f"{k}={x}" for k, x in v.items()) if isinstance(v, dict) else str(v))
def test_k_le_64_f16(shape, env, monkeypatch):
    layer = wl.LAYERS["r50_c64_56_f16"].with_(N=2, H=22, W=23, name="k64_" + str(shape["K"]), **shape)
    _full_check(layer, env=env, monkeypatch=monkeypatch)


@pytest.mark.parametrize("env", FORCED_F16, ids=lambda e: ",".join(f"{k[12:]}={v}" for k, v in e.items()))
def test_forced_plans_f16(env, monkeypatch):
    layer = wl.LAYERS["r50_c64_56_f16"].with_(N=2, H=30, W=29, C=72, K=136, name="forced16")
    _full_check(layer, env=env, monkeypatch=monkeypatch)


def test_determinism_f16():
    layer = wl.LAYERS["r50_c128_28_f16"].with_(N=3, name="det16")
    X, dY = wl.make_inputs(layer)
    _, a = _run(layer, X, dY)
    _, b = _run(layer, X, dY)
    assert np.array_equal(a, b)


FULL_F16 = wl.RESNET50_F16 + wl.VGG16_F16 + [wl.LAYERS["r50_l3_n512_f16"]]


@pytest.mark.parametrize("layer", FULL_F16, ids=lambda l: l.name)
def test_full_size_sampled_f16(layer):
    X, dY = wl.make_inputs(layer)
    p, got = _run(layer, X, dY)
    idx = wl.sample_indices(layer, 256)
    ref = O.bfc_c_sampled(X, dY, layer.R, layer.S, layer.pad, idx)
    err = O.rel_max_err(got.ravel()[idx], ref)
    record_err(f"{layer.name} full size, {len(idx)} sampled outputs", err, p.kernel_name)
    assert err <= TOL[layer.dtype], (layer.name, p, err)
    assert np.isfinite(got).all()


# ============================================================== K-sharding (strided dY)
@pytest.mark.parametrize("layer", [wl.LAYERS["r50_c128_28_f32"].with_(N=2, K=136, name="ks32"),
                                   wl.LAYERS["r50_c128_28_f16"].with_(N=2, K=200, name="ks16")],
                         ids=lambda l: l.name)
@pytest.mark.parametrize("world", [2, 3])
def test_k_sharded_slices_concatenate_to_oracle(layer, world):
    """Each rank's dW slice (channel slice of dY read in place, ldy = K) —
    concatenated along K — equals the full-batch oracle; no communication."""
    X, dY = wl.make_inputs(layer)
    Xg, Gg = torch.from_numpy(X).cuda(), torch.from_numpy(dY).cuda()
    parts = []
    for r in range(world):
        dW, k0, k1 = W.bfc_k_sharded(Xg, Gg, layer.R, layer.S, layer.pad, layer.dtype, r, world)
        parts.append((k0, dW))
    torch.cuda.synchronize()
    assert [k0 for k0, _ in parts] == sorted(k0 for k0, _ in parts)
    got = torch.cat([d for _, d in parts], dim=0).cpu().numpy()
    ref = O.bfc_c(X, dY, layer.R, layer.S, layer.pad)
    err = O.rel_max_err(got, ref)
    record_err(f"{layer.name} K-sharded x{world}", err)
    assert err <= TOL[layer.dtype]


# ============================================================== FP16 widths 2..9
@pytest.mark.parametrize("S", [2, 4, 5, 6, 7, 8, 9])
def test_f16_all_widths(S):
    layer = wl.LAYERS["wide_r5_f32"].with_(N=2, C=48, K=72, H=20, W=23, R=S, S=S, pad=S // 2, dtype="f16",
                                           name=f"f16_w{S}")
    _full_check(layer)


# ============================================================== BF16 tensor-core variant
REDUCED_BF16 = [l.with_(dtype="bf16", name=l.name.replace("f16", "bf16")) for l in REDUCED_F16[:4]]


@pytest.mark.parametrize("layer", REDUCED_BF16, ids=lambda l: l.name)
def test_reduced_bf16(layer):
    _full_check(layer)


@pytest.mark.parametrize("S", [2, 5, 7])
def test_bf16_widths(S):
    layer = wl.LAYERS["wide_r5_f32"].with_(N=2, C=48, K=72, H=20, W=23, R=S, S=S, pad=S // 2, dtype="bf16",
                                           name=f"bf16_w{S}")
    _full_check(layer)


def test_bf16_full_size_sampled():
    layer = wl.LAYERS["r50_c256_14_f16"].with_(dtype="bf16", name="r50_c256_14_bf16")
    X, dY = wl.make_inputs(layer)
    p, got = _run(layer, X, dY)
    idx = wl.sample_indices(layer, 256)
    ref = O.bfc_c_sampled(X, dY, layer.R, layer.S, layer.pad, idx)
    err = O.rel_max_err(got.ravel()[idx], ref)
    record_err(f"{layer.name} full size, {len(idx)} sampled outputs", err, p.kernel_name)
    assert err <= TOL["bf16"]


@pytest.mark.gpu
@pytest.mark.parametrize("z,tile,cs", [(4, "128x128", 8), (7, "128x128", 8), (4, "128x128", 4)])
def test_no_hang_partial_tile_alpha4_cold_l2(z, tile, cs):
    """Regression: the deep-raw-ring Omega_4(3,2) kernel (14 transformer warps,
    3 operand stages) broke the operand-ring parity bound and hung within a few
    hundred cold-L2 calls on these forced ResNet-50 L1 plans.  Run 1500 calls
    in a child process under a hard timeout so a hang fails instead of blocking."""
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, os.path.join(root, "tools", "hang_repro.py"), "r50_c64_56_f16",
                        str(z), tile, str(cs), "1500"], capture_output=True, text=True, timeout=240, cwd=root)
    assert r.returncode == 0 and "done 1500" in r.stdout, r.stdout + r.stderr
