"""GPU parity, round 2: the second-generation tensor-core kernel
(bfc_tc2.cuh), pad = 0 layers, every reachable FP32 kernel for F_W = 6 / 8,
exactness on structured inputs, and bitwise reproducibility under repeated
cold-L2 calls.  Every check compares the CUDA path (C ABI via the ctypes
binding) with the FP64 oracle on the same inputs, element by element.

Gate (BASELINE.json north_star): max|err| <= 1e-4 max|ref| (FP32 inputs),
<= 2e-2 max|ref| (FP16 / BF16 inputs, FP32 accumulation).
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
ENV_KEYS = ("WINRS_FORCE_TILE", "WINRS_FORCE_CSPLIT", "WINRS_FORCE_Z", "WINRS_FORCE_PAIR", "WINRS_TC_GEN", "WINRS_FORCE_CG",
            "WINRS_FORCE_TA", "WINRS_FP32_TC")


def _dev(a, dtype):
    t = torch.from_numpy(np.ascontiguousarray(a)).cuda()
    return t.to(torch.bfloat16) if dtype == "bf16" else t


def _plan(layer, env, monkeypatch):
    for k in ENV_KEYS:
        monkeypatch.delenv(k, raising=False)
    for k, v in (env or {}).items():
        monkeypatch.setenv(k, v)
    return W.plan(layer.N, layer.C, layer.H, layer.W, layer.K, layer.R, layer.S, layer.pad, layer.dtype)


def _check(layer, monkeypatch, env=None, dist="u01", X=None, dY=None, exact=False, expect_kernel=None):
    if X is None:
        X, dY = wl.make_inputs(layer, dist)
    p = _plan(layer, env, monkeypatch)
    if expect_kernel:
        assert expect_kernel in p.kernel_name, (p.kernel_name, expect_kernel)
    dW = W.as_krsc(W.bfc(p, _dev(X, layer.dtype), _dev(dY, layer.dtype)))
    torch.cuda.synchronize()
    got = dW.cpu().numpy().astype(np.float64)
    ref = O.bfc_c(X, dY, layer.R, layer.S, layer.pad)
    err = O.rel_max_err(got, ref)
    record_err(f"{layer.name}[{layer.dtype}] {env or ''}", err, f"{p.kernel_name} Z={p.info['Z']} cs={p.info['csplit']}")
    if exact:
        assert np.array_equal(got, ref), (layer.name, p.kernel_name, err, np.max(np.abs(got - ref)))
    assert err <= TOL[layer.dtype], (layer.name, p.kernel_name, err)
    assert np.isfinite(got).all()
    return p, err


# ====================================================== bfc_tc2.cuh (second-generation tensor-core kernel)
BASE = wl.LAYERS["r50_c64_56_f16"]
TC2 = [
    ("l1", dict(N=16), {}),
    ("l1_f2", dict(N=16), {"WINRS_FORCE_TILE": "64x64"}),
    ("l1_f1_cs2", dict(N=16), {"WINRS_FORCE_TILE": "64x128", "WINRS_FORCE_CSPLIT": "2"}),
    ("l2_nk128_cs1", dict(N=16, C=128, K=128, H=28, W=28), {"WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_CSPLIT": "1"}),
    ("l2_nk128_cs3", dict(N=16, C=128, K=128, H=28, W=28), {"WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_CSPLIT": "3"}),
    ("l2_nk128_cs4", dict(N=16, C=128, K=128, H=28, W=28), {"WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_CSPLIT": "4"}),
    ("l3", dict(N=16, C=256, K=256, H=14, W=14), {}),
    ("l3_cs6", dict(N=16, C=256, K=256, H=14, W=14), {"WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_CSPLIT": "6"}),
    ("l4_odd_wo", dict(N=16, C=512, K=512, H=7, W=7), {}),
    ("ragged_ck", dict(N=16, C=72, K=200, H=20, W=17), {}),
    ("ragged_f2", dict(N=16, C=40, K=136, H=20, W=17), {"WINRS_FORCE_TILE": "128x64"}),
    ("pad0", dict(N=16, C=64, K=64, H=20, W=20, pad=0), {}),
    ("pad0_f1", dict(N=16, C=128, K=64, H=19, W=21, pad=0), {"WINRS_FORCE_TILE": "64x128"}),
    ("s6_ftiles2", dict(N=16, C=64, K=64, H=16, W=16, R=3, S=6, pad=2), {"WINRS_FORCE_PAIR": "4,3,2,0,0,0"}),
    ("r5_f2", dict(N=16, C=64, K=128, H=16, W=16, R=5, S=3, pad=2), {"WINRS_FORCE_TILE": "128x64"}),
    ("r1", dict(N=16, C=64, K=64, H=12, W=12, R=1, S=3, pad=0), {}),
    ("n32_z5", dict(N=32, C=64, K=64, H=30, W=30), {"WINRS_FORCE_Z": "5"}),
    ("n48_cs8", dict(N=48, C=128, K=64, H=12, W=12), {"WINRS_FORCE_CSPLIT": "8"}),
    # cta_group::2 pairs: What rows split (256 c / 4 filter rows) and the swapped pair (256 k x 128 c)
    ("pair_l3", dict(N=16, C=256, K=256, H=14, W=14), {"WINRS_FORCE_CG": "2", "WINRS_FORCE_TILE": "128x256", "WINRS_FORCE_CSPLIT": "1"}),
    ("pair_f2_cs2_r5", dict(N=32, C=128, K=128, H=12, W=12, R=5, S=3, pad=2),
     {"WINRS_FORCE_CG": "2", "WINRS_FORCE_TILE": "128x64", "WINRS_FORCE_CSPLIT": "2"}),
    ("pair_cs4_ragged", dict(N=16, C=200, K=136, H=12, W=13), {"WINRS_FORCE_CG": "2", "WINRS_FORCE_TILE": "128x256", "WINRS_FORCE_CSPLIT": "4"}),
    ("swap_l3", dict(N=16, C=256, K=256, H=14, W=14), {"WINRS_FORCE_TILE": "256x128", "WINRS_FORCE_CSPLIT": "1"}),
    ("swap_cs4", dict(N=16, C=256, K=256, H=14, W=14), {"WINRS_FORCE_TILE": "256x128", "WINRS_FORCE_CSPLIT": "4"}),
    ("swap_ragged", dict(N=16, C=200, K=328, H=12, W=13), {"WINRS_FORCE_TILE": "256x128", "WINRS_FORCE_CSPLIT": "2"}),
    ("swap_pad0_s6", dict(N=16, C=128, K=256, H=12, W=14, S=6, pad=0), {"WINRS_FORCE_TILE": "256x128", "WINRS_FORCE_PAIR": "4,3,2,0,0,0"}),
]


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
@pytest.mark.parametrize("name,ov,env", TC2, ids=[c[0] for c in TC2])
def test_tc2(name, ov, env, dtype, monkeypatch):
    """Xhat in shared memory (the TA variant is covered by test_tc2_ta)."""
    layer = BASE.with_(name="tc2_" + name, dtype=dtype, **ov)
    _check(layer, monkeypatch, dict(env, WINRS_TC_GEN="2", WINRS_FORCE_TA="0"), expect_kernel="_v2")


# Xhat in TMEM (bfc_tc2.cuh TA: ldmatrix.trans -> IT -> tcgen05.st, A operand from TMEM), NK = 64 tiles
TA = [
    ("l1", dict(N=16), {"WINRS_FORCE_TILE": "64x64"}),
    ("l1_f1_cs2", dict(N=16), {"WINRS_FORCE_TILE": "64x128", "WINRS_FORCE_CSPLIT": "2"}),
    ("l1_cs8", dict(N=32), {"WINRS_FORCE_TILE": "64x64", "WINRS_FORCE_CSPLIT": "8"}),
    ("ragged_f2", dict(N=16, C=40, K=136, H=20, W=17), {"WINRS_FORCE_TILE": "64x64"}),
    ("ragged_f1", dict(N=16, C=200, K=72, H=13, W=11), {"WINRS_FORCE_TILE": "64x128", "WINRS_FORCE_CSPLIT": "3"}),
    ("pad0", dict(N=16, C=64, K=64, H=20, W=20, pad=0), {"WINRS_FORCE_TILE": "64x64"}),
    ("s6_ftiles2", dict(N=16, C=64, K=64, H=16, W=16, R=3, S=6, pad=2), {"WINRS_FORCE_PAIR": "4,3,2,0,0,0", "WINRS_FORCE_TILE": "64x64"}),
    ("r5_f2", dict(N=16, C=64, K=128, H=16, W=16, R=5, S=3, pad=2), {"WINRS_FORCE_TILE": "64x64"}),
    ("r1", dict(N=16, C=64, K=64, H=12, W=12, R=1, S=3, pad=0), {"WINRS_FORCE_TILE": "64x128"}),
    ("n32_z5", dict(N=32, C=64, K=64, H=30, W=30), {"WINRS_FORCE_Z": "5", "WINRS_FORCE_TILE": "64x64"}),
    ("n48_cs4", dict(N=48, C=128, K=64, H=12, W=12), {"WINRS_FORCE_CSPLIT": "4", "WINRS_FORCE_TILE": "64x128"}),
    ("l1_cs5", dict(N=32), {"WINRS_FORCE_TILE": "64x64", "WINRS_FORCE_CSPLIT": "5"}),
    ("ragged_f1_cs7", dict(N=16, C=200, K=72, H=13, W=11), {"WINRS_FORCE_TILE": "64x128", "WINRS_FORCE_CSPLIT": "7"}),
    ("l3_cs5", dict(N=16, C=256, K=256, H=14, W=14), {"WINRS_FORCE_TILE": "64x128", "WINRS_FORCE_CSPLIT": "5"}),
]


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
@pytest.mark.parametrize("name,ov,env", TA, ids=[c[0] for c in TA])
def test_tc2_ta(name, ov, env, dtype, monkeypatch):
    layer = BASE.with_(name="ta_" + name, dtype=dtype, **ov)
    _check(layer, monkeypatch, dict(env, WINRS_TC_GEN="2", WINRS_FORCE_TA="1"), expect_kernel="_v2t_")


# xi-split pair (bfc_tc2x.cuh: xi {0,1} / {2,3} on the two CTAs of a pair, Xhat in TMEM, NK = 128 tiles,
# the pair's partial OT tiles summed with the depth-split ranks in one DSMEM reduction)
XS = [
    ("l2", dict(N=16, C=128, K=128, H=28, W=28), {"WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_CSPLIT": "1"}),
    ("l2_cs2", dict(N=16, C=128, K=128, H=28, W=28), {"WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_CSPLIT": "2"}),
    ("l3_cs3", dict(N=16, C=256, K=256, H=14, W=14), {"WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_CSPLIT": "3"}),
    ("l3_cs4", dict(N=32, C=256, K=256, H=14, W=14), {"WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_CSPLIT": "4"}),
    ("l4_odd_wo", dict(N=16, C=512, K=512, H=7, W=7), {"WINRS_FORCE_TILE": "128x128"}),
    ("l1_f2", dict(N=16, C=64, K=128, H=20, W=20), {"WINRS_FORCE_TILE": "128x64"}),
    ("f2_cs4", dict(N=32, C=64, K=128, H=16, W=16), {"WINRS_FORCE_TILE": "128x64", "WINRS_FORCE_CSPLIT": "4"}),
    ("ragged_f1", dict(N=16, C=200, K=136, H=13, W=11), {"WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_CSPLIT": "3"}),
    ("ragged_f2", dict(N=16, C=40, K=72, H=20, W=17), {"WINRS_FORCE_TILE": "128x64"}),
    ("pad0", dict(N=16, C=128, K=128, H=20, W=20, pad=0), {"WINRS_FORCE_TILE": "128x128"}),
    ("s6_ftiles2", dict(N=16, C=64, K=128, H=16, W=16, R=3, S=6, pad=2), {"WINRS_FORCE_PAIR": "4,3,2,0,0,0", "WINRS_FORCE_TILE": "128x64"}),
    ("r5_f2", dict(N=16, C=64, K=128, H=16, W=16, R=5, S=3, pad=2), {"WINRS_FORCE_TILE": "128x64", "WINRS_FORCE_CSPLIT": "2"}),
    ("r1", dict(N=16, C=128, K=128, H=12, W=12, R=1, S=3, pad=0), {"WINRS_FORCE_TILE": "128x128"}),
    ("n32_z5", dict(N=32, C=128, K=128, H=30, W=30), {"WINRS_FORCE_Z": "5", "WINRS_FORCE_TILE": "128x128"}),
    ("n48_z3_cs2", dict(N=48, C=64, K=256, H=12, W=12), {"WINRS_FORCE_Z": "3", "WINRS_FORCE_CSPLIT": "2", "WINRS_FORCE_TILE": "128x64"}),
]


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
@pytest.mark.parametrize("name,ov,env", XS, ids=[c[0] for c in XS])
def test_tc2_xs(name, ov, env, dtype, monkeypatch):
    layer = BASE.with_(name="xs_" + name, dtype=dtype, **ov)
    _check(layer, monkeypatch, dict(env, WINRS_TC_GEN="2", WINRS_FORCE_TA="2"), expect_kernel="_v2x_")


# stream-K xi-split pairs (bfc_tc2x.cuh SK): all co-resident pairs split the concatenated tile depths;
# tiles cut between pairs are combined in dW in a fixed chain order
XSK = [
    ("l2", dict(N=16, C=128, K=128, H=28, W=28), {}),
    ("l3", dict(N=16, C=256, K=256, H=14, W=14), {}),
    ("l4_many_tiles", dict(N=16, C=512, K=512, H=7, W=7), {}),
    ("f2", dict(N=16, C=64, K=128, H=20, W=20), {"WINRS_FORCE_TILE": "128x64"}),
    ("ragged", dict(N=16, C=200, K=136, H=13, W=11), {}),
    ("tiny_fewer_chunks_than_pairs", dict(N=16, C=64, K=64, H=4, W=5), {"WINRS_FORCE_TILE": "128x128"}),
    ("pad0_s6", dict(N=16, C=128, K=128, H=16, W=16, S=6, pad=0), {"WINRS_FORCE_PAIR": "4,3,2,0,0,0"}),
    ("r5_f2", dict(N=32, C=64, K=128, H=16, W=16, R=5, S=3, pad=2), {"WINRS_FORCE_TILE": "128x64"}),
    ("vgg_like_long", dict(N=32, C=128, K=256, H=56, W=56), {}),
    # Z > 1: segments' buckets summed by the reduction launch
    ("z4", dict(N=16, C=128, K=128, H=28, W=28), {"WINRS_FORCE_Z": "4"}),
    ("z7_ragged", dict(N=16, C=200, K=136, H=30, W=29), {"WINRS_FORCE_Z": "7"}),
    ("f2_z6", dict(N=32, C=64, K=128, H=24, W=24), {"WINRS_FORCE_TILE": "128x64", "WINRS_FORCE_Z": "6"}),
]


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
@pytest.mark.parametrize("name,ov,env", XSK, ids=[c[0] for c in XSK])
def test_tc2_xsk(name, ov, env, dtype, monkeypatch):
    layer = BASE.with_(name="xsk_" + name, dtype=dtype, **ov)
    _check(layer, monkeypatch, dict(env, WINRS_TC_GEN="2", WINRS_FORCE_TA="3"), expect_kernel="_v2k_")


def test_tc2_xsk_two_streams(monkeypatch):
    """Two stream-K launches in flight on different streams (separate flag / ticket
    regions): both results equal the single-stream ones bit for bit."""
    layer = BASE.with_(name="xsk_streams", N=16, C=256, K=256, H=14, W=14)
    X, dY = wl.make_inputs(layer)
    p = _plan(layer, {"WINRS_TC_GEN": "2", "WINRS_FORCE_TA": "3"}, monkeypatch)
    assert "_v2k_" in p.kernel_name
    Xg, Gg = _dev(X, "f16"), _dev(dY, "f16")
    ref = W.bfc(p, Xg, Gg).clone()
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    torch.cuda.synchronize()
    outs = []
    for _ in range(10):
        a = W.bfc(p, Xg, Gg, stream=s1)
        b = W.bfc(p, Xg, Gg, stream=s2)
        outs += [a, b]
    torch.cuda.synchronize()
    for o in outs:
        assert torch.equal(o, ref)


def test_tc2_xsk_exact_and_repeatable(monkeypatch):
    """Integer inputs: the chained read-add-write of tiles cut between pairs is
    exact; 20 repeated calls are bitwise identical (fixed chain order)."""
    layer = BASE.with_(name="xsk_ints", N=32, C=256, K=256, H=14, W=14)
    g = np.random.Generator(np.random.PCG64(9))
    X = g.integers(0, 3, size=(layer.N, layer.H, layer.W, layer.C)).astype(np.float16)
    dY = g.integers(0, 3, size=(layer.N, layer.Ho, layer.Wo, layer.K)).astype(np.float16)
    p, _ = _check(layer, monkeypatch, {"WINRS_TC_GEN": "2", "WINRS_FORCE_TA": "3"}, X=X, dY=dY, exact=True,
                  expect_kernel="_v2k_")
    Xg, Gg = _dev(X, "f16"), _dev(dY, "f16")
    first = W.bfc(p, Xg, Gg).clone()
    for _ in range(20):
        assert torch.equal(W.bfc(p, Xg, Gg), first)


@pytest.mark.parametrize("name,ov,env", XS[:6], ids=[c[0] for c in XS[:6]])
def test_tc2_xs_signed(name, ov, env, monkeypatch):
    layer = BASE.with_(name="xss_" + name, **ov)
    _check(layer, monkeypatch, dict(env, WINRS_TC_GEN="2", WINRS_FORCE_TA="2"), dist="signed", expect_kernel="_v2x_")


def test_tc2_xs_exact_all_ones(monkeypatch):
    """Small-integer inputs: every product and partial sum is exact in FP32,
    so the xi-split result must equal the oracle bit for bit."""
    layer = BASE.with_(name="xs_ones", N=16, C=128, K=128, H=14, W=14)
    g = np.random.Generator(np.random.PCG64(5))
    X = g.integers(0, 3, size=(layer.N, layer.H, layer.W, layer.C)).astype(np.float16)
    dY = g.integers(0, 3, size=(layer.N, layer.Ho, layer.Wo, layer.K)).astype(np.float16)
    _check(layer, monkeypatch, {"WINRS_TC_GEN": "2", "WINRS_FORCE_TA": "2", "WINRS_FORCE_TILE": "128x128",
                                "WINRS_FORCE_CSPLIT": "2"}, X=X, dY=dY, exact=True, expect_kernel="_v2x_")


@pytest.mark.parametrize("ta,tag", [("2", "_v2x_"), ("3", "_v2k_")])
@pytest.mark.parametrize("shape,env", [
    (dict(N=16, C=64, K=128, H=20, W=20), {}),
    (dict(N=16, C=40, K=72, H=17, W=19), {}),
    (dict(N=32, C=64, K=128, H=24, W=24), {"WINRS_FORCE_Z": "6"}),
], ids=["f2", "f2_ragged", "f2_z6"])
def test_tc2_xs_balanced_f2_exact(ta, tag, shape, env, monkeypatch):
    """F = 2 tiles run the balanced split (xi {0,2} / {1,3}, three MMAs per half):
    small-integer inputs, so the pair sum must equal the oracle bit for bit."""
    layer = BASE.with_(name="xs_bal_ints", **shape)
    g = np.random.Generator(np.random.PCG64(11))
    X = g.integers(0, 3, size=(layer.N, layer.H, layer.W, layer.C)).astype(np.float16)
    dY = g.integers(-2, 3, size=(layer.N, layer.Ho, layer.Wo, layer.K)).astype(np.float16)
    _check(layer, monkeypatch, dict(env, WINRS_TC_GEN="2", WINRS_FORCE_TA=ta, WINRS_FORCE_TILE="128x64"),
           X=X, dY=dY, exact=True, expect_kernel=tag + "128x2fh")


@pytest.mark.parametrize("name,ov,env", TA[:4], ids=[c[0] for c in TA[:4]])
def test_tc2_ta_matches_smem_variant(name, ov, env, monkeypatch):
    """Same plan geometry, Xhat in TMEM vs in shared memory: the same packed
    16-bit IT values and the same MMA depth order, so bitwise identical dW."""
    layer = BASE.with_(name="ta_eq_" + name, **ov)
    X, dY = wl.make_inputs(layer)
    out = []
    for ta in ("0", "1"):
        p = _plan(layer, dict(env, WINRS_TC_GEN="2", WINRS_FORCE_TA=ta), monkeypatch)
        out.append(W.as_krsc(W.bfc(p, _dev(X, "f16"), _dev(dY, "f16"))).cpu().numpy())
    assert np.array_equal(out[0], out[1])


@pytest.mark.parametrize("name,ov,env", TC2[:8], ids=[c[0] for c in TC2[:8]])
def test_tc2_signed(name, ov, env, monkeypatch):
    layer = BASE.with_(name="tc2s_" + name, **ov)
    _check(layer, monkeypatch, dict(env, WINRS_TC_GEN="2"), dist="signed", expect_kernel="_v2")


def test_tc2_default_plans_use_tc2(monkeypatch):
    """The planner's picks for the ResNet-50 / VGG-16 FP16 layers are the
    second-generation kernel (the bench's headline path)."""
    for l in wl.RESNET50_F16 + wl.VGG16_F16:
        p = _plan(l, {}, monkeypatch)
        assert "_v2" in p.kernel_name, (l.name, p.kernel_name)


# ====================================================== bfc_tc3.cuh: FP32 inputs on the tensor cores (3xTF32)
BASE32 = wl.LAYERS["r50_c64_56_f32"]
TC3 = [
    ("l1", dict(N=8), {}),
    ("l1_f2", dict(N=8), {"WINRS_FORCE_TILE": "64x64"}),
    ("l1_f1_cs2", dict(N=8), {"WINRS_FORCE_TILE": "64x128", "WINRS_FORCE_CSPLIT": "2"}),
    ("l3", dict(N=8, C=256, K=256, H=14, W=14), {}),
    ("ragged", dict(N=8, C=72, K=100, H=20, W=17), {}),
    ("ragged_f2_cs3", dict(N=16, C=40, K=136, H=13, W=11), {"WINRS_FORCE_TILE": "64x64", "WINRS_FORCE_CSPLIT": "3"}),
    ("l4_cs5", dict(N=8, C=512, K=512, H=7, W=7), {"WINRS_FORCE_CSPLIT": "5"}),
    ("ragged_cs5", dict(N=8, C=72, K=100, H=20, W=17), {"WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_CSPLIT": "5"}),
    ("pad0", dict(N=8, C=64, K=64, H=20, W=20, pad=0), {}),
    ("r5", dict(N=8, C=64, K=64, H=16, W=16, R=5, S=3, pad=2), {}),
    ("r1", dict(N=8, C=64, K=64, H=12, W=12, R=1, S=3, pad=0), {}),
    ("s6", dict(N=8, C=64, K=64, H=16, W=16, R=3, S=6, pad=2), {"WINRS_FORCE_PAIR": "4,3,2,0,0,0"}),
    ("s9_r9", dict(N=8, C=32, K=64, H=20, W=20, R=9, S=9, pad=4), {}),
    ("z5", dict(N=16, C=64, K=64, H=30, W=30), {"WINRS_FORCE_Z": "5"}),
    ("cs8", dict(N=24, C=128, K=64, H=12, W=12), {"WINRS_FORCE_CSPLIT": "8"}),
    ("cs6_f2", dict(N=16, C=64, K=128, H=12, W=12), {"WINRS_FORCE_CSPLIT": "6", "WINRS_FORCE_TILE": "64x64"}),
    ("nk128", dict(N=8, C=128, K=128, H=14, W=14), {"WINRS_FORCE_TILE": "128x128"}),
    ("nk128_f2_ragged_cs3", dict(N=16, C=40, K=200, H=13, W=11), {"WINRS_FORCE_TILE": "128x64", "WINRS_FORCE_CSPLIT": "3"}),
    ("nk128_z3_cs4", dict(N=16, C=64, K=128, H=30, W=30), {"WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_Z": "3",
                                                          "WINRS_FORCE_CSPLIT": "4"}),
]


@pytest.mark.parametrize("dist", ["u01", "signed"])
@pytest.mark.parametrize("name,ov,env", TC3, ids=[c[0] for c in TC3])
def test_tc3_fp32(name, ov, env, dist, monkeypatch):
    """FP32 gate (1e-4) for the 3xTF32 tensor-core kernel, U[0,1) and signed inputs."""
    layer = BASE32.with_(name="tc3_" + name, **ov)
    _check(layer, monkeypatch, dict(env, WINRS_FP32_TC="1"), dist=dist, expect_kernel="f32tc_")


def test_tc3_exact_all_ones(monkeypatch):
    """X = dY = 1: every transformed operand is a small integer (exact in
    tf32, lo = 0), so the 3xTF32 result is the closed form bit for bit."""
    layer = BASE32.with_(N=8, C=64, K=64, H=18, W=17, name="tc3_ones")
    X = np.ones((layer.N, layer.H, layer.W, layer.C), np.float32)
    dY = np.ones((layer.N, layer.Ho, layer.Wo, layer.K), np.float32)
    _check(layer, monkeypatch, {"WINRS_FP32_TC": "1"}, X=X, dY=dY, exact=True, expect_kernel="f32tc_")


def test_fp32_default_plans_use_tc3(monkeypatch):
    """The planner's picks for the ResNet-50 FP32 layers are the tensor-core kernel."""
    for l in wl.RESNET50_F32:
        p = _plan(l, {}, monkeypatch)
        assert p.kernel_name.startswith("f32tc_"), (l.name, p.kernel_name)


# ====================================================== pad = 0 (pad=0 variants of the wide config)
PAD0 = [(l.with_(N=2, C=40, K=48, H=17, W=19, pad=0, name=l.name + "_pad0")) for l in wl.WIDE_F32] + [
    wl.LAYERS["r50_c64_56_f32"].with_(N=2, H=20, W=23, pad=0, name="r50_l1_pad0"),
    wl.LAYERS["r50_c256_14_f32"].with_(N=2, C=72, K=64, pad=0, name="r50_l3_pad0"),
]


@pytest.mark.parametrize("layer", PAD0, ids=lambda l: l.name)
@pytest.mark.parametrize("dtype", ["f32", "f16"])
def test_pad0(layer, dtype, monkeypatch):
    _check(layer.with_(dtype=dtype), monkeypatch)


def test_pad0_f16_n16_tc2(monkeypatch):
    layer = wl.LAYERS["r50_c64_56_f16"].with_(N=16, H=21, W=22, pad=0, name="r50_l1_pad0_n16")
    _check(layer, monkeypatch)


# ====================================================== FP32 kernels for F_W = 6, 8
FW68 = [
    (6, "8,6,3,0,0,0"),       # Omega_8(6,3)
    (6, "16,6,11,0,0,0"),     # Omega_16(6,11)
    (8, "16,8,9,0,0,0"),      # Omega_16(8,9)
    (8, "8,4,5,4,2,3"),       # Omega_8(4,5) + Omega_4(2,3)
    (8, "8,4,5,0,0,0"),       # Omega_8(4,5)
    (6, "8,6,3,4,3,2"),       # Omega_8(6,3) + Omega_4(3,2)
    (8, "16,8,9,8,4,5"),      # Omega_16(8,9) + Omega_8(4,5)
    (6, None),                # the planner's own choice
    (8, None),
]


@pytest.mark.parametrize("S,pair", FW68, ids=lambda v: str(v))
def test_fp32_fw6_fw8(S, pair, monkeypatch):
    layer = wl.LAYERS["wide_r5_f32"].with_(N=2, C=40, K=36, H=21, W=26, R=S, S=S, pad=S // 2, name=f"f32_w{S}")
    env = {"WINRS_FORCE_PAIR": pair} if pair else {}
    p, _ = _check(layer, monkeypatch, env)
    if pair:
        a = [int(x) for x in pair.split(",")]
        assert (p.info["alpha0"], p.info["n0"], p.info["r0"]) == tuple(a[:3])


# ====================================================== exactness on structured inputs
def _int_inputs(layer, lo=0, hi=8, seed=11):
    g = np.random.Generator(np.random.PCG64(seed))
    X = g.integers(lo, hi, size=(layer.N, layer.H, layer.W, layer.C)).astype(np.float32)
    dY = np.zeros((layer.N, layer.Ho, layer.Wo, layer.K), dtype=np.float32)
    return X, dY


EXACT = [
    ("f32", {"WINRS_FORCE_PAIR": "4,3,2,0,0,0"}),
    ("f16", {"WINRS_TC_GEN": "2"}),
    ("bf16", {"WINRS_TC_GEN": "2"}),
    ("f16", {"WINRS_TC_GEN": "2", "WINRS_FORCE_TA": "1", "WINRS_FORCE_TILE": "64x64"}),
    ("f16", {"WINRS_TC_GEN": "2", "WINRS_FORCE_TA": "2", "WINRS_FORCE_TILE": "128x64"}),
    ("bf16", {"WINRS_TC_GEN": "2", "WINRS_FORCE_TA": "2", "WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_CSPLIT": "2"}),
]


@pytest.mark.parametrize("dtype,env", EXACT, ids=lambda v: str(v))
def test_all_ones_exact(dtype, env, monkeypatch):
    """X = dY = 1: dW[k,r,s,c] = N cnt_H(r) cnt_W(s), integers < 2^24.  With
    the Omega_4(3,2) transforms (coefficients +-1, 1/2, 2) every intermediate
    is exact, so the GPU result equals the closed form bit for bit."""
    layer = wl.LAYERS["r50_c64_56_f16"].with_(N=16, C=64, K=64, H=18, W=17, dtype=dtype, name="ones")
    X = np.ones((layer.N, layer.H, layer.W, layer.C), np.float32)
    dY = np.ones((layer.N, layer.Ho, layer.Wo, layer.K), np.float32)
    _check(layer, monkeypatch, env, X=X.astype(wl.np_dtype(dtype)), dY=dY.astype(wl.np_dtype(dtype)), exact=True)


@pytest.mark.parametrize("dtype,env", EXACT, ids=lambda v: str(v))
def test_impulse_exact(dtype, env, monkeypatch):
    """dY = a few unit impulses, X = small integers: dW[k0] = the padded X
    window at each impulse (layout, correlation, padding), exactly."""
    layer = wl.LAYERS["r50_c64_56_f16"].with_(N=16, C=64, K=64, H=15, W=16, dtype=dtype, name="impulse")
    X, dY = _int_inputs(layer)
    for (n, h, w, k) in [(0, 0, 0, 0), (3, layer.Ho - 1, layer.Wo - 1, 63), (7, 5, 6, 17), (15, 0, layer.Wo - 1, 40)]:
        dY[n, h, w, k] = 1.0
    _check(layer, monkeypatch, env, X=X.astype(wl.np_dtype(dtype)), dY=dY.astype(wl.np_dtype(dtype)), exact=True)


def test_impulse_fp32_alpha8_tolerance(monkeypatch):
    """Omega_8 transforms have non-dyadic coefficients: impulse results are
    within the FP32 gate rather than bit-exact."""
    layer = wl.LAYERS["r50_c64_56_f32"].with_(N=2, H=15, W=16, name="impulse_a8")
    X, dY = _int_inputs(layer)
    dY[1, 3, 4, 5] = 1.0
    _check(layer, monkeypatch, {"WINRS_FORCE_PAIR": "8,3,6,4,3,2"}, X=X, dY=dY)


# ====================================================== reproducibility under repeated cold-L2 calls
@pytest.mark.parametrize("layer_name,env", [
    ("r50_c64_56_f16", {}),                                   # tc2, Z > 1, cluster split
    ("r50_c256_14_f16", {}),                                  # tc2, NK = 128, cs = 8
    ("r50_c512_7_f16", {}),                                   # tc2 swapped cta_group::2 pair, cs = 2
    ("r50_c64_56_f16", {"WINRS_TC_GEN": "1"}),                # round-1 kernel default plan
    ("r50_c128_28_f16", {"WINRS_TC_GEN": "1"}),
])
def test_repeated_calls_bitwise(layer_name, env, monkeypatch):
    """400 cold-L2 calls of the default plan: every dW equals the first one bit
    for bit (determinism for a fixed plan, R16; a ring-protocol race
    would show up as a changed or non-finite dW, or as a hang)."""
    layer = wl.LAYERS[layer_name]
    X, dY = wl.make_inputs(layer)
    p = _plan(layer, env, monkeypatch)
    Xg, Gg = _dev(X, layer.dtype), _dev(dY, layer.dtype)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    ws = torch.empty(max(16, p.workspace_bytes), dtype=torch.uint8, device="cuda")
    first = W.bfc(p, Xg, Gg, workspace=ws).clone()
    out = torch.empty_like(first)
    bad = 0
    for i in range(400):
        flush.fill_(i & 255)
        W.bfc(p, Xg, Gg, out, ws)
        if i % 50 == 49 or i == 399:
            torch.cuda.synchronize()
        bad += int(not torch.equal(out, first))
    assert bad == 0, (p.kernel_name, bad)
    idx = wl.sample_indices(layer, 128)
    ref = O.bfc_c_sampled(X, dY, layer.R, layer.S, layer.pad, idx)
    err = O.rel_max_err(W.as_krsc(first).cpu().numpy().astype(np.float64).ravel()[idx], ref)
    record_err(f"{layer_name} 400 cold-L2 calls bitwise equal {env}", err, p.kernel_name)
    assert err <= TOL[layer.dtype]


# ====================================================== N-D (3-D) BFC (PAPER.md P@17805)
ND = [
    # N, C, D, H, W, K, T, R, S, pad, env
    (1, 64, 16, 10, 11, 64, 3, 3, 3, 1, {}),
    (2, 32, 16, 7, 9, 48, 3, 3, 3, 1, {"WINRS_FORCE_CSPLIT": "2"}),
    (1, 128, 16, 6, 6, 128, 3, 3, 3, 1, {"WINRS_FORCE_TILE": "128x128"}),
    (1, 64, 16, 8, 8, 64, 3, 3, 3, 1, {"WINRS_FORCE_TILE": "128x64"}),          # (t, r) rows stacked per CTA
    (1, 256, 16, 5, 5, 256, 3, 3, 3, 1, {"WINRS_FORCE_TILE": "256x128"}),       # swapped CTA pair
    (1, 40, 17, 9, 8, 24, 2, 2, 3, 1, {"WINRS_FORCE_Z": "3"}),                  # Do = 18 -> padded below
    (2, 16, 18, 6, 6, 16, 3, 1, 3, 0, {}),                                      # pad 0, R = 1
    (1, 64, 16, 10, 11, 64, 3, 3, 3, 1, {"WINRS_FORCE_TA": "0"}),              # Xhat in shared memory
    (2, 64, 16, 7, 9, 64, 3, 3, 3, 1, {"WINRS_FORCE_TA": "1", "WINRS_FORCE_TILE": "64x64"}),   # Xhat in TMEM
    (2, 48, 8, 7, 9, 64, 3, 3, 3, 1, {"WINRS_FP32_TC": "1"}),                 # FP32 on the tensor cores
    (1, 64, 16, 6, 6, 64, 3, 3, 3, 1, {"WINRS_FP32_TC": "0"}),                # FP32 CUDA cores
]


@pytest.mark.parametrize("dtype", ["f16", "bf16", "f32"])
@pytest.mark.parametrize("case", ND, ids=[f"nd{i}" for i in range(len(ND))])
def test_nd_bfc(case, dtype, monkeypatch):
    N, C, D, H, Wd, K, T, R, S, pad, env = case
    Do = D + 2 * pad - T + 1
    if Do % 16:                       # the tc2 N-D path loads 16 depth slices per TMA box
        D += 16 - Do % 16
        Do = D + 2 * pad - T + 1
    for k in ENV_KEYS:
        monkeypatch.delenv(k, raising=False)
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    g = np.random.Generator(np.random.PCG64(1234 + N * 7 + C))
    X = g.random((N, D, H, Wd, C), dtype=np.float32)
    dY = (g.random((N, Do, H + 2 * pad - R + 1, Wd + 2 * pad - S + 1, K), dtype=np.float32) * 1e-2)
    if dtype == "f16":
        X, dY = X.astype(np.float16), dY.astype(np.float16)
    elif dtype == "bf16":
        X, dY = wl.round_to_bf16(X), wl.round_to_bf16(dY)
    elif "WINRS_FORCE_TILE" in env:   # the tensor-core tiles do not exist for FP32
        monkeypatch.delenv("WINRS_FORCE_TILE", raising=False)
    p = W.plan3d(N, C, D, H, Wd, K, T, R, S, pad, dtype)
    dW = W.as_krsc(W.bfc(p, _dev(X, dtype), _dev(dY, dtype)))
    torch.cuda.synchronize()
    got = dW.cpu().numpy().astype(np.float64)
    ref = O.bfc3d_numpy(X.astype(np.float64), dY.astype(np.float64), T, R, S, pad)
    err = O.rel_max_err(got, ref)
    record_err(f"3-D N{N} C{C} D{D} {H}x{Wd} K{K} T{T}R{R}S{S} p{pad} [{dtype}] {env}", err,
               f"{p.kernel_name} Z={p.info['Z']} cs={p.info['csplit']}")
    assert got.shape == (K, T, R, S, C)
    assert err <= TOL[dtype], (p.kernel_name, err)


# ====================================================== cluster-split stress at full size
STRESS = [
    ("vgg_128_128_112_f16", {"WINRS_TC_GEN": "1", "WINRS_FORCE_TILE": "128x64", "WINRS_FORCE_CSPLIT": "4"}),
    ("vgg_128_128_112_f16", {"WINRS_TC_GEN": "1", "WINRS_FORCE_PAIR": "8,3,6,4,3,2", "WINRS_FORCE_TILE": "128x32",
                             "WINRS_FORCE_CSPLIT": "2"}),
    ("vgg_128_128_112_f16", {"WINRS_FORCE_TA": "1", "WINRS_FORCE_CSPLIT": "6"}),
    ("vgg_128_128_112_f16", {"WINRS_FORCE_TA": "0", "WINRS_FORCE_TILE": "128x128", "WINRS_FORCE_CSPLIT": "8"}),
    ("vgg_256_256_56_f16", {"WINRS_FORCE_TILE": "256x128", "WINRS_FORCE_CSPLIT": "3"}),
    ("r50_c512_7_f32", {"WINRS_FORCE_CSPLIT": "6", "WINRS_FP32_TC": "0"}),
    ("r50_c256_14_f32", {"WINRS_FORCE_CSPLIT": "8", "WINRS_FP32_TC": "0"}),
    ("r50_c128_28_f32", {"WINRS_FORCE_CSPLIT": "8", "WINRS_FP32_TC": "1"}),
    ("r50_c64_56_f32", {"WINRS_FORCE_CSPLIT": "3", "WINRS_FP32_TC": "1"}),
]


@pytest.mark.parametrize("layer_name,env", STRESS, ids=[f"{s[0]}-{i}" for i, s in enumerate(STRESS)])
def test_cluster_split_stress(layer_name, env, monkeypatch):
    """40 cold-L2 calls of a full-size layer with a cluster split (a 256 MB
    buffer allocated and rewritten between calls): no launch failure and
    bitwise identical dW (the round-1 FP16 kernel's B_M = 128 tiles failed
    here and are no longer registered; its other tiles keep cs in 1, 2, 4)."""
    layer = wl.LAYERS[layer_name]
    X, dY = wl.make_inputs(layer)
    p = _plan(layer, env, monkeypatch)
    fcs = int(env.get("WINRS_FORCE_CSPLIT", "1"))
    assert p.info["csplit"] == fcs, (p.kernel_name, p.info["csplit"])
    Xg, Gg = _dev(X, layer.dtype), _dev(dY, layer.dtype)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    dW = torch.empty((layer.K, layer.R, layer.S, layer.C), device="cuda")
    ws = torch.empty(max(16, p.workspace_bytes), dtype=torch.uint8, device="cuda")
    first = None
    for i in range(40):
        flush.fill_(i & 0xFF)
        W.bfc(p, Xg, Gg, dW, ws)
        torch.cuda.synchronize()
        if first is None:
            first = dW.clone()
        else:
            assert torch.equal(dW, first), (p.kernel_name, i)
    idx = wl.sample_indices(layer, 64)
    ref = O.bfc_c_sampled(X, dY, layer.R, layer.S, layer.pad, idx)
    err = O.rel_max_err(first.cpu().numpy().astype(np.float64).ravel()[idx], ref)
    record_err(f"{layer_name} 40-call stress {env}", err, f"{p.kernel_name} cs={p.info['csplit']}")
    assert err <= TOL[layer.dtype]


# ====================================================== alpha = 16 with 16-bit inputs
C16 = [
    # layer overrides, forced pair
    (dict(N=8, C=64, K=64, H=20, W=20, R=9, S=9, pad=4), "16,9,8,0,0,0"),
    (dict(N=8, C=40, K=72, H=19, W=23, R=9, S=9, pad=4), "16,9,8,4,3,2"),      # residual Omega_4(3,2), ragged C/K
    (dict(N=8, C=64, K=64, H=20, W=20, R=7, S=7, pad=3), "16,7,10,8,7,2"),
    (dict(N=6, C=32, K=48, H=17, W=19, R=7, S=7, pad=0), "16,7,10,0,0,0"),     # pad 0, N % 16 != 0
]


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
@pytest.mark.parametrize("ov,pair", C16, ids=[f"c16_{i}" for i in range(len(C16))])
def test_alpha16_16bit_inputs(ov, pair, dtype, monkeypatch):
    """Omega_16(9,8) / Omega_16(7,10) (eq. (7)-scaled transforms) on FP16 / BF16
    inputs, gated at 2e-2 (Appendix B's FP16 check); both the U[0,1) protocol
    and signed inputs."""
    layer = wl.LAYERS["r50_c64_56_f16"].with_(name="c16", dtype=dtype, **ov)
    p, err = _check(layer, monkeypatch, {"WINRS_FORCE_PAIR": pair}, expect_kernel="cc_O16")
    _check(layer, monkeypatch, {"WINRS_FORCE_PAIR": pair}, dist="signed", expect_kernel="cc_O16")
