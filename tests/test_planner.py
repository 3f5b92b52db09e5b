"""Host-only tests of the planner (§4: kernel-pair selection §4.1
P@20377, Algorithm 1 §4.2, Algorithm 2 §4.3) through winrs_plan_for_device,
and of the C ABI surface (include/*.h)."""
import os
import re

import numpy as np
import pytest

import paper_conf_icpp_zhangc0zx0025_b200 as W
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
from paper_conf_icpp_zhangc0zx0025_b200._lib import WinrsError
from oracle import oracle as O

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_library_exports_every_declared_symbol():
    import ctypes
    L = ctypes.CDLL(os.path.join(ROOT, "paper_conf_icpp_zhangc0zx0025_b200", "libwinrs.so"))
    names = []
    for h in ("winrs.h", "winrs_debug.h"):
        src = open(os.path.join(ROOT, "include", h)).read()
        names += re.findall(r"WINRS_API\s+[\w\s\*]+?\b(winrs_\w+)\s*\(", src)
    assert len(names) >= 15
    for n in names:
        assert hasattr(L, n), n
    from paper_conf_icpp_zhangc0zx0025_b200._lib import SYMBOLS
    assert sorted(names) == sorted(s[0] for s in SYMBOLS)


def test_figure5_pair():
    """Golden: F_W=3, O_W=16 -> Omega_8(3,6) on 12 columns + Omega_4(3,2) on 4 (P@21094)."""
    for line in open(os.path.join(ROOT, "tests", "golden", "figure5_pairs.txt")):
        if line.startswith("#") or not line.strip():
            continue
        FW, OW, a0, n0, r0, k0, a1, n1, r1, k1 = map(int, line.split())
        # O_W = 16 with F_W = 3 and pad 1 -> W = 16
        p = W.plan_for_device(8, 64, OW, OW, 64, FW, FW, 1, "f32")
        i = p.info
        assert (i["alpha0"], i["n0"], i["r0"], i["k0"]) == (a0, n0, r0, k0)
        assert (i["alpha1"], i["n1"], i["r1"], i["k1"]) == (a1, n1, r1, k1)
        assert i["masked_cols"] == 0


@pytest.mark.parametrize("S,Wo,expect", [
    (3, 56, (8, 3, 6, 9, 4, 3, 2, 1, 0)),      # 56 = 9*6 + 2
    (3, 7, (8, 3, 6, 1, 4, 3, 2, 1, 1)),       # 7 = 6 + 2 - 1 masked (R6)
    (3, 14, (8, 3, 6, 2, 4, 3, 2, 1, 0)),
    (3, 28, (8, 3, 6, 4, 4, 3, 2, 2, 0)),
    (5, 32, (16, 5, 12, 2, 8, 5, 4, 2, 0)),    # SURVEY R7 example
    (7, 32, (16, 7, 10, 3, 8, 7, 2, 1, 0)),
    (9, 32, (16, 9, 8, 4, 0, 0, 0, 0, 0)),
    (2, 33, (4, 2, 3, 11, 0, 0, 0, 0, 0)),
    (4, 33, (8, 4, 5, 6, 4, 2, 3, 1, 0)),
])
def test_pair_selection(S, Wo, expect, monkeypatch):
    # the paper's step 1 (alpha-count cost); the default planner also scores
    # every valid pair with the B200 time model (R19)
    monkeypatch.setenv("WINRS_PLANNER", "paper")
    pad = S // 2
    Wd = Wo - 2 * pad + S - 1
    p = W.plan_for_device(4, 32, 8, Wd, 32, S, S, pad, "f32")
    i = p.info
    assert i["Wo"] == Wo
    got = (i["alpha0"], i["n0"], i["r0"], i["k0"], i["alpha1"], i["n1"], i["r1"], i["k1"], i["masked_cols"])
    assert got == expect


SHAPES = [(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype) for l in wl.LAYERS.values() if l.dtype == "f32"] + [
    (3, 8, 17, 23, 12, 3, 3, 1, "f32"), (2, 4, 9, 40, 8, 5, 5, 0, "f32"), (1, 4, 30, 30, 4, 6, 6, 3, "f32"),
    (2, 12, 11, 19, 16, 8, 8, 2, "f32"), (2, 4, 5, 5, 4, 2, 2, 0, "f32"), (1, 4, 3, 3, 4, 3, 3, 0, "f32"),
]


@pytest.mark.parametrize("shape", SHAPES)
def test_plan_invariants(shape):
    N, C, H, Wd, K, R, S, pad, dt = shape
    p = W.plan_for_device(N, C, H, Wd, K, R, S, pad, dt)
    i = p.info
    Ho, Wo = H + 2 * pad - R + 1, Wd + 2 * pad - S + 1
    assert (i["Ho"], i["Wo"]) == (Ho, Wo)
    # (1) n0, n1 divide F_W
    assert S % i["n0"] == 0 and (i["alpha1"] == 0 or S % i["n1"] == 0)
    assert i["alpha0"] == i["n0"] + i["r0"] - 1
    # (2) units cover O_W; masked columns only inside the last unit
    cover = i["k0"] * i["r0"] + i["k1"] * i["r1"]
    assert cover - Wo == i["masked_cols"] >= 0
    last_r = i["r1"] if i["k1"] else i["r0"]
    assert i["masked_cols"] < last_r
    # segments tile the Omega_a0 region: widths are multiples of r0
    assert i["seg_w"] % i["r0"] == 0
    assert i["seg_cols"] == -(-(i["k0"] * i["r0"]) // i["seg_w"])
    assert 1 <= i["seg_h"] <= Ho and i["bands"] == max(1, Ho // i["seg_h"])
    assert i["Z"] == i["bands"] * i["seg_cols"]
    # workspace = (Z-1)|dW| fp32 and <= 4% of the data bytes (R11)
    dw = K * R * S * C
    assert i["workspace_bytes"] == (i["Z"] - 1) * 4 * dw
    esz = 4 if dt == "f32" else 2
    data = esz * (N * H * Wd * C + N * Ho * Wo * K)
    assert i["workspace_bytes"] <= 0.04 * data + 1e-9
    # Winograd work never exceeds direct work for alpha >= 4 kernels
    assert i["ewm_flops"] > 0
    # determinism
    q = W.plan_for_device(N, C, H, Wd, K, R, S, pad, dt)
    assert q.info == i and q.kernel_name == p.kernel_name


def test_error_codes():
    with pytest.raises(WinrsError) as e:
        W.plan_for_device(0, 4, 8, 8, 4, 3, 3, 1)
    assert e.value.status == 1
    with pytest.raises(WinrsError) as e:
        W.plan_for_device(1, 4, 2, 2, 4, 5, 5, 0)           # Ho < 1
    assert e.value.status == 1
    with pytest.raises(WinrsError) as e:
        W.plan_for_device(1, 4, 8, 8, 4, 3, 3, -1)
    assert e.value.status == 1
    for S in (1, 11, 13):                                     # no kernel width divides S (P@28451)
        with pytest.raises(WinrsError) as e:
            W.plan_for_device(1, 4, 16, 16, 4, 3, S, 0)
        assert e.value.status == 2
    with pytest.raises(WinrsError) as e:
        W.plan_for_device(1, 6, 8, 8, 4, 3, 3, 1)             # C % 4 != 0
    assert e.value.status == 2
    with pytest.raises(WinrsError) as e:
        W.plan_for_device(1, 4, 8, 8, 4, 3, 3, 1, cc=(9, 0))  # not sm_100
    assert e.value.status == 2


def test_supported_widths():
    """F_W in {n*k : 2 <= k <= 9} (P@28451): every S with a divisor in 2..9 plans."""
    for S in range(2, 40):
        ok = any(S % n == 0 for n in range(2, 10))
        try:
            W.plan_for_device(1, 4, S + 4, S + 4, 4, 2, S, 0)
            assert ok, S
        except WinrsError as e:
            assert not ok and e.status == 2, S


def test_forced_overrides(monkeypatch):
    monkeypatch.setenv("WINRS_FORCE_Z", "6")
    monkeypatch.setenv("WINRS_FORCE_TILE", "32x32")
    p = W.plan_for_device(8, 64, 56, 56, 64, 3, 3, 1, "f32")
    assert p.info["tile_k0"] == 32 and p.info["Z"] >= 2
    monkeypatch.setenv("WINRS_FORCE_PAIR", "8,3,6,0,0,0")
    p = W.plan_for_device(8, 64, 56, 56, 64, 3, 3, 1, "f32")
    assert p.info["alpha1"] == 0 and p.info["k0"] == 10 and p.info["masked_cols"] == 4


def test_strided_entry_validates_ldy():
    """winrs_bfc_strided rejects ldy < K or misaligned ldy before any launch."""
    from paper_conf_icpp_zhangc0zx0025_b200 import _lib
    p = W.plan_for_device(2, 16, 8, 8, 16, 3, 3, 1, "f32")
    L = _lib.lib()
    fake = 1 << 20   # 16-byte aligned dummy addresses: rejected before use
    assert L.winrs_bfc_strided(p.handle, fake, fake, 8, fake, None, None) == 1     # ldy < K
    assert L.winrs_bfc_strided(p.handle, fake, fake, 18, fake, None, None) == 1    # ldy % 4
    p16 = W.plan_for_device(2, 16, 8, 8, 16, 3, 3, 1, "f16")
    assert L.winrs_bfc_strided(p16.handle, fake, fake, 20, fake, None, None) == 1  # ldy % 8


# --- R19: the B200 search vs the printed rules ---------------------------------
BENCH_LAYERS = wl.RESNET50_F32 + wl.RESNET50_F16 + wl.WIDE_F32 + wl.VGG16_F16


def _plan(l):
    return W.plan_for_device(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)


@pytest.mark.parametrize("l", BENCH_LAYERS, ids=lambda l: l.name)
def test_search_never_worse_than_paper_rules(l, monkeypatch):
    """The default plan minimises the model over a candidate set that contains
    the printed rules' plan, so its model time can only be lower or equal."""
    d = _plan(l)
    monkeypatch.setenv("WINRS_PLANNER", "paper")
    pp = _plan(l)
    assert 0 < d.model_us <= pp.model_us * (1 + 1e-9)
    # the printed rules: Z never exceeds Algorithm 1's (capped) Z^
    assert pp.info["Z"] <= max(pp.info["z_hat"], 1) * 2


@pytest.mark.parametrize("l", BENCH_LAYERS, ids=lambda l: l.name)
def test_search_plan_is_valid(l):
    """Whatever the model picks obeys the paper's hard constraints: criteria
    (1)-(2) for the pair, n1 | n0, and the 4% workspace cap (R11)."""
    i = _plan(l).info
    assert l.S % i["n0"] == 0
    if i["alpha1"]:
        assert l.S % i["n1"] == 0 and i["n0"] % i["n1"] == 0
    assert i["k0"] * i["r0"] + i["k1"] * i["r1"] - i["masked_cols"] == i["Wo"]
    assert 0 <= i["masked_cols"] < max(i["r0"], i["r1"] or 1)
    esz = 4 if l.dtype == "f32" else 2
    data = esz * (l.N * l.H * l.W * l.C + l.N * i["Ho"] * i["Wo"] * l.K)
    # R11: (Z - 1) buckets of |dW| <= floor(0.04 data / |dW|) buckets, i.e. <= 4 % of X + dY exactly
    assert i["workspace_bytes"] <= 0.04 * data
    assert i["csplit"] in (1, 2, 3, 4, 5, 6, 8)   # 7 ranks: forced only


# ============================================================== N-D (3-D) plans
def test_plan3d_rules():
    """winrs_plan3d: FP16 / BF16 plans on the second-generation kernel, FP32 on
    an FP32 kernel (tensor-core 3xTF32 when Do % 8 == 0, else CUDA-core); FP16
    with Do % 16 != 0 is UNSUPPORTED; bad shapes INVALID_ARG."""
    p = W.plan3d_for_device(2, 64, 16, 12, 12, 64, 3, 3, 3, 1, "f16")
    i = p.info
    assert (i["D"], i["T"], i["Do"]) == (16, 3, 16) and "_v2" in p.kernel_name
    assert i["direct_flops"] == 2.0 * 2 * 16 * 64 * 64 * 12 * 12 * 27
    assert W.plan3d_for_device(2, 64, 16, 12, 12, 64, 3, 3, 3, 1, "f32").kernel_name.startswith("f32")
    assert W.plan3d_for_device(2, 64, 11, 12, 12, 64, 3, 3, 3, 1, "f32").kernel_name.startswith("f32_")   # Do = 11
    with pytest.raises(WinrsError, match="UNSUPPORTED"):
        W.plan3d_for_device(2, 64, 10, 12, 12, 64, 3, 3, 3, 1, "f16")   # Do = 10
    with pytest.raises(WinrsError, match="INVALID_ARG"):
        W.plan3d_for_device(2, 64, 1, 12, 12, 64, 5, 3, 3, 1, "f16")    # Do < 1


@pytest.mark.parametrize("shape,env", [
    ((1, 16, 16, 6, 7, 24, 3, 3, 3, 1), {}),
    ((2, 8, 16, 5, 6, 16, 2, 2, 3, 1), {}),                       # Do = 17 -> rejected below; see D
    ((1, 24, 16, 5, 5, 8, 3, 3, 3, 1), {"WINRS_FORCE_CSPLIT": "2", "WINRS_FORCE_Z": "2"}),
    ((1, 16, 16, 5, 5, 16, 3, 3, 3, 1), {"WINRS_FORCE_TILE": "128x64"}),   # two (t, r) rows stacked per CTA
], ids=["t3", "t2", "split", "stacked"])
def test_plan3d_decomposition_emulated(shape, env, monkeypatch):
    """FP64 emulation of an N-D plan's decomposition (the T*R filter rows with
    their depth taps, N*Do images, clipping, segments, buckets, cluster ranks)
    equals the 3-D oracle."""
    N, C, D, H, Wd, K, T, R, S, pad = shape
    for k_, v_ in env.items():
        monkeypatch.setenv(k_, v_)
    Do = D + 2 * pad - T + 1
    if Do % 16:
        D += 16 - Do % 16
        Do = D + 2 * pad - T + 1
    p = W.plan3d_for_device(N, C, D, H, Wd, K, T, R, S, pad, "f16")
    g = np.random.Generator(np.random.PCG64(5))
    X = g.uniform(-1, 1, (N, D, H, Wd, C))
    dY = g.uniform(-1, 1, (N, Do, H + 2 * pad - R + 1, Wd + 2 * pad - S + 1, K))
    got = W.emulate(p, X, dY)
    ref = O.bfc3d_numpy(X, dY, T, R, S, pad)
    assert np.allclose(got, ref, rtol=1e-11, atol=1e-11), (p, np.max(np.abs(got - ref)))
    monkeypatch.delenv("WINRS_FORCE_TILE", raising=False)              # (tensor-core tile names)
    p32 = W.plan3d_for_device(N, C, D, H, Wd, K, T, R, S, pad, "f32")    # FP32 kernel decomposition
    got32 = W.emulate(p32, X, dY)
    assert np.allclose(got32, ref, rtol=1e-11, atol=1e-11), (p32, np.max(np.abs(got32 - ref)))


def test_bfc_allreduce_validates_arguments():
    """winrs_bfc_allreduce rejects a bad rank / world /
    epoch, null peers and peer_dW[rank] != dW before any launch (no GPU needed)."""
    import ctypes
    from paper_conf_icpp_zhangc0zx0025_b200 import _lib
    L = _lib.lib()
    p = W.plan_for_device(2, 16, 8, 8, 16, 3, 3, 1, "f32")
    fake = 1 << 20
    arr = ctypes.c_void_p * 2
    st, dw, fl = arr(fake, fake + 4096), arr(fake + 8192, fake + 12288), arr(fake + 16384, fake + 16512)
    call = lambda rank, world, epoch, dW=fake + 8192: L.winrs_bfc_allreduce(
        p.handle, fake, fake, dW, None, st, dw, fl, rank, world, epoch, None)
    assert call(0, 9, 1) == 1          # world > 8
    assert call(2, 2, 1) == 1          # rank >= world
    assert call(0, 2, 0) == 1          # epoch 0 would pass the flags immediately
    assert call(1, 2, 1) == 1          # peer_dW[rank] != dW
    assert L.winrs_bfc_allreduce(p.handle, fake, fake, fake, None, None, dw, fl, 0, 2, 1, None) == 1
    assert L.winrs_allreduce_flag_bytes() >= 4 * (2 * 8 + 1)


def test_xi_split_pair_picks_follow_the_measurements():
    """The xi-split pair wins only on the long VGG-16 layers
    with enough tiles (conv2_2: 454 vs 480 us, tools/ab_xs.sh); on ResNet-50 it
    measured slower, and 7-rank clusters are never picked."""
    from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
    for l in wl.RESNET50_F16 + wl.VGG16_F16:
        p = W.plan_for_device(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
        if l.name.startswith("r50"):
            assert "_v2x_" not in p.kernel_name, (l.name, p.kernel_name)
        assert p.info["csplit"] != 7, (l.name, p)   # 7-rank clusters: forced only
    l = wl.LAYERS["vgg_128_128_112_f16"]
    assert "_v2x_" in W.plan_for_device(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype).kernel_name


def test_five_rank_cluster_split_for_tensor_core_kernels_only(monkeypatch):
    """cs = 5 (three 5-CTA clusters per GPC) is searched for the tc2 / tc3
    kernels; the round-1 / CUDA-core kernels never run 5 or 7 ranks."""
    from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
    l = wl.LAYERS["r50_c256_14_f16"]
    p = W.plan_for_device(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
    assert p.info["csplit"] == 5 and "_v2t_" in p.kernel_name, p   # measured 31.7 vs 34.8 us at cs = 4
    monkeypatch.setenv("WINRS_FORCE_CSPLIT", "5")
    q = W.plan_for_device(2, 36, 13, 11, 40, 3, 3, 1, "f32")        # N % 8 != 0: FP32 CUDA-core kernel
    assert q.kernel_name.startswith("f32_") and q.info["csplit"] != 5, q
