"""Seeded synthetic BFC workloads shared by the tests, the bench and smoke().

This module holds NO arithmetic of the method: only layer shapes (the paper's
workload structure, §6 P@40608: C = K, channels doubled when the map
is halved, square maps, pad = floor(R/2)) and seeded random inputs (the
paper's accuracy protocol, P@50685: uniform [0,1] tensors, dY x 1e-2 for
FP16).  Both the oracle side and the CUDA side consume its arrays.
"""
from __future__ import annotations

from dataclasses import dataclass, asdict

import numpy as np


@dataclass(frozen=True)
class Layer:
    name: str
    N: int
    C: int
    H: int
    W: int
    K: int
    R: int
    S: int
    pad: int
    dtype: str          # "f32", "f16" or "bf16": dtype of X and dY (dW is always f32)
    index: int          # stable config index: seeds are 1000003+index / 2000003+index

    @property
    def Ho(self) -> int:
        return self.H + 2 * self.pad - self.R + 1

    @property
    def Wo(self) -> int:
        return self.W + 2 * self.pad - self.S + 1

    @property
    def direct_flops(self) -> int:
        """2*N*C*K*Ho*Wo*R*S: the paper's throughput numerator (P@43462)."""
        return 2 * self.N * self.C * self.K * self.Ho * self.Wo * self.R * self.S

    def with_(self, **kw) -> "Layer":
        d = asdict(self)
        d.update(kw)
        return Layer(**d)


def _mk():
    out = {}
    idx = 0

    def add(name, N, C, H, W, K, R, S, pad, dtype):
        nonlocal idx
        out[name] = Layer(name, N, C, H, W, K, R, S, pad, dtype, idx)
        idx += 1

    # configs[0]: tiny
    add("tiny_f32", 1, 4, 8, 8, 4, 3, 3, 1, "f32")
    # configs[1]: ResNet-50 3x3 layers, N=64, FP32 and FP16
    for dt in ("f32", "f16"):
        for c, hw in ((64, 56), (128, 28), (256, 14), (512, 7)):
            add(f"r50_c{c}_{hw}_{dt}", 64, c, hw, hw, c, 3, 3, 1, dt)
    # configs[2]: VGG-16 3x3 layers 2-13 (unique shapes), N=128, FP16
    for cin, cout, hw in ((64, 64, 224), (64, 128, 112), (128, 128, 112), (128, 256, 56),
                          (256, 256, 56), (256, 512, 28), (512, 512, 28), (512, 512, 14)):
        add(f"vgg_{cin}_{cout}_{hw}_f16", 128, cin, hw, hw, cout, 3, 3, 1, "f16")
    # configs[3]: wide dW widths, N=32, C=K=128, 32x32, R=S in {2,4,5,7,9}, FP32
    for rs in (2, 4, 5, 7, 9):
        add(f"wide_r{rs}_f32", 32, 128, 32, 32, 128, rs, rs, rs // 2, "f32")
    # configs[4]: ResNet-50 layer3 at N=512 (batch-sharded across GPUs), FP16
    add("r50_l3_n512_f16", 512, 256, 14, 14, 256, 3, 3, 1, "f16")
    return out


LAYERS = _mk()
RESNET50_F32 = [LAYERS[f"r50_c{c}_{hw}_f32"] for c, hw in ((64, 56), (128, 28), (256, 14), (512, 7))]
RESNET50_F16 = [LAYERS[f"r50_c{c}_{hw}_f16"] for c, hw in ((64, 56), (128, 28), (256, 14), (512, 7))]
VGG16_F16 = [l for n, l in LAYERS.items() if n.startswith("vgg_")]
WIDE_F32 = [l for n, l in LAYERS.items() if n.startswith("wide_")]


def np_dtype(dtype: str):
    """numpy storage dtype of the inputs (bf16 values are carried in float32)."""
    return {"f32": np.float32, "f16": np.float16, "bf16": np.float32}[dtype]


def round_to_bf16(x: np.ndarray) -> np.ndarray:
    """float32 -> nearest bfloat16 value (round to nearest even), kept in float32."""
    b = np.ascontiguousarray(x, dtype=np.float32).view(np.uint32)
    b = (b + np.uint32(0x7FFF) + ((b >> np.uint32(16)) & np.uint32(1))) & np.uint32(0xFFFF0000)
    return b.view(np.float32)


def make_inputs(layer: Layer, dist: str = "u01", seed_offset: int = 0):
    """Seeded X [N,H,W,C] and dY [N,Ho,Wo,K] (NHWC) in the layer's dtype.

    dist: "u01"    U[0,1) for both (the paper's protocol); dY x 1e-2 for f16.
          "signed" U[-1,1) for both (dY x 1e-2 for f16).
    Values are drawn in float32 from PCG64 and rounded (RN) to the dtype.
    """
    gx = np.random.Generator(np.random.PCG64(1000003 + layer.index + seed_offset))
    gy = np.random.Generator(np.random.PCG64(2000003 + layer.index + seed_offset))
    X = gx.random((layer.N, layer.H, layer.W, layer.C), dtype=np.float32)
    dY = gy.random((layer.N, layer.Ho, layer.Wo, layer.K), dtype=np.float32)
    if dist == "signed":
        X = X * 2 - 1
        dY = dY * 2 - 1
    elif dist != "u01":
        raise ValueError(dist)
    if layer.dtype in ("f16", "bf16"):
        dY = dY * np.float32(1e-2)
    if layer.dtype == "bf16":
        return round_to_bf16(X), round_to_bf16(dY)
    dt = np_dtype(layer.dtype)
    return X.astype(dt), dY.astype(dt)


def sample_indices(layer: Layer, count: int, seed: int = 7) -> np.ndarray:
    """Flat KRSC indices to check at full size: every corner/edge tap of the
    filter plus random interior positions (seeded)."""
    K, R, S, C = layer.K, layer.R, layer.S, layer.C
    total = K * R * S * C
    g = np.random.Generator(np.random.PCG64(seed + layer.index))
    fixed = []
    for k in (0, K - 1):
        for r in range(R):
            for s in range(S):
                for c in (0, C - 1):
                    fixed.append(((k * R + r) * S + s) * C + c)
    rnd = g.integers(0, total, size=max(0, count - len(fixed)))
    return np.unique(np.concatenate([np.array(fixed, dtype=np.int64), rnd.astype(np.int64)]))


# ---------------------------------------------------------------- N-D (3-D) layers
# SURVEY §8(f) row 4 (PAPER.md P@17805, Level-2 dimension reduction): C3D-style
# 3x3x3 layers, channels doubled when the map is halved (the paper's workload
# structure), 16 depth slices, pad 1.  (name, N, C, D, H, W, K, T, R, S, pad)
ND_LAYERS = [
    ("c3d_128_28_f16", 8, 128, 16, 28, 28, 128, 3, 3, 3, 1),
    ("c3d_256_14_f16", 8, 256, 16, 14, 14, 256, 3, 3, 3, 1),
]


def make_inputs_nd(shape, dtype: str = "f16", seed: int = 0):
    """Seeded X [N,D,H,W,C] and dY [N,Do,Ho,Wo,K] for an N-D layer tuple of
    ND_LAYERS: U[0,1) (dY x 1e-2 for 16-bit dtypes), rounded to the dtype."""
    _, N, C, D, H, W, K, T, R, S, pad = shape
    Do, Ho, Wo = D + 2 * pad - T + 1, H + 2 * pad - R + 1, W + 2 * pad - S + 1
    gx = np.random.Generator(np.random.PCG64(3000017 + seed))
    gy = np.random.Generator(np.random.PCG64(4000037 + seed))
    X = gx.random((N, D, H, W, C), dtype=np.float32)
    dY = gy.random((N, Do, Ho, Wo, K), dtype=np.float32)
    if dtype in ("f16", "bf16"):
        dY = dY * np.float32(1e-2)
    if dtype == "bf16":
        return round_to_bf16(X), round_to_bf16(dY)
    dt = np_dtype(dtype)
    return X.astype(dt), dY.astype(dt)
