"""GPU parity of FC and BDC (winrs_fc / winrs_bdc through the C ABI) against
the FP64 oracle definitions (oracle.fc_numpy / bdc_numpy), SURVEY §8(f) row 3.
Gate as for the BFC (BASELINE.json north_star): max|err| <= 1e-4 * max|ref|
for FP32 inputs, 2e-2 * max|ref| for 16-bit inputs; U[0,1] inputs."""
import numpy as np
import pytest
import torch

import paper_conf_icpp_zhangc0zx0025_b200 as W
from oracle import oracle as O
from conftest import record_err

pytestmark = pytest.mark.gpu

TOL = {"f32": 1e-4, "f16": 2e-2, "bf16": 2e-2}
TDT = {"f32": torch.float32, "f16": torch.float16, "bf16": torch.bfloat16}

CASES = [
    # kind, dtype, (N, C, H, W, K, R, S, pad)
    ("fc", "f32", (4, 8, 10, 12, 8, 3, 3, 1)),
    ("fc", "f32", (8, 36, 14, 14, 44, 3, 3, 1)),      # ragged channel tiles
    ("fc", "f32", (4, 12, 9, 9, 20, 5, 5, 2)),
    ("fc", "f32", (8, 16, 12, 13, 8, 2, 2, 0)),
    ("fc", "f16", (16, 32, 12, 12, 48, 3, 3, 1)),     # tensor-core kernel (3 | Wo, C % 16)
    ("fc", "f16", (24, 64, 14, 14, 64, 3, 3, 1)),     # first-generation FP16 pair (Wo = 14)
    ("fc", "bf16", (16, 32, 12, 15, 40, 3, 3, 1)),
    ("bdc", "f32", (4, 8, 10, 12, 8, 3, 3, 1)),
    ("bdc", "f32", (8, 40, 14, 14, 36, 3, 3, 1)),
    ("bdc", "f32", (4, 8, 6, 10, 12, 3, 3, 0)),
    ("bdc", "f16", (16, 48, 12, 12, 32, 3, 3, 1)),
    ("bdc", "f16", (32, 64, 14, 14, 64, 3, 3, 1)),
    ("bdc", "bf16", (8, 16, 8, 9, 32, 3, 3, 2)),
    # a ResNet-50 layer-3 shape at batch 32 (the FC batch is the BFC's channel axis)
    ("fc", "f16", (32, 256, 14, 14, 256, 3, 3, 1)),
    ("bdc", "f16", (32, 256, 14, 14, 256, 3, 3, 1)),
]


def _inputs(kind, shape, seed=3):
    N, C, H, Wd, K, R, S, pad = shape
    Ho, Wo = O.out_dims(H, Wd, R, S, pad)
    rng = np.random.default_rng(seed)
    Wt = rng.random((K, R, S, C))
    inp = rng.random((N, H, Wd, C) if kind == "fc" else (N, Ho, Wo, K))
    return inp, Wt


def _round(a, dtype):
    return torch.from_numpy(a).to(TDT[dtype]).to(torch.float64).numpy()


@pytest.mark.parametrize("kind,dtype,shape", CASES, ids=lambda c: str(c))
def test_conv_parity(kind, dtype, shape):
    N, C, H, Wd, K, R, S, pad = shape
    inp, Wt = _inputs(kind, shape)
    inp, Wt = _round(inp, dtype), _round(Wt, dtype)      # both sides see the same representable inputs
    cp = W.conv_plan(kind, *shape, dtype=dtype)
    gi = torch.from_numpy(inp).to(TDT[dtype]).cuda()
    gw = torch.from_numpy(Wt).to(TDT[dtype]).cuda()
    out = (W.fc if kind == "fc" else W.bdc)(cp, gi, gw)
    torch.cuda.synchronize()
    got = out.cpu().numpy().astype(np.float64)
    ref = O.fc_numpy(inp, Wt, pad) if kind == "fc" else O.bdc_numpy(inp, Wt, pad, H, Wd)
    err = O.rel_max_err(got, ref)
    record_err(f"{kind}{shape}[{dtype}]", err, cp.kernel_name)
    assert err <= TOL[dtype], (kind, shape, cp.kernel_name, err)


def test_conv_side_stream_and_repeat():
    """Run on a side stream, twice: identical results (the mapped BFC is
    deterministic) and nothing recycled early."""
    shape = (16, 32, 12, 12, 48, 3, 3, 1)
    inp, Wt = _inputs("fc", shape)
    cp = W.conv_plan("fc", *shape, dtype="f16")
    gi = torch.from_numpy(inp).half().cuda()
    gw = torch.from_numpy(Wt).half().cuda()
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    a = W.fc(cp, gi, gw, stream=s)
    b = W.fc(cp, gi, gw, stream=s)
    torch.cuda.current_stream().wait_stream(s)
    torch.cuda.synchronize()
    assert torch.equal(a, b)


def test_conv_wrong_kind_rejected():
    cp = W.conv_plan("fc", 4, 8, 10, 12, 8, 3, 3, 1, dtype="f32")
    with pytest.raises(AssertionError):
        W.bdc(cp, torch.zeros(4, 10, 12, 8, device="cuda"), torch.zeros(8, 3, 3, 8, device="cuda"))
