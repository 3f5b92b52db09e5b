"""FC and BDC on the BFC machinery (include/winrs.h
winrs_conv_*): host-side checks, no GPU.  The operand mapping of the C library
(FC -> BFC of the transposed problem, BDC -> FC of the flipped filter) is
emulated through winrs_debug_emulate of the mapped BFC plan and compared with
the oracle's plain FC / BDC definitions (pinned to torch in test_oracle.py)."""
import numpy as np
import pytest

import paper_conf_icpp_zhangc0zx0025_b200 as W
from paper_conf_icpp_zhangc0zx0025_b200._lib import WinrsError
from oracle import oracle as O

CASES = [
    # kind, dtype, (N, C, H, W, K, R, S, pad)
    ("fc", "f32", (4, 8, 10, 12, 8, 3, 3, 1)),
    ("fc", "f32", (8, 4, 7, 8, 4, 2, 3, 0)),
    ("fc", "f32", (4, 12, 9, 9, 20, 5, 5, 2)),
    ("fc", "f16", (16, 16, 9, 12, 16, 3, 3, 1)),     # mapped onto the tensor-core kernel (C % 16, 3 | Wo)
    ("fc", "f16", (8, 24, 7, 14, 16, 3, 3, 1)),      # Wo = 14: a first-generation FP16 pair
    ("bdc", "f32", (4, 8, 10, 12, 8, 3, 3, 1)),
    ("bdc", "f32", (4, 8, 6, 10, 12, 3, 3, 0)),
    ("bdc", "f16", (8, 16, 9, 12, 16, 3, 3, 1)),
    ("bdc", "bf16", (8, 16, 8, 9, 32, 3, 3, 2)),
]


@pytest.mark.parametrize("kind,dtype,shape", CASES, ids=lambda c: str(c))
def test_conv_mapping_emulated(kind, dtype, shape):
    N, C, H, Wd, K, R, S, pad = shape
    cp = W.conv_plan_for_device(kind, *shape, dtype=dtype)
    Ho, Wo = O.out_dims(H, Wd, R, S, pad)
    rng = np.random.default_rng(7)
    Wt = rng.standard_normal((K, R, S, C))
    if kind == "fc":
        X = rng.standard_normal((N, H, Wd, C))
        ref, got = O.fc_numpy(X, Wt, pad), W.emulate_conv(cp, X, Wt)
    else:
        dY = rng.standard_normal((N, Ho, Wo, K))
        ref, got = O.bdc_numpy(dY, Wt, pad, H, Wd), W.emulate_conv(cp, dY, Wt)
    assert got.shape == ref.shape
    assert np.abs(got - ref).max() <= 1e-12 * max(1.0, np.abs(ref).max())
    # the mapped BFC problem (include/winrs.h): N' = C (FC) / K (BDC), C' = N
    i = cp.bfc.info
    if kind == "fc":
        assert (i["N"], i["C"], i["K"], i["R"], i["S"], i["Ho"], i["Wo"]) == (C, N, K, Ho, Wo, R, S)
    else:
        assert (i["N"], i["C"], i["K"], i["R"], i["S"], i["pad"]) == (K, N, C, H, Wd, R - 1 - pad)
    assert cp.workspace_bytes > 0 and cp.launch_count == 3 + cp.bfc.launch_count


def test_conv_plan_errors():
    with pytest.raises(WinrsError):            # BDC needs one symmetric pad for the flipped filter
        W.conv_plan_for_device("bdc", 4, 8, 10, 12, 8, 3, 5, 1, "f32")
    with pytest.raises(WinrsError):            # pad > R - 1: the flipped pad would be negative
        W.conv_plan_for_device("bdc", 4, 8, 10, 12, 8, 3, 3, 3, "f32")
    with pytest.raises(WinrsError):            # FP16 FC: the batch is the BFC's channel axis (N % 8)
        W.conv_plan_for_device("fc", 12, 16, 9, 12, 16, 3, 3, 1, "f16")
    with pytest.raises(WinrsError):            # not sm_100
        W.conv_plan_for_device("fc", 8, 16, 9, 12, 16, 3, 3, 1, "f16", cc=(9, 0))
