"""Fused bucket reduction + cross-rank all-reduce over peer memory
(winrs_bfc_allreduce), two ranks.  The GPU box has one
GPU, so the two ranks are two processes sharing cuda:0: the buffers are
shared with CUDA IPC exactly as between NVLink peers, and the kernels'
cross-rank barriers run under the driver's time slicing.  Checks: every rank
and every call returns the same dW, bit-identical to the unfused path (each
rank's winrs_bfc, then an FP32 sum in rank order), and the oracle on the
whole batch within the FP32 / FP16 gates."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

CASES = [
    # dtype, per-rank layer overrides, env
    ("f32", dict(N=8, C=64, K=64, H=20, W=20), {"WINRS_FORCE_Z": "3"}),
    ("f16", dict(N=16, C=64, K=128, H=14, W=14), {"WINRS_FORCE_Z": "2"}),
    ("f32", dict(N=8, C=36, K=20, H=11, W=13), {}),          # |dW| % 4 != 0 elements: the scalar tail
]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, case, q):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dtype, ov, env = case
    os.environ.update(env)
    try:
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        import paper_conf_icpp_zhangc0zx0025_b200 as W
        from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
        layer = wl.LAYERS["r50_c64_56_f16" if dtype == "f16" else "r50_c64_56_f32"].with_(name="ar", **ov)
        X, dY = wl.make_inputs(layer, seed_offset=1000 * rank)
        p = W.plan(layer.N, layer.C, layer.H, layer.W, layer.K, layer.R, layer.S, layer.pad, dtype)
        Xg, Gg = torch.from_numpy(X).cuda(), torch.from_numpy(dY).cuda()
        par = W.PeerAllreduce(p)
        fused = []
        for _ in range(3):
            dW = par.bfc(Xg, Gg)
            torch.cuda.synchronize()
            fused.append(W.as_krsc(dW).cpu().numpy().copy())
            dist.barrier()
        unfused = W.as_krsc(W.bfc(p, Xg, Gg)).cpu().numpy()
        torch.cuda.synchronize()
        dist.barrier()
        par.close()
        q.put((rank, fused, unfused, X, dY, p.kernel_name, p.info["Z"]))
        dist.destroy_process_group()
    except Exception as e:   # report instead of hanging the parent
        q.put((rank, repr(e)))


@pytest.mark.parametrize("case", CASES, ids=[f"{c[0]}-{i}" for i, c in enumerate(CASES)])
def test_fused_reduce_allreduce_two_ranks(case):
    import multiprocessing as mp
    from oracle import oracle as O
    from conftest import record_err
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, case, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    res = {}
    for _ in range(2):
        item = q.get(timeout=300)
        assert len(item) > 2, f"rank {item[0]} failed: {item[1]}"
        res[item[0]] = item
    for pr in procs:
        pr.join(timeout=60)
    f0, f1 = res[0][1], res[1][1]
    for a in f0[1:] + f1:
        assert np.array_equal(a, f0[0])                      # every call, every rank: the same dW
    ref = res[0][2].astype(np.float32) + res[1][2].astype(np.float32)   # unfused, FP32 sum in rank order
    assert np.array_equal(f0[0], ref)
    X = np.concatenate([res[0][3], res[1][3]])
    dY = np.concatenate([res[0][4], res[1][4]])
    R, S, pad = 3, 3, 1
    err = O.rel_max_err(f0[0].astype(np.float64), O.bfc_c(X, dY, R, S, pad))
    record_err(f"fused reduce+allreduce 2 ranks [{case[0]}] {case[1]}", err, f"{res[0][5]} Z={res[0][6]}")
    assert err <= (1e-4 if case[0] == "f32" else 2e-2)
