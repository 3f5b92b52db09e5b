"""Batch-sharded data-parallel BFC: rank g takes a contiguous
N-slice, plans for its local shape, computes its partial dW, and ONE
all_reduce(SUM) combines them — the sum over n is the method's only exchange.

CPU tests (gloo, world_size 2, 127.0.0.1): each rank's partial dW comes from
the library's FP64 host emulation of its local plan (winrs_debug_emulate), so
the sharding + per-shard planning + all_reduce composition is checked against
the FP64 oracle of the full batch without a GPU.  The gpu-marked test runs
bfc_data_parallel itself (the CUDA kernels) on two ranks sharing cuda:0 with
the gloo backend."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _inputs(N, C, H, W, K, R, S, pad, seed=3):
    g = np.random.default_rng(seed)
    Ho, Wo = H + 2 * pad - R + 1, W + 2 * pad - S + 1
    return g.uniform(-1, 1, (N, H, W, C)), g.uniform(-1, 1, (N, Ho, Wo, K))


def _worker_cpu(rank, world, port, shape, q):
    import paper_conf_icpp_zhangc0zx0025_b200 as W
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    N, C, H, Wd, K, R, S, pad = shape
    X, dY = _inputs(*shape)
    a, b = W.shard_range(N, world, rank)
    p = W.plan_for_device(b - a, C, H, Wd, K, R, S, pad, "f32")
    dW = torch.from_numpy(W.emulate(p, X[a:b], dY[a:b]))
    dist.all_reduce(dW, op=dist.ReduceOp.SUM)
    if rank == 0:
        q.put(dW.numpy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("shape", [(4, 8, 10, 10, 8, 3, 3, 1), (5, 4, 9, 12, 8, 5, 5, 2)])
def test_gloo_two_ranks_equal_oracle(shape):
    from oracle import oracle as O
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_cpu, args=(r, 2, port, shape, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    got = q.get(timeout=240)
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    N, C, H, Wd, K, R, S, pad = shape
    X, dY = _inputs(*shape)
    ref = O.bfc_c(X, dY, R, S, pad)
    assert O.rel_max_err(got, ref) < 1e-12


def test_shard_range_partitions():
    import paper_conf_icpp_zhangc0zx0025_b200 as W
    for N in (1, 5, 8, 64, 511):
        for world in (1, 2, 3, 8):
            r = [W.shard_range(N, world, g) for g in range(world)]
            assert r[0][0] == 0 and r[-1][1] == N
            assert all(r[i][1] == r[i + 1][0] for i in range(world - 1))
            sizes = [b - a for a, b in r]
            assert max(sizes) - min(sizes) <= 1


def _worker_gpu(rank, world, port, q):
    import paper_conf_icpp_zhangc0zx0025_b200 as W
    from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    l = wl.LAYERS["r50_c256_14_f16"].with_(N=6, name="dp")
    X, dY = wl.make_inputs(l)
    a, b = W.shard_range(l.N, world, rank)
    dW = W.bfc_data_parallel(torch.from_numpy(X[a:b]).cuda(), torch.from_numpy(dY[a:b]).cuda(),
                             l.R, l.S, l.pad, l.dtype)
    torch.cuda.synchronize()
    if rank == 0:
        q.put(W.as_krsc(dW).cpu().numpy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.gpu
def test_gpu_data_parallel_two_ranks():
    from oracle import oracle as O
    from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_gpu, args=(r, 2, port, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    got = q.get(timeout=300)
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    l = wl.LAYERS["r50_c256_14_f16"].with_(N=6, name="dp")
    X, dY = wl.make_inputs(l)
    ref = O.bfc_c(X, dY, l.R, l.S, l.pad)
    assert O.rel_max_err(got, ref) <= 2e-2
