"""WinRS on B200: fused Winograd backward-filter convolution (PAPER.md, ICPP'25).

Thin Python binding over libwinrs.so (include/winrs.h) — argument marshalling
only; every step of the method runs in the library's sm_100a kernels.  PyTorch
supplies device memory, streams and process groups.

    p = plan(N, C, H, W, K, R, S, pad, "f32")     # winrs_plan
    dW = bfc(p, X, dY)                            # winrs_bfc  (dW: [K,R,S,C] fp32)

X is [N,H,W,C] (NHWC) or a logical [N,C,H,W] channels_last tensor; dY likewise
with (Ho, Wo, K).  dW is returned as a contiguous KRSC float32 tensor (use
`as_kcrs(dW)` for PyTorch's logical [K,C,R,S] weight view, channels_last).
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass

from . import _lib
from ._lib import WinrsError, DTYPES

__all__ = ["Plan", "plan", "plan_for_device", "plan3d", "plan3d_for_device", "bfc", "bfc_host", "as_kcrs", "as_krsc", "bfc_data_parallel", "shard_range",
           "bfc_k_sharded", "PeerAllreduce", "ConvPlan", "conv_plan", "conv_plan_for_device", "fc", "bdc", "emulate_conv",
           "WinrsError", "version", "emulate", "transform", "kernel_names"]


class Plan:
    """Owns a winrs_plan_t.  `info` mirrors winrs_plan_info_t."""

    def __init__(self, handle: ctypes.c_void_p, owned: bool = True):
        self._h = handle
        self._owned = owned
        inf = _lib.PlanInfoT()
        _lib.check(_lib.lib().winrs_plan_info(self._h, ctypes.byref(inf)), "winrs_plan_info")
        self.info = {name: getattr(inf, name) for name, _ in _lib.PlanInfoT._fields_}

    @property
    def handle(self):
        return self._h

    @property
    def workspace_bytes(self) -> int:
        return int(_lib.lib().winrs_workspace_bytes(self._h))

    @property
    def launch_count(self) -> int:
        return int(_lib.lib().winrs_launch_count(self._h))

    @property
    def kernel_name(self) -> str:
        return _lib.lib().winrs_debug_plan_kernel(self._h).decode()

    @property
    def model_us(self) -> float:
        """The planner's B200 time-model estimate (R19)."""
        return float(_lib.lib().winrs_debug_plan_model_us(self._h))

    @property
    def dtype(self) -> str:
        return {0: "f32", 1: "f16", 2: "bf16"}[self.info["dtype"]]

    def __del__(self):
        h, self._h = getattr(self, "_h", None), None
        try:
            if h and getattr(self, "_owned", False) and _lib is not None and _lib._lib is not None:
                _lib._lib.winrs_plan_destroy(h)
        except Exception:   # interpreter shutdown
            pass

    def __repr__(self):
        i = self.info
        s = (f"Plan(Omega_{i['alpha0']}({i['n0']},{i['r0']})x{i['k0']}")
        if i["alpha1"]:
            s += f" + Omega_{i['alpha1']}({i['n1']},{i['r1']})x{i['k1']}"
        return s + (f", Z={i['Z']}, tile={i['tile_k0']}x{i['tile_c0']}, csplit={i['csplit']}, "
                    f"ws={i['workspace_bytes']}B)")


def plan(N, C, H, W, K, R, S, pad, dtype: str = "f32") -> Plan:
    """winrs_plan on the current CUDA device."""
    h = ctypes.c_void_p()
    _lib.check(_lib.lib().winrs_plan(N, C, H, W, K, R, S, pad, DTYPES[dtype], ctypes.byref(h)), "winrs_plan")
    return Plan(h)


def plan_for_device(N, C, H, W, K, R, S, pad, dtype: str = "f32", num_sms: int = 148,
                    cc=(10, 0)) -> Plan:
    """winrs_plan_for_device: plan without touching a GPU (host tests)."""
    dev = _lib.DeviceT(num_sms, cc[0], cc[1])
    h = ctypes.c_void_p()
    _lib.check(_lib.lib().winrs_plan_for_device(N, C, H, W, K, R, S, pad, DTYPES[dtype], ctypes.byref(dev),
                                                ctypes.byref(h)), "winrs_plan_for_device")
    return Plan(h)


def plan3d(N, C, D, H, W, K, T, R, S, pad, dtype: str = "f16") -> Plan:
    """winrs_plan3d: N-D (3-D) BFC by Level-2 dimension reduction (PAPER.md
    P@17805).  X [N,D,H,W,C], dY [N,Do,Ho,Wo,K], dW [K,T,R,S,C]."""
    h = ctypes.c_void_p()
    _lib.check(_lib.lib().winrs_plan3d(N, C, D, H, W, K, T, R, S, pad, DTYPES[dtype], ctypes.byref(h)),
               "winrs_plan3d")
    return Plan(h)


def plan3d_for_device(N, C, D, H, W, K, T, R, S, pad, dtype: str = "f16", num_sms: int = 148, cc=(10, 0)) -> Plan:
    dev = _lib.DeviceT(num_sms, cc[0], cc[1])
    h = ctypes.c_void_p()
    _lib.check(_lib.lib().winrs_plan3d_for_device(N, C, D, H, W, K, T, R, S, pad, DTYPES[dtype], ctypes.byref(dev),
                                                  ctypes.byref(h)), "winrs_plan3d_for_device")
    return Plan(h)


def _as_cl(t, dims_last, name):
    """A tensor whose memory is channels-last `dims_last` = (b, *spatial, ch):
    that contiguous shape, or the logical (b, ch, *spatial) with channels_last
    (2-D) / channels_last_3d (3-D) strides.  No copy."""
    if tuple(t.shape) == tuple(dims_last) and t.is_contiguous():
        return t
    logical = (dims_last[0], dims_last[-1]) + tuple(dims_last[1:-1])
    if tuple(t.shape) == logical:
        perm = (0,) + tuple(range(2, len(logical))) + (1,)
        v = t.permute(*perm)
        if v.is_contiguous():
            return v
    raise ValueError(f"{name}: expected channels-last {tuple(dims_last)} (contiguous, or logical {logical} "
                     f"with channels_last strides), got shape {tuple(t.shape)} strides {t.stride()}")


def _as_nhwc(t, n, h, w, c, name):
    """Return a tensor whose memory is NHWC [n,h,w,c] (no copy)."""
    if tuple(t.shape) == (n, h, w, c) and t.is_contiguous():
        return t
    if tuple(t.shape) == (n, c, h, w):
        import torch
        if t.is_contiguous(memory_format=torch.channels_last):
            return t.permute(0, 2, 3, 1)
    raise ValueError(f"{name}: expected NHWC [{n},{h},{w},{c}] contiguous or channels_last "
                     f"[{n},{c},{h},{w}], got shape {tuple(t.shape)} strides {t.stride()}")


def _as_krsc(t, k, c, r, s_, name):
    """Return a tensor whose memory is KRSC [k,r,s,c] (no copy): a contiguous
    KRSC tensor, or a logical [K,C,R,S] channels_last tensor."""
    if tuple(t.shape) == (k, r, s_, c) and t.is_contiguous():
        return t
    if tuple(t.shape) == (k, c, r, s_):
        import torch
        if t.is_contiguous(memory_format=torch.channels_last):
            return t.permute(0, 2, 3, 1)
    raise ValueError(f"{name}: expected KRSC [{k},{r},{s_},{c}] contiguous or channels_last "
                     f"[{k},{c},{r},{s_}], got shape {tuple(t.shape)} strides {t.stride()}")


def bfc(p: Plan, X, dY, dW=None, workspace=None, stream=None):
    """winrs_bfc on torch CUDA tensors.

    X, dY: logical NCHW with channels_last strides, or NHWC-contiguous.
    Returns dW with logical [K,C,R,S] shape and channels_last strides, FP32
    (physical order KRSC, the C ABI's layout; `as_krsc` gives that view).  A
    caller-supplied dW (KRSC-contiguous or channels_last KCRS) is written in
    place and returned as given.  Everything runs on `stream` (default: the
    current stream); tensors allocated here are recorded on it."""
    import torch
    i = p.info
    tdt = {"f32": torch.float32, "f16": torch.float16, "bf16": torch.bfloat16}[p.dtype]
    nd = i["T"] > 1 or i["D"] > 1
    if nd:   # N-D plan: NDHWC / NDHWC / KTRSC
        Xn = _as_cl(X, (i["N"], i["D"], i["H"], i["W"], i["C"]), "X")
        Gn = _as_cl(dY, (i["N"], i["Do"], i["Ho"], i["Wo"], i["K"]), "dY")
        wshape = (i["K"], i["T"], i["R"], i["S"], i["C"])
    else:
        Xn = _as_nhwc(X, i["N"], i["H"], i["W"], i["C"], "X")
        Gn = _as_nhwc(dY, i["N"], i["Ho"], i["Wo"], i["K"], "dY")
        wshape = (i["K"], i["R"], i["S"], i["C"])
    if Xn.dtype != tdt or Gn.dtype != tdt:
        raise TypeError(f"X and dY must be {tdt} for this plan")
    if not (Xn.is_cuda and Gn.is_cuda) or Gn.device != Xn.device:
        raise ValueError("X and dY must be CUDA tensors on one device (use bfc_host for host buffers)")
    if stream is None:
        stream = torch.cuda.current_stream(Xn.device)
    sp = stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)
    ts = stream if isinstance(stream, torch.cuda.Stream) else None
    ret = dW
    if dW is None:
        with torch.cuda.stream(ts) if ts is not None else _nullctx():
            dk = torch.empty(wshape, dtype=torch.float32, device=Xn.device)
        ret = dk.permute(0, len(wshape) - 1, *range(1, len(wshape) - 1))   # logical K, C, spatial: channels last
    else:
        if dW.dtype != torch.float32 or not dW.is_cuda or dW.device != Xn.device:
            raise ValueError("dW must be a float32 CUDA tensor on X's device")
        dk = _as_cl(dW, wshape, "dW")
    wsb = p.workspace_bytes
    if wsb:
        if workspace is None:
            with torch.cuda.stream(ts) if ts is not None else _nullctx():
                workspace = torch.empty(wsb, dtype=torch.uint8, device=Xn.device)
        elif not workspace.is_cuda or workspace.device != Xn.device or \
                workspace.numel() * workspace.element_size() < wsb:
            raise ValueError(f"workspace must be >= {wsb} bytes on X's device")
    _lib.check(_lib.lib().winrs_bfc(p.handle, Xn.data_ptr(), Gn.data_ptr(), dk.data_ptr(),
                                    workspace.data_ptr() if wsb else None, sp), "winrs_bfc")
    if ts is not None:   # the caching allocator must not recycle these before `stream` is done with them
        dk.record_stream(ts)
        if wsb:
            workspace.record_stream(ts)
    return ret


class _nullctx:
    def __enter__(self):
        return None

    def __exit__(self, *a):
        return False


def as_krsc(dW):
    """bfc()'s logical [K,C,R,S] (or [K,C,T,R,S]) channels-last result -> its
    KRSC [K,R,S,C] (KTRSC) storage view (the C ABI / oracle layout), no copy.
    Channels-last-contiguous input passes."""
    if dW.dim() >= 4 and dW.stride(1) == 1 and not dW.is_contiguous():
        return dW.permute(0, *range(2, dW.dim()), 1)
    return dW


def bfc_k_sharded(X, dY, R: int, S: int, pad: int, dtype: str, rank: int, world: int):
    """K-sharded BFC (BASELINE.json's communication-free alternative, DESIGN.md
    §8): rank `rank` computes dW[k0:k1] for its slice of the output channels
    over the FULL batch, reading its channel slice of dY in place
    (winrs_bfc_strided, ldy = K).  Returns (dW_slice [k1-k0, R, S, C], k0, k1);
    the slices of all ranks concatenated along K are the full dW."""
    import torch
    N, H, W, C = X.shape
    K = dY.shape[-1]
    align = 4 if dtype == "f32" else 8
    if K % align:
        raise ValueError("K must be a multiple of %d" % align)
    a, b = shard_range(K // align, world, rank)
    k0, k1 = a * align, b * align
    p = plan(N, C, H, W, k1 - k0, R, S, pad, dtype)
    if not (dY.is_contiguous() and X.is_contiguous()):
        raise ValueError("X and dY must be contiguous NHWC")
    dW = torch.empty((k1 - k0, R, S, C), dtype=torch.float32, device=X.device)
    wsb = p.workspace_bytes
    ws = torch.empty(wsb, dtype=torch.uint8, device=X.device) if wsb else None
    sp = torch.cuda.current_stream(X.device).cuda_stream
    _lib.check(_lib.lib().winrs_bfc_strided(p.handle, X.data_ptr(), dY.data_ptr() + k0 * dY.element_size(), K,
                                            dW.data_ptr(), ws.data_ptr() if wsb else None, sp),
               "winrs_bfc_strided")
    return dW, k0, k1


def bfc_host(p: Plan, X_host, dY_host, dW_host, dev_X, dev_dY, dev_dW, workspace=None, stream=None):
    """winrs_bfc_host: host (ideally pinned) tensors in, host dW out; the
    H2D copies, the BFC and the D2H copy all run on `stream`, which is then
    synchronised."""
    import torch
    wsb = p.workspace_bytes
    if wsb and workspace is None:
        workspace = torch.empty(wsb, dtype=torch.uint8, device=dev_X.device)
    if stream is None:
        stream = torch.cuda.current_stream(dev_X.device)
    _lib.check(_lib.lib().winrs_bfc_host(p.handle, X_host.data_ptr(), dY_host.data_ptr(), dW_host.data_ptr(),
                                         dev_X.data_ptr(), dev_dY.data_ptr(), dev_dW.data_ptr(),
                                         workspace.data_ptr() if wsb else None, stream.cuda_stream),
               "winrs_bfc_host")
    return dW_host


def as_kcrs(dW):
    """KRSC storage -> logical [K,C,R,S] view (channels_last strides), no copy."""
    return dW.permute(0, 3, 1, 2)


def shard_range(N: int, world: int, rank: int):
    """Contiguous batch slice [start, end) of rank `rank` (NHWC => the slice of
    X and dY is contiguous in memory); the first N % world ranks get one more."""
    base, extra = divmod(N, world)
    start = rank * base + min(rank, extra)
    return start, start + base + (1 if rank < extra else 0)


def bfc_data_parallel(X_shard, dY_shard, R: int, S: int, pad: int, dtype: str = "f32", group=None,
                      p: Plan | None = None):
    """Batch-sharded BFC: each rank runs the fused BFC on
    its contiguous N-slice, then ONE all_reduce(SUM) of dW over the process
    group — the sum over n is the only exchange the method needs."""
    import torch.distributed as dist
    N, H, W, C = X_shard.shape
    K = dY_shard.shape[-1]
    if p is None:
        p = plan(N, C, H, W, K, R, S, pad, dtype)
    dW = bfc(p, X_shard, dY_shard)
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(as_krsc(dW), op=dist.ReduceOp.SUM, group=group)   # the contiguous KRSC storage
    return dW


class _CudaBuf:
    """A raw device buffer exposed to torch through __cuda_array_interface__ (no copy)."""

    def __init__(self, ptr, n):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": "<f4", "data": (int(ptr), False), "version": 2}


class PeerAllreduce:
    """Data-parallel BFC with the bucket reduction and the cross-rank sum fused
    into one kernel over peer memory (winrs_bfc_allreduce, include/winrs.h;
    SURVEY §8(f) row 1).  Collective constructor over a torch.distributed group
    (any backend: only the 64-byte CUDA IPC handles are exchanged, with
    all_gather_object).  `bfc(X, dY)` returns this rank's dW, logical [K,C,R,S]
    channels_last like `bfc()`, identical on every rank."""

    def __init__(self, p: Plan, group=None):
        import torch.distributed as dist
        self.p = p
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        i = p.info
        self.n = i["K"] * i["T"] * i["R"] * i["S"] * i["C"]
        L = _lib.lib()
        self._own, handles = [], []
        for nbytes in (4 * self.n, 4 * self.n, int(L.winrs_allreduce_flag_bytes())):   # stage, dW, flags
            ptr, h = ctypes.c_void_p(), ctypes.create_string_buffer(64)
            _lib.check(L.winrs_ipc_alloc(nbytes, ctypes.byref(ptr), h), "winrs_ipc_alloc")
            self._own.append(ptr.value)
            handles.append(h.raw)
        allh = [None] * self.world
        if self.world > 1:
            dist.all_gather_object(allh, handles, group=group)
        else:
            allh = [handles]
        self._opened = []
        peers = [[None] * self.world for _ in range(3)]
        for q in range(self.world):
            for j in range(3):
                if q == self.rank:
                    peers[j][q] = self._own[j]
                else:
                    ptr = ctypes.c_void_p()
                    _lib.check(L.winrs_ipc_open(allh[q][j], ctypes.byref(ptr)), "winrs_ipc_open")
                    self._opened.append(ptr.value)
                    peers[j][q] = ptr.value
        arr = ctypes.c_void_p * self.world
        self._stage, self._dW, self._flags = (arr(*peers[0]), arr(*peers[1]), arr(*peers[2]))
        self.epoch = 0
        self._group = group

    def bfc(self, X, dY, workspace=None, stream=None):
        import torch
        i = self.p.info
        tdt = {"f32": torch.float32, "f16": torch.float16, "bf16": torch.bfloat16}[self.p.dtype]
        Xn = _as_nhwc(X, i["N"], i["H"], i["W"], i["C"], "X")
        Gn = _as_nhwc(dY, i["N"], i["Ho"], i["Wo"], i["K"], "dY")
        if Xn.dtype != tdt or Gn.dtype != tdt:
            raise TypeError(f"X and dY must be {tdt} for this plan")
        if stream is None:
            stream = torch.cuda.current_stream(Xn.device)
        sp = stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)
        wsb = self.p.workspace_bytes
        if wsb and workspace is None:
            workspace = torch.empty(wsb, dtype=torch.uint8, device=Xn.device)
        self.epoch += 1
        _lib.check(_lib.lib().winrs_bfc_allreduce(self.p.handle, Xn.data_ptr(), Gn.data_ptr(), self._own[1],
                                                  workspace.data_ptr() if wsb else None, self._stage, self._dW,
                                                  self._flags, self.rank, self.world, self.epoch, sp),
                   "winrs_bfc_allreduce")
        dW = torch.as_tensor(_CudaBuf(self._own[1], self.n), device=Xn.device).view(i["K"], i["R"], i["S"], i["C"])
        return dW.permute(0, 3, 1, 2)

    def close(self):
        L = _lib.lib()
        for ptr in getattr(self, "_opened", []):
            L.winrs_ipc_close(ptr)
        for ptr in getattr(self, "_own", []):
            L.winrs_ipc_free(ptr)
        self._opened, self._own = [], []


class ConvPlan:
    """Owns a winrs_conv_plan_t (FC or BDC on the BFC machinery, include/winrs.h).
    `bfc` is the mapped BFC Plan (owned by this object)."""

    def __init__(self, handle: ctypes.c_void_p, kind: str, dims):
        self._h = handle
        self.kind = kind
        self.N, self.C, self.H, self.W, self.K, self.R, self.S, self.pad, self.dtype = dims
        self.Ho = self.H + 2 * self.pad - self.R + 1
        self.Wo = self.W + 2 * self.pad - self.S + 1
        b = ctypes.c_void_p()
        _lib.check(_lib.lib().winrs_conv_bfc_plan(self._h, ctypes.byref(b)), "winrs_conv_bfc_plan")
        self.bfc = Plan(b, owned=False)   # the mapped BFC plan, owned by the conv plan

    @property
    def workspace_bytes(self) -> int:
        return int(_lib.lib().winrs_conv_workspace_bytes(self._h))

    @property
    def launch_count(self) -> int:
        return int(_lib.lib().winrs_conv_launch_count(self._h))

    @property
    def kernel_name(self) -> str:
        return self.bfc.kernel_name

    def __del__(self):
        h, self._h = getattr(self, "_h", None), None
        try:
            if h and _lib is not None and _lib._lib is not None:
                _lib._lib.winrs_conv_plan_destroy(h)
        except Exception:
            pass


_CONV_KINDS = {"fc": 0, "bdc": 1}


def conv_plan(kind: str, N, C, H, W, K, R, S, pad, dtype: str = "f16") -> ConvPlan:
    """winrs_conv_plan: FC ("fc") or BDC ("bdc") of the layer on the current device."""
    h = ctypes.c_void_p()
    _lib.check(_lib.lib().winrs_conv_plan(_CONV_KINDS[kind], N, C, H, W, K, R, S, pad, DTYPES[dtype],
                                          ctypes.byref(h)), "winrs_conv_plan")
    return ConvPlan(h, kind, (N, C, H, W, K, R, S, pad, dtype))


def conv_plan_for_device(kind: str, N, C, H, W, K, R, S, pad, dtype: str = "f16", num_sms: int = 148,
                         cc=(10, 0)) -> ConvPlan:
    dev = _lib.DeviceT(num_sms, cc[0], cc[1])
    h = ctypes.c_void_p()
    _lib.check(_lib.lib().winrs_conv_plan_for_device(_CONV_KINDS[kind], N, C, H, W, K, R, S, pad, DTYPES[dtype],
                                                     ctypes.byref(dev), ctypes.byref(h)),
               "winrs_conv_plan_for_device")
    return ConvPlan(h, kind, (N, C, H, W, K, R, S, pad, dtype))


def _conv_run(cp: ConvPlan, fn: str, inp, Wt, out_shape, workspace, stream):
    import torch
    tdt = {"f32": torch.float32, "f16": torch.float16, "bf16": torch.bfloat16}[cp.dtype]
    ishape = (cp.N, cp.H, cp.W, cp.C) if cp.kind == "fc" else (cp.N, cp.Ho, cp.Wo, cp.K)
    In = _as_cl(inp, ishape, "input")
    Wn = _as_krsc(Wt, cp.K, cp.C, cp.R, cp.S, "Wt")
    if In.dtype != tdt or Wn.dtype != tdt:
        raise TypeError(f"input and Wt must be {tdt} for this plan")
    if not (In.is_cuda and Wn.is_cuda) or In.device != Wn.device:
        raise ValueError("input and Wt must be CUDA tensors on one device")
    if stream is None:
        stream = torch.cuda.current_stream(In.device)
    sp = stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)
    ts = stream if isinstance(stream, torch.cuda.Stream) else None
    with torch.cuda.stream(ts) if ts is not None else _nullctx():
        out = torch.empty(out_shape, dtype=torch.float32, device=In.device)
        if workspace is None:
            workspace = torch.empty(cp.workspace_bytes, dtype=torch.uint8, device=In.device)
    if workspace.numel() * workspace.element_size() < cp.workspace_bytes or workspace.device != In.device:
        raise ValueError(f"workspace must be >= {cp.workspace_bytes} bytes on the input's device")
    _lib.check(getattr(_lib.lib(), fn)(cp._h, In.data_ptr(), Wn.data_ptr(), out.data_ptr(), workspace.data_ptr(),
                                       sp), fn)
    if ts is not None:
        out.record_stream(ts)
        workspace.record_stream(ts)
    return out


def fc(cp: ConvPlan, X, Wt, workspace=None, stream=None):
    """winrs_fc: Y [N,Ho,Wo,K] FP32 (NHWC) = conv(X [N,H,W,C], Wt [K,R,S,C])."""
    assert cp.kind == "fc"
    return _conv_run(cp, "winrs_fc", X, Wt, (cp.N, cp.Ho, cp.Wo, cp.K), workspace, stream)


def bdc(cp: ConvPlan, dY, Wt, workspace=None, stream=None):
    """winrs_bdc: dX [N,H,W,C] FP32 (NHWC) from dY [N,Ho,Wo,K] and Wt [K,R,S,C]."""
    assert cp.kind == "bdc"
    return _conv_run(cp, "winrs_bdc", dY, Wt, (cp.N, cp.H, cp.W, cp.C), workspace, stream)


def emulate_conv(cp: ConvPlan, inp, Wt):
    """FP64 host emulation of winrs_fc / winrs_bdc: the C library's operand
    mapping (include/winrs.h) in numpy, then winrs_debug_emulate of the mapped
    BFC plan (numpy float64 in, NHWC out)."""
    import numpy as np
    inp = np.asarray(inp, dtype=np.float64)
    Wt = np.asarray(Wt, dtype=np.float64)
    Xp = np.ascontiguousarray(inp.transpose(3, 1, 2, 0))            # [ch][h][w][n]
    if cp.kind == "fc":
        Gp = np.ascontiguousarray(Wt.transpose(3, 1, 2, 0))         # [C][R][S][K]
    else:
        Gp = np.ascontiguousarray(Wt[:, ::-1, ::-1, :])             # [K][R][S][C], (r,s) reversed
    out = emulate(cp.bfc, Xp, Gp)                             # [K'][R'][S'][N]
    return np.ascontiguousarray(out.transpose(3, 1, 2, 0))


def version() -> str:
    return _lib.lib().winrs_version().decode()


def kernel_names():
    L = _lib.lib()
    return [L.winrs_debug_kernel_name(i).decode() for i in range(L.winrs_debug_kernel_count())]


def emulate(p: Plan, X, dY):
    """winrs_debug_emulate: FP64 host emulation of the plan's decomposition
    (numpy float64 NHWC in, KRSC out)."""
    import numpy as np
    i = p.info
    Xd = np.ascontiguousarray(X, dtype=np.float64)
    Gd = np.ascontiguousarray(dY, dtype=np.float64)
    if i["T"] > 1 or i["D"] > 1:   # N-D plan: NDHWC in, KTRSC out
        assert Xd.shape == (i["N"], i["D"], i["H"], i["W"], i["C"])
        assert Gd.shape == (i["N"], i["Do"], i["Ho"], i["Wo"], i["K"])
        out = np.empty((i["K"], i["T"], i["R"], i["S"], i["C"]), dtype=np.float64)
    else:
        assert Xd.shape == (i["N"], i["H"], i["W"], i["C"]) and Gd.shape == (i["N"], i["Ho"], i["Wo"], i["K"])
        out = np.empty((i["K"], i["R"], i["S"], i["C"]), dtype=np.float64)
    _lib.check(_lib.lib().winrs_debug_emulate(p.handle, Xd.ctypes.data, Gd.ctypes.data, out.ctypes.data),
               "winrs_debug_emulate")
    return out


def transform(alpha: int, n: int, r: int, which: str, vec):
    """winrs_debug_transform: apply the generated FT/IT/OT of Omega_alpha(n,r) in double."""
    import numpy as np
    w = {"ft": 0, "it": 1, "ot": 2}[which]
    x = np.ascontiguousarray(vec, dtype=np.float64)
    out = np.empty(n if w == 2 else alpha, dtype=np.float64)
    _lib.check(_lib.lib().winrs_debug_transform(alpha, n, r, w, x.ctypes.data, out.ctypes.data),
               "winrs_debug_transform")
    return out
