#!/usr/bin/env python3
"""Benchmark of the WinRS fused Winograd BFC on B200 (BASELINE.json metric:
effective TFLOPS = direct-conv FLOPs 2*N*C*K*Ho*Wo*R*S / device time, plus
workspace bytes).

A "step" is one pass of the whole hot path (plan prebuilt; fused kernel +
bucket reduction [+ one NCCL all_reduce of dW when N > 1]) over every layer of
the workload, inputs resident in HBM.  L2 is flushed (a 256 MiB write) before
every layer call and each call is timed with CUDA events on the launch stream
(the flush is outside the timed events).

Default workload: the largest single-GPU BASELINE config, VGG-16's 3x3 layers
2-13 at N=128 in FP16 (configs[2]; BASELINE's metric names no config).  The
ResNet-50 layers (configs[1], FP16 and FP32) and the wide-dW config
(configs[3], FP32) are measured alongside in the same run and reported under
config.alongside (--no-alongside skips them).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload vgg|r50|wide|r50l3]
                    [--dtype f16|bf16|f32] [--impl winrs|reference] [--parallel dp|kshard]

--gpus N > 1 without a torchrun environment re-launches itself under
torch.distributed.run (one rank per GPU, NCCL, 127.0.0.1).  dp (default):
every rank runs the per-rank workload on its own batch shard and all-reduces
each layer's dW (weak scaling: global batch = N x per-rank batch), except
--workload r50l3, BASELINE configs[4]: the FIXED global batch N=512 of
ResNet-50 layer 3 split over the ranks (strong scaling), reported with and
without the all_reduce.  kshard: every rank holds the full batch and computes
its slice of the output channels (strong, no communication).  Time = max over
ranks.  --impl reference runs the FP64 CPU oracle (the only reference this
paper-only tier has) on a bounded sample of the same workload, rank 0 only.
--dry-run exercises only the launch / rank plumbing (gloo, no GPU work).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "effective TFLOPS (direct-conv FLOPs) + workspace bytes per BFC layer"


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d, "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0, "sm_max_mhz": 1965.0}, "fallback"


def _ncu_traffic(dtype: str, layer_name: str):
    """DRAM bytes (read + write) per launch of the dominant kernel from the
    latest committed ncu --set full capture (profiles/r*/traffic.json)."""
    import glob
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", "r*", "traffic.json")))
    if not files:
        return None, None
    with open(files[-1]) as f:
        t = json.load(f)
    base = layer_name.rsplit("_", 1)[0]
    layers = t.get("layers_" + dtype, t.get("layers", []))
    if dtype in t and base in layers:
        i = layers.index(base)
        if i < len(t[dtype]):
            return t[dtype][i]["dram_bytes"], os.path.relpath(files[-1], ROOT) + " (ncu --set full)"
    return None, None


def _workload(name: str, dtype: str):
    from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
    if name == "r50":
        if dtype == "bf16":
            return [l.with_(dtype="bf16", name=l.name.replace("f16", "bf16")) for l in wl.RESNET50_F16]
        return wl.RESNET50_F32 if dtype == "f32" else wl.RESNET50_F16
    if name == "vgg":
        return wl.VGG16_F16
    if name == "wide":
        return wl.WIDE_F32
    if name == "r50l3":
        return [wl.LAYERS["r50_l3_n512_f16"]]
    raise ValueError(name)


class ClockSampler:
    """SM clocks and clock-event (throttle) reasons sampled during the timed region.

    In-process NVML (pynvml): a background thread polls every ~1 ms, and the
    timed loop calls ``sample()`` itself while it waits for the queued steps
    to drain, so even a timed region of a few milliseconds gets samples taken
    while the GPU is busy.  nvidia-smi (~100 ms minimum period, ~0.5 s start
    up) never landed a sample inside the short ResNet-50 step.
    """

    REASONS = (("hw_slowdown", 0x8), ("hw_thermal_slowdown", 0x40), ("sw_thermal_slowdown", 0x20),
               ("sw_power_cap", 0x4), ("hw_power_brake_slowdown", 0x80))

    def __init__(self, cuda_index: int):
        self.rows = []
        self.h = None
        self.nvml = None
        self.stop_flag = False
        self.t = None
        self.lock = threading.Lock()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nvml = pynvml
            self.h = self._handle(cuda_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.h = None

    def _handle(self, cuda_index):
        pynvml = self.nvml
        try:
            import torch
            p = torch.cuda.get_device_properties(cuda_index)
            bus = f"{p.pci_domain_id:08X}:{p.pci_bus_id:02X}:{p.pci_device_id:02X}.0"
            return pynvml.nvmlDeviceGetHandleByPciBusId(bus)
        except Exception:
            vis = os.environ.get("CUDA_VISIBLE_DEVICES", "")
            ids = [v.strip() for v in vis.split(",") if v.strip()]
            idx = int(ids[cuda_index]) if cuda_index < len(ids) and ids[cuda_index].isdigit() else cuda_index
            return pynvml.nvmlDeviceGetHandleByIndex(idx)

    def sample(self):
        if self.h is None:
            return
        try:
            sm = self.nvml.nvmlDeviceGetClockInfo(self.h, self.nvml.NVML_CLOCK_SM)
            rs = self.nvml.nvmlDeviceGetCurrentClocksEventReasons(self.h)
        except Exception:
            return
        with self.lock:
            self.rows.append((sm, rs))

    def _loop(self):
        while not self.stop_flag:
            self.sample()
            time.sleep(0.001)

    def start(self):
        if self.h is None:
            return
        self.t = threading.Thread(target=self._loop, daemon=True)
        self.t.start()

    def stop(self):
        if self.h is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml unavailable"], "samples": 0}
        self.stop_flag = True
        if self.t is not None:
            self.t.join(timeout=2)
        sm = [r[0] for r in self.rows]
        reasons = sorted({n for _, rs in self.rows for n, bit in self.REASONS if rs & bit})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": self.max_mhz,
                "sm_min_mhz": min(sm) if sm else None, "reasons": reasons, "samples": len(sm),
                "source": "nvml"}


# L2 -> SM fill rate used for the t_L2 diagnostic: TMA boxes of the tc2 kernel,
# 148 CTAs, tools/microbench/tma_rate3.cu mode 0 on B200 (81 B/clk/SM x 148 x 1.965 GHz).
L2_SM_GBS = 23650.0


def _rows_valid(l, fh):
    return sum(1 for h in range(l.Ho) if 0 <= h + fh - l.pad < l.H)


def _rows_union(l, fhs):
    return sum(1 for h in range(l.Ho) if any(0 <= h + f - l.pad < l.H for f in fhs))


def layer_roofline(l, p, ms, peaks):
    """The BASELINE roofline of one layer call:
    T_roof = max(algorithmic bytes / HBM, Winograd EWM FLOPs / pipe peak), and
    the diagnostic bounds t_ALU (transform lane-ops / FP32 lanes) and t_L2
    (L2 -> SM bytes / measured fill rate), all against the measured time."""
    info = p.info
    esz = 4 if l.dtype == "f32" else 2
    Z = info["Z"]
    dw = 4 * l.K * l.R * l.S * l.C
    alg_bytes = esz * (l.N * l.H * l.W * l.C + l.N * l.Ho * l.Wo * l.K) + dw * (1 if Z == 1 else 2 * Z + 1)
    ewm = info["ewm_flops"]
    clk_ghz = float(peaks.get("sm_max_mhz", 1965.0)) / 1e3
    fp32_peak = 148 * 128 * 2 * clk_ghz * 1e9            # FLOP/s (lanes x FMA)
    lanes = 148 * 128 * clk_ghz * 1e9                    # lane-ops/s
    t_hbm = alg_bytes / (peaks["hbm_gbs"] * 1e9)
    if l.dtype == "f32" and p.kernel_name.startswith("f32tc_"):
        # bfc_tc3.cuh: FP32 on the tensor cores, 3 tf32 MMAs per product (3xTF32);
        # tf32 peak = the measured bf16 dense peak x the nominal 1.13 / 2.25 ratio
        tf32 = peaks["bf16_tflops"] * 1.13 / 2.25
        t_pipe, bound, pk = 3.0 * ewm / (tf32 * 1e12), "tensor", tf32
    elif l.dtype == "f32":
        t_pipe, bound, pk = ewm / fp32_peak, "alu", fp32_peak / 1e12
    else:
        t_pipe, bound, pk = ewm / (peaks["bf16_tflops"] * 1e12), "tensor", peaks["bf16_tflops"]
    if t_hbm > t_pipe:
        bound = "hbm"
    t_roof = max(t_hbm, t_pipe)
    # depth entries x tiles the kernel walks, for the diagnostics
    name = p.kernel_name
    a, n0, r0 = info["alpha0"], info["n0"], info["r0"]
    units = info["k0"] + info["k1"]
    bn, bm = info["tile_k0"], info["tile_c0"]
    kb, cb = -(-l.K // bn), -(-l.C // bm)
    ft = l.S // n0
    if "_v2s_" in name:                                   # swapped CTA pair: 256 k x 128 c, 1 filter row
        rows = sum(_rows_valid(l, fh) for fh in range(l.R))
        depth = rows * units * l.N * kb * cb * ft
        l2_bytes = depth / 16 * 2 * (8192 + 8192)         # per pair stage: each CTA X 8 KB + dY 8 KB
        alu_ops = depth * (256 + 128 * 2)                 # FT over 256 k, IT over 128 c (half2)
    elif "_v2x_" in name or "_v2k_" in name:              # xi-split pair (k: stream-K): 128 k x 128 rows
        fhs = int(name.split("x")[-1].rstrip("fh"))
        rows = sum(_rows_union(l, range(g, min(l.R, g + fhs))) for g in range(0, l.R, fhs))
        depth = rows * units * l.N * kb * cb * ft        # depth entries x pair tiles
        l2_bytes = depth / 16 * (8192 + 16384 + 2 * 8192)  # per pair stage: X 8 + 16 KB, dY 8 KB per CTA
        alu_ops = depth * (128 + 2 * 128 * 2)             # FT: W0, W1 over 128 k; IT: 2 outputs per row per half
    elif "_v3_" in name:                                  # FP32 tensor-core kernel: 8-deep stages
        fhs = int(name.split("x")[-1].rstrip("fh"))
        rows = sum(_rows_union(l, range(g, min(l.R, g + fhs))) for g in range(0, l.R, fhs))
        depth = rows * units * l.N * kb * cb * ft
        l2_bytes = depth / 8 * (16384 + bn * 64)          # per stage: X 16 KB + dY NK x 2 cols x 8 x 4 B
        alu_ops = depth * (bn * 2 * 2 + 128 * 4 * 3)      # FT (+ lo split), IT 4 outputs (+ lo split)
    elif "_v2" in name:
        tag = name.split("_v2")[1][0]                     # CTAs per UMMA (2: cta_group::2 pair); t: Xhat in TMEM
        cg = 1 if tag == "t" else int(tag)
        fhs = int(name.split("x")[-1].rstrip("fh")) * cg if bm == 64 else 1
        rows = sum(_rows_union(l, range(g, min(l.R, g + fhs))) for g in range(0, l.R, fhs))
        depth = rows * units * l.N * kb * cb * ft        # depth entries x (pair) tiles
        l2_bytes = depth / 16 * (cg * 16384 + bn * 64)    # per 16-deep stage: X 16 KB per CTA + dY NK*64 B
        alu_ops = depth * (bn + 128 * cg * 2)             # FT: W0, W1 = w0 +- w1; IT: 4 outputs per row (half2)
    else:
        rows = sum(_rows_valid(l, fh) for fh in range(l.R))
        depth = rows * units * l.N * kb * cb * ft
        ft_ops = {2: 1, 4: 2, 8: 22, 16: 90}.get(a, a * r0)    # FT adds/FMAs per channel (generated code)
        it_ops = {2: 2, 4: 4, 8: 28, 16: 110}.get(a, a * a)
        cvt = 0 if l.dtype == "f32" else (r0 + a / 2 + a / 2 + a / 2)   # unpack + pack (FP16 path)
        alu_ops = depth * (bn * (ft_ops + cvt) + bm * (it_ops + cvt))
        l2_bytes = depth * (r0 * bn + a * bm) * esz
    t_alu = alu_ops / lanes
    t_l2 = l2_bytes / (L2_SM_GBS * 1e9)
    sec = ms * 1e-3
    return {"layer": l.name, "kernel": name, "bound": bound, "frac": t_roof / sec,
            "t_roof_us": t_roof * 1e6, "t_hbm_us": t_hbm * 1e6, "t_pipe_us": t_pipe * 1e6,
            "t_alu_us": t_alu * 1e6, "t_l2_us": t_l2 * 1e6, "measured_us": ms * 1e3,
            "alg_bytes": alg_bytes, "ewm_flops": ewm, "pipe_peak_tflops": pk}


def measure(layers, args, ctx, primary=True):
    """Time one workload: per-layer cold-L2 CUDA-event times over the steps,
    warm-L2 times, CUDA-graph replays, (N > 1) compute-only times, the dominant
    kernel alone, and the end-to-end host-buffer path.  Returns a dict."""
    import torch
    import torch.distributed as dist
    import paper_conf_icpp_zhangc0zx0025_b200 as W
    from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
    world, rank, dev, kshard, strong = ctx["world"], ctx["rank"], ctx["dev"], ctx["kshard"], ctx["strong"]
    steps = args.steps if primary else max(3, min(args.steps, 5))
    warmup = args.warmup if primary else 3
    items = []
    for l in layers:
        align = 4 if l.dtype == "f32" else 8
        k0, k1, n0, n1 = 0, l.K, 0, l.N
        if strong:     # fixed global batch: this rank's contiguous image slice (NHWC: contiguous)
            n0, n1 = W.shard_range(l.N, world, rank)
            X, dY = wl.make_inputs(l)
            X, dY = np.ascontiguousarray(X[n0:n1]), np.ascontiguousarray(dY[n0:n1])
        else:
            X, dY = wl.make_inputs(l, seed_offset=0 if kshard else 1000 * rank)
        if kshard:
            a, b = W.shard_range(l.K // align, world, rank)
            k0, k1 = a * align, b * align
        ll = l.with_(N=n1 - n0)
        p = W.plan(ll.N, l.C, l.H, l.W, k1 - k0, l.R, l.S, l.pad, l.dtype)
        Xt, Gt = torch.from_numpy(X), torch.from_numpy(dY)
        if l.dtype == "bf16":   # workloads carries bf16 values in float32
            Xt, Gt = Xt.to(torch.bfloat16), Gt.to(torch.bfloat16)
        dW = torch.empty((k1 - k0, l.R, l.S, l.C), dtype=torch.float32, device=dev)
        ws = torch.empty(max(p.workspace_bytes, 16), dtype=torch.uint8, device=dev)
        it = dict(layer=l, local=ll, plan=p, X=Xt.to(dev), dY=Gt.to(dev), dW=dW, ws=ws,
                  Xh=Xt.pin_memory(), Gh=Gt.pin_memory(), dWh=torch.empty(dW.shape).pin_memory(), k0=k0, k1=k1)
        if ctx.get("fused") and world > 1 and not kshard:
            # bucket reduction + cross-rank sum in one kernel over peer memory (winrs_bfc_allreduce);
            # dW is then the IPC-shared output buffer (collective setup: every rank, same order)
            it["par"] = W.PeerAllreduce(p)
            it["dW"] = W.as_krsc(it["par"].bfc(it["X"], it["dY"], ws))
        items.append(it)
    stream = torch.cuda.current_stream(dev)

    def bfc_only(it, s):
        if kshard:   # channel slice of dY read in place (ldy = K), no communication
            from paper_conf_icpp_zhangc0zx0025_b200 import _lib
            _lib.check(_lib.lib().winrs_bfc_strided(it["plan"].handle, it["X"].data_ptr(),
                                                    it["dY"].data_ptr() + it["k0"] * it["dY"].element_size(),
                                                    it["layer"].K, it["dW"].data_ptr(), it["ws"].data_ptr(),
                                                    s.cuda_stream), "winrs_bfc_strided")
        else:
            W.bfc(it["plan"], it["X"], it["dY"], it["dW"], it["ws"], s)

    def run_bfc(it, s):
        if "par" in it:                    # fused bucket reduction + all-reduce (one kernel, peer memory)
            it["par"].bfc(it["X"], it["dY"], it["ws"], s)
            return
        bfc_only(it, s)
        if world > 1 and not kshard:
            dist.all_reduce(it["dW"])      # the data-parallel step's one exchange (NCCL over NVLink)

    flush = ctx["flush"]

    def one_step(timed_events=None):
        for j, it in enumerate(items):
            flush.fill_(j & 0xFF)                                  # evict L2 (outside the events)
            if timed_events is not None:
                timed_events[j][0].record(stream)
            run_bfc(it, stream)
            if timed_events is not None:
                timed_events[j][1].record(stream)

    for _ in range(warmup):
        one_step()
    torch.cuda.synchronize()
    clocks = ClockSampler(ctx["local"]) if primary and rank == 0 else None
    if clocks:
        clocks.start()
    ev = [[[torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)] for _ in items]
          for _ in range(steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    for s in range(steps):
        one_step(ev[s])
        if clocks:
            clocks.sample()                                        # GPU busy with the queued layers
    if clocks:
        while not ev[-1][-1][1].query():                           # GPU still draining the steps
            clocks.sample()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop() if clocks else None
    per_layer_ms = [sum(ev[s][j][0].elapsed_time(ev[s][j][1]) for s in range(steps)) / steps
                    for j in range(len(items))]

    def time_layers(flush_l2, fn, reps=5):
        out = []
        for it2 in items:
            ts = []
            for _ in range(reps):
                if flush_l2:
                    flush.fill_(3)
                else:   # keep the GPU busy while the host launches (no memory traffic)
                    torch.cuda._sleep(100000)
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                fn(it2, stream)
                b.record(stream)
                torch.cuda.synchronize()
                ts.append(a.elapsed_time(b))
            out.append(statistics.median(ts))
        return out
    warm_ms = time_layers(False, run_bfc)
    compute_only_ms = time_layers(True, bfc_only) if world > 1 and not kshard else None

    # CUDA-graph replays: each layer's winrs_bfc launches captured
    # once, replayed cold-L2; device time per replay from CUDA events.
    graph = None
    if primary and not args.no_graphs:
        graph = []
        reps = args.graph_reps or (1000 if sum(per_layer_ms) < 1.0 else 100)
        cap = torch.cuda.Stream(dev)
        for it2 in items:
            g = torch.cuda.CUDAGraph()
            cap.wait_stream(stream)
            with torch.cuda.graph(g, stream=cap):
                bfc_only(it2, cap)
            stream.wait_stream(cap)
            for _ in range(20):
                g.replay()
            torch.cuda.synchronize()
            evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
            for a, b in evs:
                flush.fill_(5)
                a.record(stream)
                g.replay()
                b.record(stream)
            torch.cuda.synchronize()
            ts = [a.elapsed_time(b) for a, b in evs]
            graph.append({"mean_ms": statistics.fmean(ts), "median_ms": statistics.median(ts), "replays": reps})
            del g

    # The dominant layer's kernel(s) alone (no all_reduce), CUDA events on the stream.
    dom = max(range(len(items)), key=lambda j: per_layer_ms[j])
    kt = []
    for _ in range(max(3, steps)):
        flush.fill_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        bfc_only(items[dom], stream)
        e1.record(stream)
        torch.cuda.synchronize()
        kt.append(e0.elapsed_time(e1))
    dom_alone_ms = statistics.median(kt)
    # the roofline uses the dominant layer's launches measured inside the timed
    # steps (its per-step CUDA-event times, median); the separate back-to-back
    # loop above is reported beside it (it runs hotter, e.g. into sw_power_cap)
    dom_ms = per_layer_ms[dom]

    # End to end through the C ABI with host buffers (pinned), copies inside.
    e2e_ms = []
    for _ in range(max(2, min(steps, 5))):
        tot = 0.0
        for it2 in items:
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            dX = torch.empty_like(it2["X"])
            dG = torch.empty_like(it2["dY"])
            a.record(stream)
            if kshard or world > 1:   # H2D, the BFC (+ all_reduce for dp), D2H of (this rank's) dW
                dX.copy_(it2["Xh"], non_blocking=True)
                dG.copy_(it2["Gh"], non_blocking=True)
                run_bfc(dict(it2, X=dX, dY=dG), stream)
                it2["dWh"].copy_(it2["dW"], non_blocking=True)
            else:
                W.bfc_host(it2["plan"], it2["Xh"], it2["Gh"], it2["dWh"], dX, dG, it2["dW"], it2["ws"], stream)
            b.record(stream)
            torch.cuda.synchronize()
            tot += a.elapsed_time(b)
        e2e_ms.append(tot)
    e2e = statistics.median(e2e_ms)

    def max_over_ranks(v):
        if world == 1 or v is None:
            return v
        t = torch.tensor([float(v)], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())
    step_ms = max_over_ranks(sum(per_layer_ms))
    e2e = max_over_ranks(e2e)
    co = max_over_ranks(sum(compute_only_ms)) if compute_only_ms else None
    h2d = sum(it2["X"].numel() * it2["X"].element_size() + it2["dY"].numel() * it2["dY"].element_size()
              for it2 in items)
    d2h = sum(it2["dW"].numel() * 4 for it2 in items)   # this rank's dW (slice under kshard)
    # whole-job FLOPs: every rank's local work
    if strong or kshard:   # fixed global problem split over the ranks
        job_flops = sum(it2["layer"].direct_flops for it2 in items)
    else:                  # weak: every rank runs the full per-rank workload
        job_flops = sum(it2["layer"].direct_flops for it2 in items) * world
    return dict(items=items, per_layer_ms=per_layer_ms, warm_ms=warm_ms, compute_only_ms=compute_only_ms,
                graph=graph, dom=dom, dom_ms=dom_ms, dom_alone_ms=dom_alone_ms, e2e_ms=e2e, step_ms=step_ms, compute_only_step_ms=co,
                clocks=clk, h2d=h2d, d2h=d2h, job_flops=job_flops, steps=steps)


def measure_nd(args, dev, flush, peaks, reps=10):
    """N-D (3-D) BFC layers: cold-L2 CUDA-event times of
    winrs_bfc on winrs_plan3d plans, FP16, inputs resident in HBM."""
    import torch
    import paper_conf_icpp_zhangc0zx0025_b200 as W
    from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
    stream = torch.cuda.current_stream(dev)
    out, tot_ms, tot_flops = [], 0.0, 0.0
    for shape in wl.ND_LAYERS:
        name, N, C, D, H, Wd, K, T, R, S, pad = shape
        X, dY = wl.make_inputs_nd(shape, "f16")
        p = W.plan3d(N, C, D, H, Wd, K, T, R, S, pad, "f16")
        Xg, Gg = torch.from_numpy(X).to(dev), torch.from_numpy(dY).to(dev)
        dW = torch.empty((K, T, R, S, C), dtype=torch.float32, device=dev)
        ws = torch.empty(max(16, p.workspace_bytes), dtype=torch.uint8, device=dev)
        for _ in range(3):
            W.bfc(p, Xg, Gg, dW, ws, stream)
        ts = []
        for _ in range(reps):
            flush.fill_(7)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            W.bfc(p, Xg, Gg, dW, ws, stream)
            b.record(stream)
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        ms = statistics.median(ts)
        i = p.info
        Z = i["Z"]
        alg = 2 * (X.size + dY.size) + 4 * dW.numel() * (1 if Z == 1 else 2 * Z + 1)
        t_roof = max(alg / (peaks["hbm_gbs"] * 1e9), i["ewm_flops"] / (peaks["bf16_tflops"] * 1e12))
        out.append({"name": name, "ms": ms, "tflops": i["direct_flops"] / (ms * 1e-3) / 1e12,
                    "kernel": p.kernel_name, "plan": repr(p), "roofline_frac": t_roof / (ms * 1e-3),
                    "workspace_bytes": p.workspace_bytes})
        tot_ms += ms
        tot_flops += i["direct_flops"]
    return {"workload": "nd_f16 (3-D BFC, winrs_plan3d)", "value": tot_flops / (tot_ms * 1e-3) / 1e12,
            "unit": "TFLOPS", "ms_per_step": tot_ms, "steps": reps, "layers": out}


def summarize(m, peaks, args):
    items = m["items"]
    layers = []
    for j, x in enumerate(items):
        rf = layer_roofline(x["local"], x["plan"], m["per_layer_ms"][j], peaks)
        d = {"name": x["layer"].name, "ms": m["per_layer_ms"][j], "warm_ms": m["warm_ms"][j],
             "tflops": x["local"].direct_flops * (x["k1"] - x["k0"]) / x["layer"].K / (m["per_layer_ms"][j] * 1e-3) / 1e12,
             "workspace_bytes": x["plan"].workspace_bytes, "plan": repr(x["plan"]), "kernel": x["plan"].kernel_name,
             "roofline_frac": rf["frac"], "bound": rf["bound"], "t_roof_us": rf["t_roof_us"],
             "t_alu_us": rf["t_alu_us"], "t_l2_us": rf["t_l2_us"]}
        if m["graph"]:
            d["graph_replay_ms"] = m["graph"][j]["mean_ms"]
            d["graph_replay_median_ms"] = m["graph"][j]["median_ms"]
            d["graph_replays"] = m["graph"][j]["replays"]
        if m["compute_only_ms"]:
            d["compute_only_ms"] = m["compute_only_ms"][j]
        layers.append(d)
    return layers


def run_winrs(args):
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    ndev = torch.cuda.device_count()
    torch.cuda.set_device(local % ndev)
    dev = torch.device("cuda", local % ndev)
    backend = None
    if world > 1:
        # NCCL over NVLink/NVSwitch; gloo only when ranks must share a device
        # (fewer GPUs than ranks: a multi-rank check on a 1-GPU box).
        backend = os.environ.get("WINRS_DIST_BACKEND", "nccl" if ndev >= world else "gloo")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    kshard = args.parallel == "kshard" and world > 1
    strong = args.workload == "r50l3" and world > 1 and not kshard
    ctx = dict(world=world, rank=rank, local=local, dev=dev, kshard=kshard, strong=strong,
               fused=args.allreduce == "fused", flush=torch.empty(256 << 20, dtype=torch.uint8, device=dev))
    layers = _workload(args.workload, args.dtype)
    m = measure(layers, args, ctx, primary=True)
    alongside = []
    if world == 1 and not args.no_alongside and args.workload == "vgg":
        for wk, dt in (("r50", "f16"), ("r50", "f32"), ("wide", "f32")):
            a = measure(_workload(wk, dt), args, ctx, primary=False)
            alongside.append((wk, dt, a))

    if rank == 0:
        peaks, src = _peaks()
        value = m["job_flops"] / (m["step_ms"] * 1e-3) / 1e12
        per_layer = summarize(m, peaks, args)
        it = m["items"][m["dom"]]
        rf = layer_roofline(it["local"], it["plan"], m["dom_ms"], peaks)
        if rf["bound"] == "hbm":
            roof = {"bound": "hbm", "achieved": rf["alg_bytes"] / (m["dom_ms"] * 1e-3) / 1e9, "peak": peaks["hbm_gbs"],
                    "unit": "GB/s", "peak_source": src + " hbm_gbs (copy)"}
        elif rf["bound"] == "alu":
            roof = {"bound": "alu", "achieved": rf["ewm_flops"] / (m["dom_ms"] * 1e-3) / 1e12, "peak": rf["pipe_peak_tflops"],
                    "unit": "TFLOP/s", "peak_source": "148 SMs x 128 FP32 lanes x 2 x sm_max_mhz (DESIGN.md §6)"}
        else:
            roof = {"bound": "tensor", "achieved": rf["ewm_flops"] / (m["dom_ms"] * 1e-3) / 1e12,
                    "peak": peaks["bf16_tflops"], "unit": "TFLOP/s", "peak_source": src + " bf16_tflops (fp16 = bf16 rate)"}
        roof["frac"] = roof["achieved"] / roof["peak"]
        roof["traffic"], roof["traffic_source"] = _ncu_traffic(args.dtype, it["layer"].name)
        roof.update(kernel=it["plan"].kernel_name, layer=it["layer"].name, alg_bytes=rf["alg_bytes"],
                    ewm_flops=rf["ewm_flops"], kernel_ms=m["dom_ms"], kernel_alone_ms=m["dom_alone_ms"], t_alu_us=rf["t_alu_us"], t_l2_us=rf["t_l2_us"],
                    per_layer_frac={d["name"]: round(d["roofline_frac"], 4) for d in per_layer},
                    worst_layer=min(per_layer, key=lambda d: d["roofline_frac"])["name"])
        cfg = {"workload": f"{args.workload}_{args.dtype}: " + ", ".join(x["layer"].name for x in m["items"]),
               "global_batch": (m["items"][0]["layer"].N if (strong or kshard) else m["items"][0]["layer"].N * world),
               "parallelism": (f"kshard{world}" if kshard else f"dp{world}") if world > 1 else "single",
               "allreduce": (args.allreduce if world > 1 and not kshard else None),
               "backend": backend,
               "l2": "flushed (256 MiB write) before every layer call; flush outside timed events",
               "workspace_cap": float(os.environ.get("WINRS_WS_CAP", "0.04")),
               "warm_l2_ms_per_step": sum(m["warm_ms"]),
               "layers": per_layer}
        if m["graph"]:
            cfg["graph_replay_ms_per_step"] = sum(g["mean_ms"] for g in m["graph"])
            cfg["graph_replay_tflops"] = m["job_flops"] / world / (cfg["graph_replay_ms_per_step"] * 1e-3) / 1e12 \
                if world == 1 else None
        if m["compute_only_step_ms"]:
            cfg["compute_only_ms_per_step"] = m["compute_only_step_ms"]
            cfg["compute_only_tflops"] = m["job_flops"] / (m["compute_only_step_ms"] * 1e-3) / 1e12
            cfg["allreduce_share"] = 1.0 - m["compute_only_step_ms"] / m["step_ms"]
        if world == 1 and not args.no_alongside and args.workload == "vgg":
            cfg.setdefault("alongside", []).append(measure_nd(args, ctx["dev"], ctx["flush"], peaks))
        for wk, dt, a in alongside:
            cfg.setdefault("alongside", []).append({
                "workload": f"{wk}_{dt}", "value": a["job_flops"] / (a["step_ms"] * 1e-3) / 1e12, "unit": "TFLOPS",
                "ms_per_step": a["step_ms"], "steps": a["steps"],
                "e2e_tflops": a["job_flops"] / (a["e2e_ms"] * 1e-3) / 1e12,
                "layers": summarize(a, peaks, args)})
        out = {
            "metric": METRIC,
            "value": value,
            "unit": "TFLOPS",
            "n_gpus": world,
            "steps": m["steps"],
            "warmup": args.warmup,
            "ms_per_step": m["step_ms"],
            "higher_is_better": True,
            "scaling": "strong" if (kshard or strong) else "weak",
            "vs_baseline": None,
            "dtype": args.dtype,
            "data": "synthetic (seeded U[0,1), dY x 1e-2 for f16; PAPER.md P@50685)",
            "config": cfg,
            "roofline": roof,
            "e2e": {"value": m["job_flops"] / (m["e2e_ms"] * 1e-3) / 1e12, "unit": "TFLOPS",
                    "h2d_bytes_per_step": m["h2d"], "d2h_bytes_per_step": m["d2h"], "ms_per_step": m["e2e_ms"]},
            "gpu_launches": sum(x["plan"].launch_count for x in m["items"]) * m["steps"],
            "clocks": m["clocks"],
        }
        if not args.no_cpu_baseline:
            out["cpu_baseline"] = cpu_baseline(layers, budget_s=args.cpu_seconds)
        print(json.dumps(out))
    if world > 1:
        dist.destroy_process_group()


def run_dry(args):
    """--dry-run: the launch / rank plumbing only (gloo, CPU tensors)."""
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if world > 1:
        import torch
        import torch.distributed as dist
        dist.init_process_group("gloo")
        t = torch.tensor([float(rank + 1)])
        dist.all_reduce(t)
        total = float(t.item())
        dist.barrier()
        dist.destroy_process_group()
    else:
        total = 1.0
    if rank == 0:
        print(json.dumps({"metric": METRIC, "dry_run": True, "n_gpus": world, "ranks_sum": total,
                          "workload": args.workload, "parallel": args.parallel}))


def cpu_baseline(layers, budget_s: float = 8.0):
    """The FP64 oracle (oracle/, as it stands) on a bounded sample of the same
    workload: each layer with its batch cut to the first n images, n grown
    until the CPU time budget is used.  Reported in the same metric."""
    from oracle import oracle as O
    from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
    threads = len(os.sched_getaffinity(0))
    n = 1
    flops = 0.0
    elapsed = 0.0
    while True:
        t0 = time.perf_counter()
        f = 0.0
        for l in layers:
            s = l.with_(N=n)
            X, dY = wl.make_inputs(s)
            O.bfc_c(X, dY, s.R, s.S, s.pad, threads=threads)
            f += s.direct_flops
        dt = time.perf_counter() - t0
        flops, elapsed = f, dt
        if dt * 2 > budget_s or n * 2 > layers[0].N:
            break
        n *= 2
    return {"value": flops / elapsed / 1e12, "unit": "TFLOPS", "cores": threads, "kind": "oracle",
            "sample": f"every layer of the workload with N cut to {n} image(s) ({flops / 1e9:.2f} GFLOP, "
                      f"{elapsed:.1f} s, FP64 C loop, OpenMP over k)"}


def run_reference(args):
    """--impl reference: the FP64 CPU oracle timed on the box's host cores on a
    bounded sample per step; rank 0 only."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from oracle import oracle as O
    from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
    layers = _workload(args.workload, args.dtype)
    threads = len(os.sched_getaffinity(0))
    sample = [l.with_(N=1) for l in layers]
    inputs = [wl.make_inputs(s) for s in sample]
    for _ in range(args.warmup):
        O.bfc_c(*inputs[0], sample[0].R, sample[0].S, sample[0].pad, threads=threads)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        for s, (X, dY) in zip(sample, inputs):
            O.bfc_c(X, dY, s.R, s.S, s.pad, threads=threads)
    dt = (time.perf_counter() - t0) / args.steps
    flops = sum(s.direct_flops for s in sample)
    v = flops / dt / 1e12
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": v, "unit": "TFLOPS", "n_gpus": int(os.environ.get("WORLD_SIZE", "1")),
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{args.workload}_{args.dtype} (each layer at N=1)"},
        "cpu_baseline": {"value": v, "unit": "TFLOPS", "cores": threads, "kind": "oracle",
                         "sample": "every layer of the workload at N=1 per step"},
        "e2e": {"value": v, "unit": "TFLOPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }))


def _free_port():
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        return so.getsockname()[1]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="winrs", choices=["winrs", "reference"])
    ap.add_argument("--workload", default="vgg", choices=["vgg", "r50", "wide", "r50l3"])
    ap.add_argument("--dtype", default=os.environ.get("WINRS_BENCH_DTYPE", "f16"), choices=["f32", "f16", "bf16"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-alongside", action="store_true", help="skip the ResNet-50 / wide workloads measured alongside")
    ap.add_argument("--no-graphs", action="store_true", help="skip the CUDA-graph replay timing")
    ap.add_argument("--graph-reps", type=int, default=0)
    ap.add_argument("--cpu-seconds", type=float, default=8.0)
    ap.add_argument("--parallel", default="dp", choices=["dp", "kshard"],
                    help="N>1: dp = batch shards + one all_reduce of dW; kshard = output-channel "
                         "shards of the full batch, no communication (strong)")
    ap.add_argument("--allreduce", default="nccl", choices=["nccl", "fused"],
                    help="N>1 dp: nccl = bucket reduction, then one NCCL all_reduce; fused = both in one "
                         "kernel over CUDA-IPC peer memory (winrs_bfc_allreduce)")
    ap.add_argument("--ws-cap", type=float, default=None,
                    help="planner workspace cap as a fraction of X+dY bytes (default: the paper's 4%%)")
    ap.add_argument("--dry-run", action="store_true", help="launch plumbing only (gloo, no GPU work)")
    args = ap.parse_args()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        # one rank per GPU: re-launch under torch.distributed.run on this node
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), os.path.abspath(__file__)] + sys.argv[1:]
        import subprocess
        sys.exit(subprocess.call(cmd))
    if args.ws_cap is not None:
        os.environ["WINRS_WS_CAP"] = str(args.ws_cap)
    if args.warmup < 3:
        args.warmup = 3
    if args.workload in ("wide",):
        args.dtype = "f32"
    if args.workload in ("vgg", "r50l3"):
        args.dtype = "f16"
    if args.dry_run:
        run_dry(args)
    elif args.impl == "reference":
        run_reference(args)
    else:
        run_winrs(args)


if __name__ == "__main__":
    main()
