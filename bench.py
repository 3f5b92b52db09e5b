#!/usr/bin/env python3
"""Benchmark of the WinRS fused Winograd BFC on B200 (BASELINE.json metric:
effective TFLOPS = direct-conv FLOPs 2*N*C*K*Ho*Wo*R*S / device time, plus
workspace bytes).

A "step" is one pass of the whole hot path (plan is prebuilt; fused kernels +
bucket reduction) over every layer of the workload, inputs resident in HBM.
Default workload: configs[1] of BASELINE.json — the four ResNet-50 3x3 layers
at N=64 (C=K=64/128/256/512, H=W=56/28/14/7, pad 1).  L2 is flushed (a
256 MiB write) before every layer call and each call is timed with CUDA events
on the launch stream (the flush is outside the timed events).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--dtype f16|f32] [--impl winrs|reference]

N > 1 (torchrun): each rank runs the same per-rank workload on its own batch
shard (weak scaling: global batch = N * 64) followed by one NCCL all_reduce of
each layer's dW — the batch-sharded data-parallel BFC; time = max over ranks.
--impl reference runs the FP64 CPU oracle (the only reference this paper-only
tier has) on a bounded sample of the same workload, rank 0 only.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

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
    if dtype in t and base in t.get("layers", []):
        i = t["layers"].index(base)
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


def run_winrs(args):
    import torch
    import torch.distributed as dist
    import paper_conf_icpp_zhangc0zx0025_b200 as W
    from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    ndev = torch.cuda.device_count()
    torch.cuda.set_device(local % ndev)
    dev = torch.device("cuda", local % ndev)
    if world > 1:
        # NCCL over NVLink/NVSwitch; WINRS_DIST_BACKEND=gloo only to exercise the
        # multi-rank path on a single-GPU box (ranks sharing one device).
        backend = os.environ.get("WINRS_DIST_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    layers = _workload(args.workload, args.dtype)
    tdt = torch.float32 if args.dtype == "f32" else torch.float16

    # Inputs resident in HBM, plans prebuilt.  dp: each rank has its own
    # seeded batch shard (weak scaling); kshard: every rank holds the full
    # batch and computes its slice of the output channels (strong scaling, no
    # communication: BASELINE's K-sharding alternative).
    kshard = args.parallel == "kshard" and world > 1
    items = []
    for l in layers:
        X, dY = wl.make_inputs(l, seed_offset=0 if kshard else 1000 * rank)
        align = 4 if l.dtype == "f32" else 8
        if kshard:
            a, b = W.shard_range(l.K // align, world, rank)
            k0, k1 = a * align, b * align
        else:
            k0, k1 = 0, l.K
        p = W.plan(l.N, l.C, l.H, l.W, k1 - k0, l.R, l.S, l.pad, l.dtype)
        Xt, Gt = torch.from_numpy(X), torch.from_numpy(dY)
        if l.dtype == "bf16":   # workloads carries bf16 values in float32
            Xt, Gt = Xt.to(torch.bfloat16), Gt.to(torch.bfloat16)
        Xg = Xt.to(dev)
        Gg = Gt.to(dev)
        dW = torch.empty((k1 - k0, l.R, l.S, l.C), dtype=torch.float32, device=dev)
        ws = torch.empty(max(p.workspace_bytes, 16), dtype=torch.uint8, device=dev)
        items.append(dict(layer=l, plan=p, X=Xg, dY=Gg, dW=dW, ws=ws, Xh=Xt.pin_memory(),
                          Gh=Gt.pin_memory(), dWh=torch.empty(dW.shape).pin_memory(),
                          k0=k0, k1=k1, flops=l.direct_flops * (k1 - k0) / l.K))

    def run_bfc(it, stream):
        if kshard:   # channel slice of dY read in place (ldy = K), no communication
            from paper_conf_icpp_zhangc0zx0025_b200 import _lib
            _lib.check(_lib.lib().winrs_bfc_strided(it["plan"].handle, it["X"].data_ptr(),
                                                    it["dY"].data_ptr() + it["k0"] * it["dY"].element_size(),
                                                    it["layer"].K, it["dW"].data_ptr(), it["ws"].data_ptr(),
                                                    stream.cuda_stream), "winrs_bfc_strided")
        else:
            W.bfc(it["plan"], it["X"], it["dY"], it["dW"], it["ws"], stream)
            if world > 1:
                dist.all_reduce(it["dW"])
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream(dev)

    def one_step(timed_events=None):
        for j, it in enumerate(items):
            flush.fill_(j & 0xFF)                                  # evict L2 (outside the events)
            if timed_events is not None:
                timed_events[j][0].record(stream)
            run_bfc(it, stream)
            if timed_events is not None:
                timed_events[j][1].record(stream)

    for _ in range(args.warmup):
        one_step()
    torch.cuda.synchronize()

    clocks = ClockSampler(local)
    if rank == 0:
        clocks.start()
    ev = [[[torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)] for _ in items]
          for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    for s in range(args.steps):
        one_step(ev[s])
        if rank == 0:
            clocks.sample()                                        # GPU busy with the queued layers
    if rank == 0:
        while not ev[-1][-1][1].query():                           # GPU still draining the steps
            clocks.sample()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop() if rank == 0 else None

    per_layer_ms = [sum(ev[s][j][0].elapsed_time(ev[s][j][1]) for s in range(args.steps)) / args.steps
                    for j in range(len(items))]
    step_ms = sum(per_layer_ms)
    if world > 1:
        t = torch.tensor([step_ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        step_ms = float(t.item())

    # Secondary numbers: warm-L2 per-layer time (no flush between
    # calls) and, for N > 1, the compute-only time without the all_reduce.
    def time_layers(flush_l2, with_allreduce, reps=5):
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
                if with_allreduce:
                    run_bfc(it2, stream)
                elif kshard:
                    run_bfc(it2, stream)
                else:
                    W.bfc(it2["plan"], it2["X"], it2["dY"], it2["dW"], it2["ws"], stream)
                b.record(stream)
                torch.cuda.synchronize()
                ts.append(a.elapsed_time(b))
            out.append(statistics.median(ts))
        return out
    warm_ms = time_layers(False, world > 1)
    compute_only_ms = time_layers(True, False) if world > 1 else None

    # Dominant kernel's live duration: time the fused kernel alone (no
    # all_reduce) for the layer with the largest share, CUDA events on the stream.
    dom = max(range(len(items)), key=lambda j: per_layer_ms[j])
    it = items[dom]
    p = it["plan"]
    info = p.info
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    kt = []
    for _ in range(max(3, args.steps)):
        flush.fill_(1)
        e0.record(stream)
        if kshard:
            run_bfc(it, stream)
        else:
            W.bfc(p, it["X"], it["dY"], it["dW"], it["ws"], stream)
        e1.record(stream)
        torch.cuda.synchronize()
        kt.append(e0.elapsed_time(e1))
    dom_ms = statistics.median(kt)

    # End to end through the C ABI with host buffers (pinned), copies inside.
    e2e_ms = []
    for _ in range(max(2, min(args.steps, 5))):
        tot = 0.0
        for it2 in items:
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            dX = torch.empty_like(it2["X"])
            dG = torch.empty_like(it2["dY"])
            a.record(stream)
            if kshard or world > 1:   # H2D, the BFC (+ all_reduce for dp), D2H of (this rank's) dW
                dX.copy_(it2["Xh"], non_blocking=True)
                dG.copy_(it2["Gh"], non_blocking=True)
                it3 = dict(it2, X=dX, dY=dG)
                run_bfc(it3, stream)
                it2["dWh"].copy_(it2["dW"], non_blocking=True)
                stream.synchronize()
            else:
                W.bfc_host(it2["plan"], it2["Xh"], it2["Gh"], it2["dWh"], dX, dG, it2["dW"], it2["ws"], stream)
            b.record(stream)
            torch.cuda.synchronize()
            tot += a.elapsed_time(b)
        e2e_ms.append(tot)
    e2e = statistics.median(e2e_ms)
    if world > 1:
        t = torch.tensor([e2e], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e = float(t.item())

    if rank == 0:
        flops = sum(it["layer"].direct_flops for it in items) * (1 if kshard else world)
        value = flops / (step_ms * 1e-3) / 1e12
        peaks, src = _peaks()
        esz = 4 if args.dtype == "f32" else 2   # f16 / bf16
        l = it["layer"]
        alg_bytes = esz * (l.N * l.H * l.W * l.C + l.N * l.Ho * l.Wo * l.K) + 4 * l.K * l.R * l.S * l.C * (
            1 if info["Z"] == 1 else 2 * info["Z"] + 1)
        if args.dtype == "f32":
            peak = 148 * 128 * 2 * float(peaks.get("sm_max_mhz", 1965.0)) * 1e6 / 1e12
            roof = {"bound": "alu", "achieved": info["ewm_flops"] / (dom_ms * 1e-3) / 1e12, "peak": peak,
                    "unit": "TFLOP/s", "peak_source": "148 SMs x 128 FP32 lanes x 2 x sm_max_mhz (DESIGN.md)",
                    "kernel": p.kernel_name, "layer": l.name}
        else:
            t_hbm = alg_bytes / (peaks["hbm_gbs"] * 1e9)
            t_tc = info["ewm_flops"] / (peaks["bf16_tflops"] * 1e12)
            if t_hbm >= t_tc:
                roof = {"bound": "hbm", "achieved": alg_bytes / (dom_ms * 1e-3) / 1e9, "peak": peaks["hbm_gbs"],
                        "unit": "GB/s", "peak_source": src}
            else:
                roof = {"bound": "tensor", "achieved": info["ewm_flops"] / (dom_ms * 1e-3) / 1e12,
                        "peak": peaks["bf16_tflops"], "unit": "TFLOP/s", "peak_source": src + " (fp16 = bf16 rate)"}
            roof.update(kernel=p.kernel_name, layer=l.name)
        roof["frac"] = roof["achieved"] / roof["peak"]
        roof["traffic"], roof["traffic_source"] = _ncu_traffic(args.dtype, l.name)
        roof["alg_bytes"] = alg_bytes
        roof["ewm_flops"] = info["ewm_flops"]
        roof["kernel_ms"] = dom_ms
        h2d = sum(it2["X"].numel() * it2["X"].element_size() + it2["dY"].numel() * it2["dY"].element_size()
                  for it2 in items)
        d2h = sum(it2["dW"].numel() * 4 for it2 in items)   # this rank's dW (slice under kshard)
        out = {
            "metric": METRIC,
            "value": value,
            "unit": "TFLOPS",
            "n_gpus": world,
            "steps": args.steps,
            "warmup": args.warmup,
            "ms_per_step": step_ms,
            "higher_is_better": True,
            "scaling": "strong" if kshard else "weak",
            "vs_baseline": None,
            "dtype": args.dtype,
            "data": "synthetic (seeded U[0,1), dY x 1e-2 for f16; PAPER.md P@50685)",
            "config": {"workload": f"{args.workload}_{args.dtype}: " + ", ".join(x["layer"].name for x in items),
                       "global_batch": layers[0].N * (1 if kshard else world),
                       "parallelism": (f"kshard{world}" if kshard else f"dp{world}") if world > 1 else "single",
                       "l2": "flushed (256 MiB write) before every layer call; flush outside timed events",
                       "workspace_cap": float(os.environ.get("WINRS_WS_CAP", "0.04")),
                       "warm_l2_ms_per_step": sum(warm_ms),
                       "compute_only_ms_per_step": sum(compute_only_ms) if compute_only_ms else None,
                       "layers": [{"name": x["layer"].name, "ms": per_layer_ms[j], "warm_ms": warm_ms[j],
                                   "tflops": x["layer"].direct_flops / (per_layer_ms[j] * 1e-3) / 1e12,
                                   "workspace_bytes": x["plan"].workspace_bytes, "plan": repr(x["plan"]),
                                   "kernel": x["plan"].kernel_name} for j, x in enumerate(items)]},
            "roofline": roof,
            "e2e": {"value": flops / (e2e * 1e-3) / 1e12, "unit": "TFLOPS", "h2d_bytes_per_step": h2d,
                    "d2h_bytes_per_step": d2h, "ms_per_step": e2e},
            "gpu_launches": sum(x["plan"].launch_count for x in items) * args.steps,
            "clocks": clk,
        }
        if not args.no_cpu_baseline:
            out["cpu_baseline"] = cpu_baseline(layers, budget_s=args.cpu_seconds)
        print(json.dumps(out))
    if world > 1:
        dist.destroy_process_group()


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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="winrs", choices=["winrs", "reference"])
    ap.add_argument("--workload", default="r50", choices=["r50", "vgg", "wide", "r50l3"])
    ap.add_argument("--dtype", default=os.environ.get("WINRS_BENCH_DTYPE", "f16"), choices=["f32", "f16", "bf16"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=8.0)
    ap.add_argument("--parallel", default="dp", choices=["dp", "kshard"],
                    help="N>1: dp = batch shards + one all_reduce of dW (weak); kshard = output-channel "
                         "shards of the full batch, no communication (strong)")
    ap.add_argument("--ws-cap", type=float, default=None,
                    help="planner workspace cap as a fraction of X+dY bytes (default: the paper's 4%%)")
    args = ap.parse_args()
    if args.ws_cap is not None:
        os.environ["WINRS_WS_CAP"] = str(args.ws_cap)
    if args.warmup < 3:
        args.warmup = 3
    if args.workload in ("wide",):
        args.dtype = "f32"
    if args.workload in ("vgg", "r50l3"):
        args.dtype = "f16"
    if args.impl == "reference":
        run_reference(args)
    else:
        run_winrs(args)


if __name__ == "__main__":
    main()
