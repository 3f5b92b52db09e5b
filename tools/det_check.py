#!/usr/bin/env python3
"""Determinism stress: N cold-L2 calls of one plan (256 MB buffer rewritten
between calls) must give bitwise identical dW.  Prints one line per
(layer, env).  Usage: python tools/det_check.py layer[,layer] 'ENV=V;ENV=V' ... [--reps N]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_zhangc0zx0025_b200 as W  # noqa: E402
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl  # noqa: E402

KEYS = ("WINRS_TC_GEN", "WINRS_FORCE_TA", "WINRS_FORCE_CSPLIT", "WINRS_FORCE_TILE", "WINRS_FORCE_Z", "WINRS_FORCE_PAIR",
        "WINRS_FORCE_CG")


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    reps = 30
    if "--reps" in sys.argv:
        reps = int(sys.argv[sys.argv.index("--reps") + 1])
        args = [a for a in args if a != str(reps)]
    layers, envs = args[0].split(","), args[1:] or [""]
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for name in layers:
        base, *ov = name.split("@")            # layer@K=V@K=V: overrides (ints)
        l = wl.LAYERS[base].with_(name=name, **{k: int(v) for k, v in (o.split("=") for o in ov)})
        X, dY = wl.make_inputs(l)
        to = (lambda a: torch.from_numpy(a).cuda().to(torch.bfloat16)) if l.dtype == "bf16" else (lambda a: torch.from_numpy(a).cuda())
        Xg, Gg = to(X), to(dY)
        for es in envs:
            for k in KEYS:
                os.environ.pop(k, None)
            for kv in filter(None, es.split(";")):
                k, v = kv.split("=")
                os.environ[k] = v
            try:
                p = W.plan(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
            except Exception as e:
                print(f"{name:22s} {es:50s} plan: {e}", flush=True)
                continue
            dW = torch.empty((l.K, l.R, l.S, l.C), device="cuda")
            ws = torch.empty(max(16, p.workspace_bytes), dtype=torch.uint8, device="cuda")
            first, bad, maxd, ts = None, 0, 0.0, []
            try:
                for i in range(reps):
                    flush.fill_(i & 0xFF)
                    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    a.record()
                    W.bfc(p, Xg, Gg, dW, ws)
                    b.record()
                    torch.cuda.synchronize()
                    ts.append(a.elapsed_time(b))
                    if first is None:
                        first = dW.clone()
                    elif not torch.equal(dW, first):
                        bad += 1
                        maxd = max(maxd, float((dW - first).abs().max() / first.abs().max()))
                ts = sorted(ts[1:] or ts)
                status = f"mismatching calls {bad}/{reps - 1} max rel diff {maxd:.2e}  median {ts[len(ts) // 2] * 1e3:.1f} us"
            except Exception as e:
                status = f"ERROR {str(e)[:60]}"
                print(f"{name:22s} {es:50s} {p.kernel_name:30s} cs={p.info['csplit']} Z={p.info['Z']} {status}", flush=True)
                return 1
            print(f"{name:22s} {es:50s} {p.kernel_name:30s} cs={p.info['csplit']} Z={p.info['Z']} {status}", flush=True)
    return 0


if __name__ == "__main__":
    sys.exit(main())
