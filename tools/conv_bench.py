"""Time winrs_fc / winrs_bdc on a few layers, split into
the layout kernels and the mapped BFC, with cuDNN's conv2d / conv2d_input of
the same layer timed alongside as context.  Prints one JSON line per case."""
import json
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
import paper_conf_icpp_zhangc0zx0025_b200 as W  # noqa: E402

LAYERS = [
    ("r50_l3", 64, 256, 14, 14, 256, 3, 3, 1),
    ("r50_l2", 64, 128, 28, 28, 128, 3, 3, 1),
    ("r50_l4", 64, 512, 7, 7, 512, 3, 3, 1),
    ("vgg_l3", 32, 256, 56, 56, 256, 3, 3, 1),
]


def t_ms(fn, it=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(it):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / it


def main():
    dt = sys.argv[1] if len(sys.argv) > 1 else "f16"
    tdt = {"f16": torch.float16, "bf16": torch.bfloat16, "f32": torch.float32}[dt]
    for name, N, C, H, Wd, K, R, S, pad in LAYERS:
        Ho, Wo = H + 2 * pad - R + 1, Wd + 2 * pad - S + 1
        flops = 2.0 * N * C * K * Ho * Wo * R * S
        X = torch.rand(N, H, Wd, C, device="cuda").to(tdt)
        dY = torch.rand(N, Ho, Wo, K, device="cuda").to(tdt)
        Wt = torch.rand(K, R, S, C, device="cuda").to(tdt)
        Xc = X.permute(0, 3, 1, 2)
        dYc = dY.permute(0, 3, 1, 2)
        Wc = Wt.permute(0, 3, 1, 2)
        for kind in ("fc", "bdc"):
            try:
                cp = W.conv_plan(kind, N, C, H, Wd, K, R, S, pad, dtype=dt)
            except Exception as e:
                print(json.dumps({"layer": name, "kind": kind, "unsupported": str(e)}))
                continue
            ws = torch.empty(cp.workspace_bytes, dtype=torch.uint8, device="cuda")
            if kind == "fc":
                ms = t_ms(lambda: W.fc(cp, X, Wt, workspace=ws))
                ref = t_ms(lambda: torch.nn.functional.conv2d(Xc, Wc, padding=pad))
            else:
                ms = t_ms(lambda: W.bdc(cp, dY, Wt, workspace=ws))
                ref = t_ms(lambda: torch.nn.grad.conv2d_input((N, C, H, Wd), Wc, dYc, padding=pad))
            # the mapped BFC alone (the layout kernels are the difference)
            b = cp.bfc
            i = b.info
            bx = torch.empty(i["N"], i["H"], i["W"], i["C"], device="cuda", dtype=tdt)
            by = torch.empty(i["N"], i["Ho"], i["Wo"], i["K"], device="cuda", dtype=tdt)
            bms = t_ms(lambda: W.bfc(b, bx, by))
            print(json.dumps({"layer": name, "kind": kind, "dtype": dt, "ms": round(ms, 4),
                              "eff_tflops": round(flops / ms / 1e9, 1), "bfc_ms": round(bms, 4),
                              "layout_ms": round(ms - bms, 4), "kernel": cp.kernel_name,
                              "plan": repr(b), "cudnn_ms": round(ref, 4)}), flush=True)


if __name__ == "__main__":
    main()
