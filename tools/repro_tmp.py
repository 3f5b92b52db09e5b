import os, sys, time, torch, numpy as np
sys.path.insert(0, '/root/repo')
import paper_conf_icpp_zhangc0zx0025_b200 as W
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
l = wl.LAYERS[os.environ.get("LAYER", "vgg_128_128_112_f16")]
X, dY = wl.make_inputs(l)
Xg, Gg = torch.from_numpy(X).cuda(), torch.from_numpy(dY).cuda()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
seq = sys.argv[1].split(",")
for step in seq:
    name, reps = step.split(":")
    for k in ("WINRS_TC_GEN", "WINRS_FORCE_TA", "WINRS_FORCE_CSPLIT", "WINRS_FORCE_TILE"):
        os.environ.pop(k, None)
    if name == "ta": os.environ["WINRS_FORCE_TA"] = "1"
    if name == "nota": os.environ["WINRS_FORCE_TA"] = "0"
    if name == "gen1": os.environ["WINRS_TC_GEN"] = "1"
    if name.startswith("gen1cs"): os.environ.update(WINRS_TC_GEN="1", WINRS_FORCE_CSPLIT=name[6:])
    if name.startswith("gen1t"): os.environ.update(WINRS_TC_GEN="1", WINRS_FORCE_TILE="128x128", WINRS_FORCE_CSPLIT=name[5:])
    p = W.plan(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
    l_dw = torch.empty((p.info["K"], p.info["R"], p.info["S"], p.info["C"]), device="cuda")
    ws = torch.empty(max(16, p.workspace_bytes), dtype=torch.uint8, device="cuda")
    try:
        for i in range(int(reps)):
            flush.fill_(i)
            W.bfc(p, Xg, Gg, l_dw, ws)
            torch.cuda.synchronize()
        print(step, p.kernel_name, p.info["csplit"], "ok", flush=True)
    except Exception as e:
        print(step, p.kernel_name, p.info["csplit"], "FAIL", str(e)[:80], flush=True)
        break
