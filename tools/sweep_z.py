import os, sys, time, statistics, json
sys.path.insert(0, os.getcwd())
import faulthandler
import torch
import paper_conf_icpp_zhangc0zx0025_b200 as W
from paper_conf_icpp_zhangc0zx0025_b200 import workloads as wl
t0 = time.time()
names = sys.argv[1].split(",")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for name in names:
    l = wl.LAYERS[name]
    X, dY = wl.make_inputs(l)
    Xg, Gg = torch.from_numpy(X).cuda(), torch.from_numpy(dY).cuda()
    print("inputs", name, round(time.time() - t0, 1), flush=True)
    cfgs = [None] + [(z, t, cs) for z in range(1, 15) for t in ("128x64", "128x128") for cs in (2, 4, 8)]
    for cfg in cfgs:
        for k in ("WINRS_FORCE_Z", "WINRS_FORCE_TILE", "WINRS_FORCE_CSPLIT"):
            os.environ.pop(k, None)
        if cfg:
            os.environ["WINRS_FORCE_Z"], os.environ["WINRS_FORCE_TILE"], os.environ["WINRS_FORCE_CSPLIT"] = str(cfg[0]), cfg[1], str(cfg[2])
        ta = time.time()
        faulthandler.dump_traceback_later(30, exit=True)
        print('cfg', cfg, file=sys.stderr, flush=True)
        try:
            p = W.plan(l.N, l.C, l.H, l.W, l.K, l.R, l.S, l.pad, l.dtype)
        except Exception as e:
            continue
        data = l.N * (l.H * l.W * l.C + p.info["Ho"] * p.info["Wo"] * l.K) * 2
        if cfg and p.workspace_bytes > 0.04 * data:
            continue
        dW = torch.empty((l.K, l.R, l.S, l.C), device="cuda")
        ws = torch.empty(max(16, p.workspace_bytes), dtype=torch.uint8, device="cuda")
        ts = []
        for i in range(12):
            flush.fill_(i)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); W.bfc(p, Xg, Gg, dW, ws); b.record()
            torch.cuda.synchronize()
            if i >= 2:
                ts.append(a.elapsed_time(b))
        print(json.dumps({"layer": name, "cfg": cfg, "plan": repr(p), "ctas": p.info["ctas_main"],
                          "us": round(statistics.median(ts) * 1e3, 1), "wall_s": round(time.time() - ta, 2)}), flush=True)
