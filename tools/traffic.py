#!/usr/bin/env python3
"""Write profiles/<round>/traffic.json (DRAM bytes read + written per launch,
one launch per ResNet-50 layer in bench order) from the ncu --set full
captures tools/profile_round.sh brings back.  bench.py reads it for
roofline.traffic.  Usage: python tools/traffic.py [round_dir]"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def launches(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, vals = rows[0], rows[2:]
    get = lambda r, k: r[h.index(k)]
    res = []
    for r in vals:
        rd = float(get(r, "dram__bytes_read.sum"))
        wr = float(get(r, "dram__bytes_write.sum"))
        # ncu reports bytes in the unit row (rows[1]); normalise to bytes
        u_rd, u_wr = rows[1][h.index("dram__bytes_read.sum")], rows[1][h.index("dram__bytes_write.sum")]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        res.append({"kernel": get(r, "Kernel Name")[:80], "dram_bytes": rd * scale.get(u_rd, 1) + wr * scale.get(u_wr, 1),
                    "duration_us": float(get(r, "gpu__time_duration.sum")) *
                    {"usecond": 1, "nsecond": 1e-3, "msecond": 1e3}.get(rows[1][h.index("gpu__time_duration.sum")], 1)})
    return res


def main():
    rnd = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "r01")
    t = {"layers": ["r50_c64_56", "r50_c128_28", "r50_c256_14", "r50_c512_7"],
         "note": "dram__bytes_read.sum + dram__bytes_write.sum per launch, ncu --set full --clock-control none, "
                 "one launch per ResNet-50 layer in bench order (tools/profile_round.sh)"}
    for dt in ("f16", "f32"):
        rep = os.path.join(ROOT, "gpurun_out", "prof_%s.ncu-rep" % dt)
        if os.path.exists(rep):
            t[dt] = launches(rep)
    with open(os.path.join(rnd, "traffic.json"), "w") as f:
        json.dump(t, f, indent=1)
    print(json.dumps(t, indent=1))


if __name__ == "__main__":
    main()
