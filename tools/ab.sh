#!/bin/bash
# A/B the in-tree library variants on the GPU box: bench per variant (no CPU
# baseline), one JSON line each under gpurun_out/ab_<variant>_<workload>.json.
# Usage: VARIANTS="libwinrs.so libwinrs_x.so" WORKLOADS="r50 vgg" bash tools/ab.sh [extra bench args]
mkdir -p gpurun_out
for v in ${VARIANTS:-libwinrs.so}; do
  for w in ${WORKLOADS:-r50}; do
    tag=${v#libwinrs}; tag=${tag%.so}; tag=${tag#_}; tag=${tag:-main}
    WINRS_LIB=$v timeout 300 python bench.py --workload $w --no-cpu-baseline --steps 10 "$@" \
      > gpurun_out/ab_${tag}_${w}.json 2> gpurun_out/ab_${tag}_${w}.err
  done
done
python - <<'PY'
import glob, json
for f in sorted(glob.glob("gpurun_out/ab_*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "FAILED", e); continue
    print(f, "%.1f TFLOPS" % d["value"], " ".join("%s=%.1fus" % (l["name"].split("_f")[0], l["ms"] * 1e3) for l in d["config"]["layers"]))
PY
