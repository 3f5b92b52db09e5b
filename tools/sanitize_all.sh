# compute-sanitizer record (round 2): every tool over tools/sanitize.py
mkdir -p gpurun_out
for T in memcheck initcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $T --print-limit 20 python tools/sanitize.py > gpurun_out/san_$T.log 2>&1
  echo "$T rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' gpurun_out/san_$T.log | tail -1)"
done
