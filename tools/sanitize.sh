#!/bin/bash
# compute-sanitizer (memcheck, racecheck, synccheck, initcheck) over tools/sanitize_smoke.py
# (every kernel family, both spectral operator paths, DMMA spectral sizes), under gpurun.
OUT=${OUT:-gpurun_out}; mkdir -p $OUT
for t in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $t --print-limit 100000 python tools/sanitize_smoke.py > $OUT/sanitizer_$t.txt 2>&1
  echo "$t rc=$? $(tail -1 $OUT/sanitizer_$t.txt)"
done
