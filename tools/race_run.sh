#!/bin/bash
# Run tools/race_diag.py for every gpulibs/lib_*.so (race-investigation variant builds).
OUT=${OUT:-gpurun_out/race}; mkdir -p $OUT
for l in ${LIBS:-gpulibs/lib_*.so}; do
  n=$(basename $l .so)
  for f in ${FAMS:-d1,d2}; do
    BARRACUDA_LIB=$PWD/$l timeout 300 python tools/race_diag.py --repeats ${REPEATS:-100} --fams $f --dump $OUT/$n.$f.json >> $OUT/summary.jsonl 2>> $OUT/err.txt
  done
done
cat $OUT/summary.jsonl
