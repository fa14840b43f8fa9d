#!/bin/bash
# Run tools/sweep_spectral.py for every varlibs/lib_*.so (variant builds), under gpurun.
OUT=${OUT:-gpurun_out}; mkdir -p $OUT
for l in ${LIBS:-varlibs/lib_*.so}; do
  BARRACUDA_LIB=$PWD/$l timeout 600 python tools/sweep_spectral.py ${PS:-4 5 6 7 8 9 10 11 12} >> $OUT/sweep.jsonl 2>> $OUT/sweep.err
done
cat $OUT/sweep.jsonl
