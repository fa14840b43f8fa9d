#!/bin/bash
# ncu --set full of the p=12 spectral kernels (one launch each, after warm-up), under gpurun.
OUT=${OUT:-gpurun_out}; mkdir -p $OUT
for k in ${KERNELS:-sumfact3d local_grad3 sumfact2d}; do
  ncu --set full --clock-control none --import-source on -k regex:${k}_kernel -s 2 -c 1 \
     -o $OUT/prof_$k -f python tools/sweep_spectral.py 12 > $OUT/prof_$k.log 2>&1
done
ls -la $OUT
