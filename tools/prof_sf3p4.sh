#!/bin/bash
# ncu --set full of sumfact3d and local_grad3 at p = 4 (N = 4.6M, same bytes as p = 12), under gpurun.
OUT=${OUT:-gpurun_out}; mkdir -p $OUT
for k in sumfact3d local_grad3; do
  ncu --set full --clock-control none --import-source on -k regex:${k}_kernel -s 2 -c 1 \
     -o $OUT/prof_p4_$k -f python tools/sweep_spectral.py 4 > $OUT/prof_p4_$k.log 2>&1
done
