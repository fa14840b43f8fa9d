#!/bin/bash
# ncu --set full of the tile-16 fused CCSD(T) TMA kernels (one d1 and one d2 launch), under gpurun.
# tools/time_ccsdt.py (BLOCKS=1) launches d1 7 times, then d2.
OUT=${OUT:-gpurun_out}; mkdir -p $OUT
TILE=16 BLOCKS=1 ncu --set full --clock-control none --import-source on -k regex:ccsdt_tma_kernel -s 2 -c 1 \
   -o $OUT/prof_tma16_d1 -f python tools/time_ccsdt.py > $OUT/prof_tma16_d1.log 2>&1
TILE=16 BLOCKS=1 ncu --set full --clock-control none --import-source on -k regex:ccsdt_tma_kernel -s 9 -c 1 \
   -o $OUT/prof_tma16_d2 -f python tools/time_ccsdt.py > $OUT/prof_tma16_d2.log 2>&1
