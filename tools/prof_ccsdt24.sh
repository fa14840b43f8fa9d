#!/bin/bash
# ncu --set full of the tile-24 CCSD(T) kernels (one d1 and one d2 launch), run under gpurun.
# tools/time_ccsdt.py with BLOCKS=1 launches d1 7 times, then d2.
OUT=${OUT:-gpurun_out}; mkdir -p $OUT
TILE=24 BLOCKS=1 ncu --set full --clock-control none --import-source on -k regex:tma24 -s 2 -c 1 \
   -o $OUT/prof_tma24_d1 -f python tools/time_ccsdt.py > $OUT/prof_tma24_d1.log 2>&1
TILE=24 BLOCKS=1 ncu --set full --clock-control none --import-source on -k regex:tma24 -s 9 -c 1 \
   -o $OUT/prof_tma24_d2 -f python tools/time_ccsdt.py > $OUT/prof_tma24_d2.log 2>&1
ls -la $OUT
