#!/bin/bash
# ncu --set full of the streaming / tile-24 CCSD(T) kernels added in round 1 (under gpurun).
OUT=${OUT:-gpurun_out}; mkdir -p $OUT
for k in svs_kernel s1h_kernel; do
  ncu --set full --clock-control none --import-source on -k regex:$k -s 2 -c 1 -o $OUT/prof_stream_$k -f \
      python tools/prof_stream.py > $OUT/prof_stream_$k.log 2>&1
done
TILE=24 ncu --set full --clock-control none --import-source on -k regex:triples24 -s 1 -c 1 -o $OUT/prof_triples24 -f \
      python tools/prof_f4.py > $OUT/prof_triples24.log 2>&1
ls -la $OUT/*.ncu-rep
