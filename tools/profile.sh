#!/bin/bash
# Run on the GPU box (gpurun).  Launch list of the bench command + ncu --set full of the
# top kernels.  Outputs under gpurun_out/ (copy the summaries to profiles/).
set -u
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
B="python bench.py --no-cpu --no-e2e"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    $B --steps 2 --warmup 3 > $OUT/launches_bench.json 2> $OUT/launches.err
for k in ${KERNELS:-local_grad3 sumfact3d sumfact2d ccsdt_kernel}; do
  ncu --set full --clock-control none --import-source on -k regex:$k -s 2 -c 1 -o $OUT/prof_$k -f \
      $B --steps 1 --warmup 3 > /dev/null 2> $OUT/prof_$k.err
done
ls -la $OUT
