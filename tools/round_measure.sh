#!/bin/bash
# Full measurement pass (run under gpurun): bench JSON, clocks, launch list, ncu captures.
set -u
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 200 > $OUT/clocks.csv &
CLK=$!
python bench.py > $OUT/bench.json 2> $OUT/bench.err
kill $CLK
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --no-cpu --no-e2e --steps 2 --warmup 3 > /dev/null 2> $OUT/launches.err
for k in ${KERNELS:-local_grad3_kernel sumfact3d_kernel sumfact2d_kernel ccsdt_tma_kernel}; do
  ncu --set full --clock-control none --import-source on -k regex:$k -s 2 -c 1 -o $OUT/prof_$k -f \
      python bench.py --no-cpu --no-e2e --steps 1 --warmup 3 > /dev/null 2> $OUT/prof_$k.err
done
for r in $OUT/*.ncu-rep; do
  [ -e "$r" ] || continue
  ncu -i "$r" --page raw --csv > "${r%.ncu-rep}.raw.csv" 2>/dev/null && rm -f "$r"
done
ls -la $OUT
