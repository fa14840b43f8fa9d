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
    python bench.py --no-cpu --no-e2e --no-configs --steps 2 --warmup 3 > /dev/null 2> $OUT/launches.err
# (kernel regex, launches to skip): one launch each; ccsdt_tma_kernel twice (a d1 launch,
# then a d2 launch: 8 d1 then 8 d2 launches per step)
for ks in local_grad3_tma_kernel:2 sumfact_tma_kernel:2 sumfact_tma_kernel:3 ccsdt_tma_kernel:2 ccsdt_tma_kernel:10; do
  k=${ks%%:*}; s=${ks##*:}
  ncu --set full --clock-control none --import-source on -k regex:$k -s $s -c 1 -o $OUT/prof_${k}_s$s -f \
      python bench.py --no-cpu --no-e2e --no-configs --steps 1 --warmup 3 > /dev/null 2> $OUT/prof_$k.err
done
for r in $OUT/*.ncu-rep; do
  [ -e "$r" ] || continue
  ncu -i "$r" --page raw --csv > "${r%.ncu-rep}.raw.csv" 2>/dev/null && rm -f "$r"
done
ls -la $OUT
