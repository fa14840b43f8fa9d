#!/bin/bash
# Round-end measurement pass (under gpurun): GPU tests, smoke(), bench JSON + ncu launch
# list + ncu --set full of the bench kernels (tools/round_measure.sh), every row
# (tools/bench_rows.py), ncu of the streaming CCSD(T) kernels.  Outputs in gpurun_out/.
set -u
OUT=${OUT:-gpurun_out}; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.txt 2>&1; tail -2 $OUT/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $OUT/smoke.txt 2>&1; tail -1 $OUT/smoke.txt
OUT=$OUT tools/round_measure.sh > $OUT/rm.log 2>&1
cat $OUT/bench.json
python tools/bench_rows.py > $OUT/rows_full.jsonl 2> $OUT/rows_full.err; tail -2 $OUT/rows_full.err
for k in svs_kernel s1h_kernel; do
  ncu --set full --clock-control none --import-source on -k regex:$k -s 2 -c 1 -o $OUT/prof_stream_$k -f \
      python tools/prof_stream.py > /dev/null 2>&1
done
TILE=24 ncu --set full --clock-control none -k regex:triples24 -s 1 -c 1 -o $OUT/prof_triples24 -f \
      python tools/prof_f4.py > /dev/null 2>&1
ls $OUT
