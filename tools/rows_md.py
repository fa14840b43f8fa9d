"""profiles/rows_rNN.jsonl (tools/bench_rows.py) -> markdown table.
Usage: python tools/rows_md.py profiles/rows_r01.jsonl > profiles/rows_r01.md"""
import json
import sys

rows = [json.loads(l) for l in open(sys.argv[1]) if l.strip().startswith("{")]
print("# Per-row / per-config measurements (tools/bench_rows.py on one B200)\n")
print("Roofline: HBM = MEASURED_PEAKS.json hbm_gbs, FP64 37.2 TFLOP/s. `frac` = bound time / measured time "
      "(bound = max(bytes/HBM, flops/FP64), algorithmic bytes and flops of DESIGN.md §4).\n")
print("| row | config | ms | GFLOP/s | bound | frac |")
print("|---|---|---|---|---|---|")
for r in rows:
    cfg = r["config"] + (f" (graph-amortised {r['graph_us_per_call']} us/call)" if "graph_us_per_call" in r else "")
    print(f"| {r['row']} | {cfg} | {r['ms']} | {r['gflops']} | {r['bound']} | {r['roofline_frac']} |")
