"""Summarise an .ncu-rep here (no GPU): key metrics, stall reasons, top SASS lines by stall samples.
Usage: python tools/ncu_top.py <file.ncu-rep> [ntop]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
ntop = int(sys.argv[2]) if len(sys.argv) > 2 else 20
raw = list(csv.reader(io.StringIO(subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout)))
h, v = raw[0], raw[2]
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum",
        "lts__t_sector_hit_rate.pct", "lts__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"]
for w in want:
    if w in h:
        print(f"{w} = {v[h.index(w)]}")
st = []
for i, n in enumerate(h):
    if n.startswith("smsp__pcsamp_warps_issue_stalled_") and "not_issued" not in n:
        try:
            st.append((float(v[i]), n.replace("smsp__pcsamp_warps_issue_stalled_", "")))
        except ValueError:
            pass
st.sort(reverse=True)
tot = sum(x for x, _ in st) or 1
print("stalls:", ", ".join(f"{n} {100 * x / tot:.0f}%" for x, n in st[:8]))
src = list(csv.reader(io.StringIO(subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                                                 capture_output=True, text=True).stdout)))
hh = src[1]
rows = src[2:]
i_s = hh.index("Warp Stall Sampling (All Samples)")
tot = sum(float(x[i_s] or 0) for x in rows) or 1
for x in sorted(rows, key=lambda x: -float(x[i_s] or 0))[:ntop]:
    print(f"{100 * float(x[i_s]) / tot:5.1f}%  {x[1][:100]}")
