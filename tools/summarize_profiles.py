"""Summarise gpurun_out/ measurement artefacts into profiles/ (run here, no GPU).
Usage: python tools/summarize_profiles.py <round-tag>"""
import collections
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
G = os.environ.get("G") or os.path.join(ROOT, "gpurun_out")
P = os.path.join(ROOT, "profiles")
tag = sys.argv[1] if len(sys.argv) > 1 else "r01"

bench = json.load(open(os.path.join(G, "bench.json")))
cfg = bench["config"]
lines = [f"# Profile summary {tag}", "", "## bench.py (default workload)", "",
         f"- value: {bench['value']:.1f} GFLOP/s, ms_per_step {bench['ms_per_step']:.3f}, clocks {bench['clocks']}",
         f"- roofline (dominant kernel {bench['roofline']['kernel']}): achieved {bench['roofline']['achieved']:.1f} "
         f"{bench['roofline']['unit']} of {bench['roofline']['peak']} -> frac {bench['roofline']['frac']:.3f}",
         f"- e2e: {bench['e2e']['value']:.1f} GFLOP/s (H2D {bench['e2e']['h2d_bytes_per_step']/1e9:.2f} GB/step)",
         f"- cpu_baseline (oracle, {bench['cpu_baseline']['cores']} cores): {bench['cpu_baseline']['value']:.1f} GFLOP/s",
         "", "| kernel | ms/step | launches | GFLOP/s | GB/s | bound | frac |", "|---|---|---|---|---|---|---|"]
for k, v in bench["kernels"].items():
    lines.append(f"| {k} | {v['ms_per_step']:.3f} | {v['launches']} | {v['gflops']:.0f} | {v['gbs']:.0f} | {v['bound']} | {v['frac']:.3f} |")

# launch list: share of device time per kernel (ncu, cold-cache, serialised)
rows = list(csv.reader(open(os.path.join(G, "launches.csv"))))
hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
h = rows[hi]
ki, vi = h.index("Kernel Name"), h.index("Metric Value")
agg = collections.defaultdict(list)
setup = collections.defaultdict(list)
for r in rows[hi + 1:]:
    if len(r) > vi:
        try:
            name = r[ki].split("(")[0]
            v = float(r[vi].replace(",", ""))
        except ValueError:
            continue
        # the step's kernels, template variants merged (the constant-bank slot 0/1
        # instantiations); setup kernels (FP64 probes, input fills, torch) listed apart
        if "probe_" in name or "fill_kernel" in name or "at::" in name:
            setup[name].append(v)
        else:
            base = name.replace("void ", "")
            if "<" in base and ("sumfact" in base or "local_grad3" in base):
                base = base[:base.rindex(",")] + ">" if base.count(",") else base
            agg[base].append(v)
tot = sum(sum(v) for v in agg.values())
lines += ["", "## ncu launch list (gpu__time_duration, --clock-control none; bench --steps 2 --warmup 3)", "",
          "Step kernels only (warm-up + timed steps; shares of their total); setup kernels "
          "(live FP64 probes, input fills) below the table.", "",
          "| kernel | launches | total us | share |", "|---|---|---|---|"]
for k, v in sorted(agg.items(), key=lambda x: -sum(x[1])):
    lines.append(f"| {k} | {len(v)} | {sum(v)/1e3:.1f} | {sum(v)/tot*100:.1f}% |")
lines.append("")
lines.append("setup: " + ", ".join(f"{k} x{len(v)} {sum(v)/1e3:.0f} us" for k, v in setup.items()))

WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__block_size", "launch__grid_size",
        "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
        "sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "lts__throughput.avg.pct_of_peak_sustained_elapsed"]
traffic = {}
lines += ["", "## ncu --set full (one launch each)", ""]
for f in sorted(os.listdir(G)):
    # .ncu-rep (read here) or its --page raw --csv export (written on the box by
    # tools/round_measure.sh so gpurun_out/ stays under the copy-back limit)
    if f.endswith(".ncu-rep"):
        raw = subprocess.run(["ncu", "-i", os.path.join(G, f), "--page", "raw", "--csv"],
                             capture_output=True, text=True).stdout
    elif f.endswith(".raw.csv"):
        raw = open(os.path.join(G, f)).read()
    else:
        continue
    rr = list(csv.reader(io.StringIO(raw)))
    if len(rr) < 3:
        continue
    hh, uu, vv = rr[0], rr[1], rr[2]
    d = {n: (vv[i], uu[i]) for i, n in enumerate(hh)}
    name = d.get("Kernel Name", ("?", ""))[0]
    lines.append(f"### {name}")
    for w in WANT:
        if w in d:
            lines.append(f"- {w} = {d[w][0]} {d[w][1]}")
    st = [(float(vv[i].replace(",", "")), n) for i, n in enumerate(hh)
          if n.startswith("smsp__pcsamp_warps_issue_stalled") and not n.endswith("not_issued")]
    st.sort(reverse=True)
    s = sum(x for x, _ in st) or 1
    lines.append("- top stalls: " + ", ".join(f"{n.replace('smsp__pcsamp_warps_issue_stalled_', '')} {x/s*100:.0f}%"
                                                for x, n in st[:6]))
    lines.append("")
    def gb(key):
        v, u = d[key]
        v = float(v.replace(",", ""))
        return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
    if "dram__bytes_read.sum" in d:
        base = name.split("(")[0].split("<")[0].replace("void ", "").replace("bc::", "").strip()
        kn = {"local_grad3_kernel": "local_grad3", "local_grad3_tma_kernel": "local_grad3",
              "sumfact3d_kernel": "sumfact3d", "sumfact2d_kernel": "sumfact2d",
              "ccsdt_tma_kernel": "ccsdt_tma"}.get(base, base)
        if base == "sumfact_tma_kernel":  # <P1, NA, CS>: NA = 1 is the 2-D form
            targs = [a.replace("(int)", "").strip() for a in name.split("<", 1)[1].split(">", 1)[0].split(",")]
            kn = "sumfact2d" if targs[1] == "1" else "sumfact3d"
        tb = gb("dram__bytes_read.sum") + gb("dram__bytes_write.sum")
        n_elem = cfg.get("n_elem", cfg.get("n_elem_per_gpu"))
        if kn == "ccsdt_tma":
            fam = "d1" if ("<1" in name or "<(int)1" in name) else "d2"
            traffic[f"ccsdt_{fam}_fused:p{cfg['p']}:n{n_elem}:t{cfg['ccsdt_tile']}"] = tb
        else:
            traffic[f"{kn}:p{cfg['p']}:n{n_elem}:t{cfg['ccsdt_tile']}"] = tb
open(os.path.join(P, f"ncu_summary_{tag}.md"), "w").write("\n".join(lines) + "\n")
json.dump(traffic, open(os.path.join(P, "traffic.json"), "w"), indent=1)
subprocess.run(["cp", os.path.join(G, "launches.csv"), os.path.join(P, f"launches_{tag}.csv")])
subprocess.run(["cp", os.path.join(G, "bench.json"), os.path.join(P, f"bench_{tag}.json")])
print("\n".join(lines[:40]))
