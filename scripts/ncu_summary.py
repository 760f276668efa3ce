#!/usr/bin/env python
"""Summarise an ncu --set full report: key SOL metrics, stall reasons, top SASS stall sites."""
import csv, io, subprocess, sys

rep = sys.argv[1]
topn = int(sys.argv[2]) if len(sys.argv) > 2 else 25

def run(*a):
    return subprocess.run(["ncu", "-i", rep, *a], capture_output=True, text=True).stdout

raw = list(csv.reader(io.StringIO(run("--page", "raw", "--csv"))))
hdr, units = raw[0], raw[1]
want = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "sm__inst_executed.avg.per_cycle_active", "lts__t_sector_hit_rate.pct",
        "l1tex__t_sector_hit_rate.pct", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "lts__t_bytes.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "launch__shared_mem_per_block_dynamic"]
for vals in raw[2:]:  # one row per captured kernel launch
  for w in want:
    if w in hdr:
        i = hdr.index(w)
        print(f"{w:60s} {vals[i]} {units[i]}")
  stalls = []
  for i, h in enumerate(hdr):
    if h.startswith("smsp__average_warp_latency_issue_stalled_") and h.endswith(".ratio"):
        try:
            stalls.append((float(vals[i].replace(",", "")), h[len("smsp__average_warp_latency_issue_stalled_"):]))
        except ValueError:
            pass
    if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio"):
        try:
            stalls.append((float(vals[i].replace(",", "")), h[len("smsp__average_warps_issue_stalled_"):]))
        except ValueError:
            pass
  print("stalls (warps per issue):", ", ".join(f"{n}={v:.2f}" for v, n in sorted(stalls, reverse=True)[:10]))
  print()
src = list(csv.reader(io.StringIO(run("--page", "source", "--csv", "--print-source", "sass"))))
if len(src) > 2:
    h = src[1]
    ix = {k: j for j, k in enumerate(h)}
    rows = src[2:]
    key = "Warp Stall Sampling (All Samples)"
    def n(r):
        try:
            return int(r[ix[key]] or 0)
        except ValueError:
            return 0
    rows = [r for r in rows if len(r) > ix[key]]
    tot = sum(n(r) for r in rows)
    print(f"SASS instructions: {len(rows)}, stall samples: {tot}")
    for r in sorted(rows, key=lambda r: -n(r))[:topn]:
        print(f"  {r[ix['Address']][-5:]} {r[ix['Source']][:60]:60s} {n(r):6d} "
              f"exec={r[ix['Instructions Executed']]}")
