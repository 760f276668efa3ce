#!/usr/bin/env python
"""Per-CUDA-source-line summary of an ncu --set full report captured with
--import-source on and -lineinfo: warp instructions executed and stall
samples per source line (`--page source --print-source cuda,sass`).
usage: python scripts/ncu_lines.py REPORT [topn] [sort: stall|inst]"""
import csv, io, subprocess, sys

rep = sys.argv[1]
topn = int(sys.argv[2]) if len(sys.argv) > 2 else 40
key = sys.argv[3] if len(sys.argv) > 3 else "stall"
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
recs, fname = [], ""
for r in csv.reader(io.StringIO(out)):
    if len(r) == 2 and r[0] == "File Path":
        fname = r[1].rsplit("/", 1)[-1]
    if len(r) > 8 and r[0].isdigit():
        def f(i):
            try:
                return float(r[i].replace(",", ""))
            except ValueError:
                return 0.0
        recs.append((fname, int(r[0]), r[1].strip(), f(4), f(7)))
ti = sum(x[4] for x in recs)
ts = sum(x[3] for x in recs)
print(f"warp instructions executed {ti:.0f}, stall samples {ts:.0f}")
recs.sort(key=lambda x: -(x[3] if key == "stall" else x[4]))
for fn, ln, src, st, ins in recs[:topn]:
    print(f"{fn[:12]:12s}:{ln:<5d} inst={ins:>11.0f} ({100*ins/max(ti,1):4.1f}%) stall={st:>6.0f} ({100*st/max(ts,1):4.1f}%)  {src[:80]}")
