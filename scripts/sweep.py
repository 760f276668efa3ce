#!/usr/bin/env python
"""Tuning sweep (GPU box): run bench.py for each BRO_ELL_VARIANT x workload x
dtype in subprocesses and print one compact line per run.
usage: python scripts/sweep.py OUTDIR "0 1 2" "C5:f64 C5:f32:0,8 C2:f64"
(a case may carry its own comma-separated variant list)
"""
import json
import os
import subprocess
import sys

out = sys.argv[1]
variants = sys.argv[2].split()
cases = sys.argv[3].split()
extra = sys.argv[4:] if len(sys.argv) > 4 else []
os.makedirs(out, exist_ok=True)
for case in cases:
    parts = case.split(":")
    wl, dt = parts[0], parts[1]
    for v in (parts[2].split(",") if len(parts) > 2 else variants):
        env = dict(os.environ, BRO_ELL_VARIANT=v)
        cmd = [sys.executable, "bench.py", "--workload", wl, "--dtype", dt, "--steps", "300",
               "--no-cpu-baseline", "--no-e2e"] + extra
        if wl in ("C1", "C2", "C3"):
            cmd.append("--flush-l2")
        r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=900)
        tag = f"{wl}_{dt}_v{v}"
        with open(os.path.join(out, tag + ".json"), "w") as f:
            f.write(r.stdout)
        if r.returncode != 0:
            print(tag, "FAILED", r.stderr[-500:])
            continue
        d = json.loads(r.stdout.strip().splitlines()[-1])
        ro, un = d["roofline"], d["uncompressed"]
        print(f"{tag}: {d['value']:.1f} GFLOP/s  kern {ro['kernel_ms']*1e3:.1f}us  "
              f"{ro['achieved']:.0f} GB/s frac {ro['frac']:.3f} | base {un['value']:.1f} GFLOP/s "
              f"{un['achieved_GBps']:.0f} GB/s  speedup {un['speedup_bro']:.3f}  clocks {d['clocks']}",
              flush=True)
