#!/usr/bin/env python
"""Tuning sweep (GPU box): run bench.py for each variant x case in
subprocesses and print one compact line per run.

usage: python scripts/sweep.py OUTDIR "VARIANTS" "CASES" [extra bench args]
  VARIANTS: space-separated; each is comma-separated KEY=VALUE items, where
            vw=N sets --vec-words N and any other KEY is an environment
            variable of libbro (BRO_ELL_KERNEL, BRO_RING_KB, ...);
            "-" = defaults.
  CASES:    space-separated WORKLOAD:DTYPE (C1..C5 : f64|f32).
e.g. python scripts/sweep.py gpurun_out/s1 "vw=4 vw=1 vw=1,BRO_RING_KB=24" "C5:f64 C5:f32"
"""
import json
import os
import subprocess
import sys

out = sys.argv[1]
variants = sys.argv[2].split()
cases = sys.argv[3].split()
extra = sys.argv[4:]
os.makedirs(out, exist_ok=True)
for case in cases:
    wl, dt = case.split(":")[:2]
    for var in variants:
        env = dict(os.environ)
        args = []
        if var != "-":
            for item in var.split(","):
                k, v = item.split("=")
                if k == "vw":
                    args += ["--vec-words", v]
                else:
                    env[k] = v
        cmd = [sys.executable, "bench.py", "--workload", wl, "--dtype", dt, "--steps", "300",
               "--no-cpu-baseline", "--no-e2e"] + args + extra
        if wl in ("C1", "C2", "C3") and "--flush-l2" not in extra:
            cmd.append("--flush-l2")
        r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=900)
        tag = f"{wl}_{dt}_{var.replace(',', '_').replace('=', '')}"
        with open(os.path.join(out, tag + ".json"), "w") as f:
            f.write(r.stdout)
        if r.returncode != 0:
            print(tag, "FAILED", r.stderr[-800:], flush=True)
            continue
        d = json.loads(r.stdout.strip().splitlines()[-1])
        ro, un = d["roofline"], d["uncompressed"]
        ck = d.get("clocks") or {}
        print(f"{tag:40s} {d['value']:8.1f} GFLOP/s kern {ro['kernel_ms']*1e3:7.1f}us "
              f"{ro['achieved']:6.0f} GB/s frac {ro['frac']:.3f} | base {un['value']:8.1f} "
              f"{un['achieved_GBps']:6.0f} GB/s speedup {un['speedup_bro']:.3f} "
              f"sm {ck.get('sm_mhz')} {ck.get('reasons')}", flush=True)
