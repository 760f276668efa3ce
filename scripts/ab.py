#!/usr/bin/env python
"""A/B timing of BRO handle layouts / kernel instances in ONE process (gpurun):
every variant times bro_spmv with CUDA events on the launching stream (W
warm-ups, K timed calls, L2 flushed before each call for L2-resident
workloads), next to the uncompressed baseline of the same matrix.

  python scripts/ab.py C5 f64 "slice_h=32" "slice_h=64" "slice_h=64,ell_kernel=5" ...
  python scripts/ab.py C4 f32 --format coo "coo_T=8" "coo_T=16" "coo_T=32"

Each variant is a comma list of BroMatrix keyword options.  Prints one line
per variant: mean / p50 kernel us, effective GB/s (algorithmic bytes), frac
of MEASURED_PEAKS.json, speedup over the baseline.  Correctness is the
tests' job; this only checks that y matches the baseline's within 1e-9 rel.
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def parse_opts(s):
    out = {}
    for kv in filter(None, s.split(",")):
        k, v = kv.split("=")
        out[k] = int(v)
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload")
    ap.add_argument("dtype", choices=["f64", "f32"])
    ap.add_argument("variants", nargs="+")
    ap.add_argument("--format", default=None)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--baseline-opts", default="")
    a = ap.parse_args()
    import torch
    import bench
    import paper_conf_sc_tangtrwckgtw13_b200 as P
    from gen import make_x
    dtype = np.float64 if a.dtype == "f64" else np.float32
    A, fmt = bench.load_workload(a.workload, dtype, P)
    fmt = a.format or fmt
    dev = torch.device("cuda:0")
    x = torch.from_numpy(make_x(A.n, bench.WORKLOADS[a.workload][0], dtype)).to(dev)
    y = torch.empty(A.m, dtype=x.dtype, device=dev)
    stream = torch.cuda.current_stream(dev)
    with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
        peak = float(json.load(f)["hbm_gbs"])
    flush_buf = torch.empty(2 * bench.L2_BYTES // 4, dtype=torch.int32, device=dev)

    clocks = []

    def timeit(M):
        small = M.info["algorithmic_bytes"] < 4 * bench.L2_BYTES
        fl = (lambda: flush_buf.fill_(1)) if small else None
        ck = bench.ClockSampler(0)
        ck.start()
        ms = bench.time_steps(lambda: M.spmv(x, y, stream), a.steps, a.warmup, stream, fl)
        c = ck.stop() or {}
        clocks.append(f"{c.get('sm_mhz')}MHz{'/' + ','.join(c['reasons']) if c.get('reasons') else ''}")
        return ms, M.info["algorithmic_bytes"]

    base = P.BroMatrix(A, fmt=fmt, codec=0, device=0, dtype=dtype, **parse_opts(a.baseline_opts))
    bms, bbytes = timeit(base)
    yb = y.clone()
    bmean = float(bms.mean())
    print(f"{a.workload} {a.dtype} {fmt}: baseline {bmean * 1e3:.1f} us "
          f"{bbytes / (bmean * 1e-3) / 1e9:.0f} GB/s ({bbytes / 1e6:.1f} MB) {clocks[-1]}", flush=True)
    base.close()
    for v in a.variants:
        M = P.BroMatrix(A, fmt=fmt, codec=1, device=0, dtype=dtype, **parse_opts(v))
        ms, nb = timeit(M)
        ok = torch.allclose(y, yb, rtol=1e-9 if dtype == np.float64 else 1e-4, atol=1e-9)
        mean, p50 = float(ms.mean()), float(np.median(ms))
        gbs = nb / (mean * 1e-3) / 1e9
        i = M.info
        print(f"  {v:40s} {mean * 1e3:8.1f} us (p50 {p50 * 1e3:7.1f})  {gbs:6.0f} GB/s  frac {gbs / peak:.3f}  "
              f"x{bmean / mean:.3f}  h={i['slice_h']} T={i['coo_T']} inst={i['ell_kernel']} "
              f"eta={i['eta_stream']:.3f} MB={nb / 1e6:.1f} ok={bool(ok)} {clocks[-1]}", flush=True)
        M.close()


if __name__ == "__main__":
    main()
