#!/usr/bin/env python
"""Fig. 3 analog on B200 (NEXT-3): BRO-ELL GFLOP/s vs space savings eta on a
dense matrix with forced bit widths, against the in-repo ELLPACK
on the same matrix; prints one JSON object with the curve and the break-even
eta (the paper found 17% / 9% / 23% on C2070 / GTX680 / K20).

usage (GPU box): python scripts/eta_sweep.py [OUT.json] [--rows 4000000]
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_tangtrwckgtw13_b200 as P  # noqa: E402
from gen import dense_band, make_x  # noqa: E402


def timeit(fn, reps=50, warm=5):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(reps):
        fn()
    e.record()
    torch.cuda.synchronize()
    return s.elapsed_time(e) / reps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("out", nargs="?", default=None)
    ap.add_argument("--rows", type=int, default=4_000_000)
    ap.add_argument("--k", type=int, default=32)
    a = ap.parse_args()
    A = dense_band(a.rows, a.k)
    res = {"workload": f"dense {a.rows} x {a.k} (every row holds columns 0..{a.k - 1})",
           "note": "widths forced with bro_opts_t.min_bits; eta_stream = 1 - C/O (P:L246)", "curves": {}}
    for dt, tdt in ((np.float64, torch.float64), (np.float32, torch.float32)):
        x = torch.from_numpy(make_x(A.n, 0, dt)).cuda()
        y = torch.empty(A.m, dtype=tdt, device="cuda")
        base = P.BroMatrix(A, fmt="ell", codec=0, dtype=dt)
        tb = timeit(lambda: base.spmv(x, y))
        flops = 2.0 * A.nnz
        curve = {"ell": {"ms": tb, "gflops": flops / tb / 1e6,
                         "GBps": base.info["algorithmic_bytes"] / tb / 1e6}, "bro": []}
        base.close()
        for b in (1, 2, 3, 4, 6, 8, 10, 12, 14, 16, 18, 20, 22, 24, 26, 28, 31):
            M = P.BroMatrix(A, fmt="ell", codec=1, dtype=dt, min_bits=b)
            t = timeit(lambda: M.spmv(x, y))
            curve["bro"].append({"bits": b, "eta": M.info["eta_stream"], "ms": t,
                                 "gflops": flops / t / 1e6,
                                 "GBps": M.info["algorithmic_bytes"] / t / 1e6,
                                 "speedup_vs_ell": tb / t})
            M.close()
        # break-even: smallest eta at which BRO is at least as fast as ELL
        be = [p["eta"] for p in curve["bro"] if p["speedup_vs_ell"] >= 1.0]
        curve["break_even_eta"] = min(be) if be else None
        res["curves"][np.dtype(dt).name] = curve
        print(np.dtype(dt).name, "ELL", round(curve["ell"]["gflops"], 1), "GFLOP/s; break-even eta",
              curve["break_even_eta"], flush=True)
        for p in curve["bro"]:
            print(f"  b={p['bits']:2d} eta={p['eta']:.3f} {p['gflops']:8.1f} GFLOP/s {p['GBps']:7.0f} GB/s "
                  f"x{p['speedup_vs_ell']:.3f}", flush=True)
    if a.out:
        with open(a.out, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
