#!/usr/bin/env python
"""Table 5 / Fig. 9 analog (NEXT-1): compressibility and SpMV
throughput of BRO-HYB under the row orderings of bro_reorder_bar.

Orderings: the matrix as generated (C2: natural FEM order; C4: scrambled),
C4's unscrambled family order (the generator's ideal), method 0 (signature
clustering, DESIGN.md proxy), method 1 (Algorithm 2, exact; m <= 65,536 so C2
only), method 2 (Algorithm 2 with a 64-partition candidate window) and method
3 (method 2 over the signature order instead of the length sort, R27).

Reports eta_stream / eta_total (host) and, with --gpu, BRO-HYB and plain HYB
GFLOP/s (median of timed bro_spmv calls, L2 flushed before each).
usage: python scripts/bar_eval.py [--gpu] [--out FILE.json]
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_sc_tangtrwckgtw13_b200 as P  # noqa: E402
from gen import make_config, make_x, permute_rows, random_block  # noqa: E402


def orderings(cfg):
    A = make_config(cfg)
    yield "as generated", A, 0.0
    if cfg == 4:
        yield "family order (unscrambled)", random_block(seed=4, scramble=False), 0.0
    for meth in (0, 1, 2, 3):
        if meth == 1 and A.m > 65536:
            continue
        t = time.perf_counter()
        perm = P.bro_reorder_bar(A.m, A.n, A.row_ptr, A.col, method=meth)
        yield f"BAR method {meth}", permute_rows(A, perm), time.perf_counter() - t


def gpu_time(A, codec, reps=200):
    import torch
    dev = torch.device("cuda:0")
    M = P.BroMatrix(A, fmt="hyb", codec=codec, device=0)
    x = torch.from_numpy(make_x(A.n, 4)).to(dev)
    y = torch.empty(A.m, dtype=torch.float64, device=dev)
    flush = torch.empty(64 * 2**20, dtype=torch.int32, device=dev)  # 256 MB > 2x L2
    for _ in range(5):
        M.spmv(x, y)
    ts = []
    for _ in range(reps):
        flush.fill_(1)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        M.spmv(x, y)
        e.record()
        e.synchronize()
        ts.append(s.elapsed_time(e))
    M.close()
    return 2.0 * A.nnz / (float(np.median(ts)) * 1e-3) / 1e9


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpu", action="store_true")
    ap.add_argument("--out", default=None)
    ap.add_argument("--configs", default="2,4")
    args = ap.parse_args()
    rows = []
    for cfg in [int(c) for c in args.configs.split(",")]:
        for name, A, secs in orderings(cfg):
            h = P.bro_create_hyb(P.BRO_DEVICE_HOST_ONLY, A.m, A.n, A.row_ptr, A.col, A.vals)
            info = P.bro_get_info(h)
            P.bro_destroy(h)
            r = {"config": f"C{cfg}", "ordering": name, "reorder_s": round(secs, 2),
                 "eta_stream": round(info["eta_stream"], 4), "eta_total": round(info["eta_total"], 4),
                 "K": info["K"], "algorithmic_MB": round(info["algorithmic_bytes"] / 1e6, 1)}
            if args.gpu:
                r["bro_hyb_gflops"] = round(gpu_time(A, 1), 1)
                r["hyb_gflops"] = round(gpu_time(A, 0), 1)
                r["speedup"] = round(r["bro_hyb_gflops"] / r["hyb_gflops"], 3)
            rows.append(r)
            print(json.dumps(r), flush=True)
    if args.out:
        with open(args.out, "w") as f:
            json.dump(rows, f, indent=1)


if __name__ == "__main__":
    main()
