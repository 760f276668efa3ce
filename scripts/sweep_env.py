#!/usr/bin/env python
"""In-process tuning sweep (GPU box): generate a workload once, build its BRO
and uncompressed handles once, then time bro_spmv under each libbro
environment variant (the library reads its BRO_* tuning variables at every
launch).  L2 flushed before every rep for the L2-resident configs.
usage: python scripts/sweep_env.py WORKLOAD DTYPE FORMATS "VARIANTS" [reps]
  FORMATS: comma list of ell,hyb,coo;  VARIANTS: space list of K=V,K=V or "-"
e.g. python scripts/sweep_env.py C4 f64 hyb,coo "- BRO_COO_UPI=4 BRO_COO_MINB=4,BRO_COO_UPI=4"
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_sc_tangtrwckgtw13_b200 as P  # noqa: E402
from gen import make_x  # noqa: E402

wl, dt, fmts, variants = sys.argv[1], sys.argv[2], sys.argv[3].split(","), sys.argv[4].split()
reps = int(sys.argv[5]) if len(sys.argv) > 5 else 200
dtype = np.float64 if dt == "f64" else np.float32
A, _ = bench.load_workload(wl, dtype, P)
dev = torch.device("cuda:0")
x = torch.from_numpy(make_x(A.n, bench.WORKLOADS[wl][0], dtype)).to(dev)
y = torch.empty(A.m, dtype=x.dtype, device=dev)
flush_buf = torch.empty(2 * bench.L2_BYTES // 4, dtype=torch.int32, device=dev)
flush = (lambda: flush_buf.fill_(1)) if wl in ("C1", "C2", "C3") else None
stream = torch.cuda.current_stream(dev)
peak, _ = bench.measured_peaks()
base_env = {k: v for k, v in os.environ.items() if k.startswith("BRO_")}
for fmt in fmts:
    mats = {c: P.BroMatrix(A, fmt=fmt, codec=c, device=0, dtype=dtype) for c in (1, 0)}
    for var in variants:
        for k in [k for k in os.environ if k.startswith("BRO_")]:
            del os.environ[k]
        os.environ.update(base_env)
        if var != "-":
            for item in var.split(","):
                k, v = item.split("=")
                os.environ[k] = v
        res = {}
        for c, M in mats.items():
            ms = bench.time_steps(lambda: M.spmv(x, y, stream), reps, 10, stream, flush)
            res[c] = float(np.median(ms))
        ab = mats[1].info["algorithmic_bytes"]
        print(f"{wl} {dt} {fmt:3s} {var:40s} bro {res[1]*1e3:7.1f} us {ab/res[1]/1e6:6.0f} GB/s "
              f"({ab/res[1]/1e6/peak:.3f})  plain {res[0]*1e3:7.1f} us  speedup {res[0]/res[1]:.3f}", flush=True)
    for M in mats.values():
        M.close()
