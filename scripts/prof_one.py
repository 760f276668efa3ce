#!/usr/bin/env python
"""Run ONE handle variant a few times (for ncu captures under gpurun).

  python scripts/prof_one.py C5 f64 "slice_h=64,ell_kernel=10" [--format coo] [--codec 0] [--r1] [--launches 4]

--r1 runs the round-1 library (scratch_r1, built by scripts/ab_r1.py) instead."""
import argparse
import ctypes as C
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload")
    ap.add_argument("dtype")
    ap.add_argument("opts", nargs="?", default="")
    ap.add_argument("--format", default=None)
    ap.add_argument("--codec", type=int, default=1)
    ap.add_argument("--r1", action="store_true")
    ap.add_argument("--launches", type=int, default=4)
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
    s = torch.cuda.current_stream(dev)
    if a.r1:
        import ab_r1
        r1 = C.CDLL(os.path.join(ROOT, "scratch_r1", "libbro_r1.so"))
        o = ab_r1.Opts()
        r1.bro_opts_default(C.byref(o))
        h = C.c_void_p()
        rp = np.ascontiguousarray(A.row_ptr, dtype=np.int64)
        col = np.ascontiguousarray(A.col, dtype=np.int32)
        vals = np.ascontiguousarray(A.vals, dtype=dtype)
        create = r1.bro_create_hyb if fmt == "hyb" else r1.bro_create_ell
        assert create(0, 1 if dtype == np.float64 else 0, C.c_int64(A.m), C.c_int64(A.n), rp.ctypes.data_as(C.c_void_p),
                      col.ctypes.data_as(C.c_void_p), vals.ctypes.data_as(C.c_void_p), C.byref(o), C.byref(h)) == 0
        r1.bro_spmv.argtypes = [C.c_void_p] * 4
        run = lambda: r1.bro_spmv(h, x.data_ptr(), y.data_ptr(), s.cuda_stream)  # noqa: E731
    else:
        kw = {k: int(v) for k, v in (kv.split("=") for kv in a.opts.split(",") if kv)}
        M = P.BroMatrix(A, fmt=fmt, codec=a.codec, device=0, dtype=dtype, **kw)
        run = lambda: M.spmv(x, y, s)  # noqa: E731
    for _ in range(a.launches):
        run()
    torch.cuda.synchronize()
    print("done", flush=True)


if __name__ == "__main__":
    main()
