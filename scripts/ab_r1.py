#!/usr/bin/env python
"""A/B against the round-1 library in the same process/session (gpurun):
builds scratch_r1/ (the round-1 sources, git show 8295dc0) into
scratch_r1/libbro_r1.so, then times C5 bro_spmv with the round-1 library and
with the current one, clocks sampled with nvidia-smi during each."""
import ctypes as C
import os
import subprocess
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def build_r1():
    d = os.path.join(ROOT, "scratch_r1")
    lib = os.path.join(d, "libbro_r1.so")
    cmd = ["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-std=c++17", "-lineinfo", "-shared",
           "-Xcompiler", "-fPIC,-pthread,-O3", "-cudart", "static", "--expt-relaxed-constexpr",
           "-I", os.path.join(d, "include"), "-o", lib, os.path.join(d, "a", "csrc", "capi.cu"),
           os.path.join(d, "a", "csrc", "encode.cpp")]
    subprocess.run(cmd, check=True)
    return lib


class Opts(C.Structure):
    _fields_ = [("slice_h", C.c_int32), ("sym_bits", C.c_int32), ("vec_words", C.c_int32),
                ("coo_T", C.c_int32), ("hyb_K", C.c_int64), ("codec", C.c_int32), ("min_bits", C.c_int32)]


def main():
    import torch
    import bench
    import paper_conf_sc_tangtrwckgtw13_b200 as P
    from gen import make_config, make_x
    wl = sys.argv[1] if len(sys.argv) > 1 else "C5"
    dt = sys.argv[2] if len(sys.argv) > 2 else "f64"
    variants = sys.argv[3:] or ["slice_h=32", "slice_h=32,ell_kernel=7"]
    dtype = np.float64 if dt == "f64" else np.float32
    r1 = C.CDLL(build_r1())
    A, fmt = bench.load_workload(wl, dtype, P)
    dev = torch.device("cuda:0")
    x = torch.from_numpy(make_x(A.n, bench.WORKLOADS[wl][0], dtype)).to(dev)
    y = torch.empty(A.m, dtype=x.dtype, device=dev)
    stream = torch.cuda.current_stream(dev)

    def run(name, fn, nbytes):
        ck = bench.ClockSampler(0)
        ck.start()
        ms = bench.time_steps(fn, 300, 10, stream)
        c = ck.stop()
        mean = float(ms.mean())
        print(f"  {name:36s} {mean * 1e3:8.1f} us  {nbytes / (mean * 1e-3) / 1e9:6.0f} GB/s  clocks {c}", flush=True)

    o = Opts()
    r1.bro_opts_default(C.byref(o))
    h = C.c_void_p()
    rp = np.ascontiguousarray(A.row_ptr, dtype=np.int64)
    col = np.ascontiguousarray(A.col, dtype=np.int32)
    vals = np.ascontiguousarray(A.vals, dtype=dtype)
    create = r1.bro_create_hyb if fmt == "hyb" else r1.bro_create_ell
    st = create(0, 1 if dtype == np.float64 else 0, C.c_int64(A.m), C.c_int64(A.n), rp.ctypes.data_as(C.c_void_p),
                col.ctypes.data_as(C.c_void_p), vals.ctypes.data_as(C.c_void_p), C.byref(o), C.byref(h))
    assert st == 0, st
    r1.bro_spmv.argtypes = [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
    for rep in range(2):
        run(f"round-1 library (rep {rep})", lambda: r1.bro_spmv(h, x.data_ptr(), y.data_ptr(), stream.cuda_stream),
            1)
        for v in variants:
            kw = {k: int(val) for k, val in (kv.split("=") for kv in v.split(","))}
            M = P.BroMatrix(A, fmt=fmt, codec=1, device=0, dtype=dtype, **kw)
            run(f"current {v}", lambda: M.spmv(x, y, stream), M.info["algorithmic_bytes"])
            M.close()


if __name__ == "__main__":
    main()
