#!/usr/bin/env python
"""Headline benchmark: SpMV GFLOP/s and effective HBM GB/s (% of roofline) of
BRO formats vs the in-repo uncompressed ELL/HYB kernels (BASELINE.json).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload C5]
                  [--impl ours|reference] [--dtype f64|f32]

A step is one pass of the hot path: one bro_spmv (BRO-ELL: one kernel; BRO-HYB:
ELL kernel + COO kernel + fix-up) over the resident matrix.  For N > 1 a step
is one row-block iteration x_(k+1) = A.x_k of a CG-style loop: every rank's
SpMV plus the exchange that gives every rank all of x_(k+1) (--exchange:
fused P2P scatter from the kernel epilogue, overlapped NCCL allgather, or
SpMV-then-allgather; paper_conf_sc_tangtrwckgtw13_b200/dist.py).  Default
workload: C5 (3D 27-point stencil on 200^3, 8M rows, 213.8M nnz, fp64,
BRO-ELL) — the largest config, the one BASELINE.json runs at 1/2/4/8 GPUs.
Its 2.0 GB working set exceeds the 126 MB L2, so no flush is needed between
steps.  Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "SpMV GFLOP/s and effective HBM GB/s (% of roofline) vs uncompressed ELL/HYB"
WORKLOADS = {
    "C1": (1, "ell"), "C2": (2, "ell"), "C3": (3, "hyb"), "C4": (4, "hyb"), "C5": (5, "ell"),
}
L2_BYTES = 126 * 2**20
FALLBACK_HBM = 6650.0

# SMI throttle-reason bits (nvml clocks_event_reasons)
REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
           0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
           0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
           0x100: "display_clock_setting"}


def parse_args():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=2000)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--workload", default="C5", choices=sorted(WORKLOADS))
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32"])
    ap.add_argument("--format", default=None, choices=["ell", "hyb", "coo"],
                    help="override the workload's format (e.g. coo: standalone BRO-COO vs COO, Fig. 7)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--vec-words", type=int, default=0, help="0 = auto (1, the paper's multiplexing)")
    ap.add_argument("--slice-h", type=int, default=0, help="BRO-ELL slice height: 0 = auto, 32, 64")
    ap.add_argument("--coo-T", type=int, default=0, help="BRO-COO entries per lane: 0 = auto, 8, 16, 32")
    ap.add_argument("--ell-kernel", type=int, default=0, help="BRO-ELL instance: 0 = auto, 1..7 (A/B only)")
    ap.add_argument("--value-codec", type=int, default=0, choices=[0, 1],
                    help="1 = value indexing of the BRO-ELL values (P:L416 future work, DESIGN reading R28); "
                         "0 = the paper's BRO formats (default, the headline)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--flush-l2", action="store_true", help="write a 2xL2 buffer between steps")
    ap.add_argument("--exchange", default="auto", choices=["auto", "allgather", "overlap", "p2p"],
                    help="N>1 exchange of the row-block iteration (auto: p2p, else overlap, else allgather, "
                         "each verified against allgather before timing)")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="gloo only for functional checks of the N>1 path on one GPU")
    return ap.parse_args()


def workload_label(name):
    return f"{name}: " + {"C1": "2D 5-point Laplacian 64x64", "C2": "FEM banded 62,424 rows",
                          "C3": "webbase-like 1,000,005 rows", "C4": "random-block 2M rows, BAR-reordered (method 3)",
                          "C5": "3D 27-point stencil 200^3"}[name]


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    return FALLBACK_HBM, "fallback"


# BAR method for C4's input: 3 = Algorithm 2 (Eqn 1) with a
# 64-partition candidate window over the signature order (reading R27):
# measured faster than the signature order alone (method 0) on C4,
# profiles/r02/bar/bar_eval.txt
C4_BAR_METHOD = 3


def load_workload(name, dtype, lib=None):
    """Generate the config (seeded) and apply BAR (C4_BAR_METHOD) for C4."""
    from gen import make_config, permute_rows
    cfg, fmt = WORKLOADS[name]
    A = make_config(cfg, dtype)
    if cfg == 4 and lib is not None:
        perm = lib.bro_reorder_bar(A.m, A.n, A.row_ptr, A.col, dtype=dtype, method=C4_BAR_METHOD)
        A = permute_rows(A, perm)
    return A, fmt


class ClockSampler:
    """nvidia-smi sampling during the timed region (median SM clock + reasons)."""

    def __init__(self, index=0):
        self.index = index
        self.proc = None
        self.path = None

    def start(self):
        import tempfile
        fd, self.path = tempfile.mkstemp(suffix=".csv")
        self._out = os.fdopen(fd, "w")
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active")
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}", "--format=csv,noheader,nounits",
                 "-lms", "50"], stdout=self._out, stderr=subprocess.DEVNULL)
            time.sleep(0.4)
        except (OSError, FileNotFoundError):
            self.proc = None

    def stop(self):
        if self.proc is None:
            if self.path:
                self._out.close()
                os.unlink(self.path)
            return None
        time.sleep(0.1)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        self._out.close()
        rows = []
        with open(self.path) as f:
            for line in f:
                parts = [p.strip() for p in line.split(",")]
                if len(parts) < 4:
                    continue
                try:
                    rows.append((float(parts[0]), float(parts[1]), float(parts[2]), int(parts[3], 16)))
                except ValueError:
                    continue
        os.unlink(self.path)
        if not rows:
            return None
        loaded = [r for r in rows if not (r[3] & 0x1)] or rows
        sm = sorted(r[0] for r in loaded)
        mask = 0
        for r in loaded:
            mask |= r[3]
        return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": max(r[1] for r in rows),
                "power_w_max": max(r[2] for r in loaded), "samples": len(loaded),
                "reasons": [v for k, v in REASONS.items() if mask & k and k != 0x1]}


def cpu_oracle_baseline(A, x, target_s=12.0, max_rows=None):
    """The oracle's csr_spmv (as it stands, single core) on a bounded row
    sample of the same workload; GFLOP/s over the sample."""
    from oracle import spmv as ospmv
    m = A.m if max_rows is None else min(A.m, max_rows)
    rows = m
    # size the sample so one call is ~target_s/3
    probe = min(m, 200_000)
    t0 = time.perf_counter()
    ospmv.csr_spmv(A.row_ptr[:probe + 1], A.col[:A.row_ptr[probe]], A.vals[:A.row_ptr[probe]], x)
    dt = max(time.perf_counter() - t0, 1e-6)
    rows = int(min(m, probe * (target_s / 3) / dt))
    nnz = int(A.row_ptr[rows])
    times = []
    for _ in range(3):
        t0 = time.perf_counter()
        ospmv.csr_spmv(A.row_ptr[:rows + 1], A.col[:nnz], A.vals[:nnz], x)
        times.append(time.perf_counter() - t0)
    t = float(np.median(times))
    return {"value": 2.0 * nnz / t / 1e9, "unit": "GFLOP/s", "cores": 1, "kind": "oracle",
            "sample": f"rows [0,{rows}) of the workload ({nnz} nnz), median of 3 calls, "
                      f"np.longdouble accumulation, of {os.cpu_count()} host cores"}


def time_steps(fn, steps, warmup, stream, flush=None):
    """Per-step CUDA-event durations on `stream` (ms)."""
    import torch
    for _ in range(warmup):
        fn()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    for s, e in ev:
        if flush is not None:
            flush()
        s.record(stream)
        fn()
        e.record(stream)
    torch.cuda.synchronize()
    return np.array([s.elapsed_time(e) for s, e in ev])


def read_ceiling(dev, gib=2, reps=5):
    """A read-only streaming kernel on this box: best-of-N
    torch.sum over a 2 GiB fp32 buffer, CUDA events.  Context only — the
    roofline's denominator stays the driver-measured copy bandwidth, and the
    in-repo ELLPACK kernel streams faster than this library reduction."""
    import torch
    buf = torch.ones(gib * 2**30 // 4, dtype=torch.float32, device=dev)
    best = None
    for _ in range(reps + 1):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        buf.sum()
        e.record()
        torch.cuda.synchronize()
        ms = s.elapsed_time(e)
        best = ms if best is None else min(best, ms)
    del buf
    return buf_bytes(gib) / (best * 1e-3) / 1e9


def buf_bytes(gib):
    return gib * 2**30


def max_over_ranks(vals, dev, backend):
    """Element-wise max over ranks (device times are compared as the max)."""
    import torch
    import torch.distributed as dist
    t = torch.tensor(vals, dtype=torch.float64, device=dev if backend == "nccl" else "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return [float(v) for v in t.cpu()]


def run_reference(args):
    """--impl reference: the CPU oracle (the only reference this paper-only
    tier has), as it stands, on the host cores; rank 0 only."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    dtype = np.float64 if args.dtype == "f64" else np.float32
    A, fmt = load_workload(args.workload, dtype)
    from gen import make_x
    x = make_x(A.n, WORKLOADS[args.workload][0], dtype)
    from oracle import spmv as ospmv
    # each step: a bounded row sample (~1 s of oracle work)
    probe = min(A.m, 100_000)
    t0 = time.perf_counter()
    ospmv.csr_spmv(A.row_ptr[:probe + 1], A.col[:A.row_ptr[probe]], A.vals[:A.row_ptr[probe]], x)
    dt = max(time.perf_counter() - t0, 1e-6)
    rows = int(min(A.m, probe * 1.0 / dt))
    nnz = int(A.row_ptr[rows])
    for _ in range(args.warmup):
        ospmv.csr_spmv(A.row_ptr[:rows + 1], A.col[:nnz], A.vals[:nnz], x)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        ospmv.csr_spmv(A.row_ptr[:rows + 1], A.col[:nnz], A.vals[:nnz], x)
    t = time.perf_counter() - t0
    val = 2.0 * nnz * args.steps / t / 1e9
    sample = f"rows [0,{rows}) of {args.workload} ({nnz} nnz) per step"
    out = {"impl": "reference", "metric": METRIC, "value": val, "unit": "GFLOP/s", "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * t / args.steps,
           "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": args.dtype,
           "data": "synthetic", "config": {"workload": workload_label(args.workload), "format": "CSR (oracle)"},
           "cpu_baseline": {"value": val, "unit": "GFLOP/s", "cores": 1, "kind": "oracle", "sample": sample},
           "e2e": {"value": val, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)

def layout_opts(args):
    """BroMatrix layout options of the BRO handle (0 = the library's auto choice)."""
    return {"slice_h": args.slice_h, "coo_T": args.coo_T, "ell_kernel": args.ell_kernel,
            "value_codec": args.value_codec}


def build_row_block(A, rank, world, dev, fmt, dtype, bounds, args, x_host, stream):
    """The BRO row block with the fastest exchange that reproduces the
    allgather schedule on this box: p2p (fused scatter into symmetric memory),
    else overlap, else allgather.  Every rank takes the same decision."""
    import torch
    import torch.distributed as dist
    from paper_conf_sc_tangtrwckgtw13_b200.dist import RowBlockSpmv
    order = ["p2p", "overlap", "allgather"] if args.exchange == "auto" else [args.exchange]
    notes = []
    for mode in order:
        blk, err = None, ""
        if mode == "p2p":
            # every rank agrees on the preconditions before any rank enters the
            # collective symmetric-memory rendezvous (an asymmetric failure
            # inside it would leave the other ranks waiting)
            pre = 0.0
            try:
                idx = torch.device(dev).index or 0
                pre = float(torch.cuda.device_count() >= world and all(
                    torch.cuda.can_device_access_peer(idx, p) for p in range(world) if p != idx))
            except Exception:  # noqa: BLE001
                pre = 0.0
            ok_pre = torch.tensor([pre], dtype=torch.float64,
                                  device=dev if args.dist_backend == "nccl" else "cpu")
            dist.all_reduce(ok_pre, op=dist.ReduceOp.MIN)
            if ok_pre.item() != 1.0:
                notes.append({"mode": mode, "why": "no peer access between every pair of ranks' GPUs"})
                continue
        try:
            blk = RowBlockSpmv(A, rank, world, dev, fmt=fmt, codec=1, dtype=dtype, bounds=bounds,
                               vec_words=args.vec_words, exchange=mode, **layout_opts(args))
            if mode != "allgather":
                res = []
                for ex in (mode, "allgather"):
                    blk.set_x(x_host)
                    for _ in range(3):
                        blk.step(stream, ex)
                    blk.complete(stream)
                    torch.cuda.synchronize()
                    res.append(blk.X[blk.k % 2].clone())
                a, b = res
                # the modes split rows differently (overlap: three handles), so
                # summation orders differ: compare at the dtype's bound, not bitwise
                rtol = 1e-12 if dtype == np.float64 else 1e-5
                scale = torch.maximum(a.abs(), b.abs()).max().clamp_min(1e-300)
                if not (torch.isfinite(a).all() and ((a - b).abs() <= 10 * rtol * scale).all()):
                    err = "3-iteration result differs from the allgather schedule"
        except Exception as e:  # noqa: BLE001 - any setup failure moves to the next mode
            err = f"{type(e).__name__}: {e}"[:200]
        ok = torch.tensor([0.0 if err else 1.0], dtype=torch.float64,
                          device=dev if args.dist_backend == "nccl" else "cpu")
        dist.all_reduce(ok, op=dist.ReduceOp.MIN)
        if ok.item() == 1.0:
            info = {"exchange": mode, "requested": args.exchange, "rejected": notes,
                    "multicast": bool(blk.use_mc and blk.mc[0]),
                    "overlap_split": list(getattr(blk, "split", (0, 0))) if mode == "overlap" else None}
            return blk, info
        notes.append({"mode": mode, "why": err or "failed on another rank"})
        if blk is not None:
            try:
                blk.close()
            except Exception:  # noqa: BLE001
                pass
    raise SystemExit(f"no exchange mode worked: {notes}")


def main():
    args = parse_args()
    if args.impl == "reference":
        return run_reference(args)
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus and world > 1:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    # one process per GPU; ranks wrap around only in the gloo functional
    # check of the N > 1 path on a single-GPU box (never with NCCL)
    local = local % max(1, torch.cuda.device_count()) if args.dist_backend == "gloo" else local
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        if args.dist_backend == "nccl":
            if rank == 0:  # communicator setup lines (ranks, NVLS / P2P transport) in the driver's log
                os.environ.setdefault("NCCL_DEBUG", "INFO")
                os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")

    import paper_conf_sc_tangtrwckgtw13_b200 as P
    from paper_conf_sc_tangtrwckgtw13_b200.dist import RowBlockSpmv, choose_partition
    from gen import make_x

    dtype = np.float64 if args.dtype == "f64" else np.float32
    tdt = torch.float64 if dtype == np.float64 else torch.float32
    cfg, fmt = WORKLOADS[args.workload]
    A, fmt = load_workload(args.workload, dtype, P)
    fmt = args.format or fmt
    x_host = make_x(A.n, cfg, dtype)
    bounds = choose_partition(A.row_ptr, world)
    stream = torch.cuda.current_stream(dev)
    x = torch.from_numpy(x_host).to(dev)

    exch_info = None
    if world > 1:
        blk, exch_info = build_row_block(A, rank, world, dev, fmt, dtype, bounds, args, x_host, stream)
        base = RowBlockSpmv(A, rank, world, dev, fmt=fmt, codec=0, dtype=dtype, bounds=bounds,
                            exchange=blk.exchange, coo_T=args.coo_T)
        blk.set_x(x_host)
        base.set_x(x_host)
    else:
        blk = RowBlockSpmv(A, rank, world, dev, fmt=fmt, codec=1, dtype=dtype, bounds=bounds,
                           vec_words=args.vec_words, **layout_opts(args))
        base = RowBlockSpmv(A, rank, world, dev, fmt=fmt, codec=0, dtype=dtype, bounds=bounds,
                            coo_T=args.coo_T)
    info, binfo = blk.mat.info, base.mat.info
    # our kernels per step: ELL kernel, COO kernel + fix-up; the overlap
    # exchange runs one SpMV per row part (interior / head / tail); a
    # HYB/COO handle scattering to peers adds its replicate kernel
    per_spmv = (0 if fmt == "coo" else 1) + (2 if info["nnz_coo"] else 0)
    launches = per_spmv
    if world > 1 and blk.exchange == "overlap":
        launches = sum((0 if fmt == "coo" else 1) + (2 if p.info["nnz_coo"] else 0) for _, _, p in blk.parts)
    elif world > 1 and blk.exchange == "p2p" and info["nnz_coo"]:
        launches = per_spmv + 1
    flush_buf = torch.empty(2 * L2_BYTES // 4, dtype=torch.int32, device=dev) if args.flush_l2 else None
    flush = (lambda: flush_buf.fill_(1)) if args.flush_l2 else None
    y1 = torch.empty(A.m, dtype=tdt, device=dev) if world == 1 else None

    if world > 1:
        # x_{k+1} = A.x_k over the row blocks with the chosen exchange
        def step():
            blk.step(stream)

        def step_base():
            base.step(stream)

        def spmv_only():
            blk.spmv(stream=stream)

        def spmv_only_base():
            base.spmv(stream=stream)
    else:
        def step():
            blk.mat.spmv(x, y1, stream)

        def step_base():
            base.mat.spmv(x, y1, stream)

        spmv_only, spmv_only_base = step, step_base

    # --- timed region (ours) with clock sampling
    clocks = ClockSampler(local) if rank == 0 else None
    if clocks:
        clocks.start()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    per_step = time_steps(step, args.steps, args.warmup, stream, flush)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ck = clocks.stop() if clocks else None
    total_ms = float(per_step.sum())
    # kernel-only duration (SpMV launch without the allgather) for the roofline
    kern = time_steps(spmv_only, min(args.steps, 500), 3, stream, flush)
    kern_ms = float(np.mean(kern))
    base_ms = float(np.mean(time_steps(step_base, min(args.steps, 500), args.warmup, stream, flush)))
    base_kern_ms = float(np.mean(time_steps(spmv_only_base, min(args.steps, 500), 3, stream, flush)))
    ag_ms = None
    if world > 1:
        # the same iteration with the baseline schedule (SpMV, then allgather)
        ag_ms = float(np.mean(time_steps(lambda: blk.step(stream, "allgather"), min(args.steps, 500),
                                         args.warmup, stream, flush)))
        total_ms, base_ms, kern_ms_max, ag_ms = max_over_ranks([total_ms, base_ms, kern_ms, ag_ms], dev,
                                                                args.dist_backend)
        exch_info.update({"allgather_ms_per_step": ag_ms, "spmv_only_ms_max_over_ranks": kern_ms_max,
                          "spmv_only_gflops": 2.0 * A.nnz / (kern_ms_max * 1e-3) / 1e9,
                          "speedup_vs_allgather": ag_ms / (total_ms / args.steps)})

    # --- launch latency: the same bro_spmv captured once in a CUDA graph and
    # replayed (the CG-loop form; matters for the small, L2-resident C1/C2)
    graph = None
    if world == 1:
        g = torch.cuda.CUDAGraph()
        blk.mat.spmv(x, y1, stream)
        torch.cuda.synchronize()
        with torch.cuda.graph(g):
            blk.mat.spmv(x, y1, None)
        g_ms = time_steps(g.replay, min(args.steps, 500), 3, stream, flush)
        graph = {"us_per_call": float(np.median(g_ms)) * 1e3,
                 "p10_us": float(np.percentile(g_ms, 10)) * 1e3, "p90_us": float(np.percentile(g_ms, 90)) * 1e3,
                 "gflops": 2.0 * A.nnz / (float(np.median(g_ms)) * 1e-3) / 1e9}

    # --- end to end through the C ABI with pinned host buffers (rank 0 / N=1 path)
    e2e = None
    if not args.no_e2e:
        from paper_conf_sc_tangtrwckgtw13_b200.dist import global_to_padded
        xh = torch.from_numpy(global_to_padded(x_host, bounds) if world > 1 else x_host).pin_memory()
        yh = torch.empty(blk.mat.m, dtype=tdt).pin_memory()
        xh_np, yh_np = xh.numpy(), yh.numpy()
        P.bro_spmv_host(blk.mat.h, xh_np, yh_np, stream.cuda_stream)  # warm
        e2e_steps = max(3, min(args.steps, 30))
        if world > 1:
            dist.barrier()
        t0e, t1e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0e.record(stream)
        for _ in range(e2e_steps):
            P.bro_spmv_host(blk.mat.h, xh_np, yh_np, stream.cuda_stream)
        t1e.record(stream)
        torch.cuda.synchronize()
        e2e_ms = t0e.elapsed_time(t1e) / e2e_steps
        if world > 1:
            (e2e_ms,) = max_over_ranks([e2e_ms], dev, args.dist_backend)
        isz = np.dtype(dtype).itemsize
        e2e = {"value": 2.0 * A.nnz / (e2e_ms * 1e-3) / 1e9, "unit": "GFLOP/s",
               "h2d_bytes_per_step": int(blk.mat.n * isz), "d2h_bytes_per_step": int(blk.mat.m * isz),
               "ms_per_step": e2e_ms,
               "path": "bro_spmv_host: pinned x H2D + bro_spmv + y D2H + stream sync, per rank "
                       "(ELL-only handles pipeline the three over streams in 8 pieces)"}

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return

    peak, peak_kind = measured_peaks()
    rc = read_ceiling(dev) if world == 1 else None
    alg_bytes = info["algorithmic_bytes"]
    achieved = alg_bytes / (kern_ms * 1e-3) / 1e9
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        with open(tp) as f:
            tr = json.load(f).get(f"{args.workload}:{args.dtype}:bro{':vi' if args.value_codec else ''}:{world}")
        if tr:
            traffic = tr
    value = 2.0 * A.nnz / (total_ms / args.steps * 1e-3) / 1e9
    base_value = 2.0 * A.nnz / (base_ms * 1e-3) / 1e9
    cpu = None
    if not args.no_cpu_baseline and world == 1:
        cpu = cpu_oracle_baseline(A, x_host)
    bro_name = {"ell": "BRO-ELL", "hyb": "BRO-HYB", "coo": "BRO-COO"}[fmt]
    if info["value_code_bytes"]:
        bro_name += " + value index"
    out = {
        "metric": METRIC,
        "value": value,
        "unit": "GFLOP/s",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": total_ms / args.steps,
        "higher_is_better": True,
        "scaling": "strong",
        "vs_baseline": None,
        "dtype": args.dtype,
        "data": "synthetic",
        "config": {
            "workload": workload_label(args.workload),
            "format": bro_name, "m": A.m, "n": A.n, "nnz": A.nnz,
            "vec_words": info["vec_words"], "slice_h": info["slice_h"], "coo_T": info["coo_T"],
            "ell_kernel": {0: None, 1: "tiny", 2: "few-slice", 3: "small-window", 4: "mid-window",
                           5: "general", 6: "split-4", 7: "split-2"}[info["ell_kernel"]] if info["nnz_ell"] or fmt != "coo" else None,
            "l2": ("flushed (2x L2 write) before every step" if args.flush_l2 else
                   ("inputs larger than L2" if alg_bytes > L2_BYTES else "L2-resident (warm)")),
            "parallelism": f"row-block x{world}" + (f" + {exch_info['exchange']} exchange of y per step (x_(k+1) = A.x_k)"
                                                    if world > 1 else ""),
            "eta_stream": info["eta_stream"], "eta_total": info["eta_total"],
            "value_codec": ({"codes": f"{info['value_code_bytes']}-byte", "distinct_values": info["value_dict_size"]}
                            if info["value_code_bytes"] else None),
        },
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                     "frac": achieved / peak, "traffic": traffic,
                     "peak_kind": peak_kind,
                     "kernel": (f"bro_ell_{'tiny' if info['ell_kernel'] == 1 else 'od'}"
                                f"<{'double' if dtype == np.float64 else 'float'},V={info['vec_words']},"
                                f"R={info['slice_h'] // 32}>")
                     if fmt == "ell" else ("coo_spmv + coo_fixup" if fmt == "coo" else
                                           "bro_ell + coo_spmv + coo_fixup"),
                     "algorithmic_bytes_per_launch": alg_bytes, "kernel_ms": kern_ms,
                     "frac_of_8TBps_spec": achieved / 8000.0,
                     "read_stream_GBps": rc, "read_stream_how": "torch.sum over 2 GiB fp32 (a library "
                     "reduction, context only: the in-repo ELLPACK streams faster)" if rc else None},
        "uncompressed": {"format": {"ell": "ELLPACK", "hyb": "HYB", "coo": "COO"}[fmt], "value": base_value,
                         "unit": "GFLOP/s", "kernel_ms": base_kern_ms,
                         "algorithmic_bytes": binfo["algorithmic_bytes"],
                         "achieved_GBps": binfo["algorithmic_bytes"] / (base_kern_ms * 1e-3) / 1e9,
                         "speedup_bro": value / base_value},
        "step_ms_p10_p50_p90": [float(np.percentile(per_step, q)) for q in (10, 50, 90)],
        "cuda_graph": graph,
        "exchange": exch_info,
        "gpu_launches": int(launches * args.steps),
        "clocks": ck,
        "cpu_baseline": cpu,
        "e2e": e2e,
        "gflops_kernel_only": 2.0 * A.nnz / world / (kern_ms * 1e-3) / 1e9 if world == 1 else None,
    }
    print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
