#!/usr/bin/env python
"""Benchmark: the six fp32 Level-3 routines at N=8192 on B200 (BASELINE.json metric).

One STEP = one pass of the whole hot path over one batch of synthetic input:
    C <- sgemm ('N','N', a, A, B, b, C)          2 N^3 flops
    C <- ssymm ('L','L', a, A, B, b, C)          2 N^3      (A's lower triangle)
    C <- ssyrk ('L','N', a, A, b, C)             N^2 (N+1)  (lower triangle of C)
    C <- ssyr2k('L','N', a, A, B, b, C)          2 N^3 + N
    X <- strmm ('L','L','N','N', a, T, X)        N^3        (X = B copied)
    X <- strsm ('L','L','N','N', a, T, X)        N^3
with a = 1.5, b = 0.5, N = K = 8192 (configs[1..3] of BASELINE.json at N=8192),
T diagonally dominant lower-triangular.  Flops are LAWN-41 algorithmic counts
(Q1).  value = total flops / step time (GFLOPS, all ranks).

Every operand is 256 MiB > 126 MB L2, so no L2 flush is needed between steps.
At N>1 (torchrun) each rank runs the chain on its own column slab of B/C/X
(n_global = 8192 * world) after an NCCL broadcast of A and T from rank 0
inside the timed region (column-slab sharding, weak scaling).

After the headline (default 3xTF32) run, a short device-only pass of the same
chain in the opt-in TF32+BF16X mode is reported under "alt_mode" (never as
the headline; --no-alt-mode skips it), and the box's cuBLAS SGEMM (fp32 and
1-pass TF32, torch.matmul) under "context" (--no-context skips it).

--impl reference times the fp64 CPU oracle (the deliberately slow reference
arm of this tier) on a bounded column sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

N = 8192
ALPHA, BETA = 1.5, 0.5
ROUTINES = ["sgemm", "ssymm", "ssyrk", "ssyr2k", "strmm", "strsm"]


def flops(n, cols=None):
    """LAWN-41 counts for one step (cols = columns of B/C actually computed)."""
    c = n if cols is None else cols
    return {
        "sgemm": 2.0 * n * n * c,
        "ssymm": 2.0 * n * n * c,
        "ssyrk": 1.0 * n * n * (n + 1) * (c / n),
        "ssyr2k": (2.0 * n * n * n + n) * (c / n),
        "strmm": 1.0 * n * n * c,
        "strsm": 1.0 * n * n * c,
    }


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d, "measured"
    return {"bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0, "hbm_gbs": 6650.0}, "fallback"


# nominal dense TF32 / BF16 ratio (B200_PROFILING.md: 1.1 vs 2.25 PFLOP/s)
TF32_OVER_BF16 = 1.1 / 2.25


def fp32_3xtf32_peak(peaks, sustained=True):
    """fp32-via-3xTF32 peak: measured bf16 x nominal tf32/bf16 ratio / 3 UMMAs."""
    bf16 = peaks["bf16_tflops_sustained" if sustained else "bf16_tflops"]
    return bf16 * TF32_OVER_BF16 / 3.0


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region
    (every `interval_ms`; each row keeps the host time it arrived at, so a
    window of the run can be summarised on its own)."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index, interval_ms=200):
        self.index = index
        self.interval_ms = interval_ms
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                 "--format=csv,noheader,nounits", "-lms", str(self.interval_ms)],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")] + [time.time()])

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self, t0=None, t1=None):
        rows = [r for r in self.rows if (t0 is None or r[-1] >= t0) and (t1 is None or r[-1] <= t1)]
        if not rows and (t0 is not None or t1 is not None):
            rows = self.rows                    # window shorter than one sample: every sample
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        sm = [float(r[0]) for r in rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        pw = [float(r[2]) for r in rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in rows:
            for nm, v in zip(names, r[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        out = {"sm_mhz": float(np.median(sm)) if sm else None,
               "sm_max_mhz": max(mx) if mx else None,
               "samples": len(rows), "reasons": sorted(reasons)}
        if pw:
            out["power_w"] = float(np.median(pw))
        return out


# ----------------------------------------------------------------------------- inputs
def make_inputs(n, cols, rank):
    """Seeded host inputs (pinned later).  A, T are shared (broadcast at N>1);
    B, C are this rank's column slab of the global matrices."""
    import blas3_inputs as gen
    A = gen.uniform(n, n, "bench-A") if rank == 0 else None
    T = gen.triangular_dd(n, "L", "N", "bench-T") if rank == 0 else None
    B = gen.uniform(n, cols, "bench-B", rank)
    C = gen.uniform(n, cols, "bench-C", rank)
    return A, T, B, C


def pinned(arr, torch):
    """numpy Fortran (n x c) -> pinned host tensor laid out (c, n) row-major."""
    t = torch.from_numpy(np.ascontiguousarray(arr.T)).pin_memory()
    return t


# ----------------------------------------------------------------------------- our arm
def init_dist():
    """One process per GPU (torchrun env).  NCCL communicators are created
    eagerly (device_id) and exercised by a barrier, and each rank logs its
    communicator to stderr so a launch's rank count is visible in the log."""
    import torch
    import torch.distributed as dist
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    local = local % max(1, torch.cuda.device_count())   # (a 1-GPU logic check may share a device)
    torch.cuda.set_device(local)
    comm = {"backend": None, "world": world}
    if world > 1:
        backend = os.environ.get("BLAS3_BENCH_BACKEND", "nccl")   # gloo: 1-GPU logic check only
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
        dist.barrier()
        comm["backend"] = backend
        if backend == "nccl":
            v = torch.cuda.nccl.version()
            comm["nccl_version"] = ".".join(map(str, v)) if isinstance(v, tuple) else str(v)
        print(f"[bench] rank {rank}/{world} on cuda:{local}: {backend} process group up "
              f"(communicator initialised, barrier passed)", file=sys.stderr, flush=True)
    return torch, dist, world, rank, local, comm


def run_ours(args):
    torch, dist, world, rank, local, comm_info = init_dist()

    import paper_conf_ipps_cuiwxyf11_b200 as b3
    b3.set_math_mode(args.math)
    n = N if args.size is None else args.size
    cols = n                                   # per-rank slab width (weak scaling)
    A_h, T_h, B_h, C_h = make_inputs(n, cols, rank)
    dev = torch.device("cuda", local)

    def colmaj(t2d):                           # (c, n) row-major device -> (n, c) column-major view
        return t2d.t()

    # device buffers (column-major views of (cols, n) row-major storage)
    dA = torch.empty((n, n), device=dev); dT = torch.empty((n, n), device=dev)
    dB = torch.empty((cols, n), device=dev); dC0 = torch.empty((cols, n), device=dev)
    dC = torch.empty((cols, n), device=dev); dX = torch.empty((cols, n), device=dev)
    hA = pinned(A_h, torch) if rank == 0 else None
    hT = pinned(T_h, torch) if rank == 0 else None
    hB, hC = pinned(B_h, torch), pinned(C_h, torch)
    hC_out = torch.empty((cols, n), pin_memory=True); hX_out = torch.empty((cols, n), pin_memory=True)
    if rank == 0:
        dA.copy_(hA); dT.copy_(hT)
    dB.copy_(hB); dC0.copy_(hC)
    if world > 1:
        dist.broadcast(dA, 0); dist.broadcast(dT, 0)
    torch.cuda.synchronize()

    A, T = colmaj(dA), colmaj(dT)
    Bm, C0, C, X = colmaj(dB), colmaj(dC0), colmaj(dC), colmaj(dX)
    stream = torch.cuda.current_stream()
    fl = flops(n, cols)
    ev = {r: [] for r in ROUTINES}

    if world > 1:
        from paper_conf_ipps_cuiwxyf11_b200 import dist as d3
        # The exchange steps, all overlapped with compute:
        #  * A: broadcast in 8 K-panels on a comm stream, consumed by the
        #    panel GEMMs of the sgemm as they land (d3.sgemm);
        #  * T: only its lower triangle, 4 trapezoid panels, on a second comm
        #    stream, enqueued right after A's panels (needed from strmm on);
        #  * SYRK/SYR2K (no right-hand side to shard): k-split weak scaling --
        #    rank r's own k-slab (its B slab; for SYR2K its B and C0 slabs),
        #    the partial products summed by an NCCL all-reduce on a third
        #    stream that overlaps the next routines.  beta*C is applied on
        #    rank 0 only (the others start from zeros), so the sum is exact.
        # While a collective is in flight the products leave RESERVE SMs to
        # NCCL (BLAS3_OPT_MAX_SMS).
        RESERVE = 16
        # device-side panel consumption (one streamed GEMM polling per-panel
        # flags) needs its own GPU per rank: ranks sharing one device (the gloo
        # logic check) would let one rank's persistent grid take the SMs the
        # other rank's flag writes need
        DEVICE_SIDE = comm_info.get("backend") == "nccl"
        nsm = torch.cuda.get_device_properties(dev).multi_processor_count
        dCs1 = torch.empty((n, n), device=dev); dCs2 = torch.empty((n, n), device=dev)
        Cs1, Cs2 = colmaj(dCs1), colmaj(dCs2)
        comm_T = torch.cuda.Stream(device=dev)
        comm_R = torch.cuda.Stream(device=dev)
        beta_r = BETA if rank == 0 else 0.0

        def allreduce_async(buf):
            e = torch.cuda.Event(); e.record(torch.cuda.current_stream())
            with torch.cuda.stream(comm_R):
                comm_R.wait_event(e)
                d3.syrk_k_split(buf)

        def syrk_k(Bk=None):
            Bk = Bm if Bk is None else Bk
            if rank == 0:
                dCs1.copy_(dC0)
            else:
                dCs1.zero_()
            b3.ssyrk("L", "N", ALPHA, Bk, beta_r, Cs1)
            allreduce_async(dCs1)

        def syr2k_k(Bk=None, Ck=None):
            Bk = Bm if Bk is None else Bk
            Ck = C0 if Ck is None else Ck
            if rank == 0:
                dCs2.copy_(dC0)
            else:
                dCs2.zero_()
            b3.ssyr2k("L", "N", ALPHA, Bk, Ck, beta_r, Cs2)
            allreduce_async(dCs2)

        def bcast_T_async(Tv):
            e = torch.cuda.Event(); e.record(torch.cuda.current_stream())
            with torch.cuda.stream(comm_T):
                comm_T.wait_event(e)
                for p0, p1 in d3.k_panels(n, 4):
                    d3.broadcast_trapezoid(Tv, p0, p1, True)
                eT = torch.cuda.Event(); eT.record(comm_T)
            return eT

    def chain(record):
        def timed(name, fn, reserve=False):
            def run():
                if reserve and world > 1:
                    with b3.options(max_sms=nsm - RESERVE):
                        fn()
                else:
                    fn()
            if record:
                e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
                e0.record(stream); run(); e1.record(stream)
                ev[name].append((e0, e1))
            else:
                run()
        if world == 1:
            timed("sgemm", lambda: b3.sgemm("N", "N", ALPHA, A, Bm, BETA, C))
            timed("ssymm", lambda: b3.ssymm("L", "L", ALPHA, A, Bm, BETA, C))
            timed("ssyrk", lambda: b3.ssyrk("L", "N", ALPHA, A, BETA, C))
            timed("ssyr2k", lambda: b3.ssyr2k("L", "N", ALPHA, A, Bm, BETA, C))
            timed("strmm", lambda: b3.strmm("L", "L", "N", "N", ALPHA, T, X))
            timed("strsm", lambda: b3.strsm("L", "L", "N", "N", ALPHA, T, X))
            return
        # (collectives of one process group share one NCCL stream in enqueue
        # order: A's panels go first, T's triangle queues behind them)
        timed("sgemm", lambda: d3.sgemm("N", "N", ALPHA, A, Bm, BETA, C, panels=8, reserve_sms=RESERVE,
                                        device_side=DEVICE_SIDE))
        eT = bcast_T_async(T)
        timed("ssymm", lambda: b3.ssymm("L", "L", ALPHA, A, Bm, BETA, C), reserve=True)
        timed("ssyrk", syrk_k, reserve=True)
        timed("ssyr2k", syr2k_k, reserve=True)
        stream.wait_event(eT)
        timed("strmm", lambda: b3.strmm("L", "L", "N", "N", ALPHA, T, X), reserve=True)
        timed("strsm", lambda: b3.strsm("L", "L", "N", "N", ALPHA, T, X))
        stream.wait_stream(comm_R)            # the reduced SYRK/SYR2K results are part of the step

    def step_device(record=False):
        # fresh working copies so every step computes on the same data
        dC.copy_(dC0); dX.copy_(dB)
        chain(record)

    # ---- e2e leg: host (pinned) inputs -> the chain -> host results, every step.
    # Two device buffer sets and two copy streams (H2D, D2H: PCIe is full
    # duplex) so step s+1's uploads run under step s's compute and step s's
    # downloads under step s+1's; every step still moves its own inputs in and
    # its results out inside the timed region.  Within a step B/C land in
    # column chunks and the sgemm runs on each slab as it arrives; T uploads
    # behind the first routines.
    h2d_stream = torch.cuda.Stream(device=dev)
    d2h_stream = torch.cuda.Stream(device=dev)
    E2E_CHUNKS = 4
    bufs = [dict(A=dA, T=dT, B=dB, C=dC, X=dX)]
    bufs.append({k: torch.empty_like(v) for k, v in bufs[0].items()})
    free_ev = [None, None]            # set b may be overwritten once this event has passed

    def step_e2e(s):
        bset = bufs[s % 2]
        A_, T_ = colmaj(bset["A"]), colmaj(bset["T"])
        Bm_, C_, X_ = colmaj(bset["B"]), colmaj(bset["C"]), colmaj(bset["X"])
        bounds = [(i * cols // E2E_CHUNKS, (i + 1) * cols // E2E_CHUNKS) for i in range(E2E_CHUNKS)]
        with torch.cuda.stream(h2d_stream):
            if free_ev[s % 2] is not None:
                h2d_stream.wait_event(free_ev[s % 2])
            if rank == 0:
                bset["A"].copy_(hA, non_blocking=True)
            eA = torch.cuda.Event(); eA.record(h2d_stream)
            evs = []
            for c0, c1 in bounds:                   # (cols, n) row-major rows = matrix columns
                bset["B"][c0:c1].copy_(hB[c0:c1], non_blocking=True)
                bset["C"][c0:c1].copy_(hC[c0:c1], non_blocking=True)
                e = torch.cuda.Event(); e.record(h2d_stream); evs.append(e)
            if rank == 0:
                bset["T"].copy_(hT, non_blocking=True)
            eT = torch.cuda.Event(); eT.record(h2d_stream)
        stream.wait_event(eA)
        if world > 1:
            for (c0, c1), e in zip(bounds, evs):
                stream.wait_event(e)
            d3.sgemm("N", "N", ALPHA, A_, Bm_, BETA, C_, panels=8, reserve_sms=RESERVE, device_side=DEVICE_SIDE)
        else:
            for (c0, c1), e in zip(bounds, evs):
                stream.wait_event(e)
                b3.sgemm("N", "N", ALPHA, A_, Bm_[:, c0:c1], BETA, C_[:, c0:c1])
        b3.ssymm("L", "L", ALPHA, A_, Bm_, BETA, C_)
        if world == 1:
            b3.ssyrk("L", "N", ALPHA, A_, BETA, C_)
            b3.ssyr2k("L", "N", ALPHA, A_, Bm_, BETA, C_)
        else:
            syrk_k(Bm_)
            syr2k_k(Bm_, C_)
        eC = torch.cuda.Event(); eC.record(stream)
        with torch.cuda.stream(d2h_stream):
            d2h_stream.wait_event(eC)
            hC_out.copy_(bset["C"], non_blocking=True)
        stream.wait_event(eT)
        if world > 1:
            stream.wait_event(bcast_T_async(T_))
        bset["X"].copy_(bset["B"])
        b3.strmm("L", "L", "N", "N", ALPHA, T_, X_)
        b3.strsm("L", "L", "N", "N", ALPHA, T_, X_)
        if world > 1:
            stream.wait_stream(comm_R)
        eX = torch.cuda.Event(); eX.record(stream)
        with torch.cuda.stream(d2h_stream):
            d2h_stream.wait_event(eX)
            hX_out.copy_(bset["X"], non_blocking=True)
            fe = torch.cuda.Event(); fe.record(d2h_stream)
        free_ev[s % 2] = fe

    def e2e_loop(steps):
        """Time `steps` pipelined e2e steps on the device clock: from before the
        first upload to after the last download (max over ranks)."""
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        h2d_stream.wait_event(e0)
        for s_ in range(steps):
            step_e2e(s_)
        stream.wait_stream(d2h_stream)
        stream.wait_stream(h2d_stream)
        e1.record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        ms_ = e0.elapsed_time(e1)
        if world > 1:
            t = torch.tensor([ms_], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms_ = float(t.item())
        free_ev[0] = free_ev[1] = None
        return ms_

    def timed_loop(fn, steps, record=False):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(steps):
            fn(record) if record is not None else fn()
        e1.record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        ms = e0.elapsed_time(e1)
        if world > 1:
            t = torch.tensor([ms], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
        return ms

    for _ in range(args.warmup):
        step_device()
    torch.cuda.synchronize()
    launches0 = b3.launch_count()
    with ClockSampler(local, interval_ms=50) as clk:
        time.sleep(0.6)                       # nvidia-smi start-up, before the timed region
        t_clk0 = time.time()
        ms = timed_loop(lambda rec: step_device(rec), args.steps, record=True)
        t_clk1 = time.time()
    launches = b3.launch_count() - launches0

    # e2e: same metric through the public API with host buffers
    ms_e2e = float("nan")
    if not args.no_e2e:
        e2e_loop(max(1, min(2, args.warmup)))          # warm-up (both buffer sets)
        ms_e2e = e2e_loop(args.steps)

    ev_ms = {r: float(np.mean([a.elapsed_time(b) for a, b in ev[r]])) for r in ROUTINES}

    # the opt-in TF32+BF16X mode on the same data, device timing only, reported
    # beside (never instead of) the default 3xTF32 headline
    alt = None
    if world == 1 and args.math == "3xtf32" and not args.no_alt_mode:
        per_default = {r: list(v) for r, v in ev.items()}
        for r in ROUTINES:
            ev[r].clear()
        b3.set_math_mode("tf32_bf16x")
        try:
            for _ in range(args.warmup):
                step_device()
            ms_alt = timed_loop(lambda rec: step_device(rec), args.steps, record=True)
            alt_routines = {}
            for r in ROUTINES:
                avg = float(np.mean([a.elapsed_time(b) for a, b in ev[r]]))
                alt_routines[r] = {"ms": round(avg, 4), "gflops": round(fl[r] / (avg * 1e-3) / 1e9, 1)}
            alt = {"math": "tf32_bf16x",
                   "value": round(sum(fl.values()) / (ms_alt / args.steps * 1e-3) / 1e9, 1),
                   "unit": "GFLOPS", "ms_per_step": round(ms_alt / args.steps, 3),
                   "routines": alt_routines,
                   "note": "opt-in mode (DESIGN.md Q28): hi*hi as one TF32 UMMA + both cross terms "
                           "in one packed BF16 UMMA; same data, device timing, after the headline run"}
        finally:
            b3.set_math_mode(args.math)
            for r in ROUTINES:
                ev[r][:] = per_default[r]

    # per routine, in isolation: each routine back to back for ~0.5 s with the
    # clocks sampled every 50 ms (the chain's own clock record covers the whole
    # step); STRMM / STRSM restore X every call (the copy is inside the time)
    isolated = None
    if world == 1 and not args.no_routine_clocks:
        isolated = {}
        single = {
            "sgemm": lambda: b3.sgemm("N", "N", ALPHA, A, Bm, BETA, C),
            "ssymm": lambda: b3.ssymm("L", "L", ALPHA, A, Bm, BETA, C),
            "ssyrk": lambda: b3.ssyrk("L", "N", ALPHA, A, BETA, C),
            "ssyr2k": lambda: b3.ssyr2k("L", "N", ALPHA, A, Bm, BETA, C),
            "strmm": lambda: (dX.copy_(dB), b3.strmm("L", "L", "N", "N", ALPHA, T, X)),
            "strsm": lambda: (dX.copy_(dB), b3.strsm("L", "L", "N", "N", ALPHA, T, X)),
        }
        with ClockSampler(local, interval_ms=50) as clk_r:
            time.sleep(0.4)
            for r in ROUTINES:
                fn = single[r]
                fn(); torch.cuda.synchronize()
                reps = max(3, int(500.0 / max(0.1, ev_ms[r])))
                c0 = torch.cuda.Event(enable_timing=True); c1 = torch.cuda.Event(enable_timing=True)
                t0 = time.time()
                c0.record(stream)
                for _ in range(reps):
                    fn()
                c1.record(stream)
                torch.cuda.synchronize()
                t1 = time.time()
                ms_r = c0.elapsed_time(c1) / reps
                isolated[r] = {"ms": round(ms_r, 4), "gflops": round(fl[r] / (ms_r * 1e-3) / 1e9, 1),
                               "reps": reps, "clocks": clk_r.summary(t0, t1)}
        for r in ROUTINES:            # each routine in its own sustained loop (the chain's
            isolated[r]["pct_of_sgemm"] = round(   # per-routine times carry the power state of the
                100.0 * isolated[r]["gflops"] / isolated["sgemm"]["gflops"], 1)   # routine before)

    # context (north star: "reports the box's cuBLAS SGEMM as context"): torch's
    # cuBLAS fp32 SGEMM (TF32 off) and its 1-pass TF32 mode on the same A, B
    context = None
    if world == 1 and n == N and not args.no_context:
        def cublas_rate(tf32):
            prev = torch.backends.cuda.matmul.allow_tf32
            torch.backends.cuda.matmul.allow_tf32 = tf32
            try:
                out = torch.empty((n, n), device=dev)
                for _ in range(2):
                    torch.matmul(A, Bm, out=out)
                torch.cuda.synchronize()
                c0 = torch.cuda.Event(enable_timing=True); c1 = torch.cuda.Event(enable_timing=True)
                reps = 3
                c0.record(stream)
                for _ in range(reps):
                    torch.matmul(A, Bm, out=out)
                c1.record(stream)
                torch.cuda.synchronize()
                return round(2.0 * n ** 3 / (c0.elapsed_time(c1) / reps * 1e-3) / 1e9, 1)
            finally:
                torch.backends.cuda.matmul.allow_tf32 = prev
        context = {"cublas_sgemm_fp32_gflops": cublas_rate(False),
                   "cublas_sgemm_tf32_1pass_gflops": cublas_rate(True),
                   "note": "torch.matmul (cuBLAS) N=8192 NN on the bench's A, B; fp32 = TF32 off "
                           "(the fp32-accurate comparator); tf32 = 1 pass, ~1e-3 accuracy",
                   # the paper's own numbers with their hardware (quoted, not measured here;
                   # PAPER.md P:15)
                   "paper": {"max_speedup_over_cublas3.2": {"GeForce 9800": 5.4, "GTX285": 2.8,
                                                             "Tesla C2050": 3.4},
                             "gtx285_cublas3.2_sgemm_gflops": 420, "gtx285_cublas3.2_ssymm_gflops": 155,
                             "gtx285_oa_ssymm_gflops": 403, "problem": "fp32, N=4096"}}

    # fp64 family (blas3_d*): DGEMM NN and DTRSM LLNN at N = 4096 on
    # the same device, against the DFMA peak (148 SM x 64 DFMA/clk x 2 x max
    # clock; tools/probes/dmma_rate.cu measured 36.4 TF/s for DFMA and 37.1 for
    # DMMA, so the CUDA cores are the FP64 roofline)
    fp64 = None
    if world == 1 and not args.no_fp64:
        n64 = 4096
        f64t = lambda: b3.colmajor(n64, n64, dtype=torch.float64).uniform_(-1, 1)  # noqa: E731
        A64, B64, C64, X64 = f64t(), f64t(), f64t(), f64t()
        T64 = f64t().mul_(1.0 / n64)
        T64.diagonal().fill_(1.0)
        pk64 = 148 * 64 * 2 * load_peaks()[0].get("sm_max_mhz", 1965.0) * 1e6 / 1e12
        fp64 = {"n": n64, "peak_tflops": round(pk64, 1),
                "peak_source": "148 SM x 64 DFMA/clk x 2 x max SM clock (DFMA; DMMA measured no faster)"}
        for name, fn, flops64 in (("dgemm", lambda: b3.dgemm("N", "N", ALPHA, A64, B64, BETA, C64), 2.0 * n64 ** 3),
                                  ("dtrsm", lambda: b3.dtrsm("L", "L", "N", "N", ALPHA, T64, X64), 1.0 * n64 ** 3)):
            X64.copy_(B64)
            fn()
            torch.cuda.synchronize()
            c0 = torch.cuda.Event(enable_timing=True); c1 = torch.cuda.Event(enable_timing=True)
            c0.record(stream)
            for _ in range(3):
                fn()
            c1.record(stream)
            torch.cuda.synchronize()
            ms64 = c0.elapsed_time(c1) / 3
            fp64[name] = {"ms": round(ms64, 3), "gflops": round(flops64 / (ms64 * 1e-3) / 1e9, 1),
                          "frac": round(flops64 / (ms64 * 1e-3) / 1e12 / pk64, 3)}
        del A64, B64, C64, X64, T64

    total_flops = sum(fl.values()) * world
    step_ms = ms / args.steps
    value = total_flops / (step_ms * 1e-3) / 1e9
    e2e_value = total_flops / (ms_e2e / args.steps * 1e-3) / 1e9
    per = {}
    for r in ROUTINES:
        ts = [a.elapsed_time(b) for a, b in ev[r]]
        avg = float(np.mean(ts))
        per[r] = {"ms": round(avg, 4), "gflops": round(fl[r] / (avg * 1e-3) / 1e9, 1)}
    peaks, peak_src = load_peaks()
    # Peak denominator (B200_PROFILING.md): the burst figure for a kernel timed
    # alone or in a short loop, the sustained one only for a loop of >= 2 s
    # under the power cap.  The timed region here is steps x ~21 ms.
    sustained = ms >= 2000.0
    pk = fp32_3xtf32_peak(peaks, sustained=sustained)
    if args.math == "tf32_bf16x":        # 2 UMMAs per k-step: tf32 (K=8) + bf16 (K=16), equal time
        pk = pk * 3.0 / 2.0
    if args.math == "simt":
        pk = 148 * 128 * 2 * (peaks.get("sm_max_mhz", 1965.0)) * 1e6 / 1e12
    for r in ROUTINES:                   # every routine against the same kernel peak
        per[r]["frac"] = round(per[r]["gflops"] / 1e3 / pk, 3)
        per[r]["pct_of_sgemm"] = round(100.0 * per[r]["gflops"] / per["sgemm"]["gflops"], 1)
    sg_ms = per["sgemm"]["ms"]
    achieved = fl["sgemm"] / (sg_ms * 1e-3) / 1e12
    traffic, traffic_src = None, None
    tp = os.path.join(ROOT, "profiles", "ncu_sgemm_traffic.json")
    if os.path.exists(tp) and n == N and args.math == "3xtf32":   # (the capture is of the 3xTF32 kernel)
        try:
            tj = json.load(open(tp))
            # only a capture of THIS build counts (the library's content hash)
            stamp = os.path.join(ROOT, "paper_conf_ipps_cuiwxyf11_b200", "libblas3.so.sha256")
            cur = open(stamp).read().strip() if os.path.exists(stamp) else None
            if tj.get("lib_sha256") and tj.get("lib_sha256") == cur:
                traffic, traffic_src = tj.get("dram_bytes_per_launch"), tj.get("source")
            else:
                traffic_src = "stale: profiles/ncu_sgemm_traffic.json is a capture of another build"
        except (ValueError, OSError):
            traffic = None
    h2d = (2 * n * n * 4 if rank == 0 else 0) + 2 * n * cols * 4
    d2h = 2 * n * cols * 4
    if context is not None:
        context["sgemm_speedup_over_cublas_fp32"] = round(
            per["sgemm"]["gflops"] / context["cublas_sgemm_fp32_gflops"], 2)
    out = {
        "metric": "GFLOPS per routine (SGEMM/SSYMM/SSYRK/SSYR2K/STRMM/STRSM) at N=8192, "
                  "1/2/4/8 B200, % of peak",
        "value": round(value, 1),
        "unit": "GFLOPS",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": round(step_ms, 3),
        "higher_is_better": True,
        "scaling": "weak",
        "vs_baseline": None,
        "dtype": "f32",
        "data": "synthetic (seeded U(-1,1); diagonally dominant T)",
        "config": {
            "workload": "configs[1..3] at N=8192: sgemm NN, ssymm LL, ssyrk LN, ssyr2k LN "
                        "(K=8192), strmm LLNN, strsm LLNN; alpha=1.5 beta=0.5",
            "n": n, "k": n, "cols_per_rank": cols, "math": args.math,
            "l2": "no flush: every operand is 256 MiB > 126 MB L2",
            "parallelism": (f"dp{world}: column slabs of B/C/X per rank ({cols} columns each); A broadcast "
                            f"from rank 0 in 8 K-panels consumed as they land by one streamed sgemm "
                            f"(device-side panel flags; per-panel GEMMs under gloo), T's lower "
                            f"triangle in 4 trapezoid panels overlapped with sgemm..ssyr2k (NCCL, "
                            f"comm streams, 16 SMs reserved while in flight); ssyrk/ssyr2k k-split, "
                            f"partials all-reduced (NCCL) overlapped with the next routines")
            if world > 1 else "1 GPU",
        },
        "routines": per,
        "pct_of_peak": round(100.0 * value / world / 1e3 / pk, 1),
        "roofline": {
            "bound": "tensor" if args.math != "simt" else "alu",
            "kernel": "tc_structured_gemm (the sgemm launch)" if args.math != "simt"
            else "simt_structured_gemm (the sgemm launch)",
            "achieved": round(achieved, 2),
            "peak": round(pk, 1),
            "unit": "TFLOP/s",
            "frac": round(achieved / pk, 3),
            "peak_source": (f"{peak_src} bf16 {'sustained' if sustained else 'burst'} "
                            f"{peaks.get('bf16_tflops_sustained' if sustained else 'bf16_tflops')} TF/s "
                            f"(timed loop {ms / 1e3:.2f} s; sustained only for >= 2 s) x "
                            f"nominal tf32/bf16 {TF32_OVER_BF16:.3f} / "
                            + ("3 (3xTF32)" if args.math == "3xtf32" else
                               "2 (TF32 hi*hi + one BF16 K=16 cross-term UMMA per k-step)"))
            if args.math != "simt" else "148 SM x 128 FP32 lanes x 2 x max SM clock",
            "traffic": traffic,
            "traffic_source": traffic_src,
            "algorithmic_bytes": 4 * n * n * 4 if args.math != "simt" else None,
        },
        "e2e": {"value": round(e2e_value, 1), "unit": "GFLOPS",
                "h2d_bytes_per_step": h2d * world, "d2h_bytes_per_step": d2h * world},
        "gpu_launches": int(launches),
        "comm": comm_info,
        "alt_mode": alt,
        "fp64": fp64,
        "context": context,
        "gpu_launches_per_step": round(launches / args.steps, 1),
        "isolated": isolated,
        "clocks": clk.summary(t_clk0, t_clk1 + 0.05),
    }
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        out["cpu_baseline"] = cpu_baseline(args.cpu_seconds)
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


# ----------------------------------------------------------------------------- configs[4]
CFG5_N = 32768
CFG5_ROUTINES = ["sgemm", "ssymm", "strsm"]


def cfg5_inputs(torch, n, c0, c1, rank, dev):
    """Seeded device-side inputs of BASELINE configs[4] (an N = 32768 host
    generation would take minutes).  Every 256-column block of a global
    matrix has its own Philox seed (hash of name and block index), so a
    rank's slab holds the same numbers for any world size.  A: U(-1,1) n x n
    (rank 0); T: lower triangular, off-diagonal U(-1,1), a_ii = 1 + max(row,
    column) abs-sum (reading Q22), NaN in the blank triangle (never read);
    B, C: U(-1,1) column slabs [c0, c1)."""
    import hashlib

    def block(name, j, rows, cols):
        h = hashlib.sha256(repr((20111, "cfg5", name, n, j)).encode()).digest()
        g = torch.Generator(device=dev)
        g.manual_seed(int.from_bytes(h[:8], "little") & ((1 << 63) - 1))
        return torch.rand((cols, rows), generator=g, device=dev).mul_(2.0).sub_(1.0)

    def slab_of(name, a, b, out):              # out: (b - a, n) row-major storage of columns a..b
        for j in range(a // 256, -(-b // 256)):
            x0, x1 = max(a, j * 256), min(b, (j + 1) * 256)
            out[x0 - a:x1 - a] = block(name, j, n, min(256, n - j * 256))[x0 - j * 256:x1 - j * 256]
        return out

    dA = torch.empty((n, n), device=dev)
    dT = torch.empty((n, n), device=dev)
    if rank == 0:
        slab_of("A", 0, n, dA)
        slab_of("T", 0, n, dT)                 # dT[j] = column j of T
        tt = dT                                # rows of tt = columns of T; keep rows > col (strict lower)
        idx = torch.arange(n, device=dev)
        rowsum = torch.zeros(n, dtype=torch.float64, device=dev)
        colsum = torch.zeros(n, dtype=torch.float64, device=dev)
        for j0 in range(0, n, 1024):
            blk = tt[j0:j0 + 1024]             # columns j0.. of T, each a row here
            jj = idx[j0:j0 + 1024, None]
            strict = idx[None, :] > jj         # T(i, j) with i > j
            blk.masked_fill_(~strict, 0.0)
            a64 = blk.abs().double()
            colsum[j0:j0 + 1024] = a64.sum(1)
            rowsum += a64.sum(0)
            blk.masked_fill_(idx[None, :] < jj, float("nan"))
        dom = (1.0 + torch.maximum(rowsum, colsum)).float()
        tt.diagonal().copy_(dom)
    cols = c1 - c0
    dB = slab_of("B", c0, c1, torch.empty((cols, n), device=dev))
    dC0 = slab_of("C", c0, c1, torch.empty((cols, n), device=dev))
    return dA, dT, dB, dC0


def run_cfg5(args):
    """BASELINE configs[4]: N = 32768 SGEMM NN, SSYMM LL and STRSM LLNN with
    the right-hand side in column slabs of N/P columns per rank (pre-resident)
    and A (T) resident on rank 0 and broadcast INSIDE each routine's timed
    region: A in 8 K-panels for SGEMM, only the stored lower triangle in
    trapezoid panels for SSYMM (8) and STRSM (4), every broadcast pipelined
    with the products that consume it (dist.py).  Strong scaling: the global
    problem is fixed; value = its LAWN-41 flops / step time (max over ranks),
    so T1/TP = value(P) / value(1)."""
    torch, dist, world, rank, local, comm_info = init_dist()
    import paper_conf_ipps_cuiwxyf11_b200 as b3
    from paper_conf_ipps_cuiwxyf11_b200 import dist as d3
    b3.set_math_mode(args.math)
    n = CFG5_N if args.size is None else args.size
    c0, c1 = d3.slab(n, world, rank)
    cols = c1 - c0
    dev = torch.device("cuda", local)
    dA, dT, dB, dC0 = cfg5_inputs(torch, n, c0, c1, rank, dev)
    dC = torch.empty_like(dC0); dX = torch.empty_like(dB)
    A, T, Bm, C0, C, X = dA.t(), dT.t(), dB.t(), dC0.t(), dC.t(), dX.t()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    stream = torch.cuda.current_stream()
    ev = {r: [] for r in CFG5_ROUTINES}
    calls = {
        "sgemm": lambda: d3.sgemm("N", "N", ALPHA, A, Bm, BETA, C, panels=8,
                                  device_side=comm_info.get("backend") == "nccl"),
        "ssymm": lambda: d3.ssymm("L", "L", ALPHA, A, Bm, BETA, C, panels=8),
        "strsm": lambda: d3.strsm("L", "L", "N", "N", ALPHA, T, X, panels=4),
    }

    def step(record=False):
        dC.copy_(dC0); dX.copy_(dB)
        for r in CFG5_ROUTINES:
            if record:
                e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
                e0.record(stream); calls[r](); e1.record(stream)
                ev[r].append((e0, e1))
            else:
                calls[r]()

    def timed_loop(steps, record):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(steps):
            step(record)
        e1.record(stream)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        if world > 1:
            t = torch.tensor([ms], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
        return ms

    for _ in range(args.warmup):
        step()
    launches0 = b3.launch_count()
    with ClockSampler(local, interval_ms=50) as clk:
        time.sleep(0.6)
        t_clk0 = time.time()
        ms = timed_loop(args.steps, True)
        t_clk1 = time.time()
    launches = b3.launch_count() - launches0

    # e2e: the same step through the public API with host buffers: A and T
    # uploaded on rank 0, the B/C slabs on every rank, C/X slabs downloaded
    e2e = None
    if not args.no_e2e:
        try:
            hA = torch.empty_like(dA, device="cpu").pin_memory() if rank == 0 else None
            hT = torch.empty_like(dT, device="cpu").pin_memory() if rank == 0 else None
            hB = torch.empty_like(dB, device="cpu").pin_memory()
            hC = torch.empty_like(dC0, device="cpu").pin_memory()
            hCo = torch.empty_like(dC0, device="cpu").pin_memory()
            hXo = torch.empty_like(dB, device="cpu").pin_memory()
            if rank == 0:
                hA.copy_(dA); hT.copy_(dT)
            hB.copy_(dB); hC.copy_(dC0)
            e2e_steps = max(1, min(args.steps, 3))

            def e2e_step():
                if rank == 0:
                    dA.copy_(hA, non_blocking=True); dT.copy_(hT, non_blocking=True)
                dB.copy_(hB, non_blocking=True); dC0.copy_(hC, non_blocking=True)
                step()
                hCo.copy_(dC, non_blocking=True); hXo.copy_(dX, non_blocking=True)
            e2e_step()
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            t0 = torch.cuda.Event(enable_timing=True); t1 = torch.cuda.Event(enable_timing=True)
            t0.record(stream)
            for _ in range(e2e_steps):
                e2e_step()
            t1.record(stream)
            torch.cuda.synchronize()
            ms_e = t0.elapsed_time(t1)
            if world > 1:
                t = torch.tensor([ms_e], device=dev)
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
                ms_e = float(t.item())
            tot = 5.0 * n ** 3
            e2e = {"value": round(tot / (ms_e / e2e_steps * 1e-3) / 1e9, 1), "unit": "GFLOPS",
                   "h2d_bytes_per_step": int(2 * n * n * 4 + 2 * n * n * 4), "d2h_bytes_per_step": int(2 * n * n * 4),
                   "steps": e2e_steps}
        except RuntimeError as exc:            # pinned host memory of the N = 32768 operands
            e2e = {"value": None, "unit": "GFLOPS", "h2d_bytes_per_step": None, "d2h_bytes_per_step": None,
                   "unavailable": f"host buffers: {str(exc).splitlines()[0][:120]}"}

    per = {}
    fl = {"sgemm": 2.0 * n ** 3, "ssymm": 2.0 * n ** 3, "strsm": 1.0 * n ** 3}
    for r in CFG5_ROUTINES:
        avg = float(np.mean([a.elapsed_time(b) for a, b in ev[r]]))
        if world > 1:
            t = torch.tensor([avg], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            avg = float(t.item())
        per[r] = {"ms": round(avg, 3), "gflops": round(fl[r] / (avg * 1e-3) / 1e9, 1)}
    step_ms = ms / args.steps
    value = sum(fl.values()) / (step_ms * 1e-3) / 1e9
    peaks, peak_src = load_peaks()
    pk = fp32_3xtf32_peak(peaks, sustained=True)
    out = {
        "metric": "GFLOPS per routine (SGEMM/SSYMM/SSYRK/SSYR2K/STRMM/STRSM) at N=8192, "
                  "1/2/4/8 B200, % of peak",
        "value": round(value, 1), "unit": "GFLOPS", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(step_ms, 3), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic (seeded device-side U(-1,1) per 256-column block; diagonally dominant T)",
        "config": {"workload": f"configs[4]: N={n} sgemm NN, ssymm LL, strsm LLNN, right-hand side in "
                               f"column slabs of N/P columns, A/T broadcast from rank 0 inside the timed region",
                   "n": n, "cols_per_rank": cols, "math": args.math,
                   "l2": "no flush: every operand is >= 512 MiB > 126 MB L2",
                   "parallelism": (f"dp{world}: column slabs; A broadcast in 8 K-panels (sgemm), lower "
                                   f"triangle in trapezoid panels (ssymm 8, strsm 4), pipelined with the "
                                   f"consuming products, 16 SMs reserved while in flight")
                   if world > 1 else "1 GPU (T1 of the strong-scaling curve)"},
        "routines": per,
        "pct_of_peak": round(100.0 * value / world / 1e3 / pk, 1),
        "roofline": {"bound": "tensor", "kernel": "tc_structured_gemm (whole step)",
                     "achieved": round(value / world / 1e3, 2), "peak": round(pk, 1), "unit": "TFLOP/s",
                     "frac": round(value / world / 1e3 / pk, 3),
                     "peak_source": f"{peak_src} bf16 sustained x tf32/bf16 {TF32_OVER_BF16:.3f} / 3",
                     "traffic": None},
        "e2e": e2e,
        "gpu_launches": int(launches),
        "comm": comm_info,
        "clocks": clk.summary(t_clk0, t_clk1 + 0.05),
    }
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


# ----------------------------------------------------------------------------- oracle (reference arm)
_INPUT_CACHE = {}


def oracle_sample(n, ncols, seconds_hint=None):
    """Time the fp64 oracle on `ncols` sampled output columns of each routine
    of the step at size n (the same seeded inputs as our arm)."""
    import blas3_inputs as gen
    import oracle
    oracle.build()
    key = (n,)
    if key not in _INPUT_CACHE:                 # generate the 8192^2 inputs once
        _INPUT_CACHE.clear()
        _INPUT_CACHE[key] = make_inputs(n, n, 0)
    A, T, B, C = _INPUT_CACHE[key]
    sel = gen.sample_indices(n, ncols, "bench-sample")
    fl = flops(n, len(sel))
    times = {}
    calls = {
        "sgemm": lambda: oracle.sgemm("N", "N", ALPHA, A, B, BETA, C, sel=sel),
        "ssymm": lambda: oracle.ssymm("L", "L", ALPHA, A, B, BETA, C, sel=sel),
        "ssyrk": lambda: oracle.ssyrk("L", "N", ALPHA, A, BETA, C, sel=sel),
        "ssyr2k": lambda: oracle.ssyr2k("L", "N", ALPHA, A, B, BETA, C, sel=sel),
        "strmm": lambda: oracle.strmm("L", "L", "N", "N", ALPHA, T, B, sel=sel),
        "strsm": lambda: oracle.strsm("L", "L", "N", "N", ALPHA, T, B, sel=sel),
    }
    for r, f in calls.items():
        t0 = time.perf_counter(); f(); times[r] = time.perf_counter() - t0
    # LAWN-41 per-column counts; ssyrk/ssyr2k columns of the lower triangle vary
    # in length, so use the exact sampled-column count for them
    fl["ssyrk"] = float(sum(2.0 * n * (n - j) for j in sel)) / 2.0 * 2.0
    fl["ssyr2k"] = float(sum(4.0 * n * (n - j) for j in sel))
    return fl, times, len(sel)


def cpu_baseline(target_seconds):
    import oracle
    oracle.build()
    n = N
    # calibrate: a small sample first, then scale to ~target_seconds total
    fl, times, ns = oracle_sample(n, max(2, oracle.num_threads()))
    t = sum(times.values())
    ncols = int(min(n, max(ns, ns * target_seconds / max(t, 1e-3))))
    if ncols > ns:
        fl, times, ns = oracle_sample(n, ncols)
    tot = sum(times.values())
    return {"value": round(sum(fl.values()) / tot / 1e9, 3), "unit": "GFLOPS",
            "cores": oracle.num_threads(), "kind": "oracle",
            "sample": f"{ns} sampled output columns of each of the six routines at N={n} "
                      f"(fp64 C oracle, OpenMP over columns), {tot:.1f} s"}


def run_reference(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    oracle.build()
    ncols = max(2, oracle.num_threads())
    # calibrate one step to ~ (budget / (steps + warmup)) seconds
    budget = args.cpu_seconds * 3
    fl, times, ns = oracle_sample(N, ncols)
    per_step = budget / max(1, args.steps + args.warmup)
    ncols = int(min(N, max(ncols, ncols * per_step / max(sum(times.values()), 1e-3))))
    for _ in range(args.warmup):
        oracle_sample(N, ncols)
    tot_t, tot_f = 0.0, 0.0
    for _ in range(args.steps):
        fl, times, ns = oracle_sample(N, ncols)
        tot_t += sum(times.values()); tot_f += sum(fl.values())
    value = tot_f / tot_t / 1e9
    out = {
        "impl": "reference",
        "metric": "GFLOPS per routine (SGEMM/SSYMM/SSYRK/SSYR2K/STRMM/STRSM) at N=8192, "
                  "1/2/4/8 B200, % of peak",
        "value": round(value, 3), "unit": "GFLOPS", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(1e3 * tot_t / args.steps, 1),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (seeded U(-1,1); diagonally dominant T)",
        "config": {"workload": "configs[1..3] at N=8192: sgemm NN, ssymm LL, ssyrk LN, ssyr2k LN "
                               "(K=8192), strmm LLNN, strsm LLNN; alpha=1.5 beta=0.5",
                   "n": N, "k": N, "cols_per_rank": N, "math": "fp64 oracle (plain C)",
                   "l2": "n/a (host CPU)",
                   "parallelism": f"host CPU, {oracle.num_threads()} OpenMP threads over output columns"},
        "cpu_baseline": {"value": round(value, 3), "unit": "GFLOPS", "cores": oracle.num_threads(),
                         "kind": "oracle",
                         "sample": f"{ns} sampled output columns of each routine per step"},
        "e2e": {"value": round(value, 3), "unit": "GFLOPS", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(out), flush=True)


def spawn_command(gpus, argv, port=None):
    """argv for `python -m torch.distributed.run` with one process per GPU on
    127.0.0.1 (used when bench.py --gpus N > 1 is started without torchrun)."""
    if port is None:
        import socket
        s = socket.socket()
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
        s.close()
    script = os.path.abspath(argv[0])
    return [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={gpus}",
            "--master-addr", "127.0.0.1", "--master-port", str(port), script, *argv[1:]]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--math", default="3xtf32", choices=["3xtf32", "simt", "tf32_bf16x"])
    ap.add_argument("--size", type=int, default=None,
                    help="matrix order (default 8192; 32768 for --workload cfg5)")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true", help="skip the e2e leg (profiling runs)")
    ap.add_argument("--no-context", action="store_true", help="skip the cuBLAS context timing")
    ap.add_argument("--no-fp64", action="store_true", help="skip the fp64-family context timing")
    ap.add_argument("--no-alt-mode", action="store_true",
                    help="skip the extra device-only pass in the opt-in TF32+BF16X mode")
    ap.add_argument("--no-routine-clocks", action="store_true",
                    help="skip the per-routine isolated loops (~0.5 s each, clocks sampled every 50 ms)")
    ap.add_argument("--workload", default="chain", choices=["chain", "cfg5"],
                    help="chain: the six-routine N=8192 step (default, weak scaling at N>1); "
                         "cfg5: BASELINE configs[4], N=32768 column slabs (strong scaling)")
    args = ap.parse_args()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        # not under torchrun: re-launch this command with one process per GPU
        os.execv(sys.executable, spawn_command(args.gpus, sys.argv))
    if "WORLD_SIZE" in os.environ and int(os.environ["WORLD_SIZE"]) != args.gpus:
        print(f"warning: --gpus {args.gpus} but WORLD_SIZE={os.environ['WORLD_SIZE']}; "
              f"using WORLD_SIZE", file=sys.stderr)
    if args.warmup < 3:
        print("warning: --warmup < 3 violates the timing rules", file=sys.stderr)
    if args.impl == "reference":
        run_reference(args)
    elif args.workload == "cfg5":
        run_cfg5(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
