"""Sustained interleaved A/B: each case back to back for ~--ms milliseconds
with nvidia-smi clocks/power sampled every 50 ms, rounds interleaved so the
box's power/thermal state hits every case alike (the bench's isolated loops
run the same way).

python tools/sustained_ab.py [--rounds 3] [--ms 600] case ...
case: sgemm | strsm[:opt=v[,opt=v]]   (N = 8192, LLNN, X restored every call)
"""
import argparse
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_cuiwxyf11_b200 as b3  # noqa: E402
from bench import ClockSampler  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("cases", nargs="+")
ap.add_argument("--rounds", type=int, default=3)
ap.add_argument("--ms", type=float, default=600.0)
ap.add_argument("--n", type=int, default=8192)
args = ap.parse_args()
n = args.n


def mk(m, c):
    t = b3.colmajor(m, c)
    t.uniform_(-1, 1)
    return t


A, Bm, C, X, B0 = mk(n, n), mk(n, n), mk(n, n), mk(n, n), mk(n, n)
T = mk(n, n)
T.mul_(1.0 / n)
T.diagonal().fill_(1.0)


def parse(case):
    name, _, rest = case.partition(":")
    opts = {}
    for kv in filter(None, rest.split(",")):
        k, v = kv.split("=")
        opts[k] = int(v)
    if name == "sgemm":
        return (lambda: b3.sgemm("N", "N", 1.5, A, Bm, 0.5, C)), 2.0 * n ** 3, opts
    if name == "strsm":
        return (lambda: (X.copy_(B0), b3.strsm("L", "L", "N", "N", 1.5, T, X))), 1.0 * n ** 3, opts
    if name == "strmm":
        return (lambda: (X.copy_(B0), b3.strmm("L", "L", "N", "N", 1.5, T, X))), 1.0 * n ** 3, opts
    raise SystemExit(f"unknown case {case}")


cases = [(c, *parse(c)) for c in args.cases]
res = {c: [] for c, *_ in cases}
stream = torch.cuda.current_stream()
with ClockSampler(torch.cuda.current_device(), interval_ms=50) as clk:
    for rnd in range(args.rounds):
        for c, fn, fl, opts in cases:
            with b3.options(**opts):
                fn()
                torch.cuda.synchronize()
                e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
                e0.record(stream); fn(); e1.record(stream); torch.cuda.synchronize()
                reps = max(3, int(args.ms / max(0.05, e0.elapsed_time(e1))))
                t0 = time.time()
                e0.record(stream)
                for _ in range(reps):
                    fn()
                e1.record(stream)
                torch.cuda.synchronize()
                t1 = time.time()
                ms = e0.elapsed_time(e1) / reps
                res[c].append((ms, clk.summary(t0, t1)))
for c, fn, fl, opts in cases:
    ms = float(np.median([r[0] for r in res[c]]))
    mhz = [r[1].get("sm_mhz") for r in res[c]]
    pw = [r[1].get("power_w") for r in res[c]]
    print(f"{c:40s} {ms * 1e3:9.1f} us {fl / ms / 1e9:7.1f} TF/s  sm_mhz {mhz}  power_w {pw}", flush=True)
