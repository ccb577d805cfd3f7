"""Interleaved A/B timing of one library option over the bench-shaped calls.

python tools/opt_ab.py <option> <v1> <v2> ... [--math 3xtf32] [--rounds 5]
Prints the median time and TF/s of each call under each option value
(CUDA events, rounds interleaved so clock drift hits every value alike).
"""
import argparse
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("option")
ap.add_argument("values", nargs="+", type=int)
ap.add_argument("--math", default="3xtf32")
ap.add_argument("--rounds", type=int, default=5)
ap.add_argument("--cases", default="sgemm,ssymm,ssyrk,ssyr2k,strmm,strsm,ts_syrk,ts_syr2k,sgemm2048,sgemm1024")
args = ap.parse_args()
b3.set_math_mode(args.math)


def mk(m, n):
    t = b3.colmajor(m, n)
    t.uniform_(-1, 1)
    return t


n = 8192
A, B, C, X = mk(n, n), mk(n, n), mk(n, n), mk(n, n)
T = mk(n, n)
T.mul_(1.0 / n)
T.diagonal().fill_(1.0)
ts, k = 16384, 512
As, Bs, Cs = mk(ts, k), mk(ts, k), mk(ts, ts)
A2, B2, C2 = mk(2048, 2048), mk(2048, 2048), mk(2048, 2048)
A1, B1, C1 = mk(1024, 1024), mk(1024, 1024), mk(1024, 1024)
T4, X4, B4 = mk(4096, 4096), mk(4096, 4096), mk(4096, 4096)
T4.mul_(1.0 / 4096)
T4.diagonal().fill_(1.0)
T2, X2, Bx2 = mk(2048, 2048), mk(2048, 2048), mk(2048, 2048)
T2.mul_(1.0 / 2048)
T2.diagonal().fill_(1.0)
X84, B84 = mk(8192, 4096), mk(8192, 4096)
cases = {
    "sgemm": (lambda: b3.sgemm("N", "N", 1.5, A, B, 0.5, C), 2.0 * n ** 3, 5, None),
    "ssymm": (lambda: b3.ssymm("L", "L", 1.5, A, B, 0.5, C), 2.0 * n ** 3, 5, None),
    "ssyrk": (lambda: b3.ssyrk("L", "N", 1.5, A, 0.5, C), 1.0 * n * n * (n + 1), 5, None),
    "ssyr2k": (lambda: b3.ssyr2k("L", "N", 1.5, A, B, 0.5, C), 2.0 * n ** 3 + n, 5, None),
    "strmm": (lambda: b3.strmm("L", "L", "N", "N", 1.0, T, X), 1.0 * n ** 3, 5, lambda: X.copy_(B)),
    "strsm": (lambda: b3.strsm("L", "L", "N", "N", 1.0, T, X), 1.0 * n ** 3, 5, lambda: X.copy_(B)),
    "ts_syrk": (lambda: b3.ssyrk("L", "N", 1.5, As, 0.5, Cs), 1.0 * k * ts * (ts + 1), 10, None),
    "ts_syr2k": (lambda: b3.ssyr2k("L", "N", 1.5, As, Bs, 0.5, Cs), 2.0 * k * ts * ts + ts, 10, None),
    "sgemm2048": (lambda: b3.sgemm("N", "N", 1.5, A2, B2, 0.5, C2), 2.0 * 2048 ** 3, 40, None),
    "sgemm1024": (lambda: b3.sgemm("N", "N", 1.5, A1, B1, 0.5, C1), 2.0 * 1024 ** 3, 100, None),
    "strsm4096": (lambda: b3.strsm("L", "L", "N", "N", 1.0, T4, X4), 1.0 * 4096 ** 3, 10, lambda: X4.copy_(B4)),
    "strsm2048": (lambda: b3.strsm("L", "L", "N", "N", 1.0, T2, X2), 1.0 * 2048 ** 3, 20, lambda: X2.copy_(Bx2)),
    "strsm8k4k": (lambda: b3.strsm("L", "L", "N", "N", 1.0, T, X84), 1.0 * 8192 ** 2 * 4096, 5,
                  lambda: X84.copy_(B84)),
}
sel = [c for c in args.cases.split(",") if c in cases]


def timed(fn, reps, pre):
    """reps calls back to back between two events (pre() once before: the
    in-place routines' operand drifts slowly, ||T|| ~ 1)."""
    if pre:
        pre()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


res = {(c, v): [] for c in sel for v in args.values}
for rnd in range(args.rounds):
    for v in args.values:
        with b3.options(**{args.option: v}):
            for c in sel:
                fn, fl, reps, pre = cases[c]
                if rnd == 0:
                    if pre:
                        pre()
                    fn()
                res[(c, v)].append(timed(fn, reps, pre))
for c in sel:
    fl = cases[c][1]
    row = [f"{c:10s}"]
    for v in args.values:
        ms = float(np.median(res[(c, v)]))
        row.append(f"{args.option}={v}: {ms * 1e3:9.1f} us {fl / ms / 1e9:7.1f} TF/s")
    print("  ".join(row), flush=True)
