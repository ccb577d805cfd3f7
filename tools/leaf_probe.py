"""STRSM leaf-shaped problems in isolation: STRMM L L N N with a 2048-order
triangle and 8192 right-hand sides (the shape of a sweep leaf, 256 pair
tiles with triangular K) against a dense GEMM of the same flop count
(2048 x 8192 x 1024), under tile-schedule options.  CUDA events, calls
back to back, interleaved rounds.

python tools/leaf_probe.py [--rounds 5]
"""
import argparse
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--rounds", type=int, default=5)
args = ap.parse_args()


def mk(m, n):
    t = b3.colmajor(m, n)
    t.uniform_(-1, 1)
    return t


R, N = 2048, 8192
T = mk(R, R); T.mul_(1.0 / R); T.diagonal().fill_(1.0)
X = mk(R, N); B0 = mk(R, N)
A = mk(R, 1024); Bd = mk(1024, N); C = mk(R, N)
cases = {
    "trmm_leaf": (lambda: b3.strmm("L", "L", "N", "N", 1.0, T, X), 1.0 * R * R * N),
    "gemm_same_flops": (lambda: b3.sgemm("N", "N", 1.0, A, Bd, 0.0, C), 2.0 * R * N * 1024),
    "gemm_2048x8192x2048": (lambda: b3.sgemm("N", "N", 1.0, T, X, 0.0, C), 2.0 * R * N * R),
}
opts = [{}, {"tc_split": 0}, {"tc_static": 1}, {"tc_raster": 4}]
res = {}
for rnd in range(args.rounds):
    for oi, o in enumerate(opts):
        with b3.options(**o):
            for name, (fn, fl) in cases.items():
                fn(); torch.cuda.synchronize()
                e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
                e0.record()
                for _ in range(10):
                    fn()
                e1.record(); torch.cuda.synchronize()
                res.setdefault((name, oi), []).append(e0.elapsed_time(e1) / 10)
for name, (fn, fl) in cases.items():
    row = [f"{name:22s}"]
    for oi, o in enumerate(opts):
        ms = float(np.median(res[(name, oi)]))
        row.append(f"{o or 'default'}: {ms * 1e3:7.1f} us {fl / ms / 1e9:6.1f} TF/s")
    print("  ".join(row), flush=True)
