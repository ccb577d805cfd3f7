"""fp64 family timing (blas3_d*): each routine back to back between two CUDA
events after a warm-up, N = --n (default 8192), LAWN-41 flop counts, against
the FP64 FMA peak of the device (148 SMs x 64 DFMA/clk x 2 x max clock).

python tools/fp64_bench.py [--n 8192] [--reps 3]
"""
import argparse
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_cuiwxyf11_b200 as b3  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=8192)
ap.add_argument("--reps", type=int, default=3)
args = ap.parse_args()
n = args.n
f64 = torch.float64


def mk():
    t = b3.colmajor(n, n, dtype=f64)
    t.uniform_(-1, 1)
    return t


A, B, C, X = mk(), mk(), mk(), mk()
T = mk()
T.mul_(1.0 / n)
T.diagonal().fill_(1.0)
cases = {
    "dgemm": (lambda: b3.dgemm("N", "N", 1.5, A, B, 0.5, C), 2.0 * n ** 3),
    "dsymm": (lambda: b3.dsymm("L", "L", 1.5, A, B, 0.5, C), 2.0 * n ** 3),
    "dsyrk": (lambda: b3.dsyrk("L", "N", 1.5, A, 0.5, C), 1.0 * n * n * (n + 1)),
    "dsyr2k": (lambda: b3.dsyr2k("L", "N", 1.5, A, B, 0.5, C), 2.0 * n ** 3 + n),
    "dtrmm": (lambda: b3.dtrmm("L", "L", "N", "N", 1.0, T, X), 1.0 * n ** 3),
    "dtrsm": (lambda: b3.dtrsm("L", "L", "N", "N", 1.0, T, X), 1.0 * n ** 3),
}
props = torch.cuda.get_device_properties(0)
peak = props.multi_processor_count * 64 * 2 * 1.965e9 / 1e12
out = {"n": n, "fp64_fma_peak_tflops_at_1965mhz": round(peak, 1)}
for name, (fn, fl) in cases.items():
    X.copy_(B)
    fn()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(args.reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / args.reps
    out[name] = {"ms": round(ms, 3), "tflops": round(fl / ms / 1e9, 2), "frac": round(fl / ms / 1e9 / peak, 3)}
    print(name, out[name], flush=True)
print(json.dumps(out))
