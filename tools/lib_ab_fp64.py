"""Same-box A/B of libblas3.so builds on the fp64 routines (raw C ABI, one
ctypes handle per library, interleaved rounds, CUDA events, medians).
python tools/lib_ab_fp64.py LIB_A LIB_B ... [--n 8192] [--rounds 5]"""
import argparse
import ctypes

import numpy as np
import torch

ap = argparse.ArgumentParser()
ap.add_argument("libs", nargs="+")
ap.add_argument("--n", type=int, default=8192)
ap.add_argument("--rounds", type=int, default=5)
args = ap.parse_args()
n = args.n
_i64, _d, _p, _c = ctypes.c_int64, ctypes.c_double, ctypes.c_void_p, ctypes.c_char
libs = []
for path in args.libs:
    L = ctypes.CDLL(path, mode=ctypes.RTLD_LOCAL)
    L.blas3_dgemm.argtypes = [_c, _c, _i64, _i64, _i64, _d, _p, _i64, _p, _i64, _d, _p, _i64, _p]
    L.blas3_dsymm.argtypes = [_c, _c, _i64, _i64, _d, _p, _i64, _p, _i64, _d, _p, _i64, _p]
    L.blas3_dtrmm.argtypes = [_c, _c, _c, _c, _i64, _i64, _d, _p, _i64, _p, _i64, _p]
    libs.append(L)
mk = lambda: torch.empty((n, n), dtype=torch.float64, device="cuda").uniform_(-1, 1)  # noqa: E731
A, B, C, X = mk(), mk(), mk(), mk()
st = torch.cuda.current_stream().cuda_stream
P = lambda t: t.data_ptr()  # noqa: E731
cases = {
    "dgemm_NN": (lambda L: L.blas3_dgemm(b"N", b"N", n, n, n, 1.5, P(A), n, P(B), n, 0.5, P(C), n, st), 2.0 * n ** 3),
    "dgemm_TN": (lambda L: L.blas3_dgemm(b"T", b"N", n, n, n, 1.5, P(A), n, P(B), n, 0.5, P(C), n, st), 2.0 * n ** 3),
    "dsymm_LL": (lambda L: L.blas3_dsymm(b"L", b"L", n, n, 1.5, P(A), n, P(B), n, 0.5, P(C), n, st), 2.0 * n ** 3),
    "dtrmm_LLNN": (lambda L: L.blas3_dtrmm(b"L", b"L", b"N", b"N", n, n, 1.0, P(A), n, P(X), n, st), 1.0 * n ** 3),
}
res = {(c, i): [] for c in cases for i in range(len(libs))}
for rnd in range(args.rounds):
    for i, L in enumerate(libs):
        for c, (fn, fl) in cases.items():
            assert fn(L) == 0
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
            e0.record()
            for _ in range(2):
                fn(L)
            e1.record(); torch.cuda.synchronize()
            res[(c, i)].append(e0.elapsed_time(e1) / 2)
for c, (fn, fl) in cases.items():
    row = [f"{c:12s}"]
    for i, path in enumerate(args.libs):
        ms = float(np.median(res[(c, i)]))
        row.append(f"{path.split('/')[-1]}: {ms:8.3f} ms {fl / ms / 1e9:6.1f} TF/s")
    print("  ".join(row), flush=True)
