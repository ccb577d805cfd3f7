"""Same-box A/B of two builds of libblas3.so through the raw C ABI.

python tools/lib_ab.py LIB_A LIB_B [--rounds 5] [--cases sgemm,ssyrk,...]
Each library is a separate ctypes handle (RTLD_LOCAL, so their symbols do not
mix); every case runs on the same device buffers, rounds interleaved, CUDA
events, medians.  Used to compare a change against the previous round's
library on the same box (box-to-box spread is several %).
"""
import argparse
import ctypes

import numpy as np
import torch

ap = argparse.ArgumentParser()
ap.add_argument("libs", nargs="+")
ap.add_argument("--rounds", type=int, default=5)
ap.add_argument("--cases", default="sgemm,ssymm,ssyrk,ssyr2k,strmm,strsm,ts_syrk,ts_syr2k,sgemm2048")
args = ap.parse_args()

_i64, _f, _p, _c = ctypes.c_int64, ctypes.c_float, ctypes.c_void_p, ctypes.c_char
SIG = {
    "blas3_sgemm": [_c, _c, _i64, _i64, _i64, _f, _p, _i64, _p, _i64, _f, _p, _i64, _p],
    "blas3_ssymm": [_c, _c, _i64, _i64, _f, _p, _i64, _p, _i64, _f, _p, _i64, _p],
    "blas3_ssyrk": [_c, _c, _i64, _i64, _f, _p, _i64, _f, _p, _i64, _p],
    "blas3_ssyr2k": [_c, _c, _i64, _i64, _f, _p, _i64, _p, _i64, _f, _p, _i64, _p],
    "blas3_strmm": [_c, _c, _c, _c, _i64, _i64, _f, _p, _i64, _p, _i64, _p],
    "blas3_strsm": [_c, _c, _c, _c, _i64, _i64, _f, _p, _i64, _p, _i64, _p],
}
libs = []
for path in args.libs:
    h = ctypes.CDLL(path, mode=ctypes.RTLD_LOCAL)
    for k, v in SIG.items():
        getattr(h, k).argtypes = v
        getattr(h, k).restype = ctypes.c_int
    libs.append(h)


def mk(m, n):
    t = torch.empty((n, m), device="cuda").t()
    t.uniform_(-1, 1)
    return t


def P(t):
    return t.data_ptr(), t.stride(1)


n = 8192
A, B, C, X = mk(n, n), mk(n, n), mk(n, n), mk(n, n)
T = mk(n, n)
T.mul_(1.0 / n)
T.diagonal().fill_(1.0)
ts, k = 16384, 512
As, Bs, Cs = mk(ts, k), mk(ts, k), mk(ts, ts)
A2, B2, C2 = mk(2048, 2048), mk(2048, 2048), mk(2048, 2048)
T4, X4, B4 = mk(4096, 4096), mk(4096, 4096), mk(4096, 4096)
T4.mul_(1.0 / 4096)
T4.diagonal().fill_(1.0)
st = torch.cuda.current_stream().cuda_stream


def call(lib, name, *a):
    rc = getattr(lib, name)(*a)
    assert rc == 0, (name, rc)


def cases(lib):
    (pa, la), (pb, lb), (pc, lc), (px, lx), (pt, lt) = P(A), P(B), P(C), P(X), P(T)
    (pas, las), (pbs, lbs), (pcs, lcs) = P(As), P(Bs), P(Cs)
    (pa2, la2), (pb2, lb2), (pc2, lc2) = P(A2), P(B2), P(C2)
    (pt4, lt4), (px4, lx4) = P(T4), P(X4)
    return {
        "sgemm": (lambda: call(lib, "blas3_sgemm", b"N", b"N", n, n, n, 1.5, pa, la, pb, lb, 0.5, pc, lc, st),
                  2.0 * n ** 3, 5, None),
        "ssymm": (lambda: call(lib, "blas3_ssymm", b"L", b"L", n, n, 1.5, pa, la, pb, lb, 0.5, pc, lc, st),
                  2.0 * n ** 3, 5, None),
        "ssyrk": (lambda: call(lib, "blas3_ssyrk", b"L", b"N", n, n, 1.5, pa, la, 0.5, pc, lc, st),
                  1.0 * n * n * (n + 1), 5, None),
        "ssyr2k": (lambda: call(lib, "blas3_ssyr2k", b"L", b"N", n, n, 1.5, pa, la, pb, lb, 0.5, pc, lc, st),
                   2.0 * n ** 3 + n, 5, None),
        "strmm": (lambda: call(lib, "blas3_strmm", b"L", b"L", b"N", b"N", n, n, 1.0, pt, lt, px, lx, st),
                  1.0 * n ** 3, 5, lambda: X.copy_(B)),
        "strsm": (lambda: call(lib, "blas3_strsm", b"L", b"L", b"N", b"N", n, n, 1.0, pt, lt, px, lx, st),
                  1.0 * n ** 3, 5, lambda: X.copy_(B)),
        "strsm4096": (lambda: call(lib, "blas3_strsm", b"L", b"L", b"N", b"N", 4096, 4096, 1.0, pt4, lt4, px4, lx4,
                                   st), 1.0 * 4096 ** 3, 10, lambda: X4.copy_(B4)),
        "ts_syrk": (lambda: call(lib, "blas3_ssyrk", b"L", b"N", ts, k, 1.5, pas, las, 0.5, pcs, lcs, st),
                    1.0 * k * ts * (ts + 1), 10, None),
        "ts_syr2k": (lambda: call(lib, "blas3_ssyr2k", b"L", b"N", ts, k, 1.5, pas, las, pbs, lbs, 0.5, pcs, lcs,
                                  st), 2.0 * k * ts * ts + ts, 10, None),
        "sgemm2048": (lambda: call(lib, "blas3_sgemm", b"N", b"N", 2048, 2048, 2048, 1.5, pa2, la2, pb2, lb2, 0.5,
                                   pc2, lc2, st), 2.0 * 2048 ** 3, 40, None),
    }


sel = args.cases.split(",")
tabs = [cases(lib) for lib in libs]


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


res = {(c, i): [] for c in sel for i in range(len(libs))}
for rnd in range(args.rounds):
    for c in sel:
        for i, tab in enumerate(tabs):
            fn, fl, reps, pre = tab[c]
            if rnd == 0:
                if pre:
                    pre()
                fn(); torch.cuda.synchronize()
            res[(c, i)].append(timed(fn, reps, pre))
names = [p.split("/")[-1] for p in args.libs]
for c in sel:
    fl = tabs[0][c][1]
    row = [f"{c:10s}"]
    for i in range(len(libs)):
        ms = float(np.median(res[(c, i)]))
        row.append(f"{names[i]}: {ms * 1e3:9.1f} us {fl / ms / 1e9:7.1f} TF/s")
    print("  ".join(row), flush=True)
