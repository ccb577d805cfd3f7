"""Host-side cost per call (the library is asynchronous: with a tiny GPU
workload the loop is host-bound, so wall time / calls = host cost).
python tools/host_overhead.py"""
import ctypes
import sys
import time

import torch

sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3  # noqa: E402


def mk(m, n):
    t = b3.colmajor(m, n)
    t.uniform_(-1, 1)
    return t


def per_call(fn, n=500):
    for _ in range(20):
        fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(n):
        fn()
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    return (t1 - t0) / n * 1e6, (t2 - t0) / n * 1e6


A, B, C = mk(128, 128), mk(128, 128), mk(128, 128)
st = torch.cuda.current_stream().cuda_stream
lib = b3._lib
print("python wrapper sgemm 128: enqueue %.1f us/call, incl. GPU %.1f us/call" % per_call(
    lambda: b3.sgemm("N", "N", 1.0, A, B, 0.0, C)))
pa, pb, pc = A.data_ptr(), B.data_ptr(), C.data_ptr()
print("raw C ABI sgemm 128:      enqueue %.1f us/call, incl. GPU %.1f us/call" % per_call(
    lambda: lib.blas3_sgemm(b"N", b"N", 128, 128, 128, 1.0, pa, 128, pb, 128, 0.0, pc, 128, st)))
print("torch.cuda.current_stream(): %.2f us" % (per_call(lambda: torch.cuda.current_stream().cuda_stream, 2000)[0]))
S = mk(128, 128)
print("raw C ABI ssymm 128:      enqueue %.1f us/call" % per_call(
    lambda: lib.blas3_ssymm(b"L", b"L", 128, 128, 1.0, S.data_ptr(), 128, pb, 128, 0.0, pc, 128, st))[0])
print("raw C ABI ssyr2k 128:     enqueue %.1f us/call" % per_call(
    lambda: lib.blas3_ssyr2k(b"L", b"N", 128, 128, 1.0, pa, 128, pb, 128, 0.0, pc, 128, st))[0])
for n in (2048, 8192):
    T = mk(n, n); T.mul_(1.0 / n); T.diagonal().fill_(1.0)
    X = mk(n, n)
    torch.cuda.synchronize()
    ts = []
    for _ in range(5):
        t0 = time.perf_counter()
        lib.blas3_strsm(b"L", b"L", b"N", b"N", n, n, 1.0, T.data_ptr(), n, X.data_ptr(), n, st)
        ts.append((time.perf_counter() - t0) * 1e6)
        torch.cuda.synchronize()
    print(f"strsm {n}: host enqueue of the whole call {min(ts):.0f} us (min of 5)")
