"""Tall-skinny SYRK/SYR2K (BASELINE configs[3]: N=16384, K=512) and short-K
GEMM/TRSM timings, for epilogue-bound shapes.  python tools/ts_probe.py"""
import sys, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3


def t(fn, reps=5):
    for _ in range(2): fn()
    e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
    torch.cuda.synchronize(); e0.record()
    for _ in range(reps): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


n, k = 16384, 512
A = b3.colmajor(n, k); B = b3.colmajor(n, k); C = b3.colmajor(n, n)
for x in (A, B, C): x.uniform_(-1, 1)
for uplo, tr in (("L", "N"), ("U", "N")):
    ms = t(lambda: b3.ssyrk(uplo, tr, 1.5, A, 0.5, C)); print(f"ssyrk  {uplo}{tr} N=16384 K=512: {ms:.3f} ms {k*n*(n+1)/ms/1e9:.1f} TF/s")
    ms = t(lambda: b3.ssyr2k(uplo, tr, 1.5, A, B, 0.5, C)); print(f"ssyr2k {uplo}{tr} N=16384 K=512: {ms:.3f} ms {(2*k*n*n+n)/ms/1e9:.1f} TF/s")
del A, B, C
for (m, nn, kk) in [(7168, 8192, 1024), (8192, 8192, 512), (8192, 8192, 8192)]:
    A = b3.colmajor(m, kk); B = b3.colmajor(kk, nn); C = b3.colmajor(m, nn)
    for x in (A, B, C): x.uniform_(-1, 1)
    ms = t(lambda: b3.sgemm("N", "N", 1.0, A, B, 0.5, C)); print(f"sgemm m={m} n={nn} k={kk} beta=0.5: {ms:.3f} ms {2*m*nn*kk/ms/1e9:.1f} TF/s")
N = 8192
T = b3.colmajor(N, N); T.uniform_(-1, 1); T.diagonal().add_(N / 2.0); X = b3.colmajor(N, N); X0 = b3.colmajor(N, N); X0.uniform_(-1, 1)
ms = t(lambda: (X.copy_(X0), b3.strsm("L", "L", "N", "N", 1.5, T, X))); print(f"strsm N=8192 (+copy): {ms:.3f} ms {N**3/ms/1e9:.1f} TF/s")
