"""Timing of the non-bench BASELINE configs (context for DESIGN.md): tall-skinny
SYRK/SYR2K (N=16384, K=512), the SGEMM/SSYMM size sweep, TRMM/TRSM at 4096."""
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
ms = t(lambda: b3.ssyrk("L", "N", 1.5, A, 0.5, C)); print(f"ssyrk  N=16384 K=512: {ms:.3f} ms {k*n*(n+1)/ms/1e9:.1f} TF/s")
ms = t(lambda: b3.ssyr2k("L", "N", 1.5, A, B, 0.5, C)); print(f"ssyr2k N=16384 K=512: {ms:.3f} ms {(2*k*n*n+n)/ms/1e9:.1f} TF/s")
del A, B, C
for n in (1024, 2048, 4096, 8192):
    A = b3.colmajor(n, n); B = b3.colmajor(n, n); C = b3.colmajor(n, n)
    for x in (A, B, C): x.uniform_(-1, 1)
    g = t(lambda: b3.sgemm("N", "N", 1.5, A, B, 0.5, C)); s_ = t(lambda: b3.ssymm("L", "L", 1.5, A, B, 0.5, C))
    print(f"N={n:5d} sgemm {2*n**3/g/1e9:6.1f} TF/s  ssymm {2*n**3/s_/1e9:6.1f} TF/s")
n = 4096
T = b3.colmajor(n, n); T.uniform_(-1, 1); T.diagonal().add_(n / 2.0); X = b3.colmajor(n, n); X.uniform_(-1, 1)
print(f"N=4096 strmm {n**3/t(lambda: b3.strmm('L','L','N','N',1.0,T,X))/1e9:6.1f} TF/s  strsm {n**3/t(lambda: b3.strsm('L','L','N','N',1.0,T,X))/1e9:6.1f} TF/s")
