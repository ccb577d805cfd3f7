"""Store-path probe: short-K SGEMM (C write dominated) vs ldc padding and vs a
plain device copy of the same bytes."""
import sys, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
def t(fn, reps=10):
    for _ in range(3): fn()
    e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
    torch.cuda.synchronize(); e0.record()
    for _ in range(reps): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3
m = n = 8192; k = int(sys.argv[1]) if len(sys.argv) > 1 else 32
A = b3.colmajor(m, k); B = b3.colmajor(k, n)
for x in (A, B): x.uniform_(-1, 1)
for pad in (0, 32, 64, 1024):
    Cs = torch.empty(n, m + pad, device="cuda"); C = Cs[:, :m].t()
    us = t(lambda: b3.sgemm("N", "N", 1.0, A, B, 0.0, C))
    print(f"k={k} ldc={m+pad}: {us:8.1f} us  write {m*n*4/us/1e3:7.1f} GB/s", flush=True)
X = torch.empty(m * n, device="cuda"); Y = torch.empty_like(X)
us = t(lambda: Y.copy_(X)); print(f"copy 256MiB: {us:.1f} us {2*m*n*4/us/1e3:.1f} GB/s")
us = t(lambda: Y.fill_(1.0)); print(f"fill 256MiB: {us:.1f} us {m*n*4/us/1e3:.1f} GB/s")
