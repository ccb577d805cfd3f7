"""Per-tile fixed cost of the tcgen05 kernel: short-K GEMMs with beta=0 / beta!=0."""
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
for (m, n, k) in [(8192, 8192, 32), (8192, 8192, 256), (2048, 8192, 256), (2048, 8192, 2048)]:
    A = b3.colmajor(m, k); B = b3.colmajor(k, n); C = b3.colmajor(m, n)
    for x in (A, B, C): x.uniform_(-1, 1)
    r = []
    for beta in (0.0, 0.5):
        us = t(lambda: b3.sgemm("N", "N", 1.0, A, B, beta, C))
        r.append(f"beta={beta}: {us:8.1f} us ({2*m*n*k/us/1e6:6.1f} TF/s)")
    print(f"m={m} n={n} k={k}: " + "  ".join(r), flush=True)
