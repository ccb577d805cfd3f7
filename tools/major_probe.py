"""NN vs NT SGEMM (B K-major vs MN-major) under the kernel debug knobs."""
import sys, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
n = 8192
A = b3.colmajor(n, n); B = b3.colmajor(n, n); C = b3.colmajor(n, n)
for t in (A, B, C): t.uniform_(-1, 1)
out = []
for ta, tb in [("N", "N"), ("N", "T")]:
    for _ in range(2): b3.sgemm(ta, tb, 1.0, A, B, 0.5, C)
    e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
    torch.cuda.synchronize(); e0.record()
    for _ in range(5): b3.sgemm(ta, tb, 1.0, A, B, 0.5, C)
    e1.record(); torch.cuda.synchronize()
    out.append(f"{ta}{tb} {e0.elapsed_time(e1) / 5:.3f} ms")
print(" | ".join(out), flush=True)
