"""Per-phase timeline of CTA 0 for a few launch shapes (BLAS3_TRACE=1)."""
import os, sys, torch
os.environ["BLAS3_TRACE"] = "1"
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
for (m, n, k) in [(128, 128, 32), (128, 128, 128), (1024, 1024, 128), (1024, 1024, 1024), (8192, 8192, 256)]:
    A = b3.colmajor(m, k); B = b3.colmajor(k, n); C = b3.colmajor(m, n)
    for x in (A, B, C): x.uniform_(-1, 1)
    for _ in range(3):
        b3.sgemm("N", "N", 1.0, A, B, 0.0, C)
    torch.cuda.synchronize()
    print("----", flush=True)
