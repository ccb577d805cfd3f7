"""Per-stage timeline of CTA 0 for small single launches (BLAS3_TRACE=1):
python tools/trace_small.py   (prints [blas3 trace] lines on stderr)"""
import sys, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
for (m, n, k) in [(128, 128, 128), (256, 256, 256), (1024, 1024, 128), (1024, 8192, 1024)]:
    A = b3.colmajor(m, k); B = b3.colmajor(k, n); C = b3.colmajor(m, n)
    for x in (A, B, C): x.uniform_(-1, 1)
    for beta in (0.0, 1.0):
        for _ in range(3):
            b3.sgemm("N", "N", 1.0, A, B, beta, C)
        torch.cuda.synchronize()
        print(f"-- m={m} n={n} k={k} beta={beta}", file=sys.stderr, flush=True)
