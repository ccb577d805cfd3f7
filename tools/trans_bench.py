"""SGEMM rate per transpose combination (operand majorness) at 8192^3."""
import sys, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
n = 8192
A = b3.colmajor(n, n); B = b3.colmajor(n, n); C = b3.colmajor(n, n)
for t in (A, B, C): t.uniform_(-1, 1)
for ta, tb in [("N", "N"), ("T", "N"), ("N", "T"), ("T", "T")]:
    for _ in range(2): b3.sgemm(ta, tb, 1.0, A, B, 0.5, C)
    e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
    torch.cuda.synchronize(); e0.record()
    for _ in range(5): b3.sgemm(ta, tb, 1.0, A, B, 0.5, C)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 5
    print(f"{ta}{tb} (A {'K' if ta=='T' else 'MN'}-major, B {'K' if tb=='N' else 'MN'}-major): {ms:.3f} ms {2*n**3/ms/1e9:.1f} TF/s", flush=True)
