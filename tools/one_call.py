"""One call of one routine at N (for ncu captures): python tools/one_call.py sgemm 8192"""
import sys, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
r, n = sys.argv[1], int(sys.argv[2])
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 1
A = b3.colmajor(n, n); B = b3.colmajor(n, n); C = b3.colmajor(n, n)
for t in (A, B, C):
    t.uniform_(-1, 1)
T = b3.colmajor(n, n); T.uniform_(-1, 1); T.diagonal().add_(n / 2.0)
for _ in range(reps):
    if r == "sgemm": b3.sgemm("N", "N", 1.5, A, B, 0.5, C)
    elif r == "ssymm": b3.ssymm("L", "L", 1.5, A, B, 0.5, C)
    elif r == "ssyrk": b3.ssyrk("L", "N", 1.5, A, 0.5, C)
    elif r == "ssyr2k": b3.ssyr2k("L", "N", 1.5, A, B, 0.5, C)
    elif r == "strmm": b3.strmm("L", "L", "N", "N", 1.5, T, B)
    elif r == "strsm": b3.strsm("L", "L", "N", "N", 1.5, T, B)
torch.cuda.synchronize()
print("done", r, n)
