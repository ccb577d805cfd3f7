import sys, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
n = 8192
A = b3.colmajor(n, n); A.uniform_(-1, 1); B = b3.colmajor(n, n); B.uniform_(-1, 1); C = b3.colmajor(n, n)
def t(fn, reps=5):
    fn(); torch.cuda.synchronize()
    e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True); e0.record()
    for _ in range(reps): fn()
    e1.record(); torch.cuda.synchronize(); return e0.elapsed_time(e1) / reps
with b3.options(gm_map=1):
    print("ssymm gm", t(lambda: b3.ssymm("L", "L", 1.5, A, B, 0.5, C)))
with b3.options(gm_map=0):
    print("ssymm staged", t(lambda: b3.ssymm("L", "L", 1.5, A, B, 0.5, C)))
print("sgemm", t(lambda: b3.sgemm("N", "N", 1.5, A, B, 0.5, C)))
