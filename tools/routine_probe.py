"""Per-routine time at N (default 8192): python tools/routine_probe.py [n] [routines...]"""
import sys, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
which = sys.argv[2:] or ["sgemm", "ssymm", "strmm", "strsm", "ssyrk"]
A = b3.colmajor(n, n); B = b3.colmajor(n, n); C = b3.colmajor(n, n)
for t in (A, B, C): t.uniform_(-1, 1)
T = b3.colmajor(n, n); T.uniform_(-1, 1); T.diagonal().add_(n / 2.0)
calls = {"sgemm": (lambda: b3.sgemm("N", "N", 1.5, A, B, 0.5, C), 2 * n**3),
         "ssymm": (lambda: b3.ssymm("L", "L", 1.5, A, B, 0.5, C), 2 * n**3),
         "ssyrk": (lambda: b3.ssyrk("L", "N", 1.5, A, 0.5, C), n**3),
         "strmm": (lambda: b3.strmm("L", "L", "N", "N", 1.5, T, B), n**3),
         "strsm": (lambda: b3.strsm("L", "L", "N", "N", 1.5, T, B), n**3)}
out = []
for r in which:
    fn, fl = calls[r]
    fn(); torch.cuda.synchronize()
    e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
    e0.record()
    for _ in range(3): fn()
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 3
    out.append(f"{r} {ms:.3f} ms {fl / ms / 1e9:.1f}")
print(" | ".join(out), flush=True)
