"""SSYRK / SSYR2K lower vs upper, interleaved medians (thermal drift cancels):
python tools/uplo_probe.py"""
import statistics, sys, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
n = k = 8192
A = b3.colmajor(n, k); B = b3.colmajor(n, k); C = b3.colmajor(n, n)
for x in (A, B, C): x.uniform_(-1, 1)
def t(fn, reps=3):
    fn(); e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
    torch.cuda.synchronize(); e0.record()
    for _ in range(reps): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps
cases = {f"{r} {u}{tr}": (lambda r=r, u=u, tr=tr: b3.ssyrk(u, tr, 1.5, A, 0.5, C) if r == "ssyrk"
                          else b3.ssyr2k(u, tr, 1.5, A, B, 0.5, C))
         for r in ("ssyrk", "ssyr2k") for u in "LU" for tr in "NT"}
cases["sgemm NN"] = lambda: b3.sgemm("N", "N", 1.5, A, B, 0.5, C)
res = {k_: [] for k_ in cases}
for _ in range(4):
    for name, fn in cases.items():
        res[name].append(t(fn))
for name, v in res.items():
    ms = statistics.median(v)
    fl = 2 * n ** 3 if name.startswith("sgemm") else (n * n * (n + 1) if name.startswith("ssyrk") else 2 * k * n * n + n)
    print(f"{name:12s} {ms:.3f} ms {fl / ms / 1e9:7.1f} TF/s", flush=True)
