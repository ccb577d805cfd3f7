"""FP32 SIMT kernel throughput (row A10): python tools/simt_probe.py"""
import sys, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
b3.set_math_mode("simt")
for n in (4096, 8192):
    A = b3.colmajor(n, n); B = b3.colmajor(n, n); C = b3.colmajor(n, n)
    for t in (A, B, C): t.uniform_(-1, 1)
    b3.sgemm("N", "N", 1.5, A, B, 0.5, C); torch.cuda.synchronize()
    e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True); e0.record()
    for _ in range(3): b3.sgemm("N", "N", 1.5, A, B, 0.5, C)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 3
    print(f"simt sgemm N={n}: {ms:.3f} ms {2 * n**3 / ms / 1e9:.1f} TF/s", flush=True)
    for r, fn, fl in [("ssymm", lambda: b3.ssymm("L", "L", 1.5, A, B, 0.5, C), 2 * n**3),
                      ("strmm", lambda: b3.strmm("L", "L", "N", "N", 1.0, A, B), n**3)]:
        fn(); torch.cuda.synchronize(); e0.record()
        for _ in range(3): fn()
        e1.record(); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 3
        print(f"simt {r} N={n}: {ms:.3f} ms {fl / ms / 1e9:.1f} TF/s", flush=True)
