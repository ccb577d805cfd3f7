"""Per-shape GEMM timing (CUDA events, no profiler): python tools/shape_bench.py"""
import sys, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
shapes = [(8192, 8192, 8192), (7168, 8192, 1024), (1024, 8192, 1024), (768, 8192, 128),
          (128, 8192, 128), (8192, 8192, 32), (4096, 4096, 4096)]
for mode in sys.argv[1:] or ["3xtf32"]:
    b3.set_math_mode(mode)
    for (m, n, k) in shapes:
        A = b3.colmajor(m, k); B = b3.colmajor(k, n); C = b3.colmajor(m, n)
        for t in (A, B, C): t.uniform_(-1, 1)
        for _ in range(3): b3.sgemm("N", "N", 1.0, A, B, 0.5, C)
        reps = max(3, int(2e11 / (2 * m * n * k)))
        e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
        torch.cuda.synchronize(); e0.record()
        for _ in range(reps): b3.sgemm("N", "N", 1.0, A, B, 0.5, C)
        e1.record(); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / reps
        print(f"{mode:7s} m={m:5d} n={n:5d} k={k:5d}  {ms*1e3:9.1f} us  {2*m*n*k/ms/1e9:8.1f} TF/s", flush=True)
