import sys, numpy as np, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
for mode in ("3xtf32", "tf32_bf16x"):
    b3.set_math_mode(mode)
    for (m, n, k, ta, tb) in [(300, 260, 270, "N", "N"), (1024, 1024, 4096, "T", "N"), (2048, 512, 8192, "N", "T")]:
        A = b3.colmajor(m if ta == "N" else k, k if ta == "N" else m); A.uniform_(-1, 1)
        B = b3.colmajor(k if tb == "N" else n, n if tb == "N" else k); B.uniform_(-1, 1)
        C = b3.colmajor(m, n); C.uniform_(-1, 1)
        ref = 1.5 * (A.double().T if ta == "T" else A.double()) @ (B.double().T if tb == "T" else B.double()) + 0.5 * C.double()
        b3.sgemm(ta, tb, 1.5, A, B, 0.5, C); torch.cuda.synchronize()
        rel = ((C.double() - ref).norm() / ref.norm()).item()
        print(f"{mode:11s} {ta}{tb} m={m} n={n} k={k}: rel err {rel:.2e}", flush=True)
