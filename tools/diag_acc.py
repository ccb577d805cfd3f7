"""Accuracy vs K: tcgen05 3xTF32 vs SIMT FP32 vs cuBLAS (fp32 / 1xTF32), e_rel to fp64."""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
import blas3_inputs as gen
m = n = 512
for k in [256, 1024, 4096, 16384]:
    A = gen.uniform(m, k, "acc-a", k); B = gen.uniform(k, n, "acc-b", k)
    ref = A.astype(np.float64) @ B.astype(np.float64)
    row = [f"k={k:6d}"]
    for mode in ["3xtf32", "simt"]:
        b3.set_math_mode(mode)
        dC = b3.colmajor(m, n, fill=0.0)
        b3.sgemm("N", "N", 1.0, b3.from_fortran(A), b3.from_fortran(B), 0.0, dC)
        got = dC.cpu().numpy().astype(np.float64)
        row.append(f"{mode}={np.linalg.norm(got-ref)/np.linalg.norm(ref):.2e}")
    tA, tB = torch.from_numpy(np.ascontiguousarray(A)).cuda(), torch.from_numpy(np.ascontiguousarray(B)).cuda()
    for tf in [False, True]:
        torch.backends.cuda.matmul.allow_tf32 = tf
        got = (tA @ tB).cpu().numpy().astype(np.float64)
        row.append(f"cublas_{'tf32' if tf else 'fp32'}={np.linalg.norm(got-ref)/np.linalg.norm(ref):.2e}")
    print("  ".join(row), flush=True)
