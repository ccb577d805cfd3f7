"""Diagnostic: error pattern of the tcgen05 GEMM vs fp64 numpy on small shapes."""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
import blas3_inputs as gen

def run(m, n, k, ta="N", tb="N", integer=True):
    mk = (m, k) if ta == "N" else (k, m)
    kn = (k, n) if tb == "N" else (n, k)
    f = gen.integers if integer else gen.uniform
    A = f(*mk, "da"); B = f(*kn, "db"); C = np.zeros((m, n), np.float32, order="F")
    dC = b3.from_fortran(C)
    b3.sgemm(ta, tb, 1.0, b3.from_fortran(A), b3.from_fortran(B), 0.0, dC)
    torch.cuda.synchronize()
    got = dC.cpu().numpy().astype(np.float64)
    oA = A.astype(np.float64) if ta == "N" else A.astype(np.float64).T
    oB = B.astype(np.float64) if tb == "N" else B.astype(np.float64).T
    ref = oA @ oB
    bad = np.abs(got - ref) > 1e-3 * (1 + np.abs(ref))
    msg = f"m={m} n={n} k={k} {ta}{tb}: bad={bad.sum()}/{bad.size}"
    if bad.any():
        r, c = np.nonzero(bad)
        msg += f" rows[{r.min()},{r.max()}] cols[{c.min()},{c.max()}]"
        # try to explain: which k-blocks are missing/duplicated? solve for per-kblock weights
        nkb = (k + 31) // 32
        parts = []
        for kb in range(nkb):
            sl = slice(kb * 32, min(k, kb * 32 + 32))
            parts.append((oA[:, sl] @ oB[sl, :]).ravel())
        X = np.stack(parts, 1)
        w, *_ = np.linalg.lstsq(X, got.ravel(), rcond=None)
        msg += " kblock-weights=" + np.array2string(np.round(w, 3), max_line_width=300)
    print(msg, flush=True)

for (m, n, k) in [(128, 256, 32), (128, 256, 64), (128, 256, 128), (128, 256, 160), (128, 256, 192),
                  (128, 256, 256), (256, 256, 256), (128, 512, 64), (300, 131, 520)]:
    for ta, tb in [("N", "N"), ("T", "N"), ("N", "T"), ("T", "T")]:
        run(m, n, k, ta, tb)
