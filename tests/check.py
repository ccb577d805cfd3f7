"""Shared helpers for the GPU parity tests: run a routine through the public
binding (-> C ABI -> CUDA kernels) on numpy inputs and compute the error
metrics of DESIGN.md §Parity (north-star tolerances)."""
import numpy as np

F64 = np.float64


def f64(x):
    return np.asarray(x, dtype=F64)


def to_dev(buf):
    import paper_conf_ipps_cuiwxyf11_b200 as b3
    return b3.from_fortran(buf)


def to_host(t):
    return np.asfortranarray(t.cpu().numpy())


def bits_equal(a, b):
    a = np.ascontiguousarray(np.asarray(a, dtype=np.float32))
    b = np.ascontiguousarray(np.asarray(b, dtype=np.float32))
    return a.shape == b.shape and np.array_equal(a.view(np.uint32), b.view(np.uint32))


def op(X, t):
    return X.T if t.upper() != "N" else X


def sym_full(A, uplo, n):
    A = np.nan_to_num(f64(A[:n, :n]))
    if uplo.upper() == "L":
        L = np.tril(A)
        return L + np.tril(L, -1).T
    U = np.triu(A)
    return U + np.triu(U, 1).T


def tri_full(A, uplo, diag, n):
    A = np.nan_to_num(f64(A[:n, :n]))
    T = np.tril(A) if uplo.upper() == "L" else np.triu(A)
    if diag.upper() == "U":
        np.fill_diagonal(T, 1.0)
    return T


def fro(x):
    return float(np.linalg.norm(f64(x)))


def e_nw(got, ref, scale):
    """normwise ||C - C_ref||_F / scale (scale = |a| ||opA|| ||opB|| + |b| ||C||)."""
    return fro(f64(got) - f64(ref)) / max(scale, 1e-300)


def e_rel(got, ref):
    return fro(f64(got) - f64(ref)) / max(fro(ref), 1e-300)


# binding tolerance (north star)
TOL_NW = 1e-5

# Output-relative diagnostic: the GPU result
# must be as accurate as a plain fp32 evaluation of the same expression on the
# same inputs, up to a factor 4, with a floor of 2e-6:
#     e_rel(got) <= max(4 * e_rel(plain fp32), 2e-6).
# The comparator is numpy's float32 matmul on the materialised effective
# operands (fp32 products, fp32 sums) -- it shares nothing with the kernels
# and does not depend on their design (no chunk sizes, no split model).  For
# U(-1,1) data it sits near 3e-7, so the bound is 2e-6 in practice, an order
# of magnitude below a 1xTF32 result (~2.6e-4) and below a 3xTF32 kernel that
# lets its truncating TMEM accumulator run over long K (3.9e-6 at KC = 16).
REL_FLOOR = 2e-6


def f32_eval(alpha, X, Y, beta=0.0, C=None):
    """alpha * X @ Y (+ beta * C) computed in float32 throughout."""
    X32 = np.asarray(X, dtype=np.float32)
    Y32 = np.asarray(Y, dtype=np.float32)
    P = np.float32(alpha) * (X32 @ Y32)
    if C is not None and beta != 0.0:
        P = P + np.float32(beta) * np.asarray(C, dtype=np.float32)
    return P


def rel_bound(fp32_result, ref):
    """max(4 * e_rel(plain fp32 result), REL_FLOOR) against the fp64 ref."""
    return max(4.0 * e_rel(fp32_result, ref), REL_FLOOR)


def syr2k_f32(alpha, opA, opB, beta, C):
    """alpha*(opA opB^T + opB opA^T) + beta*C in float32 (full square)."""
    a32, b32 = np.asarray(opA, np.float32), np.asarray(opB, np.float32)
    P = np.float32(alpha) * (a32 @ b32.T + b32 @ a32.T)
    if beta != 0.0:
        P = P + np.float32(beta) * np.nan_to_num(np.asarray(C, np.float32))
    return P


# ---- plain fp32 evaluations on sampled output columns (large-size parity) ----
def sym_f32(A, uplo):
    """sym(A) from its uplo triangle, float32 (the other triangle never read)."""
    A = np.nan_to_num(np.asarray(A, np.float32))
    if uplo.upper() == "L":
        L = np.tril(A)
        return L + np.tril(L, -1).T
    U = np.triu(A)
    return U + np.triu(U, 1).T


def tri_f32(A, uplo, diag):
    A = np.nan_to_num(np.asarray(A, np.float32))
    T = np.tril(A) if uplo.upper() == "L" else np.triu(A)
    if diag.upper() == "U":
        np.fill_diagonal(T, 1.0)
    return T


def sel_f32(routine, args, sel):
    """Plain fp32 result of `routine` on the output columns `sel` (rows for
    nothing: every sampled routine here samples columns), same argument order
    as the oracle / binding."""
    f = np.float32
    if routine == "sgemm":
        ta, tb, al, A, B, be, C = args
        oA = op(np.asarray(A, f), ta)
        oB = op(np.asarray(B, f), tb)[:, sel]
        return f32_eval(al, oA, oB, be, np.asarray(C, f)[:, sel])
    if routine == "ssymm":
        side, uplo, al, A, B, be, C, S = args          # S = sym_f32(A, uplo), precomputed
        B = np.asarray(B, f)
        if side.upper() == "L":
            return f32_eval(al, S, B[:, sel], be, np.asarray(C, f)[:, sel])
        return f32_eval(al, B, S[:, sel], be, np.asarray(C, f)[:, sel])
    if routine in ("ssyrk", "ssyr2k"):
        uplo, trans, al, A, B, be, C = args
        oA = op(np.asarray(A, f), trans)              # n x k
        oB = oA if B is None else op(np.asarray(B, f), trans)
        P = oA @ oB[sel, :].T
        if routine == "ssyr2k":
            P = P + oB @ oA[sel, :].T
        P = f(al) * P
        if be != 0.0:
            P = P + f(be) * np.nan_to_num(np.asarray(C, f)[:, sel])
        return P
    if routine == "strmm":
        side, ta, al, T, B = args                      # T = tri_f32(A, uplo, diag)
        oT = op(T, ta)
        B = np.asarray(B, f)
        return f32_eval(al, oT, B[:, sel]) if side.upper() == "L" else f32_eval(al, B, oT[:, sel])
    raise ValueError(routine)
