"""Parity at BASELINE.json configs[4]'s order, N = 32768, on one GPU: SGEMM NN,
SSYMM LL and STRSM LLNN (the routines of the column-slab scaling run), the
seeded inputs of blas3_inputs, alpha = 1.5, beta = 0.5.  Each matrix is 4 GiB;
the fp64 oracle computes a sample of output columns exactly (columns are
independent) and the north-star metrics are restricted to that sample.  Norms
of the 4 GiB operands are accumulated in fp64 over row chunks (no 8 GiB
temporaries).  The STRSM residual ||T X_s - alpha B_s|| / (||T|| ||X_s||) is
the binding criterion (<= 1e-5 sqrt(N)), plus the forward error vs the oracle.
"""
import numpy as np
import pytest

import blas3_inputs as gen
from check import TOL_NW, f64, to_dev, to_host

pytestmark = pytest.mark.gpu

N = 32768
AL, BE = 1.5, 0.5
CH = 2048                                  # row chunk for fp64 reductions


def fro_big(X, rows=None):
    """Frobenius norm in fp64 over row chunks (X: fp32, any shape)."""
    s = 0.0
    for r0 in range(0, X.shape[0], CH):
        blk = X[r0:r0 + CH].astype(np.float64)
        s += float(np.sum(blk * blk))
    return s ** 0.5


def fro_tri_sym(A):
    """||sym(A)||_F from A's lower triangle: 2 ||strict lower||^2 + ||diag||^2."""
    s = 0.0
    for r0 in range(0, A.shape[0], CH):
        blk = A[r0:r0 + CH].astype(np.float64)
        rr = np.arange(r0, r0 + blk.shape[0])[:, None]
        cc = np.arange(A.shape[1])[None, :]
        s += 2.0 * float(np.sum(np.where(cc < rr, blk * blk, 0.0)))
        s += float(np.sum(np.where(cc == rr, blk * blk, 0.0)))
    return s ** 0.5


def tri_matmul(T, X):
    """tril(T) @ X in fp64 over row chunks (NaN blank triangle ignored)."""
    out = np.empty((T.shape[0], X.shape[1]))
    X64 = f64(X)
    for r0 in range(0, T.shape[0], CH):
        blk = T[r0:r0 + CH].astype(np.float64)
        rr = np.arange(r0, r0 + blk.shape[0])[:, None]
        cc = np.arange(T.shape[1])[None, :]
        out[r0:r0 + CH] = np.where(cc <= rr, blk, 0.0) @ X64
    return out


@pytest.fixture(scope="module")
def env():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    free, _ = torch.cuda.mem_get_info()
    if free < 20 * 2**30:
        pytest.skip("needs ~20 GiB of device memory")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_cuiwxyf11_b200 as b3
    import oracle
    oracle.build()
    b3.set_math_mode("3xtf32")
    sel = gen.sample_indices(N, 8, "cfg5-parity")
    return b3, oracle, sel


def test_sgemm_ssymm_32768(env):
    import torch
    b3, oracle, sel = env
    A = gen.uniform(N, N, "cfg5-A")
    B = gen.uniform(N, N, "cfg5-B")
    C = gen.uniform(N, N, "cfg5-C")
    dA, dB = to_dev(A), to_dev(B)
    nA, nBs, nCs = fro_big(A), fro_big(B[:, sel]), fro_big(C[:, sel])
    # SGEMM NN
    dC = to_dev(C)
    before = b3.launch_count("tc")
    b3.sgemm("N", "N", AL, dA, dB, BE, dC)
    got = to_host(dC[:, sel])
    assert b3.launch_count("tc") > before
    ref = oracle.sgemm("N", "N", AL, A, B, BE, C, sel=sel)
    err = np.linalg.norm(f64(got) - ref) / (AL * nA * nBs + BE * nCs)
    assert err <= TOL_NW, err
    # SSYMM LL: only A's lower triangle is read (sym(A) from it)
    dC.copy_(to_dev(C))
    b3.ssymm("L", "L", AL, dA, dB, BE, dC)
    got = to_host(dC[:, sel])
    ref = oracle.ssymm("L", "L", AL, A, B, BE, C, sel=sel)
    err = np.linalg.norm(f64(got) - ref) / (AL * fro_tri_sym(A) * nBs + BE * nCs)
    assert err <= TOL_NW, err
    del dA, dB, dC
    torch.cuda.empty_cache()


def test_strsm_32768(env):
    import torch
    b3, oracle, sel = env
    T = gen.triangular_dd(N, "L", "N", "cfg5-T")
    B = gen.uniform(N, N, "cfg5-B")
    dX = to_dev(B)
    b3.strsm("L", "L", "N", "N", AL, to_dev(T), dX)
    Xs = f64(to_host(dX[:, sel]))
    Bs = f64(B[:, sel])
    nT = 0.0
    for r0 in range(0, N, CH):                          # ||tril(T)|| (blank triangle is NaN)
        blk = np.nan_to_num(T[r0:r0 + CH].astype(np.float64))
        rr = np.arange(r0, r0 + blk.shape[0])[:, None]
        nT += float(np.sum(np.where(np.arange(N)[None, :] <= rr, blk * blk, 0.0)))
    nT **= 0.5
    resid = np.linalg.norm(tri_matmul(np.nan_to_num(T), Xs) - AL * Bs) / (nT * np.linalg.norm(Xs))
    assert resid <= 1e-5 * np.sqrt(N), resid
    ref = oracle.strsm("L", "L", "N", "N", AL, T, B, sel=sel)
    assert np.linalg.norm(Xs - ref) / np.linalg.norm(ref) <= 1e-5
    del dX
    torch.cuda.empty_cache()
