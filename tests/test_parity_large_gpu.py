"""Parity at BASELINE.json's full size, in the configuration bench.py times.

N = K = 8192, alpha = 1.5, beta = 0.5, the bench's seeded inputs and variants
(sgemm NN, ssymm LL, ssyrk LN, ssyr2k LN, strmm LLNN, strsm LLNN, plus the
transposed / right-side / upper variants below).  The fp64 oracle computes a
sample of output columns exactly (columns are independent), and the metrics
are restricted to that sample consistently.
"""
import numpy as np
import pytest

import blas3_inputs as gen
from check import TOL_NW, e_nw, f64, fro, to_dev, to_host, tol_rel

pytestmark = pytest.mark.gpu

N = 8192
AL, BE = 1.5, 0.5


@pytest.fixture(scope="module")
def env():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_cuiwxyf11_b200 as b3
    import oracle
    oracle.build()
    b3.set_math_mode("3xtf32")
    A = gen.uniform(N, N, "bench-A")
    T = gen.triangular_dd(N, "L", "N", "bench-T")
    B = gen.uniform(N, N, "bench-B", 0)
    C = gen.uniform(N, N, "bench-C", 0)
    sel = gen.sample_indices(N, 24, "large-parity")
    return b3, oracle, A, T, B, C, sel, {k: to_dev(v) for k, v in dict(A=A, T=T, B=B).items()}


def _tc_used(b3, before):
    assert b3.launch_count("tc") > before, "expected the tcgen05 route"


@pytest.mark.parametrize("ta,tb", [("N", "N"), ("T", "N"), ("N", "T")])
def test_sgemm_8192(env, ta, tb):
    b3, oracle, A, T, B, C, sel, d = env
    before = b3.launch_count("tc")
    dC = to_dev(C)
    b3.sgemm(ta, tb, AL, d["A"], d["B"], BE, dC)
    got = to_host(dC)[:, sel]
    _tc_used(b3, before)
    ref = oracle.sgemm(ta, tb, AL, A, B, BE, C, sel=sel)
    opB_S = B[:, sel] if tb == "N" else B[sel, :]
    scale = AL * fro(A) * fro(opB_S) + BE * fro(C[:, sel])
    assert e_nw(got, ref, scale) <= TOL_NW
    assert fro(f64(got) - ref) / fro(ref) <= tol_rel(N, "3xtf32")


@pytest.mark.parametrize("side,uplo", [("L", "L"), ("R", "U")])
def test_ssymm_8192(env, side, uplo):
    b3, oracle, A, T, B, C, sel, d = env
    dC = to_dev(C)
    b3.ssymm(side, uplo, AL, d["A"], d["B"], BE, dC)     # only A's uplo triangle is read
    got = to_host(dC)[:, sel]
    ref = oracle.ssymm(side, uplo, AL, A, B, BE, C, sel=sel)
    Af = f64(A)
    S = (np.tril(Af) + np.tril(Af, -1).T) if uplo == "L" else (np.triu(Af) + np.triu(Af, 1).T)
    # side=L: column j of C uses B(:,j); side=R: column j uses Asym(:,j)
    scale = (AL * fro(S) * fro(B[:, sel]) if side == "L" else AL * fro(B) * fro(S[:, sel])) \
        + BE * fro(C[:, sel])
    assert e_nw(got, ref, scale) <= TOL_NW


@pytest.mark.parametrize("two", [False, True])
@pytest.mark.parametrize("uplo,trans", [("L", "N"), ("U", "T")])
def test_syrk_syr2k_8192(env, two, uplo, trans):
    b3, oracle, A, T, B, C, sel, d = env
    dC = to_dev(C)
    if two:
        b3.ssyr2k(uplo, trans, AL, d["A"], d["B"], BE, dC)
        ref = oracle.ssyr2k(uplo, trans, AL, A, B, BE, C, sel=sel)
    else:
        b3.ssyrk(uplo, trans, AL, d["A"], BE, dC)
        ref = oracle.ssyrk(uplo, trans, AL, A, BE, C, sel=sel)
    got = to_host(dC)[:, sel]
    mask = np.zeros((N, len(sel)), bool)
    for t, j in enumerate(sel):
        if uplo == "L":
            mask[j:, t] = True
        else:
            mask[: j + 1, t] = True
    opA_S = A[sel, :] if trans == "N" else A[:, sel]
    opB_S = B[sel, :] if trans == "N" else B[:, sel]
    scale = (AL * (fro(A) * fro(opB_S) + fro(B) * fro(opA_S)) if two else AL * fro(A) * fro(opA_S)) \
        + BE * fro(C[:, sel][mask])
    assert e_nw(got[mask], ref[mask], scale) <= TOL_NW
    assert np.array_equal(got[~mask].view(np.uint32), C[:, sel][~mask].view(np.uint32))


@pytest.mark.parametrize("side,ta", [("L", "N"), ("R", "T")])
def test_strmm_8192(env, side, ta):
    b3, oracle, A, T, B, C, sel, d = env
    dX = to_dev(B)
    b3.strmm(side, "L", ta, "N", AL, d["T"], dX)
    got = to_host(dX)[:, sel]
    ref = oracle.strmm(side, "L", ta, "N", AL, T, B, sel=sel)
    Tf = np.tril(np.nan_to_num(f64(T)))
    opT = Tf if ta == "N" else Tf.T
    scale = AL * fro(opT) * fro(B[:, sel]) if side == "L" else AL * fro(B) * fro(opT[:, sel])
    assert e_nw(got, ref, scale) <= TOL_NW


@pytest.mark.parametrize("ta", ["N", "T"])
def test_strsm_8192(env, ta):
    b3, oracle, A, T, B, C, sel, d = env
    dX = to_dev(B)
    b3.strsm("L", "L", ta, "N", AL, d["T"], dX)
    X = f64(to_host(dX)[:, sel])
    Tf = np.tril(np.nan_to_num(f64(T)))
    opT = Tf if ta == "N" else Tf.T
    resid = fro(opT @ X - AL * f64(B[:, sel])) / (fro(opT) * fro(X))
    assert resid <= 1e-5 * np.sqrt(N)
    ref = oracle.strsm("L", "L", ta, "N", AL, T, B, sel=sel)
    assert fro(X - ref) / fro(ref) <= 1e-5


@pytest.mark.parametrize("ta,tb", [("N", "N"), ("T", "N")])
def test_sgemm_8192_tf32_bf16x(env, ta, tb):
    """The opt-in TF32+BF16X mode (packed bf16 cross terms) at the bench size."""
    b3, oracle, A, T, B, C, sel, d = env
    b3.set_math_mode("tf32_bf16x")
    try:
        dC = to_dev(C)
        b3.sgemm(ta, tb, AL, d["A"], d["B"], BE, dC)
        got = to_host(dC)[:, sel]
    finally:
        b3.set_math_mode("3xtf32")
    ref = oracle.sgemm(ta, tb, AL, A, B, BE, C, sel=sel)
    scale = AL * fro(A) * fro(B[:, sel]) + BE * fro(C[:, sel])
    assert e_nw(got, ref, scale) <= TOL_NW
    assert fro(f64(got) - ref) / fro(ref) <= tol_rel(N, "tf32_bf16x")
