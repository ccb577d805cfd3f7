"""Parity at BASELINE.json's full size, in the configuration bench.py times.

N = K = 8192, alpha = 1.5, beta = 0.5, the bench's seeded inputs, and EVERY
variant of every routine at that size: SGEMM x 4 transa/transb, SSYMM x 4
side/uplo (the default staged route and GM_map forced on), SSYRK and
SSYR2K x 4 uplo/trans (configs[3] at N = K = 8192), STRMM and STRSM x 16
side/uplo/trans/diag (configs[2] at 8192).  The fp64 oracle computes a sample
of output columns exactly (columns are independent; rows for STRSM side=R),
and the metrics are restricted to that sample consistently:
normwise <= 1e-5 (north star), the output-relative diagnostic
max(4 * e_rel(plain fp32), 2e-6) (check.rel_bound), STRSM
residual <= 1e-5 sqrt(N) and forward error <= 1e-5.
"""
import itertools

import numpy as np
import pytest

import blas3_inputs as gen
from check import (TOL_NW, e_nw, e_rel, f64, fro, op, rel_bound, sel_f32, sym_f32, to_dev, to_host,
                   tri_f32)

pytestmark = pytest.mark.gpu

N = 8192
AL, BE = 1.5, 0.5
NSEL = 24


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
    B = gen.uniform(N, N, "bench-B", 0)
    C = gen.uniform(N, N, "bench-C", 0)
    sel = gen.sample_indices(N, NSEL, "large-parity")
    return dict(b3=b3, oracle=oracle, A=A, B=B, C=C, sel=sel, dA=to_dev(A), dB=to_dev(B))


_TRI = {}


def tri(uplo, diag):
    """The bench's T (lower, diag N) and the other three stored forms."""
    key = (uplo, diag)
    if key not in _TRI:
        _TRI.clear()                     # one 256 MiB triangle (+ device copy) at a time
        T = gen.triangular_dd(N, "L", "N", "bench-T") if key == ("L", "N") else \
            gen.triangular_dd(N, uplo, diag, "large-T")
        _TRI[key] = (T, to_dev(T), tri_f32(T, uplo, diag))
    return _TRI[key]


def _tc_used(b3, before):
    assert b3.launch_count("tc") > before, "expected the tcgen05 route"


def _col_mask(sel, uplo):
    mask = np.zeros((N, len(sel)), bool)
    for t, j in enumerate(sel):
        if uplo == "L":
            mask[j:, t] = True
        else:
            mask[: j + 1, t] = True
    return mask


@pytest.mark.parametrize("ta,tb", list(itertools.product("NT", "NT")))
def test_sgemm_8192(env, ta, tb):
    b3, A, B, C, sel = env["b3"], env["A"], env["B"], env["C"], env["sel"]
    before = b3.launch_count("tc")
    dC = to_dev(C)
    b3.sgemm(ta, tb, AL, env["dA"], env["dB"], BE, dC)
    got = to_host(dC)[:, sel]
    _tc_used(b3, before)
    ref = env["oracle"].sgemm(ta, tb, AL, A, B, BE, C, sel=sel)
    opB_S = B[:, sel] if tb == "N" else B[sel, :]
    scale = AL * fro(A) * fro(opB_S) + BE * fro(C[:, sel])
    assert e_nw(got, ref, scale) <= TOL_NW
    assert e_rel(got, ref) <= rel_bound(sel_f32("sgemm", (ta, tb, AL, A, B, BE, C), sel), ref)


@pytest.mark.parametrize("gm_map", [-1, 1])
@pytest.mark.parametrize("side,uplo", list(itertools.product("LR", "LU")))
def test_ssymm_8192(env, side, uplo, gm_map):
    """gm_map=-1: the default, staged route (sym(A) merged while staging from
    both stored orientations, never materialised); 1: GM_map forced on."""
    b3, A, B, C, sel = env["b3"], env["A"], env["B"], env["C"], env["sel"]
    dC = to_dev(C)
    with b3.options(gm_map=gm_map):
        b3.ssymm(side, uplo, AL, env["dA"], env["dB"], BE, dC)   # only A's uplo triangle is read
    got = to_host(dC)[:, sel]
    ref = env["oracle"].ssymm(side, uplo, AL, A, B, BE, C, sel=sel)
    S = sym_f32(A, uplo)
    # side=L: column j of C uses B(:,j); side=R: column j uses Asym(:,j)
    scale = (AL * fro(S) * fro(B[:, sel]) if side == "L" else AL * fro(B) * fro(S[:, sel])) \
        + BE * fro(C[:, sel])
    assert e_nw(got, ref, scale) <= TOL_NW
    assert e_rel(got, ref) <= rel_bound(sel_f32("ssymm", (side, uplo, AL, A, B, BE, C, S), sel), ref)


@pytest.mark.parametrize("two", [False, True])
@pytest.mark.parametrize("uplo,trans", list(itertools.product("LU", "NT")))
def test_syrk_syr2k_8192(env, two, uplo, trans):
    b3, A, B, C, sel = env["b3"], env["A"], env["B"], env["C"], env["sel"]
    dC = to_dev(C)
    if two:
        b3.ssyr2k(uplo, trans, AL, env["dA"], env["dB"], BE, dC)
        ref = env["oracle"].ssyr2k(uplo, trans, AL, A, B, BE, C, sel=sel)
    else:
        b3.ssyrk(uplo, trans, AL, env["dA"], BE, dC)
        ref = env["oracle"].ssyrk(uplo, trans, AL, A, BE, C, sel=sel)
    got = to_host(dC)[:, sel]
    mask = _col_mask(sel, uplo)
    opA_S = A[sel, :] if trans == "N" else A[:, sel]
    opB_S = B[sel, :] if trans == "N" else B[:, sel]
    scale = (AL * (fro(A) * fro(opB_S) + fro(B) * fro(opA_S)) if two else AL * fro(A) * fro(opA_S)) \
        + BE * fro(C[:, sel][mask])
    assert e_nw(got[mask], ref[mask], scale) <= TOL_NW
    f32 = sel_f32("ssyr2k" if two else "ssyrk", (uplo, trans, AL, A, B if two else None, BE, C), sel)
    assert e_rel(got[mask], ref[mask]) <= rel_bound(f32[mask], ref[mask])
    assert np.array_equal(got[~mask].view(np.uint32), C[:, sel][~mask].view(np.uint32))


V16 = list(itertools.product("LU", "NU", "LR", "NT"))     # (uplo, diag) outer: one T at a time


@pytest.mark.parametrize("uplo,diag,side,ta", V16)
def test_strmm_8192(env, uplo, diag, side, ta):
    b3, B, sel = env["b3"], env["B"], env["sel"]
    T, dT, T32 = tri(uplo, diag)
    dX = to_dev(B)
    b3.strmm(side, uplo, ta, diag, AL, dT, dX)
    got = to_host(dX)[:, sel]
    ref = env["oracle"].strmm(side, uplo, ta, diag, AL, T, B, sel=sel)
    opT = op(T32, ta)
    scale = AL * fro(opT) * fro(B[:, sel]) if side == "L" else AL * fro(B) * fro(opT[:, sel])
    assert e_nw(got, ref, scale) <= TOL_NW
    assert e_rel(got, ref) <= rel_bound(sel_f32("strmm", (side, ta, AL, T32, B), sel), ref)


@pytest.mark.parametrize("uplo,diag,side,ta", V16)
def test_strsm_8192(env, uplo, diag, side, ta):
    b3, B, sel = env["b3"], env["B"], env["sel"]
    T, dT, T32 = tri(uplo, diag)
    dX = to_dev(B)
    b3.strsm(side, uplo, ta, diag, AL, dT, dX)
    X = to_host(dX)
    opT = f64(op(T32, ta))
    if side == "L":
        Xs = f64(X[:, sel])
        resid = fro(opT @ Xs - AL * f64(B[:, sel])) / (fro(opT) * fro(Xs))
    else:
        Xs = f64(X[sel, :])
        resid = fro(Xs @ opT - AL * f64(B[sel, :])) / (fro(opT) * fro(Xs))
    assert resid <= 1e-5 * np.sqrt(N)
    ref = env["oracle"].strsm(side, uplo, ta, diag, AL, T, B, sel=sel)
    assert fro(Xs - ref) / fro(ref) <= 1e-5


@pytest.mark.parametrize("ta,tb", [("N", "N"), ("T", "N")])
def test_sgemm_8192_tf32_bf16x(env, ta, tb):
    """The opt-in TF32+BF16X mode (packed bf16 cross terms) at the bench size."""
    b3, A, B, C, sel = env["b3"], env["A"], env["B"], env["C"], env["sel"]
    b3.set_math_mode("tf32_bf16x")
    try:
        dC = to_dev(C)
        b3.sgemm(ta, tb, AL, env["dA"], env["dB"], BE, dC)
        got = to_host(dC)[:, sel]
    finally:
        b3.set_math_mode("3xtf32")
    ref = env["oracle"].sgemm(ta, tb, AL, A, B, BE, C, sel=sel)
    scale = AL * fro(A) * fro(B[:, sel]) + BE * fro(C[:, sel])
    assert e_nw(got, ref, scale) <= TOL_NW
    assert e_rel(got, ref) <= rel_bound(sel_f32("sgemm", (ta, tb, AL, A, B, BE, C), sel), ref)
