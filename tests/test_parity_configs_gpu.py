"""Parity on the other BASELINE.json configurations (sampled oracle columns).

configs[1]: SGEMM and SSYMM square sweep N = 1024..8192 (sampled sizes), all
            transa/transb and side/uplo variants;
configs[2]: STRMM and STRSM at N = 4096, all 16 side/uplo/trans/diag, with
            diagonally dominant A (reading Q22);
configs[3]: SSYRK and SSYR2K tall-skinny N = 16384, K = 512, both uplo/trans.
The oracle computes 12 sampled output columns exactly (rows for STRSM
side='R'); metrics are restricted to the sample.
"""
import itertools

import numpy as np
import pytest

import blas3_inputs as gen
from check import (TOL_NW, e_nw, e_rel, f64, fro, rel_bound, sel_f32, sym_f32, to_dev, to_host,
                   tri_f32, tri_full)

pytestmark = pytest.mark.gpu
AL, BE = 1.5, 0.5
NS = 12


@pytest.fixture(scope="module")
def b3():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_cuiwxyf11_b200 as m
    m.set_math_mode("3xtf32")
    return m


@pytest.mark.parametrize("n", [1024, 3072, 7168])
def test_cfg2_sgemm_ssymm_sweep(b3, oracle_mod, n):
    A = gen.uniform(n, n, "c2-A", n); B = gen.uniform(n, n, "c2-B", n); C = gen.uniform(n, n, "c2-C", n)
    sel = gen.sample_indices(n, NS, "c2", n)
    dA, dB = to_dev(A), to_dev(B)
    for ta, tb in itertools.product("NT", "NT"):
        dC = to_dev(C)
        b3.sgemm(ta, tb, AL, dA, dB, BE, dC)
        got = to_host(dC)[:, sel]
        ref = oracle_mod.sgemm(ta, tb, AL, A, B, BE, C, sel=sel)
        opB_S = B[:, sel] if tb == "N" else B[sel, :]
        assert e_nw(got, ref, AL * fro(A) * fro(opB_S) + BE * fro(C[:, sel])) <= TOL_NW, (ta, tb)
        f32 = sel_f32("sgemm", (ta, tb, AL, A, B, BE, C), sel)
        assert e_rel(got, ref) <= rel_bound(f32, ref), (ta, tb)
    Af = f64(A)
    for side, uplo in itertools.product("LR", "LU"):
        dC = to_dev(C)
        b3.ssymm(side, uplo, AL, dA, dB, BE, dC)
        got = to_host(dC)[:, sel]
        ref = oracle_mod.ssymm(side, uplo, AL, A, B, BE, C, sel=sel)
        S = (np.tril(Af) + np.tril(Af, -1).T) if uplo == "L" else (np.triu(Af) + np.triu(Af, 1).T)
        scale = (AL * fro(S) * fro(B[:, sel]) if side == "L" else AL * fro(B) * fro(S[:, sel])) \
            + BE * fro(C[:, sel])
        assert e_nw(got, ref, scale) <= TOL_NW, (side, uplo)
        f32 = sel_f32("ssymm", (side, uplo, AL, A, B, BE, C, sym_f32(A, uplo)), sel)
        assert e_rel(got, ref) <= rel_bound(f32, ref), (side, uplo)


@pytest.fixture(scope="module")
def cfg3():
    n = 4096
    B = gen.uniform(n, n, "c3-B")
    tris = {(u, d): gen.triangular_dd(n, u, d, "c3") for u in "LU" for d in "NU"}
    return n, B, tris


@pytest.mark.parametrize("side,uplo,ta,diag", list(itertools.product("LR", "LU", "NT", "NU")))
def test_cfg3_strmm_strsm_4096(b3, oracle_mod, cfg3, side, uplo, ta, diag):
    n, B, tris = cfg3
    A = tris[(uplo, diag)]
    sel = gen.sample_indices(n, NS, "c3", side, uplo, ta, diag)
    T = tri_full(A, uplo, diag, n)
    opT = T if ta == "N" else T.T
    dA = to_dev(A)
    # STRMM
    dX = to_dev(B)
    b3.strmm(side, uplo, ta, diag, AL, dA, dX)
    got = to_host(dX)[:, sel]
    ref = oracle_mod.strmm(side, uplo, ta, diag, AL, A, B, sel=sel)
    scale = AL * fro(opT) * fro(B[:, sel]) if side == "L" else AL * fro(B) * fro(opT[:, sel])
    assert e_nw(got, ref, scale) <= TOL_NW
    f32 = sel_f32("strmm", (side, ta, AL, tri_f32(A, uplo, diag), B), sel)
    assert e_rel(got, ref) <= rel_bound(f32, ref)
    # STRSM: residual + forward error on the sample (rows for side=R)
    dX = to_dev(B)
    b3.strsm(side, uplo, ta, diag, AL, dA, dX)
    X = to_host(dX)
    if side == "L":
        Xs = f64(X[:, sel])
        resid = fro(opT @ Xs - AL * f64(B[:, sel])) / (fro(opT) * fro(Xs))
    else:
        Xs = f64(X[sel, :])
        resid = fro(Xs @ opT - AL * f64(B[sel, :])) / (fro(opT) * fro(Xs))
    assert resid <= 1e-5 * np.sqrt(n)
    ref = oracle_mod.strsm(side, uplo, ta, diag, AL, A, B, sel=sel)
    assert fro(Xs - ref) / fro(ref) <= 1e-5


@pytest.fixture(scope="module")
def cfg4():
    n, k = 16384, 512
    C = gen.uniform(n, n, "c4-C")
    return n, k, C


@pytest.mark.parametrize("two", [False, True])
@pytest.mark.parametrize("uplo,trans", list(itertools.product("LU", "NT")))
def test_cfg4_tall_skinny_syrk_syr2k(b3, oracle_mod, cfg4, two, uplo, trans):
    n, k, C = cfg4
    shp = (n, k) if trans == "N" else (k, n)
    A, B = gen.uniform(*shp, "c4-A"), gen.uniform(*shp, "c4-B")
    sel = gen.sample_indices(n, NS, "c4", uplo, trans)
    dC = to_dev(C)
    if two:
        b3.ssyr2k(uplo, trans, AL, to_dev(A), to_dev(B), BE, dC)
        ref = oracle_mod.ssyr2k(uplo, trans, AL, A, B, BE, C, sel=sel)
    else:
        b3.ssyrk(uplo, trans, AL, to_dev(A), BE, dC)
        ref = oracle_mod.ssyrk(uplo, trans, AL, A, BE, C, sel=sel)
    got = to_host(dC)[:, sel]
    mask = np.zeros((n, len(sel)), bool)
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
    f32 = sel_f32("ssyr2k" if two else "ssyrk", (uplo, trans, AL, A, B if two else None, BE, C), sel)
    assert e_rel(got[mask], ref[mask]) <= rel_bound(f32[mask], ref[mask])
    assert np.array_equal(got[~mask].view(np.uint32), C[:, sel][~mask].view(np.uint32))
