"""BLAS3_MATH_1XTF32: the opt-in fast mode (Q25).

One TF32 pass (hi*hi only; the tensor core truncates each fp32 input to its
top 10 mantissa bits).  The binding accuracy claim is the TF32 one, derived
from the arithmetic: every product a*b is formed from hi(a)*hi(b) with
|x - hi(x)| < 2^-10 |x|, so |ab - hi(a)hi(b)| < (2^-9 + 2^-20)|a||b| and
    ||C - C_ref||_F <= |alpha| (2^-9 + 2^-20) || |op(A)| |op(B)| ||_F + fp32 terms
                    <= (2^-9 + 2^-20) |alpha| ||A||_F ||B||_F + ...,
i.e. normwise error <= 2^-9 (+ a 1e-5 margin for the fp32 accumulation).
Two pins that the mode is what it claims:
  * random data: the error is far above the 3xTF32 level (the lo terms are
    really dropped), but within the bound;
  * integer data |x| <= 4 (exactly representable in TF32): bit-exact, as the
    truncation drops nothing.
"""
import itertools

import numpy as np
import pytest

import blas3_inputs as gen
from check import bits_equal, e_nw, f64, fro, op, sym_full, to_dev, to_host, tri_full

pytestmark = pytest.mark.gpu
AL, BE = 1.5, 0.5
BOUND = 2.0 ** -9 + 1e-5


@pytest.fixture(scope="module")
def b3():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_cuiwxyf11_b200 as m
    m.set_math_mode("1xtf32")
    yield m
    m.set_math_mode("3xtf32")


@pytest.mark.parametrize("ta,tb", list(itertools.product("NT", "NT")))
def test_sgemm_1xtf32(b3, oracle_mod, ta, tb):
    m, n, k = 300, 520, 516
    A = gen.uniform(*((m, k) if ta == "N" else (k, m)), "fm-a", ta)
    B = gen.uniform(*((k, n) if tb == "N" else (n, k)), "fm-b", tb)
    C = gen.uniform(m, n, "fm-c")
    before = b3.launch_count("tc")
    dC = to_dev(C)
    b3.sgemm(ta, tb, AL, to_dev(A), to_dev(B), BE, dC)
    assert b3.launch_count("tc") > before
    ref = oracle_mod.sgemm(ta, tb, AL, A, B, BE, C)
    e = e_nw(to_host(dC), ref, AL * fro(A) * fro(B) + BE * fro(C))
    assert 1e-6 < e <= BOUND, e


@pytest.mark.parametrize("side,uplo", list(itertools.product("LR", "LU")))
def test_ssymm_1xtf32(b3, oracle_mod, side, uplo):
    m, n = 400, 260
    ka = m if side == "L" else n
    A = gen.symmetric_stored(ka, uplo, "fm-s")
    B = gen.uniform(m, n, "fm-sb")
    C = gen.uniform(m, n, "fm-sc")
    dC = to_dev(C)
    b3.ssymm(side, uplo, AL, to_dev(A), to_dev(B), BE, dC)
    ref = oracle_mod.ssymm(side, uplo, AL, A, B, BE, C)
    e = e_nw(to_host(dC), ref, AL * fro(sym_full(A, uplo, ka)) * fro(B) + BE * fro(C))
    assert 1e-6 < e <= BOUND, e


@pytest.mark.parametrize("uplo,trans", list(itertools.product("LU", "NT")))
def test_ssyrk_ssyr2k_1xtf32(b3, oracle_mod, uplo, trans):
    n, k = 332, 272                 # ld % 4 == 0: the tcgen05 route (else SIMT, exact fp32)
    A = gen.uniform(*((n, k) if trans == "N" else (k, n)), "fm-k", trans)
    B = gen.uniform(*((n, k) if trans == "N" else (k, n)), "fm-k2", trans)
    C = gen.uniform(n, n, "fm-kc")
    mask = np.tril(np.ones((n, n), bool)) if uplo == "L" else np.triu(np.ones((n, n), bool))
    dC = to_dev(C)
    b3.ssyrk(uplo, trans, AL, to_dev(A), BE, dC)
    got = to_host(dC)
    ref = oracle_mod.ssyrk(uplo, trans, AL, A, BE, C)
    e = e_nw(got[mask], ref[mask], AL * fro(A) ** 2 + BE * fro(C[mask]))
    assert 1e-6 < e <= BOUND and bits_equal(got[~mask], C[~mask]), e
    dC = to_dev(C)
    b3.ssyr2k(uplo, trans, AL, to_dev(A), to_dev(B), BE, dC)
    got = to_host(dC)
    ref = oracle_mod.ssyr2k(uplo, trans, AL, A, B, BE, C)
    e = e_nw(got[mask], ref[mask], 2 * AL * fro(A) * fro(B) + BE * fro(C[mask]))
    assert 1e-6 < e <= BOUND, e


@pytest.mark.parametrize("side,uplo,ta,diag", list(itertools.product("LR", "LU", "NT", "N")))
def test_strmm_strsm_1xtf32(b3, oracle_mod, side, uplo, ta, diag):
    m, n = 600, 280
    ka = m if side == "L" else n
    A = gen.triangular_dd(ka, uplo, diag, "fm-t")
    B = gen.uniform(m, n, "fm-tb")
    T = op(tri_full(A, uplo, diag, ka), ta)
    dB = to_dev(B)
    b3.strmm(side, uplo, ta, diag, AL, to_dev(A), dB)
    ref = oracle_mod.strmm(side, uplo, ta, diag, AL, A, B)
    e = e_nw(to_host(dB), ref, AL * fro(T) * fro(B))
    assert 1e-6 < e <= BOUND, e
    dB = to_dev(B)
    b3.strsm(side, uplo, ta, diag, AL, to_dev(A), dB)
    X = f64(to_host(dB))
    R = (T @ X if side == "L" else X @ T) - AL * f64(B)
    resid = fro(R) / (fro(T) * fro(X))
    assert resid <= BOUND, resid


def test_integer_inputs_exact_in_1xtf32(b3, oracle_mod):
    """|x| <= 4 integers are exact in TF32: the fast mode drops nothing."""
    m, n, k = 260, 300, 140
    A = gen.integers(m, k, "fm-ia")
    B = gen.integers(k, n, "fm-ib")
    C = gen.integers(m, n, "fm-ic")
    dC = to_dev(C)
    b3.sgemm("N", "N", 1.0, to_dev(A), to_dev(B), 1.0, dC)
    ref = oracle_mod.sgemm("N", "N", 1.0, A, B, 1.0, C)
    assert bits_equal(to_host(dC), ref.astype(np.float32))
