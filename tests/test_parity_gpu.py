"""GPU parity: the CUDA path (via the C ABI) against the fp64 oracle.

Binding tolerances are the north star's (BASELINE.json): normwise relative
error <= 1e-5 for the product routines, STRSM residual <= 1e-5*sqrt(N) on
diagonally dominant A.  Because 1xTF32 would also pass those at N >= 1024
(SURVEY EXP-1), every case also checks the output-relative error against a
kernel-independent bound, max(4 * e_rel(plain fp32 evaluation), 2e-6)
(check.rel_bound), and STRSM's forward error <= 1e-5.
Integer-valued inputs must reproduce the oracle bit for bit (one correct
answer, Q18).  Sizes span several tiles and ragged tails.
All three fp32-accurate math modes (3xTF32 and TF32+BF16X on tcgen05, FP32
SIMT) are exercised.
"""
import itertools

import numpy as np
import pytest

import blas3_inputs as gen
from check import (TOL_NW, bits_equal, e_nw, e_rel, f32_eval, f64, fro, op, rel_bound, sym_full,
                   syr2k_f32, to_dev, to_host, tri_full)

pytestmark = pytest.mark.gpu

MODES = ["3xtf32", "simt", "tf32_bf16x"]
AL, BE = 1.5, 0.5


@pytest.fixture(scope="module")
def b3():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_cuiwxyf11_b200 as m
    return m


@pytest.fixture(params=MODES)
def mode(request, b3):
    b3.set_math_mode(request.param)
    yield request.param
    b3.set_math_mode("3xtf32")


@pytest.fixture
def route(b3, mode):
    """route(*lds) after a call: in 3xtf32 mode, TMA-eligible leading
    dimensions (all % 4 == 0) must have run on the tcgen05 kernel; anything
    else (or SIMT mode) must not have."""
    before = {p: b3.launch_count(p) for p in ("tc", "simt")}

    def check(*lds):
        tc = b3.launch_count("tc") > before["tc"]
        if mode != "simt" and all(ld % 4 == 0 for ld in lds):
            assert tc, "expected the tcgen05 route"
        else:
            assert not tc, "tcgen05 route taken unexpectedly"
    return check


# ------------------------------------------------------------------------------------ SGEMM
GEMM_SIZES = [(1, 1, 1), (33, 17, 45), (132, 260, 100), (256, 256, 256), (300, 132, 520),
              (516, 1000, 260)]


@pytest.mark.parametrize("ta,tb", list(itertools.product("NT", "NT")))
@pytest.mark.parametrize("m,n,k", GEMM_SIZES)
def test_sgemm(b3, oracle_mod, mode, route, ta, tb, m, n, k):
    A = gen.uniform(*((m, k) if ta == "N" else (k, m)), "pg-a", ta)
    B = gen.uniform(*((k, n) if tb == "N" else (n, k)), "pg-b", tb)
    C = gen.uniform(m, n, "pg-c")
    dC = to_dev(C)
    b3.sgemm(ta, tb, AL, to_dev(A), to_dev(B), BE, dC)
    got = to_host(dC)
    route(A.shape[0], B.shape[0], m)
    ref = oracle_mod.sgemm(ta, tb, AL, A, B, BE, C)
    assert e_nw(got, ref, AL * fro(A) * fro(B) + BE * fro(C)) <= TOL_NW
    assert e_rel(got, ref) <= rel_bound(f32_eval(AL, op(A, ta), op(B, tb), BE, C), ref)


@pytest.mark.parametrize("k", [512, 8192])
def test_same_sign_accumulation(b3, oracle_mod, mode, k):
    """Worst case for the tensor core's truncating fp32 accumulator (reading
    Q24): with all products positive every truncation biases the sum the same
    way, so the error adds up coherently over the UMMAs of one TMEM partial
    instead of as a random walk.  The plain fp32 evaluation (round to nearest)
    has no such bias; the kernel must stay within the same diagnostic bound."""
    m, n = 256, 260
    A = gen.uniform(m, k, "pos-a", lo=0.0, hi=1.0)
    B = gen.uniform(k, n, "pos-b", lo=0.0, hi=1.0)
    C = gen.uniform(m, n, "pos-c", lo=0.0, hi=1.0)
    dC = to_dev(C)
    b3.sgemm("N", "N", AL, to_dev(A), to_dev(B), BE, dC)
    got = to_host(dC)
    ref = oracle_mod.sgemm("N", "N", AL, A, B, BE, C)
    assert e_nw(got, ref, AL * fro(A) * fro(B) + BE * fro(C)) <= TOL_NW
    assert e_rel(got, ref) <= rel_bound(f32_eval(AL, A, B, BE, C), ref)


@pytest.mark.parametrize("ta,tb", list(itertools.product("NT", "NT")))
@pytest.mark.parametrize("m,n,k", [(132, 260, 1000), (64, 300, 36)])
def test_sgemm_integer_bitexact(b3, oracle_mod, mode, ta, tb, m, n, k):
    A = gen.integers(*((m, k) if ta == "N" else (k, m)), "ig-a")
    B = gen.integers(*((k, n) if tb == "N" else (n, k)), "ig-b")
    C = gen.integers(m, n, "ig-c")
    dC = to_dev(C)
    b3.sgemm(ta, tb, AL, to_dev(A), to_dev(B), BE, dC)
    ref = oracle_mod.sgemm(ta, tb, AL, A, B, BE, C).astype(np.float32)
    assert bits_equal(to_host(dC), ref)


def test_sgemm_beta0_nan_c_and_alpha0(b3, mode):
    m = n = k = 70
    A, B = gen.uniform(m, k, "z-a"), gen.uniform(k, n, "z-b")
    Cn = np.full((m, n), np.nan, np.float32, order="F")
    dC = to_dev(Cn)
    b3.sgemm("N", "N", 1.0, to_dev(A), to_dev(B), 0.0, dC)
    assert np.isfinite(to_host(dC)).all()
    An = np.full((m, k), np.nan, np.float32, order="F")
    C = gen.uniform(m, n, "z-c")
    dC = to_dev(C)
    b3.sgemm("N", "N", 0.0, to_dev(An), to_dev(An), 0.5, dC)
    assert bits_equal(to_host(dC), (f64(C) * 0.5).astype(np.float32))
    dC = to_dev(Cn)
    b3.sgemm("N", "N", 0.0, to_dev(An), to_dev(An), 0.0, dC)
    assert (to_host(dC) == 0).all()


@pytest.mark.parametrize("pad", [3, 2])
def test_sgemm_padded_ld(b3, oracle_mod, mode, route, pad):
    """ld > rows with NaN padding: padding must not leak into C and the
    padding rows of C must stay untouched (pad=3: ld = 153 / 81 breaks TMA's
    16-B rule -> SIMT route; pad=2: ld = 152 / 80 keeps the tcgen05 route)."""
    m, n, k = 150, 90, 78
    A = gen.uniform(m, k, "pd-a", ld=m + pad); B = gen.uniform(k, n, "pd-b", ld=k + pad)
    C = gen.uniform(m, n, "pd-c", ld=m + pad)
    dA, dB, dCf = to_dev(A), to_dev(B), to_dev(C)
    b3.sgemm("N", "N", AL, dA[:m], dB[:k], BE, dCf[:m])
    route(m + pad, k + pad, m + pad)
    full = to_host(dCf)
    ref = oracle_mod.sgemm("N", "N", AL, A[:m], B[:k], BE, C[:m])
    assert e_nw(full[:m], ref, AL * fro(A[:m]) * fro(B[:k]) + BE * fro(C[:m])) <= TOL_NW
    assert np.isnan(full[m:]).all()


@pytest.mark.parametrize("big_on", ["A", "B"])
@pytest.mark.parametrize("ta,tb", list(itertools.product("NT", "NT")))
def test_split_is_real(b3, oracle_mod, route, mode, big_on, ta, tb):
    """Decisive pin for the 3xTF32 split: one operand holds 15-bit integers
    (|x| < 2^14, needs hi + lo: TF32 keeps 11 significant bits), the other
    3-bit integers (lo = 0).  Then hi*hi + lo*hi (+ hi*lo = 0) is the exact
    product, every partial sum is an integer < 2^24, so the result must be
    bit-exact -- a 1xTF32 (or a dropped lo term) cannot be."""
    m, n, k = 260, 132, 64
    big = lambda *s: gen.integers(*s, "big", lo=-(2 ** 14) + 1, hi=2 ** 14 - 1)  # noqa: E731
    small = lambda *s: gen.integers(*s, "small", lo=-4, hi=4)                    # noqa: E731
    shpA = (m, k) if ta == "N" else (k, m)
    shpB = (k, n) if tb == "N" else (n, k)
    A = big(*shpA) if big_on == "A" else small(*shpA)
    B = big(*shpB) if big_on == "B" else small(*shpB)
    C = np.zeros((m, n), np.float32, order="F")
    dC = to_dev(C)
    b3.sgemm(ta, tb, 1.0, to_dev(A), to_dev(B), 0.0, dC)
    got = to_host(dC)
    route(A.shape[0], B.shape[0], m)
    assert bits_equal(got, oracle_mod.sgemm(ta, tb, 1.0, A, B, 0.0, C).astype(np.float32))


def test_determinism(b3):
    m = n = k = 384
    A, B, C = gen.uniform(m, k, "d-a"), gen.uniform(k, n, "d-b"), gen.uniform(m, n, "d-c")
    outs = []
    for _ in range(2):
        dC = to_dev(C)
        b3.sgemm("N", "T", AL, to_dev(A), to_dev(B), BE, dC)
        outs.append(to_host(dC))
    assert bits_equal(outs[0], outs[1])


# ------------------------------------------------------------------------------------ SSYMM
@pytest.mark.parametrize("side,uplo", list(itertools.product("LR", "LU")))
@pytest.mark.parametrize("m,n", [(1, 1), (44, 68), (200, 132), (256, 300), (516, 260)])
@pytest.mark.parametrize("gm_map", [-1, 0])
def test_ssymm(b3, oracle_mod, mode, route, side, uplo, m, n, gm_map):
    """gm_map=-1: the default policy (below order 4096: sym(A) materialised,
    then the GEMM); gm_map=0: mirrored while staging, the route from 4096."""
    ka = m if side == "L" else n
    A = gen.symmetric_stored(ka, uplo, "ps", side)        # other triangle = NaN sentinel
    B, C = gen.uniform(m, n, "ps-b"), gen.uniform(m, n, "ps-c")
    dC = to_dev(C)
    with b3.options(gm_map=gm_map):
        b3.ssymm(side, uplo, AL, to_dev(A), to_dev(B), BE, dC)
    got = to_host(dC)
    route(ka, m)
    ref = oracle_mod.ssymm(side, uplo, AL, A, B, BE, C)
    S = sym_full(A, uplo, ka)
    assert e_nw(got, ref, AL * fro(S) * fro(B) + BE * fro(C)) <= TOL_NW
    f32 = f32_eval(AL, S, B, BE, C) if side == "L" else f32_eval(AL, B, S, BE, C)
    assert e_rel(got, ref) <= rel_bound(f32, ref)


@pytest.mark.parametrize("side,uplo", list(itertools.product("LR", "LU")))
@pytest.mark.parametrize("gm_map", [-1, 0])
def test_ssymm_integer_bitexact_and_equals_gemm(b3, oracle_mod, mode, side, uplo, gm_map):
    m, n = 300, 172
    ka = m if side == "L" else n
    A = gen.symmetric_stored(ka, uplo, "is", integer=True)
    B, C = gen.integers(m, n, "is-b"), gen.integers(m, n, "is-c")
    dC = to_dev(C)
    with b3.options(gm_map=gm_map):
        b3.ssymm(side, uplo, AL, to_dev(A), to_dev(B), BE, dC)
    got = to_host(dC)
    assert bits_equal(got, oracle_mod.ssymm(side, uplo, AL, A, B, BE, C).astype(np.float32))
    # SYMM == GEMM on the explicitly symmetrised A (north-star identity)
    S = np.asfortranarray(sym_full(A, uplo, ka).astype(np.float32))
    dG = to_dev(C)
    if side == "L":
        b3.sgemm("N", "N", AL, to_dev(S), to_dev(B), BE, dG)
    else:
        b3.sgemm("N", "N", AL, to_dev(B), to_dev(S), BE, dG)
    assert bits_equal(got, to_host(dG))


# ------------------------------------------------------------------------------------ SYRK / SYR2K
@pytest.mark.parametrize("two", [False, True])
@pytest.mark.parametrize("uplo,trans", list(itertools.product("LU", "NT")))
@pytest.mark.parametrize("n,k", [(1, 1), (68, 32), (300, 200), (260, 520)])
def test_syrk_syr2k(b3, oracle_mod, mode, route, two, uplo, trans, n, k):
    shp = (n, k) if trans == "N" else (k, n)
    A, B = gen.uniform(*shp, "pk-a"), gen.uniform(*shp, "pk-b")
    C = gen.uniform(n, n, "pk-c")
    mask = np.tril(np.ones((n, n), bool)) if uplo == "L" else np.triu(np.ones((n, n), bool))
    C[~mask] = np.nan                                  # the other triangle: never read, never written
    dC = to_dev(C)
    if two:
        b3.ssyr2k(uplo, trans, AL, to_dev(A), to_dev(B), BE, dC)
        ref = oracle_mod.ssyr2k(uplo, trans, AL, A, B, BE, C)
        scale = AL * fro(A) * fro(B) + BE * fro(C[mask])
    else:
        b3.ssyrk(uplo, trans, AL, to_dev(A), BE, dC)
        ref = oracle_mod.ssyrk(uplo, trans, AL, A, BE, C)
        scale = AL * fro(A) ** 2 + BE * fro(C[mask])
    got = to_host(dC)
    route(A.shape[0], n)
    assert e_nw(got[mask], ref[mask], scale) <= TOL_NW
    oA, oB = op(A, trans), op(B, trans)             # n x k
    f32 = syr2k_f32(AL, oA, oB, BE, C) if two else f32_eval(AL, oA, oA.T, BE, np.nan_to_num(C))
    assert e_rel(got[mask], ref[mask]) <= rel_bound(f32[mask], ref[mask])
    assert bits_equal(got[~mask], C[~mask])


@pytest.mark.parametrize("uplo,trans", list(itertools.product("LU", "NT")))
@pytest.mark.parametrize("n,k", [(292, 152), (520, 1000)])
def test_syrk_integer_bitexact(b3, oracle_mod, mode, uplo, trans, n, k):
    """Integer inputs: every product and partial sum is exact in fp32, so the
    uplo triangle must equal the fp64 oracle bit for bit (one correct answer,
    Q18) and the other triangle must be untouched."""
    shp = (n, k) if trans == "N" else (k, n)
    A, C = gen.integers(*shp, "ik-a"), gen.integers(n, n, "ik-c")
    mask = np.tril(np.ones((n, n), bool)) if uplo == "L" else np.triu(np.ones((n, n), bool))
    dC = to_dev(C)
    b3.ssyrk(uplo, trans, AL, to_dev(A), BE, dC)
    got = to_host(dC)
    ref = oracle_mod.ssyrk(uplo, trans, AL, A, BE, C).astype(np.float32)
    assert bits_equal(got[mask], ref[mask])
    assert bits_equal(got[~mask], C[~mask])


@pytest.mark.parametrize("uplo,trans", list(itertools.product("LU", "NT")))
@pytest.mark.parametrize("n,k", [(292, 152), (520, 1000)])
def test_syr2k_integer_bitexact_and_two_gemms(b3, oracle_mod, mode, uplo, trans, n, k):
    shp = (n, k) if trans == "N" else (k, n)
    A, B, C = gen.integers(*shp, "i2-a"), gen.integers(*shp, "i2-b"), gen.integers(n, n, "i2-c")
    mask = np.tril(np.ones((n, n), bool)) if uplo == "L" else np.triu(np.ones((n, n), bool))
    dC = to_dev(C)
    b3.ssyr2k(uplo, trans, AL, to_dev(A), to_dev(B), BE, dC)
    got = to_host(dC)
    # the fp64 oracle, bit for bit (integer data: one correct answer)
    ref = oracle_mod.ssyr2k(uplo, trans, AL, A, B, BE, C).astype(np.float32)
    assert bits_equal(got[mask], ref[mask])
    assert bits_equal(got[~mask], C[~mask])
    # north-star identity SYR2K == two GEMMs, also through the oracle
    ta, tb = ("N", "T") if trans == "N" else ("T", "N")
    g1 = oracle_mod.sgemm(ta, tb, AL, A, B, BE, C)
    g2 = oracle_mod.sgemm(ta, tb, AL, B, A, 1.0, np.asfortranarray(g1.astype(np.float32)))
    assert bits_equal(got[mask], g2.astype(np.float32)[mask])


# ------------------------------------------------------------------------------------ STRMM
V16 = list(itertools.product("LR", "LU", "NT", "NU"))


@pytest.mark.parametrize("side,uplo,ta,diag", V16)
@pytest.mark.parametrize("m,n", [(1, 1), (68, 44), (260, 300), (516, 132)])
def test_strmm(b3, oracle_mod, mode, route, side, uplo, ta, diag, m, n):
    ka = m if side == "L" else n
    A = gen.triangular_dd(ka, uplo, diag, "pt")          # NaN blank triangle (+ NaN unit diagonal)
    B = gen.uniform(m, n, "pt-b")
    dB = to_dev(B)
    b3.strmm(side, uplo, ta, diag, AL, to_dev(A), dB)
    got = to_host(dB)
    route(ka, m)
    ref = oracle_mod.strmm(side, uplo, ta, diag, AL, A, B)
    T = tri_full(A, uplo, diag, ka)
    assert e_nw(got, ref, AL * fro(T) * fro(B)) <= TOL_NW
    oT = op(T, ta)
    assert e_rel(got, ref) <= rel_bound(f32_eval(AL, oT, B) if side == "L" else f32_eval(AL, B, oT), ref)


@pytest.mark.parametrize("side,uplo,ta,diag", V16)
def test_strmm_integer_bitexact(b3, oracle_mod, mode, side, uplo, ta, diag):
    m, n = 292, 200
    ka = m if side == "L" else n
    A = gen.triangular_integer(ka, uplo, diag, "it")
    B = gen.integers(m, n, "it-b")
    dB = to_dev(B)
    b3.strmm(side, uplo, ta, diag, AL, to_dev(A), dB)
    assert bits_equal(to_host(dB), oracle_mod.strmm(side, uplo, ta, diag, AL, A, B).astype(np.float32))


# ------------------------------------------------------------------------------------ STRSM
def trsm_metrics(got, A, B, side, uplo, ta, diag, alpha, oracle_mod):
    ka = A.shape[1]
    T = op(tri_full(A, uplo, diag, ka), ta)
    X = f64(got)
    R = (T @ X if side == "L" else X @ T) - alpha * f64(B)
    resid = fro(R) / (fro(T) * fro(X))
    ref = oracle_mod.strsm(side, uplo, ta, diag, alpha, A, B)
    return resid, e_rel(X, ref)


@pytest.mark.parametrize("side,uplo,ta,diag", V16)
@pytest.mark.parametrize("m,n", [(1, 1), (68, 44), (300, 260), (1100, 64)])
def test_strsm(b3, oracle_mod, mode, route, side, uplo, ta, diag, m, n):
    if side == "R":
        m, n = n, m            # keep the triangular order large for side=R too
    ka = m if side == "L" else n
    A = gen.triangular_dd(ka, uplo, diag, "px")
    B = gen.uniform(m, n, "px-b")
    dB = to_dev(B)
    b3.strsm(side, uplo, ta, diag, AL, to_dev(A), dB)
    route(ka, m)
    resid, fwd = trsm_metrics(to_host(dB), A, B, side, uplo, ta, diag, AL, oracle_mod)
    assert resid <= 1e-5 * np.sqrt(ka)
    assert fwd <= 1e-5


@pytest.mark.parametrize("side,uplo,ta", list(itertools.product("LR", "LU", "NT")))
def test_strsm_integer_exact_solution(b3, mode, side, uplo, ta):
    """A unit bidiagonal with +-1 off-diagonal, X integer, B = op(A) X exactly:
    the blocked inverse-based solve must return X bit for bit."""
    ka, other = 400, 70
    g = gen.rng("bidiag", side, uplo, ta)
    Tm = np.eye(ka)
    sub = g.choice([-1.0, 1.0], size=ka - 1)
    if uplo == "L":
        Tm[np.arange(1, ka), np.arange(ka - 1)] = sub
    else:
        Tm[np.arange(ka - 1), np.arange(1, ka)] = sub
    A = np.asfortranarray(Tm.astype(np.float32))
    gen.nan_outside(A, uplo, keep_diag=False)           # unit diagonal is never read
    X = gen.integers(*((ka, other) if side == "L" else (other, ka)), "bidiag-x")
    opT = op(Tm, ta)
    Bx = (opT @ f64(X)) if side == "L" else (f64(X) @ opT)
    B = np.asfortranarray(Bx.astype(np.float32))
    dB = to_dev(B)
    b3.strsm(side, uplo, ta, "U", 1.0, to_dev(A), dB)
    assert bits_equal(to_host(dB), X)


def test_strsm_after_strmm_returns_b(b3):
    m, n = 600, 300
    A = gen.triangular_dd(m, "U", "N", "rt")
    B = gen.uniform(m, n, "rt-b")
    dA, dB = to_dev(A), to_dev(B)
    b3.strmm("L", "U", "T", "N", 1.0, dA, dB)
    b3.strsm("L", "U", "T", "N", 1.0, dA, dB)
    assert e_rel(to_host(dB), B) <= 1e-5


def test_tr_alpha_zero(b3):
    m, n = 50, 40
    An = np.full((m, m), np.nan, np.float32, order="F")
    B = gen.uniform(m, n, "a0")
    for f in (b3.strmm, b3.strsm):
        dB = to_dev(B)
        f("L", "L", "N", "N", 0.0, to_dev(An), dB)
        assert (to_host(dB) == 0).all()
