"""GPU parity of the fp64 family (blas3_d*) against the
fp64 oracle, through the C ABI.

The oracle (oracle/oracle.c) takes fp32 inputs and accumulates in fp64. On
fp32-representable inputs every product is exact in fp64 (24 + 24 bits), so
the oracle and the DFMA kernels both compute the exact BLAS result up to
fp64 summation rounding, K * 2^-53 relative at most. The tolerance below is
4 * K * 2^-53 on the normwise error, which is ~1e-13 at these sizes and eight
orders of magnitude below what a dropped term, a wrong mirror or a wrong
triangle would give. Integer-valued inputs have an exact, unique fp64
result: it must be reproduced bit for bit. The unreferenced triangle of A
and, for SYRK/SYR2K, of C hold NaN sentinels (never read, never written).
Sizes span several 128 x 128 tiles with ragged tails.
"""
import itertools

import numpy as np
import pytest

import blas3_inputs as gen
from check import f64, fro, op, sym_full, to_host, tri_full

pytestmark = pytest.mark.gpu

AL, BE = 1.5, 0.5
U53 = 2.0 ** -53


@pytest.fixture(scope="module")
def b3():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_cuiwxyf11_b200 as m
    return m


def dev(b3, X):
    return b3.from_fortran(f64(X), f64=True)


def tol(k):
    return 4.0 * max(k, 1) * U53


def enw(got, ref, scale):
    return fro(f64(got) - f64(ref)) / max(scale, 1e-300)


def launched_fp64(b3, before):
    """the DFMA kernels ran (SIMT path counter; the tcgen05 path never)."""
    return b3.launch_count("simt") > before["simt"] and b3.launch_count("tc") == before["tc"]


def counts(b3):
    return {p: b3.launch_count(p) for p in ("tc", "simt")}


@pytest.mark.parametrize("ta,tb", list(itertools.product("NT", "NT")))
@pytest.mark.parametrize("m,n,k", [(1, 1, 1), (33, 17, 45), (200, 131, 77), (300, 260, 520)])
def test_dgemm(b3, oracle_mod, ta, tb, m, n, k):
    A = gen.uniform(*((m, k) if ta == "N" else (k, m)), "dg-a", ta)
    B = gen.uniform(*((k, n) if tb == "N" else (n, k)), "dg-b", tb)
    C = gen.uniform(m, n, "dg-c")
    dC = dev(b3, C)
    before = counts(b3)
    b3.dgemm(ta, tb, AL, dev(b3, A), dev(b3, B), BE, dC)
    got = to_host(dC)
    assert launched_fp64(b3, before)
    ref = oracle_mod.sgemm(ta, tb, AL, A, B, BE, C)
    assert enw(got, ref, AL * fro(A) * fro(B) + BE * fro(C)) <= tol(k)


@pytest.mark.parametrize("side,uplo", list(itertools.product("LR", "LU")))
@pytest.mark.parametrize("m,n", [(70, 45), (200, 131), (129, 300)])
def test_dsymm(b3, oracle_mod, side, uplo, m, n):
    ka = m if side == "L" else n
    A = gen.symmetric_stored(ka, uplo, "ds-a", side)       # NaN outside the stored triangle
    B = gen.uniform(m, n, "ds-b")
    C = gen.uniform(m, n, "ds-c")
    dC = dev(b3, C)
    b3.dsymm(side, uplo, AL, dev(b3, A), dev(b3, B), BE, dC)
    got = to_host(dC)
    ref = oracle_mod.ssymm(side, uplo, AL, A, B, BE, C)
    S = sym_full(A, uplo, ka)
    assert enw(got, ref, AL * fro(S) * fro(B) + BE * fro(C)) <= tol(ka)


@pytest.mark.parametrize("two", [False, True])
@pytest.mark.parametrize("uplo,trans", list(itertools.product("LU", "NT")))
@pytest.mark.parametrize("n,k", [(70, 33), (200, 131), (257, 64)])
def test_dsyrk_dsyr2k(b3, oracle_mod, two, uplo, trans, n, k):
    A = gen.uniform(*((n, k) if trans == "N" else (k, n)), "dk-a", trans)
    B = gen.uniform(*((n, k) if trans == "N" else (k, n)), "dk-b", trans)
    C = gen.nan_outside(gen.uniform(n, n, "dk-c"), uplo)   # the other triangle: NaN, untouched
    dC = dev(b3, C)
    if two:
        b3.dsyr2k(uplo, trans, AL, dev(b3, A), dev(b3, B), BE, dC)
        ref = oracle_mod.ssyr2k(uplo, trans, AL, A, B, BE, C)
        scale = 2 * AL * fro(A) * fro(B)
    else:
        b3.dsyrk(uplo, trans, AL, dev(b3, A), BE, dC)
        ref = oracle_mod.ssyrk(uplo, trans, AL, A, BE, C)
        scale = AL * fro(A) ** 2
    got = to_host(dC)
    mask = np.tril(np.ones((n, n), bool)) if uplo == "L" else np.triu(np.ones((n, n), bool))
    assert np.isnan(got[~mask]).all(), "the opposite triangle was written"
    Cm = np.where(mask, np.nan_to_num(f64(C)), 0.0)
    assert enw(np.where(mask, got, 0.0), np.where(mask, ref, 0.0), scale + BE * fro(Cm)) <= tol(2 * k)


V16 = list(itertools.product("LR", "LU", "NT", "NU"))


@pytest.mark.parametrize("side,uplo,ta,diag", V16)
def test_dtrmm(b3, oracle_mod, side, uplo, ta, diag):
    m, n = (200, 131) if side == "L" else (131, 200)
    ka = m if side == "L" else n
    A = gen.nan_outside(gen.uniform(ka, ka, "dt-a", side, uplo), uplo, keep_diag=diag == "N")
    B = gen.uniform(m, n, "dt-b")
    dB = dev(b3, B)
    b3.dtrmm(side, uplo, ta, diag, AL, dev(b3, A), dB)
    got = to_host(dB)
    ref = oracle_mod.strmm(side, uplo, ta, diag, AL, A, B)
    T = tri_full(A, uplo, diag, ka)
    assert enw(got, ref, AL * fro(T) * fro(B)) <= tol(ka)


@pytest.mark.parametrize("side,uplo,ta,diag", V16)
@pytest.mark.parametrize("order,rhs", [(200, 131), (64, 65), (331, 40), (1100, 37)])
def test_dtrsm(b3, oracle_mod, side, uplo, ta, diag, order, rhs):
    """Diagonally dominant A (cond ~ 1): forward error vs the oracle and the
    residual, both at fp64 level. Orders up to 512 are one panel launch
    (331 = five 64-blocks + a ragged one); 1100 recurses (576 + 524 -> panels
    of 512, 64 and a ragged 524 split again), with the GEMM updates between."""
    m, n = (order, rhs) if side == "L" else (rhs, order)
    A = gen.triangular_dd(order, uplo, diag, "dr-a")
    B = gen.uniform(m, n, "dr-b")
    dB = dev(b3, B)
    b3.dtrsm(side, uplo, ta, diag, AL, dev(b3, A), dB)
    X = f64(to_host(dB))
    ref = oracle_mod.strsm(side, uplo, ta, diag, AL, A, B)
    assert fro(X - ref) / fro(ref) <= 64 * order * U53
    T = op(tri_full(A, uplo, diag, order), ta)
    R = (T @ X if side == "L" else X @ T) - AL * f64(B)
    assert fro(R) / (fro(T) * fro(X)) <= 64 * order * U53


# ------------------------------------------------------------------ bit-exact on integers
def test_integer_inputs_bit_exact(b3, oracle_mod):
    """Small integers: every product and partial sum is an exact fp64 integer,
    so the result is unique -- equal to the oracle's bit for bit."""
    m, n, k = 150, 97, 70
    A = gen.integers(m, k, "di-a")
    B = gen.integers(k, n, "di-b")
    C = gen.integers(m, n, "di-c")
    dC = dev(b3, C)
    b3.dgemm("N", "N", 2.0, dev(b3, A), dev(b3, B), 3.0, dC)
    assert np.array_equal(to_host(dC), oracle_mod.sgemm("N", "N", 2.0, A, B, 3.0, C))
    S = gen.symmetric_stored(m, "U", "di-s", integer=True)
    Bs = gen.integers(m, n, "di-bs")
    dC = dev(b3, C)
    b3.dsymm("L", "U", 2.0, dev(b3, S), dev(b3, Bs), 3.0, dC)
    assert np.array_equal(to_host(dC), oracle_mod.ssymm("L", "U", 2.0, S, Bs, 3.0, C))
    Cs = gen.nan_outside(gen.integers(m, m, "di-cs"), "L")
    dC = dev(b3, Cs)
    b3.dsyr2k("L", "T", 2.0, dev(b3, gen.integers(k, m, "di-k1")), dev(b3, gen.integers(k, m, "di-k2")), 3.0, dC)
    ref = oracle_mod.ssyr2k("L", "T", 2.0, gen.integers(k, m, "di-k1"), gen.integers(k, m, "di-k2"), 3.0, Cs)
    got = to_host(dC)
    low = np.tril(np.ones((m, m), bool))
    assert np.array_equal(got[low], ref[low])
    T = gen.triangular_integer(m, "L", "U", "di-t")
    dB = dev(b3, Bs)
    b3.dtrmm("L", "L", "T", "U", 2.0, dev(b3, T), dB)
    assert np.array_equal(to_host(dB), oracle_mod.strmm("L", "L", "T", "U", 2.0, T, Bs))


# ------------------------------------------------------------------ special cases and errors
def test_special_cases(b3):
    import torch
    C = b3.colmajor(50, 40, dtype=torch.float64)
    C.fill_(float("nan"))
    A = b3.colmajor(50, 30, dtype=torch.float64)
    A.fill_(float("nan"))
    B = b3.colmajor(30, 40, dtype=torch.float64)
    B.fill_(1.0)
    b3.dgemm("N", "N", 0.0, A, B, 0.0, C)         # alpha = 0: A, B not read; beta = 0: C not read
    assert torch.all(C == 0)
    Bt = b3.colmajor(50, 40, dtype=torch.float64)
    Bt.fill_(float("nan"))
    T = b3.colmajor(50, 50, dtype=torch.float64)
    T.fill_(float("nan"))
    b3.dtrsm("L", "L", "N", "N", 0.0, T, Bt)       # alpha = 0: B <- 0, A not read
    assert torch.all(Bt == 0)
    rc = b3.blas3_dgemm(b"X", b"N", 1, 1, 1, 1.0, 0, 1, 0, 1, 0.0, 0, 1, 0)
    assert rc == 1
    rc = b3.blas3_dtrsm(b"L", b"L", b"N", b"N", 10, 5, 1.0, 0, 9, 0, 10, 0)
    assert rc == 9
    with pytest.raises(TypeError):
        b3.dgemm("N", "N", 1.0, b3.colmajor(4, 4), b3.colmajor(4, 4), 0.0, b3.colmajor(4, 4))


def test_large_dgemm_and_dtrsm_sampled(b3, oracle_mod):
    """N = 2048: 16 x 32 tiles, K = 2048; and a 2048-order DTRSM (five levels
    of the recursive split), both checked on sampled oracle columns."""
    import torch
    n = 2048
    A = gen.uniform(n, n, "dl-a")
    B = gen.uniform(n, n, "dl-b")
    C = gen.uniform(n, n, "dl-c")
    sel = gen.sample_indices(n, 24, "dl-s")
    dC = dev(b3, C)
    b3.dgemm("T", "N", AL, dev(b3, A), dev(b3, B), BE, dC)
    torch.cuda.synchronize()
    got = to_host(dC)[:, sel]
    ref = oracle_mod.sgemm("T", "N", AL, A, B, BE, C, sel=sel)
    assert enw(got, ref, AL * fro(A) * fro(B[:, sel]) + BE * fro(C[:, sel])) <= tol(n)
    T = gen.triangular_dd(n, "U", "N", "dl-t")
    dB = dev(b3, B)
    b3.dtrsm("L", "U", "N", "N", AL, dev(b3, T), dB)
    X = f64(to_host(dB))[:, sel]
    ref = oracle_mod.strsm("L", "U", "N", "N", AL, T, B, sel=sel)
    assert fro(X - ref) / fro(ref) <= 64 * n * U53


@pytest.mark.parametrize("routine", ["dgemm", "dsyrk", "dtrmm", "dtrsm"])
def test_padded_ld_untouched(b3, oracle_mod, routine):
    """Outputs inside larger NaN-filled allocations with odd leading dimensions
    (ld = rows + 5): only the m x n block changes, the padding rows and the
    columns beyond n keep their NaN sentinels, and the block is correct
    (a bounds check in place of a memory checker)."""
    import torch
    m, n, k = 150, 97, 70
    ld = m + 5
    full = torch.full((n + 2, ld), float("nan"), dtype=torch.float64, device="cuda")
    view = full[:n].t()[:m]                          # m x n, column-major, ld = m + 5
    if routine == "dtrsm" or routine == "dtrmm":
        T = gen.triangular_dd(m, "L", "N", "pad-t")
        B = gen.uniform(m, n, "pad-b")
        view.copy_(torch.from_numpy(f64(B)))
        getattr(b3, routine)("L", "L", "N", "N", AL, dev(b3, T), view)
        ref = getattr(oracle_mod, "s" + routine[1:])("L", "L", "N", "N", AL, T, B)
        tolr = 64 * m * U53
    elif routine == "dgemm":
        A = gen.uniform(m, k, "pad-a"); B = gen.uniform(k, n, "pad-b2"); C = gen.uniform(m, n, "pad-c")
        view.copy_(torch.from_numpy(f64(C)))
        b3.dgemm("N", "N", AL, dev(b3, A), dev(b3, B), BE, view)
        ref = oracle_mod.sgemm("N", "N", AL, A, B, BE, C)
        tolr = tol(k) * 10
    else:                                            # dsyrk on an n x n block
        n = m
        full = torch.full((n + 2, ld), float("nan"), dtype=torch.float64, device="cuda")
        view = full[:n].t()[:m]
        A = gen.uniform(m, k, "pad-k"); C = gen.nan_outside(gen.uniform(m, m, "pad-kc"), "U")
        view.copy_(torch.from_numpy(f64(C)))
        b3.dsyrk("U", "N", AL, dev(b3, A), BE, view)
        ref = oracle_mod.ssyrk("U", "N", AL, A, BE, C)
        up = np.triu(np.ones((m, m), bool))
        got = view.cpu().numpy()
        assert fro(np.where(up, got, 0) - np.where(up, ref, 0)) / fro(np.where(up, ref, 0)) <= tol(k) * 10
        host = full.cpu().numpy()
        assert np.isnan(host[:n, m:]).all() and np.isnan(host[n:]).all()
        assert np.isnan(got[~up]).all()
        return
    got = view.cpu().numpy()
    assert fro(got - ref) / fro(ref) <= tolr
    host = full.cpu().numpy()
    assert np.isnan(host[:n, m:]).all(), "padding rows written"
    assert np.isnan(host[n:]).all(), "columns beyond n written"


@pytest.mark.parametrize("routine", ["dsymm", "dsyrk", "dsyr2k", "dtrmm", "dtrsm_R"])
def test_large_structured_sampled(b3, oracle_mod, routine):
    """N = 4096 (32 x 32 tiles of 128, the fp64 bench size) on sampled oracle
    columns (rows for side = R): the structured routines at scale, where every
    region class (real / shadow / blank / diagonal-crossing) occurs many times."""
    import torch
    n = 4096
    sel = gen.sample_indices(n, 12, "dL-s", routine)
    B = gen.uniform(n, n, "dL-b")
    C = gen.uniform(n, n, "dL-c")
    if routine == "dsymm":
        S = gen.symmetric_stored(n, "U", "dL-a")
        dC = dev(b3, C)
        b3.dsymm("L", "U", AL, dev(b3, S), dev(b3, B), BE, dC)
        torch.cuda.synchronize()
        got = to_host(dC)[:, sel]
        ref = oracle_mod.ssymm("L", "U", AL, S, B, BE, C, sel=sel)
        scale = AL * fro(sym_full(S, "U", n)) * fro(B[:, sel]) + BE * fro(C[:, sel])
        assert enw(got, ref, scale) <= tol(n)
    elif routine in ("dsyrk", "dsyr2k"):
        k = 512
        A = gen.uniform(n, k, "dL-ka"); A2 = gen.uniform(n, k, "dL-kb")
        Cl = gen.nan_outside(C, "L")
        dC = dev(b3, Cl)
        if routine == "dsyrk":
            b3.dsyrk("L", "N", AL, dev(b3, A), BE, dC)
            ref = oracle_mod.ssyrk("L", "N", AL, A, BE, Cl, sel=sel)
        else:
            b3.dsyr2k("L", "N", AL, dev(b3, A), dev(b3, A2), BE, dC)
            ref = oracle_mod.ssyr2k("L", "N", AL, A, A2, BE, Cl, sel=sel)
        torch.cuda.synchronize()
        got = to_host(dC)[:, sel]
        low = np.array([[i >= j for j in sel] for i in range(n)])
        assert np.isnan(got[~low]).all()
        d = np.where(low, np.nan_to_num(f64(got)) - np.nan_to_num(f64(ref)), 0.0)
        assert fro(d) / fro(np.where(low, np.nan_to_num(f64(ref)), 0.0)) <= tol(2 * k) * 10
    elif routine == "dtrmm":
        T = gen.nan_outside(gen.uniform(n, n, "dL-t"), "L", keep_diag=False)
        dB = dev(b3, B)
        b3.dtrmm("L", "L", "T", "U", AL, dev(b3, T), dB)
        torch.cuda.synchronize()
        got = to_host(dB)[:, sel]
        ref = oracle_mod.strmm("L", "L", "T", "U", AL, T, B, sel=sel)
        assert enw(got, ref, AL * fro(tri_full(T, "L", "U", n)) * fro(B[:, sel])) <= tol(n)
    else:                                            # DTRSM side = R, sampled rows
        T = gen.triangular_dd(n, "U", "N", "dL-tr")
        dB = dev(b3, B)
        b3.dtrsm("R", "U", "T", "N", AL, dev(b3, T), dB)
        torch.cuda.synchronize()
        X = f64(to_host(dB))[sel, :]
        ref = oracle_mod.strsm("R", "U", "T", "N", AL, T, B, sel=sel)
        assert fro(X - ref) / fro(ref) <= 64 * n * U53
