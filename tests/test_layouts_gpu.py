"""Leading dimensions and base pointers of the structured routines (SURVEY §4
"ABI unit tests"): every operand is a view into a larger NaN-filled buffer,
with padding rows (ld > rows) and optionally a one-row offset of the view's
start.  ld % 4 == 0 with an aligned base keeps TMA's 16-byte rules -> the
tcgen05 route; ld % 4 == 1, or a view starting one float into the buffer,
breaks them -> the SIMT route for the offending operands' problems.  Either way the result must
match the fp64 oracle, NaN padding must not leak into the result, and every
padding row / untouched element of the output buffer must stay bit-identical.
"""
import numpy as np
import pytest

import blas3_inputs as gen
from check import TOL_NW, e_nw, f64, fro, op, sym_full, to_dev, to_host, tri_full

pytestmark = pytest.mark.gpu
AL, BE = 1.5, 0.5
CASES = [("tma_ok", 0), ("ld_odd", 0), ("base_misaligned", 1)]   # (kind, row offset of the view)
IDS = [c[0] for c in CASES]


def ld_for(rows, kind, off):
    """ld % 4 == 0 with >= 4 padding rows, except kind 'ld_odd' (ld % 4 == 1)."""
    ld = -(-(off + rows) // 4) * 4 + 4
    return ld + 1 if kind == "ld_odd" else ld


@pytest.fixture(scope="module", params=["3xtf32", "tf32_bf16x"])
def b3(request):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_cuiwxyf11_b200 as m
    m.set_math_mode(request.param)
    yield m
    m.set_math_mode("3xtf32")


def embed(X, kind, off, tag):
    """X (rows x cols) inside a NaN buffer (ld from ld_for), starting at row off."""
    rows, cols = X.shape
    buf = np.full((cols, ld_for(rows, kind, off)), np.nan, np.float32).T   # F-order (ld x cols)
    buf[off:off + rows, :] = X
    return buf


def run(b3, fn, bufs, off, rows):
    """Device copies of the buffers, views starting at row `off`, call, host result buffers."""
    devs = [to_dev(b) for b in bufs]
    views = [d[off:off + r] for d, r in zip(devs, rows)]
    tc0 = b3.launch_count("tc")
    fn(*views)
    return [to_host(d) for d in devs], b3.launch_count("tc") > tc0


def check_pad(full, orig, off, rows):
    """rows outside [off, off + rows) of the output buffer untouched (bitwise)."""
    keep = np.ones(full.shape[0], bool)
    keep[off:off + rows] = False
    a, b = full[keep], orig[keep]
    assert np.array_equal(np.isnan(a), np.isnan(b))
    assert np.array_equal(np.nan_to_num(a), np.nan_to_num(b))


@pytest.mark.parametrize("kind,off", CASES, ids=IDS)
@pytest.mark.parametrize("side,uplo", [("L", "L"), ("R", "U")])
def test_ssymm_layouts(b3, oracle_mod, kind, off, side, uplo):
    m, n = 150, 97
    ka = m if side == "L" else n
    S = gen.symmetric_stored(ka, uplo, "lay-s")
    B, C = gen.uniform(m, n, "lay-b"), gen.uniform(m, n, "lay-c")
    bufs = [embed(S, kind, off, "s"), embed(B, kind, off, "b"), embed(C, kind, off, "c")]
    (_, _, Cf), tc = run(b3, lambda s, b, c: b3.ssymm(side, uplo, AL, s, b, BE, c), bufs, off, [ka, m, m])
    ref = oracle_mod.ssymm(side, uplo, AL, S, B, BE, C)
    got = Cf[off:off + m]
    Sf = sym_full(S, uplo, ka)
    assert e_nw(got, ref, AL * fro(Sf) * fro(B) + BE * fro(C)) <= TOL_NW
    check_pad(Cf, bufs[2], off, m)
    assert tc == (kind == "tma_ok")


@pytest.mark.parametrize("kind,off", CASES, ids=IDS)
@pytest.mark.parametrize("two", [False, True], ids=["syrk", "syr2k"])
def test_syrk_syr2k_layouts(b3, oracle_mod, kind, off, two):
    n, k = 133, 70
    A, B = gen.uniform(n, k, "lay-a"), gen.uniform(n, k, "lay-b2")
    C = gen.uniform(n, n, "lay-c2")
    bufs = [embed(A, kind, off, "a"), embed(B, kind, off, "b"), embed(C, kind, off, "c")]
    if two:
        fn = lambda a, b, c: b3.ssyr2k("L", "N", AL, a, b, BE, c)
        ref = oracle_mod.ssyr2k("L", "N", AL, A, B, BE, C)
        scale = 2 * AL * fro(A) * fro(B) + BE * fro(C)
    else:
        fn = lambda a, b, c: b3.ssyrk("L", "N", AL, a, BE, c)
        ref = oracle_mod.ssyrk("L", "N", AL, A, BE, C)
        scale = AL * fro(A) ** 2 + BE * fro(C)
    (_, _, Cf), tc = run(b3, fn, bufs, off, [n, n, n])
    got = Cf[off:off + n]
    low = np.tril(np.ones((n, n), bool))
    assert e_nw(np.where(low, got, 0), np.where(low, ref, 0), scale) <= TOL_NW
    assert np.array_equal(got[~low], C[~low])                         # upper triangle untouched
    check_pad(Cf, bufs[2], off, n)
    assert tc == (kind == "tma_ok")


@pytest.mark.parametrize("kind,off", CASES, ids=IDS)
@pytest.mark.parametrize("routine", ["strmm", "strsm"])
@pytest.mark.parametrize("side,uplo,ta,diag", [("L", "L", "N", "N"), ("R", "U", "T", "U")])
def test_trmm_trsm_layouts(b3, oracle_mod, kind, off, routine, side, uplo, ta, diag):
    m, n = 141, 90
    ka = m if side == "L" else n
    T = gen.triangular_dd(ka, uplo, diag, "lay-t")
    B = gen.uniform(m, n, "lay-b3")
    bufs = [embed(T, kind, off, "t"), embed(B, kind, off, "b")]
    fn = getattr(b3, routine)
    (_, Bf), tc = run(b3, lambda t, b: fn(side, uplo, ta, diag, AL, t, b), bufs, off, [ka, m])
    got = f64(Bf[off:off + m])
    Top = op(tri_full(T, uplo, diag, ka), ta)
    if routine == "strmm":
        ref = oracle_mod.strmm(side, uplo, ta, diag, AL, T, B)
        assert e_nw(got, ref, AL * fro(Top) * fro(B)) <= TOL_NW
    else:
        resid = (Top @ got if side == "L" else got @ Top) - AL * f64(B)
        assert fro(resid) / (fro(Top) * fro(got)) <= 1e-5 * np.sqrt(ka)
        ref = oracle_mod.strsm(side, uplo, ta, diag, AL, T, B)
        assert fro(got - ref) / fro(ref) <= 1e-5
    check_pad(Bf, bufs[1], off, m)
    if kind == "tma_ok":
        assert tc
