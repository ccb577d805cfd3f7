"""dist.py executor on one GPU: "virtual ranks" run every rank's slab in turn
on the same device (the broadcast of A is the identity at world size 1); the
assembled result must equal the single-call result bit for bit, since each
output column's arithmetic (k-blocks in order, same UMMA sequence) does not
depend on the slab it is computed in.  The pipelined K-panel SGEMM changes the
summation grouping (C is rounded between panels), so it is checked with the
north-star tolerance instead."""
import numpy as np
import pytest

import blas3_inputs as gen
from check import TOL_NW, e_nw, fro, to_dev, to_host

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def mods():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_cuiwxyf11_b200 as b3
    from paper_conf_ipps_cuiwxyf11_b200 import dist as d3
    b3.set_math_mode("3xtf32")
    return b3, d3


def bits(a):
    return np.ascontiguousarray(a, dtype=np.float32).view(np.uint32)


@pytest.mark.parametrize("world", [2, 3, 8])
def test_virtual_ranks_side_left(mods, world):
    b3, d3 = mods
    n, cols = 520, 1000
    A = gen.uniform(n, n, "vr-A"); S = gen.symmetric_stored(n, "L", "vr-S")
    T = gen.triangular_dd(n, "U", "N", "vr-T")
    B = gen.uniform(n, cols, "vr-B"); C = gen.uniform(n, cols, "vr-C")
    dA, dS, dT = to_dev(A), to_dev(S), to_dev(T)
    calls = {
        "sgemm": lambda Bv, Cv: d3.sgemm("N", "N", 1.5, dA, Bv, 0.5, Cv),
        "ssymm": lambda Bv, Cv: d3.ssymm("L", "L", 1.5, dS, Bv, 0.5, Cv),
        "strmm": lambda Bv, Cv: d3.strmm("L", "U", "T", "N", 1.5, dT, Cv),
        "strsm": lambda Bv, Cv: d3.strsm("L", "U", "N", "N", 1.5, dT, Cv),
    }
    for name, f in calls.items():
        init = C if name in ("sgemm", "ssymm") else B
        dB, dfull = to_dev(B), to_dev(init)
        f(dB, dfull)                                   # one call on all columns
        dsl = to_dev(init)
        for r in range(world):                         # every rank's slab in turn
            c0, c1 = d3.slab(cols, world, r)
            if c1 > c0:
                f(dB[:, c0:c1], dsl[:, c0:c1])
        assert np.array_equal(bits(to_host(dfull)), bits(to_host(dsl))), name


@pytest.mark.parametrize("two", [False, True])
@pytest.mark.parametrize("uplo,trans", [("L", "N"), ("U", "T")])
def test_virtual_ranks_syrk_balanced(mods, two, uplo, trans):
    b3, d3 = mods
    n, k, world = 1000, 300, 4
    shp = (n, k) if trans == "N" else (k, n)
    A, B, C = gen.uniform(*shp, "vs-A"), gen.uniform(*shp, "vs-B"), gen.uniform(n, n, "vs-C")
    dA, dB = to_dev(A), to_dev(B)
    dfull = to_dev(C)
    if two:
        b3.ssyr2k(uplo, trans, 1.5, dA, dB, 0.5, dfull)
    else:
        b3.ssyrk(uplo, trans, 1.5, dA, 0.5, dfull)
    dsl = to_dev(C)
    for r in range(world):
        d3._tri_slab_products(two, uplo, trans, 1.5, dA, dB if two else None, 0.5, dsl,
                              d3.balanced_tri_slabs(n, world, r))
    full, sl = to_host(dfull), to_host(dsl)
    if two:
        # off-diagonal slabs = two SGEMMs (C rounded in between): same product,
        # different rounding grouping -> compare with the north-star tolerance
        mask = np.tril(np.ones((n, n), bool)) if uplo == "L" else np.triu(np.ones((n, n), bool))
        scale = 1.5 * fro(A) * fro(B) + 0.5 * fro(C[mask])
        assert e_nw(sl[mask], full[mask].astype(np.float64), scale) <= TOL_NW
        assert np.array_equal(bits(sl[~mask]), bits(full[~mask]))
    else:
        assert np.array_equal(bits(full), bits(sl))


def test_pipelined_sgemm_panels(mods, oracle_mod):
    b3, d3 = mods
    m, n, k = 512, 768, 4096
    A, B, C = gen.uniform(m, k, "pp-A"), gen.uniform(k, n, "pp-B"), gen.uniform(m, n, "pp-C")
    dC = to_dev(C)
    d3.sgemm("N", "N", 1.5, to_dev(A), to_dev(B), 0.5, dC, panels=8, pipeline=True)
    ref = oracle_mod.sgemm("N", "N", 1.5, A, B, 0.5, C)
    assert e_nw(to_host(dC), ref, 1.5 * fro(A) * fro(B) + 0.5 * fro(C)) <= TOL_NW


@pytest.mark.parametrize("uplo", ["L", "U"])
def test_pipelined_ssymm_trapezoid_panels(mods, oracle_mod, uplo):
    """SSYMM as consumed from trapezoid panels (dist.symm_plan: diagonal block
    by SSYMM, the off-diagonal rectangle by an NN and a TN SGEMM) with the
    SM reservation of the overlapped broadcast: the north-star tolerance and
    the fp32-class diagnostic against the fp64 oracle."""
    from check import e_rel, rel_bound, sym_f32, f32_eval
    b3, d3 = mods
    n, cols = 1000, 520
    A = gen.symmetric_stored(n, uplo, "pt-S")
    B, C = gen.uniform(n, cols, "pt-B"), gen.uniform(n, cols, "pt-C")
    dC = to_dev(C)
    d3.ssymm("L", uplo, 1.5, to_dev(A), to_dev(B), 0.5, dC, panels=4, pipeline=True)
    got = to_host(dC)
    ref = oracle_mod.ssymm("L", uplo, 1.5, A, B, 0.5, C)
    S = sym_f32(A, uplo)
    assert e_nw(got, ref, 1.5 * fro(S) * fro(B) + 0.5 * fro(C)) <= TOL_NW
    assert e_rel(got, ref) <= rel_bound(f32_eval(1.5, S, B, 0.5, C), ref)


@pytest.mark.parametrize("uplo", ["L", "U"])
def test_pipelined_strsm_trapezoid_panels(mods, oracle_mod, uplo):
    """STRSM as the right-looking sweep over trapezoid panels (dist.trsm_plan)."""
    from check import f64, e_rel
    b3, d3 = mods
    n, cols = 1100, 300
    A = gen.triangular_dd(n, uplo, "N", "pt-T")
    B = gen.uniform(n, cols, "pt-X")
    dX = to_dev(B)
    d3.strsm("L", uplo, "N", "N", 1.5, to_dev(A), dX, panels=4, pipeline=True)
    X = f64(to_host(dX))
    T = np.nan_to_num(f64(A))
    T = np.tril(T) if uplo == "L" else np.triu(T)
    assert fro(T @ X - 1.5 * f64(B)) / (fro(T) * fro(X)) <= 1e-5 * np.sqrt(n)
    assert e_rel(X, oracle_mod.strsm("L", uplo, "N", "N", 1.5, A, B)) <= 1e-5


def test_max_sms_option_same_result(mods):
    """BLAS3_OPT_MAX_SMS (SMs left to NCCL) changes only the grid size (tile
    shape and k-splitting pinned, so every tile's arithmetic is the same)."""
    b3, d3 = mods
    m, n, k = 1536, 1024, 1024
    A, B, C = gen.uniform(m, k, "ms-A"), gen.uniform(k, n, "ms-B"), gen.uniform(m, n, "ms-C")
    outs = []
    for cap in (0, 132, 20):
        dC = to_dev(C)
        with b3.options(max_sms=cap, tc_cta=2, tc_split=0):
            b3.sgemm("N", "N", 1.5, to_dev(A), to_dev(B), 0.5, dC)
        outs.append(bits(to_host(dC)))
    assert np.array_equal(outs[0], outs[1]) and np.array_equal(outs[0], outs[2])
