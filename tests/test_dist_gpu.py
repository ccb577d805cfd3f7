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
