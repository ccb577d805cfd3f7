"""GPU parity of the k-sliced tail (wave quantisation, tc_kernel.cu plan_split).

When a launch has fewer tiles than producers, or its last wave is a small
remainder, those tiles are cut into up to 16 k-slices whose fp32 partials are
reduced by the last-arriving slice in slice order.  These shapes force deep
splits: a long K on very few tiles, a ragged tile grid, a slice range that
crosses the SYR2K segment boundary, TRI operands whose tiles have different
k-ranges, and C updated in place with beta != 0.  Same bars as
test_parity_gpu.py (normwise 1e-5 and the output-relative diagnostic),
integer inputs bit-exact, and the reduction order must be deterministic.
"""
import numpy as np
import pytest

import blas3_inputs as gen
from check import (TOL_NW, bits_equal, e_nw, e_rel, f32_eval, fro, op, rel_bound, syr2k_f32, to_dev,
                   to_host, tri_full)

pytestmark = pytest.mark.gpu
AL, BE = 1.5, 0.5


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


@pytest.mark.parametrize("ta,tb,m,n,k", [("N", "N", 256, 256, 4096), ("T", "N", 260, 300, 1000),
                                         ("N", "T", 128, 1000, 3000), ("T", "T", 1100, 132, 2052)])
def test_sgemm_split(b3, oracle_mod, ta, tb, m, n, k):
    A = gen.uniform(*((m, k) if ta == "N" else (k, m)), "st-a", ta)
    B = gen.uniform(*((k, n) if tb == "N" else (n, k)), "st-b", tb)
    C = gen.uniform(m, n, "st-c")
    dC = to_dev(C)
    before = b3.launch_count("tc")
    b3.sgemm(ta, tb, AL, to_dev(A), to_dev(B), BE, dC)
    assert b3.launch_count("tc") > before
    got = to_host(dC)
    ref = oracle_mod.sgemm(ta, tb, AL, A, B, BE, C)
    assert e_nw(got, ref, AL * fro(A) * fro(B) + BE * fro(C)) <= TOL_NW
    assert e_rel(got, ref) <= rel_bound(f32_eval(AL, op(A, ta), op(B, tb), BE, C), ref)


def test_sgemm_split_integer_bitexact_and_deterministic(b3, oracle_mod):
    m, n, k = 200, 300, 2500
    A, B, C = gen.integers(m, k, "si-a"), gen.integers(k, n, "si-b"), gen.integers(m, n, "si-c")
    outs = []
    for _ in range(2):
        dC = to_dev(C)
        b3.sgemm("N", "N", 1.0, to_dev(A), to_dev(B), 1.0, dC)
        outs.append(to_host(dC))
    assert bits_equal(outs[0], outs[1])
    ref = oracle_mod.sgemm("N", "N", 1.0, A, B, 1.0, C).astype(np.float32)
    assert bits_equal(outs[0], ref)


@pytest.mark.parametrize("uplo,trans", [("L", "N"), ("U", "T")])
def test_syr2k_split_across_segments(b3, oracle_mod, uplo, trans):
    n, k = 300, 1500
    shp = (n, k) if trans == "N" else (k, n)
    A, B = gen.uniform(*shp, "ss-a"), gen.uniform(*shp, "ss-b")
    C = gen.uniform(n, n, "ss-c")
    mask = np.tril(np.ones((n, n), bool)) if uplo == "L" else np.triu(np.ones((n, n), bool))
    C[~mask] = np.nan
    dC = to_dev(C)
    b3.ssyr2k(uplo, trans, AL, to_dev(A), to_dev(B), BE, dC)
    got = to_host(dC)
    ref = oracle_mod.ssyr2k(uplo, trans, AL, A, B, BE, C)
    scale = AL * fro(A) * fro(B) + BE * fro(C[mask])
    assert e_nw(got[mask], ref[mask], scale) <= TOL_NW
    f32 = syr2k_f32(AL, op(A, trans), op(B, trans), BE, C)
    assert e_rel(got[mask], ref[mask]) <= rel_bound(f32[mask], ref[mask])
    assert bits_equal(got[~mask], C[~mask])


@pytest.mark.parametrize("side,uplo,ta", [("L", "L", "N"), ("L", "U", "T"), ("R", "U", "N")])
def test_strmm_split(b3, oracle_mod, side, uplo, ta):
    m, n = (1500, 200) if side == "L" else (200, 1500)
    ka = m if side == "L" else n
    A = gen.triangular_dd(ka, uplo, "N", "sm")
    B = gen.uniform(m, n, "sm-b")
    dB = to_dev(B)
    b3.strmm(side, uplo, ta, "N", AL, to_dev(A), dB)
    got = to_host(dB)
    ref = oracle_mod.strmm(side, uplo, ta, "N", AL, A, B)
    T = tri_full(A, uplo, "N", ka)
    assert e_nw(got, ref, AL * fro(T) * fro(B)) <= TOL_NW
    oT = op(T, ta)
    assert e_rel(got, ref) <= rel_bound(f32_eval(AL, oT, B) if side == "L" else f32_eval(AL, B, oT), ref)
