"""Variant search (tune.py): the paper's generator measures several
optimisation scripts per routine and keeps the fastest; here
the candidates are C-ABI tuning options that all compute the same result.

CPU: the candidate grids are well formed and every candidate is accepted by
blas3_set_option (host-only); the options() context manager restores values.
GPU: tune_problem times every candidate through the C ABI, returns the fastest,
applies it only when asked, and the routine stays correct under the winner.
"""
import numpy as np
import pytest

import blas3_inputs as gen


@pytest.fixture(scope="module")
def b3():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_cuiwxyf11_b200 as m
    return m


def test_grid_is_the_cartesian_product(b3):
    from paper_conf_ipps_cuiwxyf11_b200 import tune
    g = tune.grid(a=[1, 2], b=[3, 4, 5])
    assert len(g) == 6
    assert {(d["a"], d["b"]) for d in g} == {(x, y) for x in (1, 2) for y in (3, 4, 5)}
    assert tune.grid() == [{}]


@pytest.mark.parametrize("routine", ["sgemm", "ssymm", "ssyrk", "ssyr2k", "strmm", "strsm"])
def test_default_candidates_are_valid_options(b3, routine):
    from paper_conf_ipps_cuiwxyf11_b200 import tune
    cands = tune.default_candidates(routine)
    assert len(cands) >= 2
    assert len({tuple(sorted(c.items())) for c in cands}) == len(cands)   # no duplicates
    before = {k: b3.get_option(k) for c in cands for k in c}
    for c in cands:
        with b3.options(**c):                   # raises ValueError on an invalid value
            for k, v in c.items():
                assert b3.get_option(k) == v
    assert {k: b3.get_option(k) for k in before} == before                # restored


@pytest.mark.gpu
@pytest.mark.parametrize("apply", [False, True])
def test_tune_problem_picks_a_candidate_and_stays_correct(b3, oracle_mod, apply):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ipps_cuiwxyf11_b200 import tune
    from check import TOL_NW, e_nw, f64, fro, to_dev, to_host
    b3.set_math_mode("3xtf32")
    n = 1024
    A, B, C = (gen.uniform(n, n, "tune", x) for x in "ABC")
    dA, dB, dC = to_dev(A), to_dev(B), to_dev(C)
    cands = tune.default_candidates("sgemm")
    before = {k: b3.get_option(k) for c in cands for k in c}
    try:
        best, table = tune.tune_problem("sgemm", ("N", "N", 1.5, dA, dB, 0.5, dC), apply=apply,
                                        reps=1, rounds=1)
        assert best in cands
        assert [c for c, _ in table] == cands and all(ms > 0 for _, ms in table)
        assert min(table, key=lambda t: t[1])[0] == best
        now = {k: b3.get_option(k) for k in before}
        assert now == ({**before, **best} if apply else before)
        dC = to_dev(C)                          # the tuning calls overwrote C
        b3.sgemm("N", "N", 1.5, dA, dB, 0.5, dC)
        got = f64(to_host(dC))
        ref = oracle_mod.sgemm("N", "N", 1.5, A, B, 0.5, C)
        assert e_nw(got, ref, 1.5 * fro(A) * fro(B) + 0.5 * fro(C)) <= TOL_NW
    finally:
        for k, v in before.items():
            b3.set_option(k, v)
