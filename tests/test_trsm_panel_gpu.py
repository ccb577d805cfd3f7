"""STRSM's diagonal-panel solver (csrc/panel_kernel.cu; DESIGN.md §7,
profiles/r02_strsm_panel.md) against the fp64 oracle.

BLAS3_OPT_TRSM_PANEL = 2 forces the solver at any right-hand-side count. By
default it is used only when its teams fill the machine, which at test sizes
would leave it unexercised. The cases below cover:
* every side/uplo/trans/diag variant, which means forward and backward panel
  order, both layouts of M, and X stored by rows or by columns;
* right-hand-side counts that are not multiples of the 256-wide team slab;
* panels of one block and of several blocks;
* several slabs per team (BLAS3_OPT_MAX_SMS shrinks the grid, so each team
  loops over slabs with the counters running on);
* the in-place contract: only B changes, and X is bit-identical to the same
  call with fewer SMs.
Metrics are test_parity_gpu.py's: residual <= 1e-5 sqrt(N) and forward error
<= 1e-5 (north star) on diagonally dominant A.
"""
import itertools

import numpy as np
import pytest

import blas3_inputs as gen
from check import f64, fro, op, to_dev, to_host, tri_full

pytestmark = pytest.mark.gpu

AL = 1.5
V16 = list(itertools.product("LR", "LU", "NT", "NU"))


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


def solve(b3, side, uplo, ta, diag, A, B, **opts):
    dB = to_dev(B)
    before = b3.launch_count("panel")
    with b3.options(trsm_panel=2, **opts):
        b3.strsm(side, uplo, ta, diag, AL, to_dev(A), dB)
    return to_host(dB), b3.launch_count("panel") - before


def check(oracle_mod, X, A, B, side, uplo, ta, diag):
    ka = A.shape[0]
    T = op(tri_full(A, uplo, diag, ka), ta)
    Xd = f64(X)
    R = (T @ Xd if side == "L" else Xd @ T) - AL * f64(B)
    assert fro(R) / (fro(T) * fro(Xd)) <= 1e-5 * np.sqrt(ka)
    ref = oracle_mod.strsm(side, uplo, ta, diag, AL, A, B)
    assert fro(Xd - ref) / fro(ref) <= 1e-5


@pytest.mark.parametrize("side,uplo,ta,diag", V16)
@pytest.mark.parametrize("order,rhs", [(1024, 300), (256, 520), (1536, 76)])
def test_panel_solver(b3, oracle_mod, side, uplo, ta, diag, order, rhs):
    """order: the triangle's order (one panel: 256, 1024 or 1536 = 1-6 blocks);
    rhs: right-hand sides (ragged against the 256-wide slab; ldb % 4 == 0 for
    side=R, where the right-hand sides are B's rows -- TMA needs it)."""
    m, n = (order, rhs) if side == "L" else (rhs, order)
    A = gen.triangular_dd(order, uplo, diag, "pn")
    B = gen.uniform(m, n, "pn-b")
    X, launched = solve(b3, side, uplo, ta, diag, A, B)
    assert launched == 1, "expected one diagonal-panel launch"
    check(oracle_mod, X, A, B, side, uplo, ta, diag)


@pytest.mark.parametrize("side,uplo,ta", [("L", "L", "N"), ("L", "U", "N"), ("R", "L", "T"), ("R", "U", "N")])
def test_panel_solver_multi_panel(b3, oracle_mod, side, uplo, ta):
    """order 4096 = two 2048 panels: the solver takes the first processed
    panel (forward or backward), the sweep the rest."""
    order, rhs = 4096, 600
    m, n = (order, rhs) if side == "L" else (rhs, order)
    A = gen.triangular_dd(order, uplo, "N", "pm")
    B = gen.uniform(m, n, "pm-b")
    X, launched = solve(b3, side, uplo, ta, "N", A, B)
    assert launched == 1
    check(oracle_mod, X, A, B, side, uplo, ta, "N")


@pytest.mark.parametrize("side", "LR")
def test_panel_solver_slab_loop_bitwise(b3, oracle_mod, side):
    """With 16 SMs a team covers several 256-wide slabs in turn. The
    per-slab arithmetic does not depend on the grid, so X must be
    bit-identical to the full-grid solve, and correct."""
    order, rhs = 1024, 2100
    m, n = (order, rhs) if side == "L" else (rhs, order)
    A = gen.triangular_dd(order, "L", "N", "ps")
    B = gen.uniform(m, n, "ps-b")
    X_full, l1 = solve(b3, side, "L", "N", "N", A, B)
    X_small, l2 = solve(b3, side, "L", "N", "N", A, B, max_sms=16)
    assert l1 == 1 and l2 == 1
    assert np.array_equal(X_full.view(np.uint32), X_small.view(np.uint32))
    check(oracle_mod, X_small, A, B, side, "L", "N", "N")


def test_panel_solver_leaves_outside_untouched(b3):
    """Only B's n columns change: a larger allocation's padding rows (ldb > m)
    and the columns beyond n keep their NaN sentinels."""
    import torch
    order, rhs, ldb = 512, 260, 520
    A = gen.triangular_dd(order, "L", "N", "pu")
    B = gen.uniform(order, rhs, "pu-b")
    full = torch.full((rhs + 3, ldb), float("nan"), device="cuda")
    full[:rhs, :order] = torch.from_numpy(np.ascontiguousarray(B.T)).cuda()
    dB = full[:rhs].t()[:order]                 # order x rhs view, column-major, ld = ldb
    with b3.options(trsm_panel=2):
        b3.strsm("L", "L", "N", "N", AL, to_dev(A), dB)
    host = full.cpu().numpy()
    assert np.isnan(host[:rhs, order:]).all()   # padding rows of each column
    assert np.isnan(host[rhs:]).all()           # columns beyond n
    assert np.isfinite(host[:rhs, :order]).all()


def test_panel_solver_concurrent_streams(b3):
    """Two solves on two streams at once, each with more teams than fit beside
    the other: the second grid's CTAs become resident as the first one's
    retire, a team's pairs are consecutive in launch order, and both results
    match the same solves run one after the other (bit for bit)."""
    import torch
    order, rhs = 2048, 8192
    A = gen.triangular_dd(order, "L", "N", "pc")
    Bs = [gen.uniform(order, rhs, f"pc-b{i}") for i in range(2)]
    dA = to_dev(A)
    seq = []
    for B in Bs:
        X, _ = solve(b3, "L", "L", "N", "N", A, B)
        seq.append(X)
    dX = [to_dev(B) for B in Bs]
    streams = [torch.cuda.Stream() for _ in range(2)]
    torch.cuda.synchronize()
    with b3.options(trsm_panel=2):
        for X, st in zip(dX, streams):
            with torch.cuda.stream(st):
                b3.strsm("L", "L", "N", "N", AL, dA, X)
    torch.cuda.synchronize()
    for X, ref in zip(dX, seq):
        assert np.array_equal(to_host(X).view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("side", "LR")
def test_panel_solver_extra_members_fold_bitwise(b3, oracle_mod, side):
    """8192 right-hand sides = 32 slabs: the full device gives each team two
    core pairs and spreads the ten leftover pairs over the teams as extra
    members (each helping three or four teams). A launch limited to 132 SMs
    cannot place them; the last core member then computes the extra's partial
    itself. The group split is the device's either way, so X is bit-identical."""
    order, rhs = 1024, 8192
    m, n = (order, rhs) if side == "L" else (rhs, order)
    A = gen.triangular_dd(order, "U", "N", "px")
    B = gen.uniform(m, n, "px-b")
    X_full, l1 = solve(b3, side, "U", "N", "N", A, B)
    X_lim, l2 = solve(b3, side, "U", "N", "N", A, B, max_sms=132)
    assert l1 == 1 and l2 == 1
    assert np.array_equal(X_full.view(np.uint32), X_lim.view(np.uint32))
    check(oracle_mod, X_full, A, B, side, "U", "N", "N")


@pytest.mark.parametrize("side,uplo,ta", [("L", "L", "N"), ("L", "U", "T"), ("R", "L", "N"), ("R", "U", "T")])
def test_panel_solver_second_panel(b3, oracle_mod, side, uplo, ta):
    """BLAS3_OPT_TRSM_PANEL2: order 6144 = three 2048 panels, forward or
    backward; the first two processed panels by the solver (two launches),
    the last by the doubling leaf, the update before the second in place."""
    order, rhs = 6144, 520
    m, n = (order, rhs) if side == "L" else (rhs, order)
    A = gen.triangular_dd(order, uplo, "N", "p2")
    B = gen.uniform(m, n, "p2-b")
    X, launched = solve(b3, side, uplo, ta, "N", A, B, trsm_panel2=1)
    assert launched == 2
    check(oracle_mod, X, A, B, side, uplo, ta, "N")
