"""STRSM sweep structure (rows A7/A8): several diagonal panels, the side-stream
doubling of all but the first processed panel, and the per-slab sweeps on
their own streams.

* in process, at the default panel width (2048): ragged orders > 2048 with
  >= 4096 right-hand sides (two slabs, a ragged last slab and panel), every
  side/uplo/trans/diag variant, residual and forward error on sampled
  columns (side=L) / rows (side=R) against the fp64 oracle;
* in a subprocess with a 256-wide panel, up to 4 slabs and a 256-wide slab
  minimum (env knobs read once per process), the whole small-size STRSM
  parity suite -- many panels, forward and backward orders, several slabs --
  once on the fused single-launch path and once on the multi-launch path.
"""
import itertools
import os
import subprocess
import sys

import numpy as np
import pytest

import blas3_inputs as gen
from check import f64, fro, op, to_dev, to_host, tri_full

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
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


@pytest.mark.parametrize("split", [0, 512, 1024, "all"], ids=["chain", "first_split512", "first_split1024",
                                                              "first_all"])
@pytest.mark.parametrize("side,uplo,ta,diag", V16)
def test_strsm_multi_panel_multi_slab(b3, oracle_mod, side, uplo, ta, diag, split):
    """split=1: BLAS3_OPT_TRSM_FIRST_SPLIT (first panel's second half by a bulk
    update + one leaf instead of the chain)."""
    ka, other = 2600, 4500                 # 2 panels (ragged), 2 slabs (ragged last)
    m, n = (ka, other) if side == "L" else (other, ka)
    A = gen.triangular_dd(ka, uplo, diag, "sweep-a")
    B = gen.uniform(m, n, "sweep-b")
    dB = to_dev(B)
    opts = dict(trsm_first_all=1) if split == "all" else dict(trsm_first_split=split)
    opts["trsm_slab_min"] = 2048          # two RHS slabs at 4500 (the default minimum is 4096)
    with b3.options(**opts):
        b3.strsm(side, uplo, ta, diag, AL, to_dev(A), dB)
    X = f64(to_host(dB))
    T = op(tri_full(A, uplo, diag, ka), ta)
    # samples straddle the slab boundary (2048 + 256 k) and the ragged tail
    sel = np.unique(np.concatenate([gen.sample_indices(other, 20, "sweep-sel"),
                                    [0, 2047, 2048, 2303, 2304, other - 1]]))
    if side == "L":
        Xs, Bs = X[:, sel], f64(B[:, sel])
        resid = fro(T @ Xs - AL * Bs) / (fro(T) * fro(Xs))
    else:
        Xs, Bs = X[sel, :], f64(B[sel, :])
        resid = fro(Xs @ T - AL * Bs) / (fro(T) * fro(Xs))
    assert resid <= 1e-5 * np.sqrt(ka)
    ref = oracle_mod.strsm(side, uplo, ta, diag, AL, A, B, sel=sel)
    assert fro(Xs - ref) / fro(ref) <= 1e-5


@pytest.mark.parametrize("side", ["L", "R"])
def test_strsm_fused_is_one_launch(b3, oracle_mod, side):
    """BLAS3_OPT_TRSM_FUSED=1: the doubling and the sweep are ONE persistent
    tcgen05 launch after the 128-block inverses; the multi-launch path (the
    default, option 0) gives the same answer to rounding."""
    ka, other = 2600, 4500
    m, n = (ka, other) if side == "L" else (other, ka)
    A = gen.triangular_dd(ka, "L", "N", "fuse-a")
    B = gen.uniform(m, n, "fuse-b")
    dA = to_dev(A)
    dB = to_dev(B)
    with b3.options(trsm_fused=1):
        tc0, all0 = b3.launch_count("tc"), b3.launch_count()
        b3.strsm(side, "L", "N", "N", AL, dA, dB)
        X1 = f64(to_host(dB))
        assert b3.launch_count("tc") - tc0 == 1 and b3.launch_count() - all0 == 2
    with b3.options(trsm_fused=0):
        dB2 = to_dev(B)
        b3.strsm(side, "L", "N", "N", AL, dA, dB2)
        X0 = f64(to_host(dB2))
    assert fro(X1 - X0) / fro(X0) <= 1e-6


@pytest.mark.parametrize("nb,fused,split", [("256", "0", "0"), ("256", "1", "0"), ("1024", "0", "512"),
                                            ("8192", "0", "512")],
                         ids=["multi_launch", "fused", "nb1024_first_split", "one_panel_first_split"])
def test_strsm_small_panels_many_slabs(nb, fused, split):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    env = {**os.environ, "BLAS3_TRSM_NB": nb, "BLAS3_TRSM_SLABS": "4", "BLAS3_TRSM_SLAB_MIN": "256",
           "BLAS3_TRSM_FUSED": fused, "BLAS3_TRSM_FIRST_SPLIT": split}
    cmd = [sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", "-k", "strsm",
           os.path.join(ROOT, "tests", "test_parity_gpu.py")]
    r = subprocess.run(cmd, env=env, cwd=ROOT, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
    assert " passed" in r.stdout


@pytest.mark.parametrize("side,uplo,ta", [("L", "L", "N"), ("R", "U", "T"), ("L", "U", "T")])
def test_strsm_multi_panel_tf32_bf16x(b3, oracle_mod, side, uplo, ta):
    """The TF32+BF16X mode on the multi-panel path, whose fused first-panel
    launch then runs the BX kernel instantiation too."""
    ka, other = 2600, 4500
    m, n = (ka, other) if side == "L" else (other, ka)
    A = gen.triangular_dd(ka, uplo, "N", "bx-a")
    B = gen.uniform(m, n, "bx-b")
    dB = to_dev(B)
    b3.set_math_mode("tf32_bf16x")
    try:
        b3.strsm(side, uplo, ta, "N", AL, to_dev(A), dB)
    finally:
        b3.set_math_mode("3xtf32")
    X = f64(to_host(dB))
    T = op(tri_full(A, uplo, "N", ka), ta)
    sel = gen.sample_indices(other, 16, "bx-sel")
    Xs, Bs = (X[:, sel], f64(B[:, sel])) if side == "L" else (X[sel, :], f64(B[sel, :]))
    resid = (T @ Xs - AL * Bs) if side == "L" else (Xs @ T - AL * Bs)
    assert fro(resid) / (fro(T) * fro(Xs)) <= 1e-5 * np.sqrt(ka)
    ref = oracle_mod.strsm(side, uplo, ta, "N", AL, A, B, sel=sel)
    assert fro(Xs - ref) / fro(ref) <= 1e-5
