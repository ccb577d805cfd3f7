"""Multi-GPU sharding logic on CPU (-m "not gpu"): the planner, and the
collectives on a world_size-2 gloo group (127.0.0.1).  The per-rank local
products here are computed by the TEST with numpy on the broadcast data, to
check the slab index math; the product path (dist.py executor) always runs
the CUDA library and is checked on the GPU in test_dist_gpu.py."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_cuiwxyf11_b200 import dist as d3


# ------------------------------------------------------------------ planner
@pytest.mark.parametrize("n,world", [(8192, 1), (8192, 2), (8192, 8), (1000, 3), (7, 4), (0, 2)])
def test_slab_partition_covers_once(n, world):
    cols = []
    for r in range(world):
        c0, c1 = d3.slab(n, world, r)
        assert c0 == c1 or (c0 % 4 == 0 and (c1 % 4 == 0 or c1 == n))
        cols.extend(range(c0, c1))
    assert cols == list(range(n))
    sizes = [d3.slab(n, world, r)[1] - d3.slab(n, world, r)[0] for r in range(world)]
    assert max(sizes) - min(sizes) <= 4 or n < 4 * world


@pytest.mark.parametrize("n,world", [(8192, 2), (8192, 8), (1000, 4)])
@pytest.mark.parametrize("lower", [True, False])
def test_balanced_triangle_slabs(n, world, lower):
    seen = []
    areas = []
    for r in range(world):
        sl = d3.balanced_tri_slabs(n, world, r)
        for c0, c1 in sl:
            seen.extend(range(c0, c1))
        areas.append(sum(d3.tri_area(n, c0, c1, lower) for c0, c1 in sl))
    assert sorted(seen) == list(range(n))
    assert sum(areas) == n * (n + 1) // 2
    assert max(areas) / min(areas) < (1.001 if n % (8 * world) == 0 else 1.05)   # balanced


@pytest.mark.parametrize("k,panels", [(8192, 8), (1000, 8), (100, 8), (32, 8), (4097, 3)])
def test_uniform_panels(k, panels):
    """The streamed GEMM maps k-block -> panel by division: one width, a
    multiple of 32, the last panel ragged, every column once."""
    pan = d3.uniform_panels(k, panels)
    w = pan[0][1] - pan[0][0]
    assert w % 32 == 0 and all(b - a == w for a, b in pan[:-1]) and 0 < pan[-1][1] - pan[-1][0] <= w
    assert [c for a, b in pan for c in range(a, b)] == list(range(k))
    assert len(pan) <= panels


def test_k_panels():
    assert d3.k_panels(8192, 8) == [(i * 1024, (i + 1) * 1024) for i in range(8)]
    p = d3.k_panels(100, 8)
    assert p[0][0] == 0 and p[-1][1] == 100 and all(b - a > 0 for a, b in p)


# ------------------------------------------------------------------ panel plans (pure)
def _sym(A, lower):
    T = np.tril(A) if lower else np.triu(A)
    return T + (np.tril(T, -1).T if lower else np.triu(T, 1).T)


def _run_symm_plan(A, B, C, alpha, beta, lower, panels):
    """Execute symm_plan's op list with numpy (fp64), reading ONLY the stored
    triangle's trapezoids of A, as the executor does with the library."""
    n = A.shape[0]
    pan, ops = d3.symm_plan(n, panels, lower)
    stored = np.tril(A) if lower else np.triu(A)           # what the broadcast delivers
    out = C.copy()
    for op in ops:
        be = beta if op[-1] else 1.0
        if op[0] == "symm":
            _, p0, p1, _ = op
            out[p0:p1] = alpha * _sym(stored[p0:p1, p0:p1], lower) @ B[p0:p1] + be * out[p0:p1]
        elif op[1] == "N":
            _, _, r0, r1, q0, q1, _ = op
            out[r0:r1] = alpha * stored[r0:r1, q0:q1] @ B[q0:q1] + be * out[r0:r1]
        else:
            _, _, q0, q1, r0, r1, _ = op
            out[q0:q1] = alpha * stored[r0:r1, q0:q1].T @ B[r0:r1] + be * out[q0:q1]
    return pan, out


@pytest.mark.parametrize("n,panels", [(256, 4), (1000, 8), (96, 1), (130, 3)])
@pytest.mark.parametrize("lower", [True, False])
def test_symm_plan_reproduces_symm(n, panels, lower):
    g = np.random.default_rng(7)
    A, B, C = g.uniform(-1, 1, (n, n)), g.uniform(-1, 1, (n, 40)), g.uniform(-1, 1, (n, 40))
    pan, out = _run_symm_plan(A, B, C, 1.5, 0.5, lower, panels)
    ref = 1.5 * _sym(A, lower) @ B + 0.5 * C
    assert np.allclose(out, ref, rtol=1e-12, atol=1e-12)
    # panels tile the order exactly once, in broadcast order
    assert [c for a, b in pan for c in range(a, b)] == list(range(n))


@pytest.mark.parametrize("n,panels", [(256, 4), (1000, 8), (96, 1), (130, 3)])
@pytest.mark.parametrize("lower", [True, False])
def test_trsm_plan_reproduces_solve(n, panels, lower):
    g = np.random.default_rng(11)
    A = g.uniform(-1, 1, (n, n)) / n + np.eye(n) * 2.0
    stored = np.tril(A) if lower else np.triu(A)
    B = g.uniform(-1, 1, (n, 30))
    pan, ops = d3.trsm_plan(n, panels, lower)
    X = B.copy()
    for op in ops:
        a1 = 1.5 if op[-1] else 1.0
        if op[0] == "trsm":
            _, p0, p1, _ = op
            X[p0:p1] = np.linalg.solve(stored[p0:p1, p0:p1], a1 * X[p0:p1])
        else:
            _, r0, r1, q0, q1, _ = op
            X[r0:r1] = a1 * X[r0:r1] - stored[r0:r1, q0:q1] @ X[q0:q1]
    assert np.allclose(X, np.linalg.solve(stored, 1.5 * B), rtol=1e-10, atol=1e-12)
    # processing order: forward for lower, backward for upper
    starts = [a for a, _ in pan]
    assert starts == sorted(starts, reverse=not lower)
    # every panel only needs its own trapezoid (rows of the stored triangle)
    for op in ops:
        if op[0] == "upd":
            _, r0, r1, q0, q1, _ = op
            t0, t1 = d3.trapezoid_rows(n, q0, q1, lower)
            assert t0 <= r0 and r1 <= t1


# ------------------------------------------------------------------ gloo, world 2
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _colmajor(arr):
    return torch.from_numpy(np.ascontiguousarray(arr.T)).t()      # (m, n) view, strides (1, m)


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import blas3_inputs as gen
        n, k = 96, 64
        A_np = gen.uniform(n, k, "dist-A")
        A = _colmajor(A_np) if rank == 0 else _colmajor(np.zeros((n, k), np.float32))
        seen = []
        d3.broadcast_panels(A, root=0, panels=3, on_panel=lambda c0, c1: seen.append((c0, c1)))
        ok_bcast = np.array_equal(A.numpy(), A_np) and seen == d3.k_panels(k, 3, 1)
        # padded-ld panel broadcast
        P_np = gen.uniform(n, k, "dist-P", ld=n + 3)
        full = torch.from_numpy(np.ascontiguousarray(P_np.T)).t() if rank == 0 else \
            torch.zeros((k, n + 3)).t()
        d3.broadcast_panels(full[:n], root=0, panels=2)
        ok_pad = np.array_equal(full[:n].numpy(), P_np[:n])
        # column-slab SGEMM composition (numpy stand-in for the local product)
        Bf = gen.uniform(k, 40, "dist-B"); Cf = gen.uniform(n, 40, "dist-C")
        c0, c1 = d3.slab(40, world, rank)
        part = 1.5 * A.numpy().astype(np.float64) @ Bf[:, c0:c1] + 0.5 * Cf[:, c0:c1]
        parts = [None] * world
        dist.all_gather_object(parts, (c0, c1, part))
        ok_slab = True
        if rank == 0:
            ref = 1.5 * A_np.astype(np.float64) @ Bf + 0.5 * Cf
            got = np.zeros_like(ref)
            for a, b, p in parts:
                got[:, a:b] = p
            ok_slab = np.array_equal(got, ref)
        # k-split SYRK reduction: sum of per-rank partial A_r A_r^T == A A^T
        k0, k1 = d3.slab(k, world, rank)
        Cp = torch.from_numpy(A_np[:, k0:k1].astype(np.float64) @ A_np[:, k0:k1].T.astype(np.float64))
        d3.syrk_k_split(Cp)
        ok_red = np.allclose(Cp.numpy(), A_np.astype(np.float64) @ A_np.T.astype(np.float64),
                             rtol=1e-12, atol=1e-12)
        # trapezoid (triangle-only) broadcast: the receiver gets the stored
        # triangle; of the other triangle only the panels' diagonal blocks travel
        nt = 128
        T_np = gen.uniform(nt, nt, "dist-T")
        ok_tri = True
        for lower in (True, False):
            Tt = _colmajor(T_np) if rank == 0 else _colmajor(np.full((nt, nt), -7.0, np.float32))
            sent = np.zeros((nt, nt), bool)
            for p0, p1 in d3.k_panels(nt, 4):
                d3.broadcast_trapezoid(Tt, p0, p1, lower, root=0)
                r0, r1 = d3.trapezoid_rows(nt, p0, p1, lower)
                sent[r0:r1, p0:p1] = True
            got = Tt.numpy()
            keep = np.tril(np.ones((nt, nt), bool)) if lower else np.triu(np.ones((nt, nt), bool))
            ok_tri &= bool(keep[~sent].sum() == 0)               # the whole stored triangle travels
            ok_tri &= np.array_equal(got[sent], T_np[sent])
            if rank == 1:
                ok_tri &= bool((got[~sent] == -7.0).all())
            ok_tri &= sent.sum() < 0.7 * nt * nt                 # about half the matrix
        q.put((rank, ok_bcast, ok_pad, ok_slab, ok_red, ok_tri))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_broadcast_slabs_reduce():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    for rank, *oks in res:
        assert all(oks), (rank, oks)
