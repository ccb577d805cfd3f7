"""Multi-GPU sharding of the six routines (row E1 of the hot-path table).

Every routine acts independently on each column of its right-hand side
(side='L'; each row for side='R'), so the path shards by COLUMN SLABS of B/C
with A replicated (BASELINE.json north star; the paper leaves multi-GPU as
future work).  The one exchange step is a broadcast of A from the root
over NCCL / NVLink.  No reduction and no gather: outputs stay sharded.

SYRK/SYR2K have no right-hand side; their C is split into column slabs of the
referenced triangle, and slab j is paired with slab 2P-1-j so every rank owns
the same triangle area (balanced), with A replicated.  (`syrk_k_split` is the
alternative for a k-distributed A: partial products + one all-reduce.)

Three layers:
  * planner   -- pure functions (`slab`, `balanced_tri_slabs`, `k_panels`),
                 no torch, no CUDA; unit-tested on CPU;
  * comms     -- `broadcast_panels` (torch.distributed; NCCL on GPUs, gloo on
                 CPU in tests), `syrk_k_split` reduction;
  * executor  -- `sgemm`, `ssymm`, `ssyrk`, `ssyr2k`, `strmm`, `strsm` on the
                 rank's slab; local work is ALWAYS the CUDA library
                 (paper_conf_ipps_cuiwxyf11_b200), never a CPU path.

SGEMM with transa='N' overlaps the broadcast with compute: A is sent in
column panels on a side stream and the compute stream consumes panel p
(K-range p of the product) as soon as it has landed; beta applies to the
first panel only.
"""
from __future__ import annotations

from typing import List, Tuple


# =============================================================== planner
def slab(n: int, world: int, rank: int, align: int = 4) -> Tuple[int, int]:
    """[c0, c1) columns of an n-column matrix owned by `rank` (contiguous,
    sizes differ by at most `align`; boundaries multiples of `align` so every
    slab keeps 16-byte TMA alignment when ld % 4 == 0)."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    units = -(-n // align)
    base, extra = divmod(units, world)
    u0 = rank * base + min(rank, extra)
    u1 = u0 + base + (1 if rank < extra else 0)
    return min(n, u0 * align), min(n, u1 * align)


def balanced_tri_slabs(n: int, world: int, rank: int, align: int = 4) -> List[Tuple[int, int]]:
    """Column slabs of an n x n triangle owned by `rank`: the triangle is cut
    into 2*world slabs and slab j is paired with slab 2*world-1-j, so each
    rank's share of triangle area is nearly equal."""
    parts = [slab(n, 2 * world, j, align) for j in range(2 * world)]
    return [p for p in (parts[rank], parts[2 * world - 1 - rank]) if p[1] > p[0]]


def tri_area(n: int, c0: int, c1: int, lower: bool = True) -> int:
    """Number of referenced entries of columns [c0, c1) of an n x n triangle."""
    return sum((n - j) if lower else (j + 1) for j in range(c0, c1))


def k_panels(k: int, panels: int, align: int = 32) -> List[Tuple[int, int]]:
    """K-range panels for the pipelined broadcast (multiples of the k-block)."""
    panels = max(1, min(panels, -(-k // align)))
    return [p for p in (slab(k, panels, i, align) for i in range(panels)) if p[1] > p[0]]


# =============================================================== comms
def _dist():
    import torch.distributed as dist
    return dist


def world_rank(group=None):
    dist = _dist()
    if not dist.is_available() or not dist.is_initialized():
        return 1, 0
    return dist.get_world_size(group), dist.get_rank(group)


def broadcast_panels(A, root: int = 0, group=None, panels: int = 1, on_panel=None):
    """Broadcast the columns of A (a column-major tensor view) from `root` in
    `panels` column panels; `on_panel(c0, c1)` is called after each panel has
    arrived (on every rank) so the caller can consume it.  With NCCL the
    broadcasts are enqueued on the current stream; the pipelined SGEMM below
    puts them on a side stream instead."""
    dist = _dist()
    world, _ = world_rank(group)
    n = A.shape[1]
    for c0, c1 in k_panels(n, panels, 1):
        if world > 1:
            _bcast(A[:, c0:c1], root, group)
        if on_panel is not None:
            on_panel(c0, c1)


def _bcast(view, root, group):
    """Broadcast a column-major panel in place (NCCL/gloo need a contiguous
    tensor: a column-major panel with ld == rows is contiguous as its
    transpose; a padded-ld panel is packed, sent and unpacked)."""
    dist = _dist()
    if view.is_contiguous():
        dist.broadcast(view, root, group=group)
    elif view.t().is_contiguous():
        dist.broadcast(view.t(), root, group=group)
    else:
        buf = view.t().contiguous()
        dist.broadcast(buf, root, group=group)
        view.t().copy_(buf)


def syrk_k_split(C_partial, group=None):
    """Sum the per-rank partial products of a k-distributed SYRK/SYR2K."""
    dist = _dist()
    if world_rank(group)[0] > 1:
        dist.all_reduce(C_partial, op=dist.ReduceOp.SUM, group=group)
    return C_partial


# =============================================================== executor
def _b3():
    import paper_conf_ipps_cuiwxyf11_b200 as b3     # CUDA library; raises if missing
    return b3


def sgemm(transa, transb, alpha, A, B_slab, beta, C_slab, root=0, group=None, panels=8,
          pipeline=None):
    """C_slab <- alpha*op(A)*op(B)_slab + beta*C_slab on this rank's columns.

    A is replicated from `root` (NCCL broadcast).  For transa='N' the
    broadcast is pipelined in K panels on a side stream, overlapped with the
    panel GEMMs on the compute stream (`pipeline` defaults to world > 1)."""
    import torch
    b3 = _b3()
    world, _ = world_rank(group)
    if pipeline is None:
        pipeline = world > 1
    if not pipeline or transa.upper() != "N" or transb.upper() != "N" or panels <= 1:
        broadcast_panels(A, root, group, 1)
        b3.sgemm(transa, transb, alpha, A, B_slab, beta, C_slab)
        return
    compute = torch.cuda.current_stream()
    comm = torch.cuda.Stream()
    comm.wait_stream(compute)
    k = A.shape[1]
    first = True
    for c0, c1 in k_panels(k, panels):
        with torch.cuda.stream(comm):
            if world > 1:
                _bcast(A[:, c0:c1], root, group)
            ev = torch.cuda.Event()
            ev.record(comm)
        compute.wait_event(ev)
        b3.sgemm("N", "N", alpha, A[:, c0:c1], B_slab[c0:c1], beta if first else 1.0, C_slab)
        first = False


def ssymm(side, uplo, alpha, A, B_slab, beta, C_slab, root=0, group=None):
    """side='L': C_slab <- alpha*A*B_slab + beta*C_slab (column slabs);
    side='R': row slabs (C_slab, B_slab are row blocks of C, B)."""
    broadcast_panels(A, root, group, 1)
    _b3().ssymm(side, uplo, alpha, A, B_slab, beta, C_slab)


def strmm(side, uplo, transa, diag, alpha, A, B_slab, root=0, group=None):
    broadcast_panels(A, root, group, 1)
    _b3().strmm(side, uplo, transa, diag, alpha, A, B_slab)


def strsm(side, uplo, transa, diag, alpha, A, B_slab, root=0, group=None):
    broadcast_panels(A, root, group, 1)
    _b3().strsm(side, uplo, transa, diag, alpha, A, B_slab)


def _tri_slab_products(two, uplo, trans, alpha, A, B, beta, C, slabs):
    """C columns [c0, c1) of the uplo triangle: the diagonal block through
    SSYRK/SSYR2K, the rest of the column slab through SGEMM(s)."""
    b3 = _b3()
    n = C.shape[0]
    lower = uplo.upper() == "L"
    tN = trans.upper() == "N"
    rows = (lambda X, r0, r1: X[r0:r1]) if tN else (lambda X, r0, r1: X[:, r0:r1])
    ta, tb = ("N", "T") if tN else ("T", "N")
    for c0, c1 in slabs:
        Cd = C[c0:c1, c0:c1]
        if two:
            b3.ssyr2k(uplo, trans, alpha, rows(A, c0, c1), rows(B, c0, c1), beta, Cd)
        else:
            b3.ssyrk(uplo, trans, alpha, rows(A, c0, c1), beta, Cd)
        r0, r1 = (c1, n) if lower else (0, c0)
        if r1 > r0:
            Co = C[r0:r1, c0:c1]
            if two:
                b3.sgemm(ta, tb, alpha, rows(A, r0, r1), rows(B, c0, c1), beta, Co)
                b3.sgemm(ta, tb, alpha, rows(B, r0, r1), rows(A, c0, c1), 1.0, Co)
            else:
                b3.sgemm(ta, tb, alpha, rows(A, r0, r1), rows(A, c0, c1), beta, Co)


def ssyrk(uplo, trans, alpha, A, beta, C, root=0, group=None):
    """Balanced column-slab sharding of C's uplo triangle, A replicated.
    C is the full n x n buffer on every rank; rank r writes only the columns
    of its two paired slabs (outputs stay sharded)."""
    broadcast_panels(A, root, group, 1)
    world, rank = world_rank(group)
    _tri_slab_products(False, uplo, trans, alpha, A, None, beta, C,
                       balanced_tri_slabs(C.shape[0], world, rank))


def ssyr2k(uplo, trans, alpha, A, B, beta, C, root=0, group=None):
    broadcast_panels(A, root, group, 1)
    broadcast_panels(B, root, group, 1)
    world, rank = world_rank(group)
    _tri_slab_products(True, uplo, trans, alpha, A, B, beta, C,
                       balanced_tri_slabs(C.shape[0], world, rank))
