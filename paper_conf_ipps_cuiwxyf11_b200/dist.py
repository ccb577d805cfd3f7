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

Pipelined broadcast: A travels in column panels on a side
(comm) stream while the compute stream consumes each panel as soon as it has
landed, so the exposed broadcast is about one panel.  For a structured A only
the stored triangle travels, one TRAPEZOID per column panel (columns [p0, p1),
rows [p0, n) of a lower / [0, p1) of an upper triangle), packed into a
contiguous staging buffer for NCCL: half the NVLink bytes.  The consumers:
  * SGEMM NN   -- panel p is the K-range p.  Default: ONE streamed GEMM whose
                  producer waits per k-block for its panel's flag (device-side
                  consumption, blas3_sgemm_streamed); alternative: one GEMM per
                  landed panel, C += alpha A[:, p] B[p, :];
  * SSYMM L    -- panel p contributes its diagonal block by SSYMM and its
                  off-diagonal rectangle R twice, C_below += R B_p (NN) and
                  C_p += R^T B_below (TN): sym(A) = sum of those (planner
                  `symm_plan`);
  * STRSM L, N -- the right-looking blocked solve in processing order: X_p by
                  the library's STRSM on the diagonal block, then one SGEMM
                  update of the rows after it (planner `trsm_plan`).
While panels are still in flight the local kernels leave `reserve_sms` SMs
free (BLAS3_OPT_MAX_SMS), so NCCL's kernels are never starved by the
persistent GEMM grid.  Every plan is a pure list of operations, unit-tested
on CPU by executing it with numpy against the unpartitioned product.
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


def uniform_panels(k: int, panels: int, align: int = 32) -> List[Tuple[int, int]]:
    """K-range panels of ONE width (a multiple of `align`; the last one
    ragged), as the streamed GEMM expects: panel p = k-block // width."""
    if k <= 0:
        return []
    w = -(-(-(-k // max(1, panels))) // align) * align
    return [(c0, min(k, c0 + w)) for c0 in range(0, k, w)]


def trapezoid_rows(n: int, p0: int, p1: int, lower: bool) -> Tuple[int, int]:
    """Rows of the stored triangle in columns [p0, p1) (diagonal block included)."""
    return (p0, n) if lower else (0, p1)


def symm_plan(n: int, panels: int, lower: bool, align: int = 32):
    """SSYMM side='L' as column panels of the stored triangle, in broadcast
    order.  Ops (alpha everywhere; `first` = apply beta, else 1.0):
      ("symm", p0, p1, first)               C[p0:p1] (+)= sym(A_pp) B[p0:p1]
      ("gemm", "N", r0, r1, p0, p1, first)  C[r0:r1] (+)= A[r0:r1, p0:p1] B[p0:p1]
      ("gemm", "T", p0, p1, r0, r1, first)  C[p0:p1] (+)= A[r0:r1, p0:p1]^T B[r0:r1]
    where [r0, r1) is the panel's off-diagonal rectangle ([p1, n) lower,
    [0, p0) upper).  Every row of C receives beta from exactly its first op."""
    ops, pan = [], k_panels(n, panels, align)
    for i, (p0, p1) in enumerate(pan):
        r0, r1 = (p1, n) if lower else (0, p0)
        if lower:
            ops.append(("symm", p0, p1, i == 0))
            if r1 > r0:
                ops.append(("gemm", "N", r0, r1, p0, p1, i == 0))
                ops.append(("gemm", "T", p0, p1, r0, r1, False))
        else:
            ops.append(("symm", p0, p1, True))           # panel i is the first to touch its rows
            if r1 > r0:
                ops.append(("gemm", "N", r0, r1, p0, p1, False))
                ops.append(("gemm", "T", p0, p1, r0, r1, False))
    return pan, ops


def trsm_plan(n: int, panels: int, lower: bool, align: int = 32):
    """STRSM side='L', transa='N' as the right-looking blocked solve over
    column panels of the stored triangle, in processing (= broadcast) order:
    forward for lower, backward for upper.  Ops:
      ("trsm", p0, p1, first)               X_p = inv(A_pp) (alpha if first else 1) B_p
      ("upd", r0, r1, p0, p1, first)        B[r0:r1] = (alpha if first else 1) B[r0:r1] - A[r0:r1, p0:p1] X_p
    alpha is folded into the first operation that touches each row."""
    pan = k_panels(n, panels, align)
    if not lower:
        pan = pan[::-1]
    ops = []
    for i, (p0, p1) in enumerate(pan):
        ops.append(("trsm", p0, p1, i == 0))
        r0, r1 = (p1, n) if lower else (0, p0)
        if r1 > r0:
            ops.append(("upd", r0, r1, p0, p1, i == 0))
    return pan, ops


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


def broadcast_trapezoid(A, p0: int, p1: int, lower: bool, root: int = 0, group=None):
    """Broadcast the stored-triangle part of columns [p0, p1) of the n x n
    column-major A (rows [p0, n) lower / [0, p1) upper) from `root`.  The
    trapezoid is packed into a contiguous buffer (NCCL / gloo need one),
    sent, and unpacked on the receivers only."""
    world, rank = world_rank(group)
    if world <= 1:
        return
    r0, r1 = trapezoid_rows(A.shape[0], p0, p1, lower)
    view = A[r0:r1, p0:p1]
    if view.t().is_contiguous():
        _dist().broadcast(view.t(), root, group=group)
        return
    buf = view.t().contiguous() if rank == root else view.new_empty((p1 - p0, r1 - r0))
    _dist().broadcast(buf, root, group=group)
    if rank != root:
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


class _Pipeline:
    """Comm-stream broadcast of A's panels, each consumed on the compute
    stream once it has landed; local kernels leave `reserve_sms` SMs to NCCL
    while panels are in flight."""

    def __init__(self, b3, reserve_sms):
        import torch
        self.torch = torch
        self.b3 = b3
        self.compute = torch.cuda.current_stream()
        self.comm = torch.cuda.Stream()
        self.comm.wait_stream(self.compute)
        self.reserve = max(0, int(reserve_sms))

    def run(self, panels, send, consume):
        torch = self.torch
        evs = []
        for p0, p1 in panels:                      # enqueue every broadcast up front
            with torch.cuda.stream(self.comm):
                send(p0, p1)
                ev = torch.cuda.Event()
                ev.record(self.comm)
            evs.append(ev)
        nsm = torch.cuda.get_device_properties(self.compute.device).multi_processor_count
        for i, ((p0, p1), ev) in enumerate(zip(panels, evs)):
            self.compute.wait_event(ev)
            last = i == len(panels) - 1
            if self.reserve and not last:
                with self.b3.options(max_sms=max(2, nsm - self.reserve)):
                    consume(i, p0, p1)
            else:
                consume(i, p0, p1)


_FLAGS = {}


def _panel_flags(device, n):
    """Per-device uint32 panel flags and a monotonically growing call value
    (the library never resets them: every call waits for a larger value)."""
    import torch
    key = str(device)
    if key not in _FLAGS or _FLAGS[key][0].numel() < n:
        _FLAGS[key] = [torch.zeros(max(64, n), dtype=torch.int32, device=device), 0]
    _FLAGS[key][1] += 1
    return _FLAGS[key][0], _FLAGS[key][1]


def sgemm(transa, transb, alpha, A, B_slab, beta, C_slab, root=0, group=None, panels=8,
          pipeline=None, reserve_sms=16, device_side=True):
    """C_slab <- alpha*op(A)*op(B)_slab + beta*C_slab on this rank's columns.

    A is replicated from `root` (NCCL broadcast).  For transa='N' the
    broadcast is pipelined in K panels on a comm stream (`pipeline` defaults
    to world > 1):
      * device_side=True (default, row F1): ONE streamed GEMM
        (blas3_sgemm_streamed) starts at once; its producer waits, per
        k-block, for the flag of the panel holding it, which the comm stream
        sets (blas3_signal) after each panel's broadcast.  Same result as a
        plain SGEMM bit for bit, C read and written once.  The GEMM leaves
        `reserve_sms` SMs to NCCL for its whole run (the broadcast cannot
        progress without SMs: the persistent grid would otherwise wait on it
        forever -- the 4 s trap of the panel wait);
      * device_side=False: one GEMM per panel as it lands (host-sequenced),
        beta on the first panel, SMs reserved while panels are in flight."""
    b3 = _b3()
    world, _ = world_rank(group)
    if pipeline is None:
        pipeline = world > 1
    if not pipeline or transa.upper() != "N" or transb.upper() != "N" or panels <= 1:
        broadcast_panels(A, root, group, 1)
        b3.sgemm(transa, transb, alpha, A, B_slab, beta, C_slab)
        return
    pan = k_panels(A.shape[1], panels)
    if device_side and b3.get_math_mode() != b3.MATH_SIMT_FP32:
        import torch
        pan = uniform_panels(A.shape[1], panels)        # the kernel maps k-block -> panel by division
        flags, value = _panel_flags(A.device, len(pan))
        compute = torch.cuda.current_stream()
        comm = torch.cuda.Stream()
        comm.wait_stream(compute)                  # A's buffer / flags free on both streams
        with torch.cuda.stream(comm):
            for i, (c0, c1) in enumerate(pan):
                if world > 1:
                    _bcast(A[:, c0:c1], root, group)
                b3.signal(flags, i, value)
        nsm = torch.cuda.get_device_properties(compute.device).multi_processor_count
        with b3.options(max_sms=max(2, nsm - max(0, int(reserve_sms)))):
            b3.sgemm_streamed("N", "N", alpha, A, B_slab, beta, C_slab, flags, pan[0][1] - pan[0][0], value)
        compute.wait_stream(comm)                  # the comm stream's work is part of the call
        return

    def consume(i, c0, c1):
        b3.sgemm("N", "N", alpha, A[:, c0:c1], B_slab[c0:c1], beta if i == 0 else 1.0, C_slab)

    _Pipeline(b3, reserve_sms).run(pan, lambda c0, c1: _bcast(A[:, c0:c1], root, group) if world > 1 else None,
                                   consume)


def ssymm(side, uplo, alpha, A, B_slab, beta, C_slab, root=0, group=None, panels=8,
          pipeline=None, reserve_sms=16):
    """side='L': C_slab <- alpha*A*B_slab + beta*C_slab (column slabs);
    side='R': row slabs (C_slab, B_slab are row blocks of C, B).
    For side='L' (world > 1 by default) only the uplo triangle of A travels,
    in trapezoid panels consumed as they land (`symm_plan`)."""
    b3 = _b3()
    world, _ = world_rank(group)
    lower = uplo.upper() == "L"
    if pipeline is None:
        pipeline = world > 1
    n = A.shape[0]
    if not pipeline or side.upper() != "L" or panels <= 1:
        for p0, p1 in k_panels(n, 1, 1):
            broadcast_trapezoid(A, p0, p1, lower, root, group)
        b3.ssymm(side, uplo, alpha, A, B_slab, beta, C_slab)
        return
    pan, ops = symm_plan(n, panels, lower)
    by_panel = {}
    for op in ops:
        key = (op[1], op[2]) if op[0] == "symm" else ((op[4], op[5]) if op[1] == "N" else (op[2], op[3]))
        by_panel.setdefault(key, []).append(op)

    def consume(i, p0, p1):
        for op in by_panel[(p0, p1)]:
            be = beta if op[-1] else 1.0
            if op[0] == "symm":
                b3.ssymm("L", uplo, alpha, A[p0:p1, p0:p1], B_slab[p0:p1], be, C_slab[p0:p1])
            elif op[1] == "N":
                _, _, r0, r1, q0, q1, _ = op
                b3.sgemm("N", "N", alpha, A[r0:r1, q0:q1], B_slab[q0:q1], be, C_slab[r0:r1])
            else:
                _, _, q0, q1, r0, r1, _ = op
                b3.sgemm("T", "N", alpha, A[r0:r1, q0:q1], B_slab[r0:r1], be, C_slab[q0:q1])

    _Pipeline(b3, reserve_sms).run(
        pan, lambda p0, p1: broadcast_trapezoid(A, p0, p1, lower, root, group), consume)


def strmm(side, uplo, transa, diag, alpha, A, B_slab, root=0, group=None):
    broadcast_panels(A, root, group, 1)
    _b3().strmm(side, uplo, transa, diag, alpha, A, B_slab)


def strsm(side, uplo, transa, diag, alpha, A, B_slab, root=0, group=None, panels=4,
          pipeline=None, reserve_sms=16):
    """Solve op(A) X = alpha B_slab on this rank's columns (side='L'; rows
    for side='R').  For side='L', transa='N' (world > 1 by default) only the
    stored triangle travels, in trapezoid panels, and the solve is the
    right-looking blocked sweep over those panels (`trsm_plan`): each
    panel's diagonal solve by the library's STRSM and its update of the
    remaining rows by SGEMM start as soon as the panel has landed."""
    b3 = _b3()
    world, _ = world_rank(group)
    lower = uplo.upper() == "L"
    if pipeline is None:
        pipeline = world > 1
    n = A.shape[0]
    if not pipeline or side.upper() != "L" or transa.upper() != "N" or panels <= 1:
        broadcast_trapezoid(A, 0, n, lower, root, group)
        b3.strsm(side, uplo, transa, diag, alpha, A, B_slab)
        return
    pan, ops = trsm_plan(n, panels, lower)
    by_panel = {}
    for op in ops:
        by_panel.setdefault((op[1], op[2]) if op[0] == "trsm" else (op[3], op[4]), []).append(op)

    def consume(i, p0, p1):
        for op in by_panel[(p0, p1)]:
            a1 = alpha if op[-1] else 1.0
            if op[0] == "trsm":
                b3.strsm("L", uplo, "N", diag, a1, A[p0:p1, p0:p1], B_slab[p0:p1])
            else:
                _, r0, r1, q0, q1, _ = op
                b3.sgemm("N", "N", -1.0, A[r0:r1, q0:q1], B_slab[q0:q1], a1, B_slab[r0:r1])

    _Pipeline(b3, reserve_sms).run(
        pan, lambda p0, p1: broadcast_trapezoid(A, p0, p1, lower, root, group), consume)


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
