"""Variant search over the library's tuning options.

The paper's generator picks, per routine, the best of several optimisation
scripts by measuring them: e.g. staging a transposed or
symmetric operand in shared memory versus pre-materialising it in global
memory (GM_map).  Here every such choice is a runtime option of the
C ABI (``blas3_set_option``), all of which compute the same result, and this
module measures candidate settings on the caller's problem and keeps the
fastest.  Host-side orchestration only: every candidate runs through the same
C-ABI entry points and CUDA kernels.

Timing: CUDA events on the current stream; candidates are INTERLEAVED over
``rounds`` rounds (1 warm-up + ``reps`` calls each, the visiting order rotated
every round) and compared by their median, so slow drifts of the clock under
the power cap and position effects hit all candidates alike.
"""
from __future__ import annotations

import itertools
import statistics

import paper_conf_ipps_cuiwxyf11_b200 as b3


def _time(fn, reps):
    import torch
    fn()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    e1.synchronize()
    return e0.elapsed_time(e1) / reps


def search(fn, candidates, reps=3, rounds=3):
    """Time `fn` under every option setting in `candidates` (dicts of option
    name -> value), interleaved.  Returns (best setting, [(setting, median ms)])."""
    samples = [[] for _ in candidates]
    nc = len(candidates)
    for r in range(rounds):
        # rotate the visiting order every round, so position effects (clock /
        # thermal state left by the previous candidate) do not favour any one
        for j in range(nc):
            i = (r + j) % nc
            with b3.options(**candidates[i]):
                samples[i].append(_time(fn, reps))
    table = [(c, statistics.median(s)) for c, s in zip(candidates, samples)]
    best = min(table, key=lambda t: t[1])[0]
    return best, table


def grid(**axes):
    """Cartesian product of option values: grid(tc_cta=[1, 2], gm_map=[0, 1])."""
    keys = list(axes)
    return [dict(zip(keys, vals)) for vals in itertools.product(*(axes[k] for k in keys))]


def tune_problem(routine, args, candidates=None, apply=True, **kw):
    """Search the default candidate grid for one call ``b3.<routine>(*args)``
    (column-major CUDA tensors, as for the tensor-level binding) and, if
    `apply`, set the winning options process-wide.  Returns (best, table)."""
    fn = getattr(b3, routine)
    if candidates is None:
        candidates = default_candidates(routine)
    best, table = search(lambda: fn(*args), candidates, **kw)
    if apply:
        for k, v in best.items():
            b3.set_option(k, v)
    return best, table


def default_candidates(routine):
    """The search space per routine: GM_map on/off, 1- vs 2-CTA tiles, and the
    STRSM panel width / slab count / first-panel halving."""
    if routine == "strsm":
        return grid(gm_map=[-1, 1], trsm_nb=[1024, 2048, 4096], trsm_slabs=[1, 2])
    if routine in ("sgemm", "ssymm", "strmm"):
        return grid(gm_map=[0, 1], tc_cta=[0, 1])
    return grid(tc_cta=[0, 1], tc_split=[0, 1])
