"""Concurrent host threads (ctypes releases the GIL during library calls), each
on its own CUDA stream, issuing all six routines -- including STRSM with its
shared side streams and the fused first-panel launch -- must produce exactly
the single-threaded results (the computation of each tile does not depend on
which CTA or stream runs it).  Exercises the host-side caches, locks, the
dynamic-scheduler counter ring and the per-stream library state."""
import threading

import numpy as np
import pytest

import blas3_inputs as gen
from check import bits_equal, to_dev, to_host

pytestmark = pytest.mark.gpu


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


def chain(b3, A, T, B, C, X):
    b3.sgemm("N", "N", 1.5, A, B, 0.5, C)
    b3.ssymm("L", "L", 1.5, A, B, 0.5, C)
    b3.ssyrk("L", "T", 1.5, A, 0.5, C)
    b3.ssyr2k("U", "N", 1.5, A, B, 0.5, C)
    b3.strmm("R", "L", "N", "N", 1.5, T, X)
    b3.strsm("L", "L", "N", "N", 1.5, T, X)


def test_threads_on_own_streams_match_serial(b3):
    import torch
    n, nthreads, reps = 2304, 4, 3
    inputs = [dict(A=gen.uniform(n, n, "thr-a", t), T=gen.triangular_dd(n, "L", "N", "thr-t", t),
                   B=gen.uniform(n, n, "thr-b", t), C=gen.uniform(n, n, "thr-c", t))
              for t in range(nthreads)]
    # serial reference, one input set at a time
    ref = []
    for inp in inputs:
        A, T, B, C = (to_dev(inp[k]) for k in "ATBC")
        X = B.clone()
        chain(b3, A, T, B, C, X)
        torch.cuda.synchronize()
        ref.append((to_host(C), to_host(X)))
    results = [[None] * reps for _ in range(nthreads)]
    errors = []
    barrier = threading.Barrier(nthreads)

    def worker(t):
        try:
            dev = {k: to_dev(inputs[t][k]) for k in "ATBC"}
            s = torch.cuda.Stream()
            barrier.wait()
            for r in range(reps):
                with torch.cuda.stream(s):
                    C = dev["C"].clone()
                    X = dev["B"].clone()
                    chain(b3, dev["A"], dev["T"], dev["B"], C, X)
                s.synchronize()
                results[t][r] = (to_host(C), to_host(X))
        except Exception as e:                  # reported below (threads cannot raise)
            errors.append(repr(e))

    threads = [threading.Thread(target=worker, args=(t,)) for t in range(nthreads)]
    for th in threads:
        th.start()
    for th in threads:
        th.join()
    assert not errors, errors
    for t in range(nthreads):
        for r in range(reps):
            C, X = results[t][r]
            assert bits_equal(C, ref[t][0]), f"thread {t} rep {r}: C differs"
            assert bits_equal(X, ref[t][1]), f"thread {t} rep {r}: X differs"
