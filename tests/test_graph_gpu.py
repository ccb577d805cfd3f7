"""CUDA-graph capture of the hot path.

Every entry point is stream-ordered and host-sync-free (include/blas3.h
"Streams"), so a caller can capture a whole chain of calls -- including
STRSM's fork/join over side streams and its stream-ordered scratch -- into a
CUDA graph and replay it.  The dynamic tile scheduler's claim counters are
reset on the device by each launch's last claim, so replays start from the
same state as eager launches.  Replays must reproduce the eager results bit
for bit (the tile -> value computation does not depend on which CTA claims
the tile, and split-k tails reduce their slices in a fixed order), on fresh
inputs copied into the captured buffers, and again on a second replay.
"""
import numpy as np
import pytest

import blas3_inputs as gen
from check import bits_equal, to_dev, to_host

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
    return m


def _chain(b3, A, T, B, C, X):
    b3.sgemm("N", "T", AL, A, B, BE, C)
    b3.ssymm("L", "U", AL, A, B, BE, C)
    b3.ssyrk("L", "N", AL, A, BE, C)
    b3.ssyr2k("U", "T", AL, A, B, BE, C)
    b3.strmm("L", "L", "N", "N", AL, T, X)
    b3.strsm("L", "L", "N", "N", AL, T, X)
    b3.strsm("R", "U", "T", "N", AL, T, X)


@pytest.mark.parametrize("mode", ["3xtf32", "simt", "tf32_bf16x"])
def test_chain_graph_replay_bit_identical(b3, mode):
    import torch
    b3.set_math_mode(mode)
    n = 2304                               # several tiles, 2 STRSM panels (ragged)
    inputs = []
    for s in range(2):                     # two input sets: capture on one, replay both
        inputs.append(dict(A=gen.uniform(n, n, f"g-a{s}"), T=gen.triangular_dd(n, "L", "N", f"g-t{s}"),
                           B=gen.uniform(n, n, f"g-b{s}"), C=gen.uniform(n, n, f"g-c{s}")))
    # eager reference results
    eager = []
    for inp in inputs:
        A, T, B, C = (to_dev(inp[k]) for k in "ATBC")
        X = B.clone()
        _chain(b3, A, T, B, C, X)
        torch.cuda.synchronize()
        eager.append((to_host(C), to_host(X)))
    # static buffers; warm up eagerly ON THE CAPTURE STREAM (per-stream library
    # state is allocated on first use, which a capture does not allow)
    sA, sT, sB, sC = (to_dev(inputs[0][k]) for k in "ATBC")
    sX = sB.clone()
    cs = torch.cuda.Stream()
    cs.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(cs):
        _chain(b3, sA, sT, sB, sC, sX)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=cs):
        _chain(b3, sA, sT, sB, sC, sX)
    for rep in range(2):
        for s, inp in enumerate(inputs):
            for k, buf in zip("ATBC", (sA, sT, sB, sC)):
                buf.copy_(to_dev(inp[k]))
            sX.copy_(sB)
            g.replay()
            torch.cuda.synchronize()
            assert bits_equal(to_host(sC), eager[s][0]), f"C differs (set {s}, replay {rep})"
            assert bits_equal(to_host(sX), eager[s][1]), f"X differs (set {s}, replay {rep})"
    b3.set_math_mode("3xtf32")


def test_tile_counters_survive_many_launches(b3):
    """More launches than the scheduler's 256 counter slots, on sizes whose
    claim counts differ per launch: every result still matches the first."""
    import torch
    b3.set_math_mode("3xtf32")
    ref = None
    for i in range(300):
        m = 640 + 128 * (i % 5)            # 1-3 waves, with and without a split tail
        A = gen.uniform(m, 512, "cnt-a")
        B = gen.uniform(512, 384, "cnt-b")
        dC = torch.zeros((384, m), device="cuda").t()
        b3.sgemm("N", "N", 1.0, to_dev(A), to_dev(B), 0.0, dC)
        if i % 5 == 0:
            out = to_host(dC)
            if ref is None:
                ref = out
            assert np.array_equal(out.view(np.uint32), ref.view(np.uint32))


def test_graph_replay_concurrent_with_eager_calls(b3):
    """A captured graph owns its scheduler counters and split-tail workspace
    (allocated inside the graph), so replaying it on another stream while eager
    calls run on the capture stream -- and two graphs at once -- never mixes
    their tile claims."""
    import torch
    b3.set_math_mode("3xtf32")
    m, n, k = 1536, 1280, 2304                 # several waves + a split tail
    A, B, C = gen.uniform(m, k, "cc-a"), gen.uniform(k, n, "cc-b"), gen.uniform(m, n, "cc-c")
    dA, dB = to_dev(A), to_dev(B)
    want = to_dev(C)
    b3.sgemm("N", "N", AL, dA, dB, BE, want)
    torch.cuda.synchronize()
    want = to_host(want)
    cs = torch.cuda.Stream()
    outs = [to_dev(C) for _ in range(2)]
    graphs = []
    for o in outs:
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=cs):
            b3.sgemm("N", "N", AL, dA, dB, BE, o)
        graphs.append(g)
    side = [torch.cuda.Stream() for _ in range(2)]
    eager = [to_dev(C) for _ in range(4)]
    for rep in range(3):
        for o in outs:
            o.copy_(to_dev(C))
        for e in eager:
            e.copy_(to_dev(C))
        torch.cuda.synchronize()
        for g, s in zip(graphs, side):
            with torch.cuda.stream(s):
                g.replay()
        with torch.cuda.stream(cs):
            for e in eager:
                b3.sgemm("N", "N", AL, dA, dB, BE, e)
        torch.cuda.synchronize()
        for o in outs + eager:
            assert bits_equal(to_host(o), want), f"replay {rep}"


def test_strsm_panel_solver_graph_replay(b3):
    """The STRSM diagonal-panel solver (forced) inside a captured graph: its
    team counters are zeroed by a memset node and its partial workspace comes
    from the call's stream-ordered scratch.  Replays on two input sets must
    match the eager results bit for bit (first panel forward, and backward)."""
    import torch
    b3.set_math_mode("3xtf32")
    n = 2304                                      # first panel 2048 (forward) / 256 (backward)

    def solve(T, X):
        with b3.options(trsm_panel=2):
            b3.strsm("L", "L", "N", "N", AL, T, X)
            b3.strsm("R", "U", "T", "N", AL, T, X)

    inputs = [dict(T=gen.triangular_dd(n, "L", "N", f"gp-t{s}"), B=gen.uniform(n, 768, f"gp-b{s}"))
              for s in range(2)]
    before = b3.launch_count("panel")
    eager = []
    for inp in inputs:
        T = to_dev(inp["T"])
        X = to_dev(inp["B"])
        Tr = to_dev(inp["T"][:768, :768].copy())
        with b3.options(trsm_panel=2):
            b3.strsm("L", "L", "N", "N", AL, T, X)
        Y = b3.colmajor(768, 768)
        Y.copy_(X[:768])
        with b3.options(trsm_panel=2):
            b3.strsm("R", "U", "T", "N", AL, Tr, Y)
        torch.cuda.synchronize()
        eager.append((to_host(X), to_host(Y)))
    assert b3.launch_count("panel") - before == 4, "expected the panel solver in every call"
    sT, sX = to_dev(inputs[0]["T"]), to_dev(inputs[0]["B"])
    sTr = to_dev(inputs[0]["T"][:768, :768].copy())
    sY = b3.colmajor(768, 768)
    cs = torch.cuda.Stream()
    cs.wait_stream(torch.cuda.current_stream())

    def captured():
        with b3.options(trsm_panel=2):
            b3.strsm("L", "L", "N", "N", AL, sT, sX)
            sY.copy_(sX[:768])
            b3.strsm("R", "U", "T", "N", AL, sTr, sY)

    with torch.cuda.stream(cs):
        captured()                                # per-stream state allocated eagerly first
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=cs):
        captured()
    for rep in range(2):
        for s, inp in enumerate(inputs):
            sT.copy_(to_dev(inp["T"]))
            sTr.copy_(to_dev(inp["T"][:768, :768].copy()))
            sX.copy_(to_dev(inp["B"]))
            g.replay()
            torch.cuda.synchronize()
            assert bits_equal(to_host(sX), eager[s][0]), f"left solve differs (set {s}, replay {rep})"
            assert bits_equal(to_host(sY), eager[s][1]), f"right solve differs (set {s}, replay {rep})"
