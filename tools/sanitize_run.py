"""Small-N workload for compute-sanitizer (memcheck / synccheck / initcheck):
every routine, several variants, both math modes, ragged sizes, and the STRSM
multi-panel sweep (256-wide panels via BLAS3_TRSM_NB, set by the caller) on both
the multi-launch and the fused path, the STRSM diagonal-panel solver, plus a
split-k tail.  Prints one line.

BLAS3_TRSM_NB=256 compute-sanitizer --tool memcheck python tools/sanitize_run.py
"""
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3


def rnd(m, n):
    t = b3.colmajor(m, n)
    t.uniform_(-1, 1)
    return t


calls = 0
for mode in ("3xtf32", "simt", "tf32_bf16x"):
    b3.set_math_mode(mode)
    m, n, k = 300, 260, 270
    A, B, C = rnd(m, k), rnd(k, n), rnd(m, n)
    b3.sgemm("N", "N", 1.5, A, B, 0.5, C)
    b3.sgemm("T", "T", 1.5, rnd(k, m), rnd(n, k), 0.0, C)
    S = rnd(m, m)
    b3.ssymm("L", "L", 1.5, S, rnd(m, n), 0.5, C)
    b3.ssymm("R", "U", 1.5, rnd(n, n), rnd(m, n), 0.5, C)
    Cs = rnd(m, m)
    b3.ssyrk("L", "N", 1.5, rnd(m, k), 0.5, Cs)
    b3.ssyr2k("U", "T", 1.5, rnd(k, m), rnd(k, m), 0.5, Cs)
    T = rnd(m, m)
    T.diagonal().add_(float(m))
    X = rnd(m, n)
    b3.strmm("L", "L", "N", "N", 1.5, T, X)
    b3.strmm("R", "U", "T", "U", 1.5, rnd(n, n), X)
    for fused in (0, 1):
        with b3.options(trsm_fused=fused):
            Tn = rnd(900, 900)
            Tn.diagonal().add_(900.0)
            b3.strsm("L", "L", "N", "N", 1.5, Tn, rnd(900, 300))
            b3.strsm("R", "U", "T", "N", 1.5, Tn, rnd(300, 900))
    calls += 12
b3.set_math_mode("3xtf32")
# the STRSM diagonal-panel solver (forced): forward / backward, both sides, a
# ragged right-hand side, and a shrunken grid whose teams loop over slabs
for opts in ({"trsm_panel": 2}, {"trsm_panel": 2, "max_sms": 16}):
    with b3.options(**opts):
        Tp = rnd(768, 768)
        Tp.diagonal().add_(768.0)
        b3.strsm("L", "L", "N", "N", 1.5, Tp, rnd(768, 600))
        b3.strsm("L", "U", "N", "U", 1.5, Tp, rnd(768, 260))
        b3.strsm("R", "L", "T", "N", 1.5, Tp, rnd(300, 768))
        calls += 3
with b3.options(gm_map=1):                                       # GM_map SSYMM beside the staged default
    b3.ssymm("L", "U", 1.5, rnd(300, 300), rnd(300, 260), 0.5, rnd(300, 260))
# a captured graph (graph-private scheduler state / split workspace), replayed twice
cs = torch.cuda.Stream()
Cg = rnd(1024, 768)
Ag, Bg = rnd(1024, 2048), rnd(2048, 768)
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g, stream=cs):
    b3.sgemm("N", "N", 1.0, Ag, Bg, 0.5, Cg)
g.replay(); g.replay()
C2 = rnd(1024, 768)
b3.sgemm("N", "N", 1.0, rnd(1024, 2048), rnd(2048, 768), 0.0, C2)   # few tiles: split-k tail
torch.cuda.synchronize()
print(f"sanitize_run ok: {calls + 1} calls, {b3.launch_count()} kernel launches", flush=True)
