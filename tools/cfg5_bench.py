"""BASELINE configs[4] at one GPU: N=32768 SGEMM NN, SSYMM LL, STRSM LLNN
(the single-GPU base of the column-slab scaling run), CUDA events, median of
`reps` calls after a warm-up.  Also prints STRSM / SGEMM.

python tools/cfg5_bench.py [n] [reps]
"""
import statistics
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3

n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
A = b3.colmajor(n, n); A.uniform_(-1, 1)
B = b3.colmajor(n, n); B.uniform_(-1, 1)
C = b3.colmajor(n, n); C.uniform_(-1, 1)


def timed(fn, pre=None):
    out = []
    for i in range(reps + 1):
        if pre:
            pre()
        e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        if i:
            out.append(e0.elapsed_time(e1))
    return statistics.median(out)


res = {}
res["sgemm"] = 2 * n**3 / timed(lambda: b3.sgemm("N", "N", 1.5, A, B, 0.5, C)) / 1e9
res["ssymm"] = 2 * n**3 / timed(lambda: b3.ssymm("L", "L", 1.5, A, B, 0.5, C)) / 1e9
del C
T = A                                          # reuse the buffer: diagonally dominant lower T
T.uniform_(-1, 1); T.diagonal().add_(n / 2.0)
X = b3.colmajor(n, n)
res["strsm"] = n**3 / timed(lambda: b3.strsm("L", "L", "N", "N", 1.5, T, X), pre=lambda: X.copy_(B)) / 1e9
for k, v in res.items():
    print(f"N={n} {k}: {v:.1f} TF/s ({100 * v / res['sgemm']:.0f}% of SGEMM)", flush=True)
