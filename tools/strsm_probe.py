"""STRSM option sweep at N=8192 (isolated, and right after an SGEMM as in the
bench chain), interleaved medians via tune.search.

python tools/strsm_probe.py [n]
"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_cuiwxyf11_b200 as b3
from paper_conf_ipps_cuiwxyf11_b200 import tune

n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
A = b3.colmajor(n, n); A.uniform_(-1, 1)
T = b3.colmajor(n, n); T.uniform_(-1, 1); T.diagonal().add_(n / 2.0)
B = b3.colmajor(n, n); B.uniform_(-1, 1)
C = b3.colmajor(n, n); C.uniform_(-1, 1)
X = b3.colmajor(n, n)


def iso():
    X.copy_(B)
    b3.strsm("L", "L", "N", "N", 1.5, T, X)


def after_gemm():
    b3.sgemm("N", "N", 1.5, A, B, 0.5, C)
    X.copy_(B)
    b3.strsm("L", "L", "N", "N", 1.5, T, X)


def gemm_only():
    b3.sgemm("N", "N", 1.5, A, B, 0.5, C)
    X.copy_(B)


extra = json.loads(os.environ.get("PROBE_CANDS", "null"))
cands = extra or [
    {},
    {"trsm_first_fused": 0},
    {"trsm_first_fused": 0, "trsm_first_ym": 0},
    {"trsm_fused": 1},
    {"trsm_reserve": 32},
    {"trsm_reserve": 64},
    {"trsm_slabs": 1},
    {"trsm_nb": 1024},
    {"trsm_geo_leaf": 512},
]
flop = float(n) ** 3
_, tg = tune.search(gemm_only, [{}], reps=3, rounds=3)
g_ms = tg[0][1]
for name, fn, base in (("isolated", iso, 0.0), ("after_gemm", after_gemm, g_ms)):
    _, table = tune.search(fn, cands, reps=3, rounds=int(os.environ.get("PROBE_ROUNDS", "3")))
    for c, ms in table:
        t = ms - base
        print(json.dumps({"mode": name, "opts": c, "ms": round(t, 4), "tflops": round(flop / t / 1e9, 1)}))
