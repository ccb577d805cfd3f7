"""STRSM option grid at one size (tune.search, interleaved medians).
python tools/strsm_search.py [n]"""
import itertools
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_cuiwxyf11_b200 as b3  # noqa: E402
from paper_conf_ipps_cuiwxyf11_b200 import tune  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
T = b3.colmajor(n, n); T.uniform_(-1.0 / n, 1.0 / n); T.diagonal().fill_(1.0)
B = b3.colmajor(n, n); B.uniform_(-1, 1)
X = b3.colmajor(n, n); X.copy_(B)


def fn():
    b3.strsm("L", "L", "N", "N", 1.0, T, X)


cands = [dict(trsm_nb=nb, trsm_first_split=fs, trsm_geo_leaf=gl, trsm_reserve=rv)
         for nb, fs, gl, rv in itertools.product([1024, 2048], [0, 512, 1024], [128, 256], [0, 16, 32])
         if fs < nb]
best, table = tune.search(fn, cands, reps=3, rounds=4)
table.sort(key=lambda x: x[1])
fl = float(n) ** 3
for c, ms in table[:12]:
    print(json.dumps({"n": n, **c, "ms": round(ms, 4), "tflops": round(fl / ms / 1e9, 1)}))
print("default:", json.dumps({k: b3.get_option(k) for k in ("trsm_nb", "trsm_first_split", "trsm_geo_leaf", "trsm_reserve")}))
