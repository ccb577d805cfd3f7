"""Grouped-raster height (BLAS3_OPT_TC_RASTER) vs time: SGEMM NN and the chain's
other full-grid routines at N=8192, interleaved medians (tune.search).
python tools/raster_probe.py"""
import json, sys
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
from paper_conf_ipps_cuiwxyf11_b200 import tune
n = 8192
A = b3.colmajor(n, n); B = b3.colmajor(n, n); C = b3.colmajor(n, n)
for x in (A, B, C): x.uniform_(-1, 1)
cands = [{"tc_raster": g} for g in (0, 4, 8, 12, 24, 32)]
for name, fn in (("sgemm", lambda: b3.sgemm("N", "N", 1.5, A, B, 0.5, C)),
                 ("ssymm", lambda: b3.ssymm("L", "L", 1.5, A, B, 0.5, C))):
    _, table = tune.search(fn, cands, reps=3, rounds=4)
    for c, ms in table:
        print(json.dumps({"routine": name, "opts": c, "ms": round(ms, 4), "tflops": round(2 * n**3 / ms / 1e9, 1)}))
