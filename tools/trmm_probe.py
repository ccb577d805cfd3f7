import json, sys
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
from paper_conf_ipps_cuiwxyf11_b200 import tune
for n in (4096, 8192):
    T = b3.colmajor(n, n); T.uniform_(-1, 1); T.diagonal().add_(1.0)
    X = b3.colmajor(n, n); X.uniform_(-1, 1)
    cands = [{}, {"tc_cta": 1}, {"tc_cta": 2}, {"gm_map": 1}, {"tc_split": 0}, {"tc_cta": 1, "gm_map": 1}]
    _, table = tune.search(lambda: b3.strmm("L", "L", "N", "N", 1.0, T, X), cands, reps=3, rounds=4)
    for c, ms in table:
        print(json.dumps({"n": n, "opts": c, "ms": round(ms, 4), "tflops": round(n**3 / ms / 1e9, 1)}), flush=True)
