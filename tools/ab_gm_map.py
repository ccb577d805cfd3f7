"""GM_map (pre-materialised operand) versus in-kernel staging, interleaved A/B
per variant at N = 4096 and 8192 (tune.search).  Writes profiles/<tag>_gm_map.md.

python tools/ab_gm_map.py [tag] [routines,comma,separated] [sizes,comma,separated]
"""
import itertools, json, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import paper_conf_ipps_cuiwxyf11_b200 as b3
from paper_conf_ipps_cuiwxyf11_b200 import tune

tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
only = set(sys.argv[2].split(",")) if len(sys.argv) > 2 else None
sizes = [int(x) for x in sys.argv[3].split(",")] if len(sys.argv) > 3 else [4096, 8192]
rows = []
for n in sizes:
    A = b3.colmajor(n, n); A.uniform_(-1, 1)
    B = b3.colmajor(n, n); B.uniform_(-1, 1)
    C = b3.colmajor(n, n); C.uniform_(-1, 1)
    T = b3.colmajor(n, n); T.uniform_(-1.0 / n, 1.0 / n); T.diagonal().fill_(1.0)   # ||T|| ~ 1: X stays O(1) over repeated in-place calls
    X = b3.colmajor(n, n); X.copy_(B)
    cases = [("sgemm", ta + tb, 2.0 * n ** 3, lambda ta=ta, tb=tb: b3.sgemm(ta, tb, 1.5, A, B, 0.5, C))
             for ta, tb in itertools.product("NT", "NT")]
    cases += [("ssymm", sd + ul, 2.0 * n ** 3, lambda sd=sd, ul=ul: b3.ssymm(sd, ul, 1.5, A, B, 0.5, C))
              for sd, ul in itertools.product("LR", "LU")]
    for sd, ul, ta in itertools.product("LR", "LU", "NT"):
        cases.append(("strmm", sd + ul + ta + "N", 1.0 * n ** 3,
                      lambda sd=sd, ul=ul, ta=ta: b3.strmm(sd, ul, ta, "N", 1.0, T, X)))
        cases.append(("strsm", sd + ul + ta + "N", 1.0 * n ** 3,
                      lambda sd=sd, ul=ul, ta=ta: b3.strsm(sd, ul, ta, "N", 1.0, T, X)))
    for routine, var, fl, fn in cases:
        if only and routine not in only:
            continue
        best, table = tune.search(fn, [{"gm_map": 0}, {"gm_map": 1}], reps=3, rounds=4)
        t0, t1 = table[0][1], table[1][1]
        r = {"routine": routine, "variant": var, "n": n, "staged_tflops": round(fl / t0 / 1e9, 1),
             "gm_map_tflops": round(fl / t1 / 1e9, 1), "gain_pct": round(100 * (t0 / t1 - 1), 1)}
        rows.append(r)
        print(json.dumps(r), flush=True)
    del A, B, C, T, X
    torch.cuda.empty_cache()

with open(os.path.join(ROOT, "profiles", f"{tag}_gm_map.md"), "w") as f:
    f.write(f"# {tag}: GM_map (operand pre-materialised in HBM) vs staged in shared memory\n\n"
            "Interleaved A/B on one B200 (tools/ab_gm_map.py: 4 rounds x (1 warm-up + 3 calls), "
            "median).  gain > 0: GM_map faster.\n\n| routine | variant | N | staged TF/s | "
            "GM_map TF/s | gain % |\n|---|---|---|---|---|---|\n")
    for r in rows:
        f.write(f"| {r['routine']} | {r['variant']} | {r['n']} | {r['staged_tflops']} | "
                f"{r['gm_map_tflops']} | {r['gain_pct']} |\n")
