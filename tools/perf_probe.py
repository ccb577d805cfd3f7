"""Perf experiments for the structured routines (not a bench; run on the GPU box).

python tools/perf_probe.py            -> runs every experiment below, each in a
                                          subprocess (env knobs are read once)
python tools/perf_probe.py one <exp>  -> one experiment in this process
"""
import json, os, subprocess, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def timeit(fn, reps=5):
    import torch
    fn(); torch.cuda.synchronize()
    e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def one(exp):
    import torch
    import paper_conf_ipps_cuiwxyf11_b200 as b3
    n = 8192
    out = {}
    A = b3.colmajor(n, n); B = b3.colmajor(n, n); C = b3.colmajor(n, n)
    for x in (A, B, C): x.uniform_(-1, 1)
    T = b3.colmajor(n, n); T.uniform_(-1, 1); T.diagonal().add_(n / 2.0)
    if exp == "ktiles":
        for k in (512, 1024, 2048, 4096, 8192):
            ms = timeit(lambda: b3.sgemm("N", "N", 1.5, A[:, :k], B[:k, :], 0.5, C))
            out[f"sgemm_k{k}"] = (round(ms, 4), round(2 * n * n * k / ms / 1e9, 1))
    elif exp == "trmm":
        ms = timeit(lambda: b3.strmm("L", "L", "N", "N", 1.5, T, B))
        out["strmm"] = (round(ms, 4), round(n ** 3 / ms / 1e9, 1))
        for m in (2048, 4096):
            Bs = b3.colmajor(m, n); Bs.uniform_(-1, 1)
            ms = timeit(lambda: b3.strmm("L", "L", "N", "N", 1.5, T[:m, :m], Bs))
            out[f"strmm_m{m}"] = (round(ms, 4), round(m * m * n / ms / 1e9, 1))
            ms = timeit(lambda: b3.sgemm("N", "N", 1.5, A[:m, :m], B[:m, :], 0.5, C[:m, :]))
            out[f"sgemm_m{m}_k{m}"] = (round(ms, 4), round(2 * m * m * n / ms / 1e9, 1))
    elif exp == "trsm":
        ms = timeit(lambda: b3.strsm("L", "L", "N", "N", 1.5, T, B))
        out["strsm"] = (round(ms, 4), round(n ** 3 / ms / 1e9, 1))
        for c in (64, 1024):
            ms = timeit(lambda: b3.strsm("L", "L", "N", "N", 1.5, T, B[:, :c]))
            out[f"strsm_n{c}"] = (round(ms, 4), round(n * n * c / ms / 1e9, 1))
    print("RESULT " + json.dumps({"exp": exp, "env": {k: v for k, v in os.environ.items()
                                                     if k.startswith("BLAS3")}, **out}), flush=True)


def main():
    runs = [("trmm", {}), ("trmm", {"BLAS3_DEBUG_TC": "32"}),
            ("trsm", {"BLAS3_TRSM_SLABS": "1"}), ("trsm", {"BLAS3_TRSM_SLABS": "2"}),
            ("trsm", {"BLAS3_TRSM_SLABS": "4"}), ("trsm", {"BLAS3_TRSM_SLABS": "2", "BLAS3_TRSM_NB": "1024"}),
            ("trsm", {"BLAS3_TRSM_SLABS": "4", "BLAS3_TRSM_NB": "1024"})]
    if len(sys.argv) > 1:
        runs = [(a.split(":")[0], dict(kv.split("=") for kv in a.split(":")[1:])) for a in sys.argv[1:]]
    for exp, env in runs:
        e = dict(os.environ); e.update(env)
        r = subprocess.run([sys.executable, __file__, "one", exp], env=e, capture_output=True, text=True)
        for line in r.stdout.splitlines():
            if line.startswith("RESULT "):
                print(line[7:], flush=True)
        if r.returncode:
            print(exp, env, "FAILED", r.stderr[-2000:], flush=True)


if __name__ == "__main__":
    if len(sys.argv) > 2 and sys.argv[1] == "one":
        one(sys.argv[2])
    else:
        main()
