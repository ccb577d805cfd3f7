"""Throughput of every routine variant at BASELINE.json's configs[1..3] on one
B200 (context for DESIGN.md §7; the headline number is bench.py's).

  configs[1]: SGEMM (4 trans combos) and SSYMM (4 side/uplo) at N = 1024..8192
  configs[2]: STRMM / STRSM, all 16 side/uplo/trans/diag, N = 4096 and 8192
  configs[3]: SSYRK / SSYR2K, both uplo/trans, N = K = 8192 and N = 16384, K = 512

Also times the box's cuBLAS SGEMM (torch.matmul, fp32 with TF32 disabled, and
TF32 1-pass) at each SGEMM size as context (the paper compared against CUBLAS).
Times: CUDA events on the current stream, 1 warm-up + `reps` back-to-back calls,
inputs resident in HBM.  Prints one JSON line per measurement and writes
`profiles/<tag>_variants.json` + `.md` when --out is given.

python tools/variant_bench.py [--quick] [--out r01]
"""
import argparse, itertools, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_cuiwxyf11_b200 as b3

AL, BE = 1.5, 0.5


def timeit(fn, reps):
    fn(); torch.cuda.synchronize()
    e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def mats(n, k=None):
    k = n if k is None else k
    out = {}
    for nm, (r, c) in {"A": (n, n), "B": (n, n), "C": (n, n)}.items():
        t = b3.colmajor(r, c); t.uniform_(-1, 1); out[nm] = t
    # unit diagonal, off-diagonal U(-1/n, 1/n): diagonally dominant and ||T|| ~ 1, so
    # repeated in-place STRMM/STRSM calls keep X at O(1) (data-dependent power:
    # exploding or vanishing X would raise the clock under the power cap)
    T = b3.colmajor(n, n); T.uniform_(-1.0 / n, 1.0 / n); T.diagonal().fill_(1.0)
    out["T"] = T
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--out", default=None)
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    rows = []

    def rec(cfg, routine, variant, n, ms, flops, **extra):
        r = {"config": cfg, "routine": routine, "variant": variant, "n": n, "ms": round(ms, 4),
             "tflops": round(flops / ms / 1e9, 1), **extra}
        rows.append(r)
        print(json.dumps(r), flush=True)

    sizes = [1024, 4096, 8192] if args.quick else list(range(1024, 8193, 1024))
    # ---- configs[1]: SGEMM / SSYMM sweep + cuBLAS context
    for n in sizes:
        M = mats(n)
        A, B, C = M["A"], M["B"], M["C"]
        for ta, tb in itertools.product("NT", "NT"):
            ms = timeit(lambda: b3.sgemm(ta, tb, AL, A, B, BE, C), args.reps)
            rec(1, "sgemm", ta + tb, n, ms, 2.0 * n ** 3)
        for side, uplo in itertools.product("LR", "LU"):
            ms = timeit(lambda: b3.ssymm(side, uplo, AL, A, B, BE, C), args.reps)
            rec(1, "ssymm", side + uplo, n, ms, 2.0 * n ** 3)
        a, bb = torch.rand(n, n, device="cuda"), torch.rand(n, n, device="cuda")
        torch.backends.cuda.matmul.allow_tf32 = False
        ms = timeit(lambda: torch.matmul(a, bb), args.reps)
        rec(1, "cublas_sgemm_fp32", "NN", n, ms, 2.0 * n ** 3)
        torch.backends.cuda.matmul.allow_tf32 = True
        ms = timeit(lambda: torch.matmul(a, bb), args.reps)
        rec(1, "cublas_sgemm_tf32_1pass", "NN", n, ms, 2.0 * n ** 3)
        torch.backends.cuda.matmul.allow_tf32 = False
        del M, A, B, C, a, bb
        torch.cuda.empty_cache()
    # ---- configs[2]: STRMM / STRSM, 16 variants
    for n in ([4096, 8192]):
        M = mats(n)
        T, B = M["T"], M["B"]
        X = b3.colmajor(n, n)
        for side, uplo, ta, diag in itertools.product("LR", "LU", "NT", "NU"):
            v = side + uplo + ta + diag
            X.copy_(B)
            ms = timeit(lambda: b3.strmm(side, uplo, ta, diag, AL, T, X), args.reps)
            rec(2, "strmm", v, n, ms, 1.0 * n ** 3)
            X.copy_(B)
            ms = timeit(lambda: b3.strsm(side, uplo, ta, diag, AL, T, X), args.reps)
            rec(2, "strsm", v, n, ms, 1.0 * n ** 3)
        del M, T, B, X
        torch.cuda.empty_cache()
    # ---- configs[3]: SSYRK / SSYR2K
    for n, k in [(8192, 8192), (16384, 512)]:
        A = b3.colmajor(n, k); A.uniform_(-1, 1)
        Bm = b3.colmajor(n, k); Bm.uniform_(-1, 1)
        At = b3.colmajor(k, n); At.uniform_(-1, 1)
        Bt = b3.colmajor(k, n); Bt.uniform_(-1, 1)
        C = b3.colmajor(n, n); C.uniform_(-1, 1)
        for uplo, tr in itertools.product("LU", "NT"):
            a_, b_ = (A, Bm) if tr == "N" else (At, Bt)
            ms = timeit(lambda: b3.ssyrk(uplo, tr, AL, a_, BE, C), args.reps)
            rec(3, "ssyrk", uplo + tr, n, ms, 1.0 * k * n * (n + 1), k=k)
            ms = timeit(lambda: b3.ssyr2k(uplo, tr, AL, a_, b_, BE, C), args.reps)
            rec(3, "ssyr2k", uplo + tr, n, ms, 2.0 * k * n * n + n, k=k)
        del A, Bm, At, Bt, C
        torch.cuda.empty_cache()

    if args.out:
        root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
        base = os.path.join(root, "profiles", f"{args.out}_variants")
        json.dump(rows, open(base + ".json", "w"), indent=1)
        sg = {r["n"]: r["tflops"] for r in rows if r["routine"] == "sgemm" and r["variant"] == "NN"}
        with open(base + ".md", "w") as f:
            f.write(f"# {args.out}: every variant at BASELINE configs[1..3], 1 B200 "
                    f"(tools/variant_bench.py, CUDA events, {args.reps} reps after 1 warm-up)\n\n")
            f.write("TF/s = LAWN-41 algorithmic flops / time; `% SGEMM` = vs this library's SGEMM NN "
                    "at the same N.\n\n| cfg | routine | variant | N | K | ms | TF/s | % SGEMM |\n"
                    "|---|---|---|---|---|---|---|---|\n")
            for r in rows:
                ref = sg.get(r["n"])
                pct = f"{100 * r['tflops'] / ref:.0f}" if ref else "-"
                f.write(f"| {r['config']} | {r['routine']} | {r['variant']} | {r['n']} | "
                        f"{r.get('k', r['n'])} | {r['ms']} | {r['tflops']} | {pct} |\n")


if __name__ == "__main__":
    main()
