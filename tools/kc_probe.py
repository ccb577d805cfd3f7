"""TMEM chunk length (BLAS3_OPT_TC_KC) vs accuracy and speed.

Accuracy: SGEMM m = n = 1024, K in {512, 2048, 8192, 16384}, U(-1,1), e_rel
against fp64 (numpy) for each kc in both tensor modes, beside the SIMT FP32
path and numpy's fp32 matmul (the comparator of tests/check.rel_bound).
Speed: interleaved CUDA-event medians of SGEMM N = 8192 and tall-skinny
SSYRK / SSYR2K (N = 16384, K = 512) for each kc.
python tools/kc_probe.py [acc] [speed]
"""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import blas3_inputs as gen  # noqa: E402
import paper_conf_ipps_cuiwxyf11_b200 as b3  # noqa: E402

KCS = [1, 2, 3, 4, 8, 16]
what = sys.argv[1:] or ["acc", "speed"]

if "acc" in what:
    m = n = 1024
    for k, lo in [(512, -1.0), (2048, -1.0), (8192, -1.0), (16384, -1.0), (512, 0.0), (8192, 0.0)]:
        A = gen.uniform(m, k, "kc-a", k, lo=lo); B = gen.uniform(k, n, "kc-b", k, lo=lo)
        ref = A.astype(np.float64) @ B.astype(np.float64)
        rel = lambda got: float(np.linalg.norm(np.asarray(got, np.float64) - ref) / np.linalg.norm(ref))  # noqa
        row = [f"k={k:6d}{' U(0,1)' if lo == 0.0 else ' U(-1,1)'}", f"np_fp32={rel(A @ B):.2e}"]
        dA, dB = b3.from_fortran(A), b3.from_fortran(B)
        for cta in (2, 1):                                # pair (paired issue) vs single-CTA kernel
            with b3.options(tc_cta=cta, tc_split=0):
                dC = b3.colmajor(m, n, fill=0.0)
                b3.sgemm("N", "N", 1.0, dA, dB, 0.0, dC)
                row.append(f"3x_default_cta{cta}={rel(dC.cpu().numpy()):.2e}")
        b3.set_math_mode("simt")
        dC = b3.colmajor(m, n, fill=0.0)
        b3.sgemm("N", "N", 1.0, dA, dB, 0.0, dC)
        row.append(f"simt={rel(dC.cpu().numpy()):.2e}")
        for mode in ["3xtf32", "tf32_bf16x"]:
            b3.set_math_mode(mode)
            for kc in KCS:
                with b3.options(tc_kc=kc):
                    dC = b3.colmajor(m, n, fill=0.0)
                    b3.sgemm("N", "N", 1.0, dA, dB, 0.0, dC)
                row.append(f"{'3x' if mode == '3xtf32' else 'bx'}kc{kc}={rel(dC.cpu().numpy()):.2e}")
        b3.set_math_mode("3xtf32")
        print("  ".join(row), flush=True)

if "speed" in what:
    def bench(fn, reps):
        e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
        e0.record()
        for _ in range(reps):
            fn()
        e1.record(); torch.cuda.synchronize()
        return e0.elapsed_time(e1) / reps

    n = 8192
    A = b3.colmajor(n, n); B = b3.colmajor(n, n); C = b3.colmajor(n, n)
    for t in (A, B, C):
        t.uniform_(-1, 1)
    ts, k = 16384, 512
    As = b3.colmajor(ts, k); Bs = b3.colmajor(ts, k); Cs = b3.colmajor(ts, ts)
    for t in (As, Bs, Cs):
        t.uniform_(-1, 1)
    cases = {
        "sgemm8192": (lambda: b3.sgemm("N", "N", 1.5, A, B, 0.5, C), 2.0 * n ** 3, 5),
        "ssyrk16384x512": (lambda: b3.ssyrk("L", "N", 1.5, As, 0.5, Cs), 1.0 * k * ts * (ts + 1), 10),
        "ssyr2k16384x512": (lambda: b3.ssyr2k("L", "N", 1.5, As, Bs, 0.5, Cs), 2.0 * k * ts * ts + ts, 10),
    }
    for mode in ["3xtf32", "tf32_bf16x"]:
        b3.set_math_mode(mode)
        res = {(c, kc): [] for c in cases for kc in KCS}
        for rnd in range(5):
            for kc in KCS:
                with b3.options(tc_kc=kc):
                    for c, (fn, fl, reps) in cases.items():
                        fn(); torch.cuda.synchronize()
                        res[(c, kc)].append(bench(fn, reps))
        for c, (fn, fl, reps) in cases.items():
            row = [f"{mode:10s} {c:16s}"]
            for kc in KCS:
                ms = float(np.median(res[(c, kc)]))
                row.append(f"kc{kc}={ms * 1e3:8.1f}us {fl / ms / 1e9:6.1f}TF/s")
            print("  ".join(row), flush=True)
    b3.set_math_mode("3xtf32")
