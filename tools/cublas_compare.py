"""The B200 analogue of the paper's Figs 10-12: every one of the
paper's 24 variants (4 GEMM, 4 SYMM, 8 TRMM, 8 TRSM with diag='N')
plus SYRK/SYR2K, this library against the box's cuBLAS at the same call, as
speedup = cuBLAS time / our time.

cuBLAS is called through ctypes on the torch-bundled libcublas (v2 API, same
device buffers, same stream), in two math modes: CUBLAS_DEFAULT_MATH (fp32,
the CUBLAS 3.2 role of the paper) and CUBLAS_TF32_TENSOR_OP_MATH (1-pass TF32:
context only -- it does not meet the fp32 accuracy of our 3xTF32 path).
Interleaved timing (tune.search-style medians).  Writes profiles/<tag>_cublas.md.

python tools/cublas_compare.py [n] [tag]
"""
import ctypes, glob, itertools, json, os, statistics, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import paper_conf_ipps_cuiwxyf11_b200 as b3

n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
tag = sys.argv[2] if len(sys.argv) > 2 else "r01"


def load_cublas():
    cands = glob.glob(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cublas", "lib",
                                   "libcublas.so*")) + ["libcublas.so.12", "libcublas.so"]
    for c in cands:
        try:
            return ctypes.CDLL(c)
        except OSError:
            continue
    raise OSError("libcublas not found")


cb = load_cublas()
h = ctypes.c_void_p()
assert cb.cublasCreate_v2(ctypes.byref(h)) == 0
assert cb.cublasSetStream_v2(h, ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)) == 0
P, I, F = ctypes.c_void_p, ctypes.c_int, ctypes.c_float
al, be = F(1.5), F(0.5)
pa, pb = ctypes.byref(al), ctypes.byref(be)
OP = {"N": 0, "T": 1}
SIDE = {"L": 0, "R": 1}
UPLO = {"L": 0, "U": 1}
DIAG = {"N": 0, "U": 1}


def ptr(t):
    return P(t.data_ptr())


def chk(rc):
    assert rc == 0, f"cuBLAS status {rc}"


A = b3.colmajor(n, n); A.uniform_(-1, 1)
B = b3.colmajor(n, n); B.uniform_(-1, 1)
C = b3.colmajor(n, n); C.uniform_(-1, 1)
T = b3.colmajor(n, n); T.uniform_(-1.0 / n, 1.0 / n); T.diagonal().fill_(1.0)
X = b3.colmajor(n, n); X.copy_(B)
X2 = b3.colmajor(n, n)


def t_ms(fn, reps=3):
    fn()
    e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record(); e1.synchronize()
    return e0.elapsed_time(e1) / reps


cases = []
for ta, tb in itertools.product("NT", "NT"):
    cases.append(("sgemm", ta + tb, 2.0 * n ** 3, lambda ta=ta, tb=tb: b3.sgemm(ta, tb, 1.5, A, B, 0.5, C),
                  lambda ta=ta, tb=tb: chk(cb.cublasSgemm_v2(h, I(OP[ta]), I(OP[tb]), I(n), I(n), I(n), pa,
                                                               ptr(A), I(n), ptr(B), I(n), pb, ptr(C), I(n)))))
for sd, ul in itertools.product("LR", "LU"):
    cases.append(("ssymm", sd + ul, 2.0 * n ** 3, lambda sd=sd, ul=ul: b3.ssymm(sd, ul, 1.5, A, B, 0.5, C),
                  lambda sd=sd, ul=ul: chk(cb.cublasSsymm_v2(h, I(SIDE[sd]), I(UPLO[ul]), I(n), I(n), pa, ptr(A),
                                                             I(n), ptr(B), I(n), pb, ptr(C), I(n)))))
for sd, ul, ta in itertools.product("LR", "LU", "NT"):
    v = sd + ul + ta + "N"
    one = F(1.0)
    cases.append(("strmm", v, 1.0 * n ** 3, lambda sd=sd, ul=ul, ta=ta: b3.strmm(sd, ul, ta, "N", 1.0, T, X),
                  lambda sd=sd, ul=ul, ta=ta, one=one: chk(cb.cublasStrmm_v2(
                      h, I(SIDE[sd]), I(UPLO[ul]), I(OP[ta]), I(0), I(n), I(n), ctypes.byref(one), ptr(T), I(n),
                      ptr(X), I(n), ptr(X2), I(n)))))
    cases.append(("strsm", v, 1.0 * n ** 3, lambda sd=sd, ul=ul, ta=ta: b3.strsm(sd, ul, ta, "N", 1.0, T, X),
                  lambda sd=sd, ul=ul, ta=ta, one=one: chk(cb.cublasStrsm_v2(
                      h, I(SIDE[sd]), I(UPLO[ul]), I(OP[ta]), I(0), I(n), I(n), ctypes.byref(one), ptr(T), I(n),
                      ptr(X), I(n)))))
for ul, tr in itertools.product("LU", "NT"):
    cases.append(("ssyrk", ul + tr, 1.0 * n * n * (n + 1), lambda ul=ul, tr=tr: b3.ssyrk(ul, tr, 1.5, A, 0.5, C),
                  lambda ul=ul, tr=tr: chk(cb.cublasSsyrk_v2(h, I(UPLO[ul]), I(OP[tr]), I(n), I(n), pa, ptr(A),
                                                             I(n), pb, ptr(C), I(n)))))
    cases.append(("ssyr2k", ul + tr, 2.0 * n ** 3 + n,
                  lambda ul=ul, tr=tr: b3.ssyr2k(ul, tr, 1.5, A, B, 0.5, C),
                  lambda ul=ul, tr=tr: chk(cb.cublasSsyr2k_v2(h, I(UPLO[ul]), I(OP[tr]), I(n), I(n), pa, ptr(A),
                                                              I(n), ptr(B), I(n), pb, ptr(C), I(n)))))

rows = []
for routine, var, fl, ours, theirs in cases:
    s = {"ours": [], "fp32": [], "tf32": []}
    for _ in range(3):
        s["ours"].append(t_ms(ours))
        chk(cb.cublasSetMathMode(h, I(0)))
        s["fp32"].append(t_ms(theirs, reps=1 if n >= 8192 else 3))
        chk(cb.cublasSetMathMode(h, I(3)))
        s["tf32"].append(t_ms(theirs))
        chk(cb.cublasSetMathMode(h, I(0)))
    med = {k: statistics.median(v) for k, v in s.items()}
    r = {"routine": routine, "variant": var, "n": n,
         "ours_tflops": round(fl / med["ours"] / 1e9, 1),
         "cublas_fp32_tflops": round(fl / med["fp32"] / 1e9, 1),
         "cublas_tf32_1pass_tflops": round(fl / med["tf32"] / 1e9, 1),
         "speedup_vs_fp32": round(med["fp32"] / med["ours"], 2)}
    rows.append(r)
    print(json.dumps(r), flush=True)

with open(os.path.join(ROOT, "profiles", f"{tag}_cublas.md"), "w") as f:
    f.write(f"# {tag}: this library vs the box's cuBLAS, N = {n}, 1 B200 (tools/cublas_compare.py)\n\n"
            "Paper analogue: Figs 10-12 (speedup over CUBLAS 3.2 per variant).  `cuBLAS fp32` = "
            "CUBLAS_DEFAULT_MATH (fp32 accuracy, the comparator); `cuBLAS TF32` = "
            "CUBLAS_TF32_TENSOR_OP_MATH (1 TF32 pass, ~1e-3 accuracy: context, not a like-for-like "
            "comparison with our fp32-accurate 3xTF32).  Medians of 3 interleaved rounds.\n\n"
            "| routine | variant | ours TF/s | cuBLAS fp32 TF/s | speedup | cuBLAS TF32 1-pass TF/s |\n"
            "|---|---|---|---|---|---|\n")
    for r in rows:
        f.write(f"| {r['routine']} | {r['variant']} | {r['ours_tflops']} | {r['cublas_fp32_tflops']} | "
                f"{r['speedup_vs_fp32']}x | {r['cublas_tf32_1pass_tflops']} |\n")
