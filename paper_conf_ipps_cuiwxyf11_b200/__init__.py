"""B200-native (sm_100a) fp32 Level-3 BLAS derived from one tuned GEMM.

Thin Python binding over the C ABI in ``include/blas3.h`` (``libblas3.so``,
built in-tree by ``build.py``).  This module only marshals arguments: every
step of every routine runs in the library's CUDA kernels.  There is no CPU
fallback: importing the package fails loudly if the library is missing, and
every routine raises on a non-zero return code.

Two layers, same names as the C ABI:
  * ``blas3_sgemm(...)`` etc. -- the raw C entry points (ctypes), BLAS
    argument order, device pointers as ints, stream as int (0 = default).
  * ``sgemm(transa, transb, alpha, A, B, beta, C)`` etc. -- the same call on
    column-major CUDA ``torch.Tensor`` views (stride(0) == 1, ld = stride(1)),
    issued on torch's current stream.  PyTorch provides memory and streams
    only.
Matrices are column-major as in BLAS3.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libblas3.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
        "(there is deliberately no CPU fallback)")

_lib = ctypes.CDLL(LIB_PATH)

_i64, _f, _p, _c, _i = ctypes.c_int64, ctypes.c_float, ctypes.c_void_p, ctypes.c_char, ctypes.c_int
_d = ctypes.c_double

_SIGS = {
    "blas3_sgemm": [_c, _c, _i64, _i64, _i64, _f, _p, _i64, _p, _i64, _f, _p, _i64, _p],
    "blas3_ssymm": [_c, _c, _i64, _i64, _f, _p, _i64, _p, _i64, _f, _p, _i64, _p],
    "blas3_ssyrk": [_c, _c, _i64, _i64, _f, _p, _i64, _f, _p, _i64, _p],
    "blas3_ssyr2k": [_c, _c, _i64, _i64, _f, _p, _i64, _p, _i64, _f, _p, _i64, _p],
    "blas3_strmm": [_c, _c, _c, _c, _i64, _i64, _f, _p, _i64, _p, _i64, _p],
    "blas3_strsm": [_c, _c, _c, _c, _i64, _i64, _f, _p, _i64, _p, _i64, _p],
    "blas3_dgemm": [_c, _c, _i64, _i64, _i64, _d, _p, _i64, _p, _i64, _d, _p, _i64, _p],
    "blas3_dsymm": [_c, _c, _i64, _i64, _d, _p, _i64, _p, _i64, _d, _p, _i64, _p],
    "blas3_dsyrk": [_c, _c, _i64, _i64, _d, _p, _i64, _d, _p, _i64, _p],
    "blas3_dsyr2k": [_c, _c, _i64, _i64, _d, _p, _i64, _p, _i64, _d, _p, _i64, _p],
    "blas3_dtrmm": [_c, _c, _c, _c, _i64, _i64, _d, _p, _i64, _p, _i64, _p],
    "blas3_dtrsm": [_c, _c, _c, _c, _i64, _i64, _d, _p, _i64, _p, _i64, _p],
    "blas3_sgemm_streamed": [_c, _c, _i64, _i64, _i64, _f, _p, _i64, _p, _i64, _f, _p, _i64, _p, _i64,
                             ctypes.c_uint32, _p],
    "blas3_signal": [_p, ctypes.c_uint32, _p],
    "blas3_set_math_mode": [_i],
    "blas3_get_math_mode": [],
    "blas3_set_workspace": [_p, ctypes.c_size_t],
    "blas3_set_option": [_i, _i64],
    "blas3_get_option": [_i],
    "blas3_launch_count": [],
    "blas3_launch_count_by_path": [_i],
    "blas3_error_string": [_i],
    "blas3_version": [],
}
_RES = {"blas3_get_option": _i64, "blas3_launch_count": _i64, "blas3_launch_count_by_path": _i64, "blas3_error_string": ctypes.c_char_p}

for _name, _args in _SIGS.items():
    _fn = getattr(_lib, _name)
    _fn.argtypes = _args
    _fn.restype = _RES.get(_name, _i)
    globals()[_name] = _fn

EXPORTED = tuple(_SIGS)
MATH_3XTF32, MATH_SIMT_FP32, MATH_1XTF32, MATH_TF32_BF16X = 0, 1, 2, 3


class Blas3Error(RuntimeError):
    def __init__(self, routine, code):
        self.code = code
        msg = blas3_error_string(code).decode()  # noqa: F821
        super().__init__(f"{routine} returned {code}: {msg}")


def _chk(name, rc):
    if rc != 0:
        raise Blas3Error(name, rc)


def _ch(x):
    return x.encode() if isinstance(x, str) else x


# ----------------------------------------------------------------- tensor helpers
def _mat(X, name, f64=False):
    """(pointer, rows, cols, ld) of a column-major fp32 (fp64) CUDA tensor view."""
    import torch
    if not isinstance(X, torch.Tensor):
        raise TypeError(f"{name} must be a torch.Tensor")
    dt = torch.float64 if f64 else torch.float32
    if X.dtype != dt or not X.is_cuda or X.dim() != 2:
        raise TypeError(f"{name} must be a 2-D {str(dt)[6:]} CUDA tensor")
    m, n = X.shape
    if m > 1 and X.stride(0) != 1:
        raise ValueError(f"{name} must be column-major (stride(0) == 1)")
    ld = X.stride(1) if n > 1 else max(1, m)
    return X.data_ptr(), m, n, max(ld, 1)


def _stream():
    import torch
    return torch.cuda.current_stream().cuda_stream


def colmajor(m, n, ld=None, device="cuda", fill=None, dtype=None):
    """Allocate an m x n column-major fp32 (or `dtype`) tensor (strides (1, ld))."""
    import torch
    ld = max(1, m) if ld is None else ld
    buf = torch.empty((n, ld), dtype=torch.float32 if dtype is None else dtype, device=device)
    if fill is not None:
        buf.fill_(fill)
    return buf.t()[:m]


def from_fortran(arr, device="cuda", f64=False):
    """Copy a numpy Fortran-ordered (ld x n) buffer to a column-major device
    tensor with the same ld; returns the full (ld x n) view (fp32, or fp64)."""
    import numpy as np
    import torch
    a = np.asfortranarray(arr, dtype=np.float64 if f64 else np.float32)
    t = torch.from_numpy(a.T.copy()).to(device)     # (n, ld) row-major == (ld, n) col-major
    return t.t()


# ----------------------------------------------------------------- routines
# Shape checks: the C ABI only sees pointers and leading dimensions, so a
# tensor smaller than the problem needs would be read (or written) past its
# allocation.  Each wrapper derives the problem size from C (or B) and op(A)
# as in BLAS and requires every operand to hold at least the leading block
# the routine reads (extra rows / columns are ignored, as with BLAS's ld).
def _need(name, X, rows, cols):
    if X.shape[0] < rows or X.shape[1] < cols:
        raise ValueError(f"{name} is {tuple(X.shape)}, the call needs at least {rows} x {cols}")


def _t(c):
    return c.upper() != "N" if isinstance(c, str) else c.upper() != b"N"


def _gemm(f64, transa, transb, alpha, A, B, beta, C):
    pc, m, n, ldc = _mat(C, "C", f64)
    pa, ar, ac, lda = _mat(A, "A", f64)
    pb, br, bc, ldb = _mat(B, "B", f64)
    k = ac if not _t(transa) else ar
    _need("A", A, *((k, m) if _t(transa) else (m, k)))
    _need("B", B, *((n, k) if _t(transb) else (k, n)))
    name = "blas3_dgemm" if f64 else "blas3_sgemm"
    _chk(name, globals()[name](_ch(transa), _ch(transb), m, n, k, alpha, pa, lda, pb, ldb, beta, pc, ldc,
                               _stream()))


def sgemm(transa, transb, alpha, A, B, beta, C):
    """C <- alpha*op(A)*op(B) + beta*C (GEMM-NN/-TN)."""
    _gemm(False, transa, transb, alpha, A, B, beta, C)


def dgemm(transa, transb, alpha, A, B, beta, C):
    """fp64 GEMM (F4): C <- alpha*op(A)*op(B) + beta*C on float64 tensors."""
    _gemm(True, transa, transb, alpha, A, B, beta, C)


def sgemm_streamed(transa, transb, alpha, A, B, beta, C, ready, panel_k, value):
    """C <- alpha*A*op(B) + beta*C with A arriving in column panels of panel_k
    columns: panel p is read once ready[p] >= value (ready: a 1-D int32 CUDA
    tensor of uint32 flags, written by another stream, e.g. via signal())."""
    import torch
    pc, m, n, ldc = _mat(C, "C")
    pa, ar, ac, lda = _mat(A, "A")
    pb, br, bc, ldb = _mat(B, "B")
    k = ac
    _need("A", A, m, k)
    _need("B", B, *((n, k) if _t(transb) else (k, n)))
    if not isinstance(ready, torch.Tensor) or not ready.is_cuda or ready.dtype != torch.int32:
        raise TypeError("ready must be an int32 CUDA tensor")
    if ready.numel() < -(-k // int(panel_k)):
        raise ValueError("ready holds fewer flags than A has panels")
    _chk("blas3_sgemm_streamed", blas3_sgemm_streamed(  # noqa: F821
        _ch(transa), _ch(transb), m, n, k, alpha, pa, lda, pb, ldb, beta, pc, ldc, ready.data_ptr(),
        int(panel_k), int(value) & 0xFFFFFFFF, _stream()))


def signal(ready, index, value):
    """Stream-ordered release write ready[index] = value on the current stream."""
    _chk("blas3_signal", blas3_signal(ready.data_ptr() + 4 * int(index), int(value) & 0xFFFFFFFF,  # noqa: F821
                                      _stream()))


def _symm(f64, side, uplo, alpha, A, B, beta, C):
    pc, m, n, ldc = _mat(C, "C", f64)
    pa, _, _, lda = _mat(A, "A", f64)
    pb, _, _, ldb = _mat(B, "B", f64)
    ka = m if (side.upper() if isinstance(side, str) else side.decode().upper()) == "L" else n
    _need("A", A, ka, ka)
    _need("B", B, m, n)
    name = "blas3_dsymm" if f64 else "blas3_ssymm"
    _chk(name, globals()[name](_ch(side), _ch(uplo), m, n, alpha, pa, lda, pb, ldb, beta, pc, ldc, _stream()))


def ssymm(side, uplo, alpha, A, B, beta, C):
    """side=L: C <- alpha*A*B + beta*C; side=R: C <- alpha*B*A + beta*C."""
    _symm(False, side, uplo, alpha, A, B, beta, C)


def dsymm(side, uplo, alpha, A, B, beta, C):
    """fp64 SYMM (F4)."""
    _symm(True, side, uplo, alpha, A, B, beta, C)


def _syrk(f64, uplo, trans, alpha, A, beta, C):
    pc, n, _, ldc = _mat(C, "C", f64)
    pa, ar, ac, lda = _mat(A, "A", f64)
    k = ac if not _t(trans) else ar
    _need("C", C, n, n)
    _need("A", A, *((k, n) if _t(trans) else (n, k)))
    name = "blas3_dsyrk" if f64 else "blas3_ssyrk"
    _chk(name, globals()[name](_ch(uplo), _ch(trans), n, k, alpha, pa, lda, beta, pc, ldc, _stream()))


def ssyrk(uplo, trans, alpha, A, beta, C):
    """C <- alpha*op(A)*op(A)^T + beta*C on the uplo triangle."""
    _syrk(False, uplo, trans, alpha, A, beta, C)


def dsyrk(uplo, trans, alpha, A, beta, C):
    """fp64 SYRK (F4)."""
    _syrk(True, uplo, trans, alpha, A, beta, C)


def _syr2k(f64, uplo, trans, alpha, A, B, beta, C):
    pc, n, _, ldc = _mat(C, "C", f64)
    pa, ar, ac, lda = _mat(A, "A", f64)
    pb, _, _, ldb = _mat(B, "B", f64)
    k = ac if not _t(trans) else ar
    _need("C", C, n, n)
    _need("A", A, *((k, n) if _t(trans) else (n, k)))
    _need("B", B, *((k, n) if _t(trans) else (n, k)))
    name = "blas3_dsyr2k" if f64 else "blas3_ssyr2k"
    _chk(name, globals()[name](_ch(uplo), _ch(trans), n, k, alpha, pa, lda, pb, ldb, beta, pc, ldc, _stream()))


def ssyr2k(uplo, trans, alpha, A, B, beta, C):
    """C <- alpha*(op(A)op(B)^T + op(B)op(A)^T) + beta*C on the uplo triangle."""
    _syr2k(False, uplo, trans, alpha, A, B, beta, C)


def dsyr2k(uplo, trans, alpha, A, B, beta, C):
    """fp64 SYR2K (F4)."""
    _syr2k(True, uplo, trans, alpha, A, B, beta, C)


def _order(side, m, n):
    return m if (side.upper() if isinstance(side, str) else side.decode().upper()) == "L" else n


def _tr(f64, solve, side, uplo, transa, diag, alpha, A, B):
    pb, m, n, ldb = _mat(B, "B", f64)
    pa, _, _, lda = _mat(A, "A", f64)
    ka = _order(side, m, n)
    _need("A", A, ka, ka)
    name = "blas3_" + ("d" if f64 else "s") + ("trsm" if solve else "trmm")
    _chk(name, globals()[name](_ch(side), _ch(uplo), _ch(transa), _ch(diag), m, n, alpha, pa, lda, pb, ldb,
                               _stream()))


def strmm(side, uplo, transa, diag, alpha, A, B):
    """B <- alpha*op(A)*B (L) or alpha*B*op(A) (R), in place."""
    _tr(False, False, side, uplo, transa, diag, alpha, A, B)


def strsm(side, uplo, transa, diag, alpha, A, B):
    """Solve op(A)X = alpha*B (L) or X op(A) = alpha*B (R); X overwrites B."""
    _tr(False, True, side, uplo, transa, diag, alpha, A, B)


def dtrmm(side, uplo, transa, diag, alpha, A, B):
    """fp64 TRMM (F4), in place."""
    _tr(True, False, side, uplo, transa, diag, alpha, A, B)


def dtrsm(side, uplo, transa, diag, alpha, A, B):
    """fp64 TRSM (F4); X overwrites B."""
    _tr(True, True, side, uplo, transa, diag, alpha, A, B)


def set_math_mode(mode):
    if isinstance(mode, str):
        mode = {"3xtf32": MATH_3XTF32, "simt": MATH_SIMT_FP32, "1xtf32": MATH_1XTF32,
                "tf32_bf16x": MATH_TF32_BF16X}[mode.lower()]
    _chk("blas3_set_math_mode", blas3_set_math_mode(mode))  # noqa: F821


def get_math_mode():
    return blas3_get_math_mode()  # noqa: F821


PATH_TCGEN05, PATH_SIMT, PATH_AUX, PATH_TRSM_PANEL = 0, 1, 2, 3

# tuning options (include/blas3.h BLAS3_OPT_*): name -> key
OPTIONS = {"gm_map": 0, "gm_min_gemm": 1, "gm_min_symm": 2, "gm_min_trmm": 3, "gm_min_trsm": 4,
           "tc_cta": 5, "tc_split": 6, "tc_static": 7, "pdl": 8, "trsm_nb": 9, "trsm_slabs": 10,
           "trsm_slab_min": 11, "trsm_reserve": 12, "trsm_geo_leaf": 13, "trsm_fused": 14,
           "trsm_first_ym": 15, "trsm_first_fused": 16, "trsm_first_split": 17, "trsm_first_all": 18, "tc_raster": 19,
           "tc_kc": 20, "tc_vec_store": 21, "max_sms": 22,
           "tc_c_prefetch": 23, "tc_c_async": 24, "trsm_panel": 25, "trsm_panel2": 26}


def set_option(name, value):
    """Set a tuning option (see include/blas3.h); raises on an invalid name/value."""
    key = OPTIONS[name] if isinstance(name, str) else int(name)
    if blas3_set_option(key, int(value)) != 0:  # noqa: F821
        raise ValueError(f"invalid option {name}={value}")


def get_option(name):
    key = OPTIONS[name] if isinstance(name, str) else int(name)
    return int(blas3_get_option(key))  # noqa: F821


class options:
    """Context manager: temporarily set tuning options, restore on exit."""

    def __init__(self, **kv):
        self.kv = kv
        self.old = {}

    def __enter__(self):
        for k, v in self.kv.items():
            self.old[k] = get_option(k)
            set_option(k, v)
        return self

    def __exit__(self, *a):
        for k, v in self.old.items():
            set_option(k, v)


def launch_count(path=None):
    """Kernels launched since load (all, or one route: 'tc', 'simt', 'aux', 'panel')."""
    if path is None:
        return int(blas3_launch_count())  # noqa: F821
    if isinstance(path, str):
        path = {"tc": PATH_TCGEN05, "simt": PATH_SIMT, "aux": PATH_AUX, "panel": PATH_TRSM_PANEL}[path]
    return int(blas3_launch_count_by_path(path))  # noqa: F821


__all__ = ["sgemm", "sgemm_streamed", "signal", "ssymm", "ssyrk", "ssyr2k", "strmm", "strsm", "set_math_mode",
           "get_math_mode", "launch_count", "colmajor", "from_fortran", "Blas3Error",
           "MATH_3XTF32", "MATH_SIMT_FP32", *EXPORTED]
