"""fp64 CPU oracle for the six fp32 Level-3 BLAS routines -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and the ``--impl reference`` arm) may import this module.
The product package ``paper_conf_ipps_cuiwxyf11_b200`` never imports it and
shares no code with it ("Oracle").

The arithmetic lives in ``oracle.c`` (plain C, fp64 accumulation, BLAS
definitions; citations to /root/reference/PAPER.md are in that file).  This
module only builds the shared library and marshals numpy arrays.

Every function takes fp32 numpy arrays in column-major ("Fortran") order, as
BLAS3 does, and returns an fp64 array holding the selected
output columns (rows for ``strsm`` with side='R').  ``sel=None`` means all.

Parity status: all six functions are pinned (tests/test_oracle.py); none is
"parity unpinned".
"""
from __future__ import annotations

import ctypes
import hashlib
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

_i64 = ctypes.c_int64
_dbl = ctypes.c_double
_ptr = ctypes.c_void_p
_chr = ctypes.c_char


_CMD = ["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c99", "-Wall"]


def build(force: bool = False) -> str:
    """Compile oracle.c into liboracle.so (gcc -O2 -fopenmp); rebuilt when the
    SHA-256 of the source and command (stored in liboracle.so.sha256) changes."""
    with open(_SRC, "rb") as f:
        digest = hashlib.sha256(f.read() + repr(_CMD).encode()).hexdigest()
    stamp = _LIB + ".sha256"
    fresh = os.path.exists(_LIB) and os.path.exists(stamp) and open(stamp).read().strip() == digest
    if force or not fresh:
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call([*_CMD, "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
        with open(stamp, "w") as f:
            f.write(digest + "\n")
    return _LIB


def _load():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        _lib.oracle_num_threads.restype = ctypes.c_int
    return _lib


def num_threads() -> int:
    return int(_load().oracle_num_threads())


def _f32(x):
    x = np.asarray(x)
    if x.dtype != np.float32:
        raise TypeError("oracle inputs must be float32")
    if x.ndim != 2:
        raise ValueError("oracle inputs must be 2-D")
    return np.asfortranarray(x)


def _ld(x):
    return max(1, x.shape[0])


def _p(x):
    return x.ctypes.data_as(_ptr)


def _sel(sel, count):
    if sel is None:
        return None, count, None
    s = np.ascontiguousarray(np.asarray(sel, dtype=np.int64))
    if s.size and (s.min() < 0 or s.max() >= count):
        raise IndexError("sample index out of range")
    return s, s.size, s.ctypes.data_as(_ptr)


def _c(ch):
    return _chr(ch.encode() if isinstance(ch, str) else ch)


def sgemm(transa, transb, alpha, A, B, beta, C, sel=None):
    """C <- alpha*op(A)*op(B) + beta*C. Returns fp64 m x nsel."""
    A, B, C = _f32(A), _f32(B), _f32(C)
    m, n = C.shape
    k = A.shape[0] if transa.upper() != "N" else A.shape[1]
    s, ns, sp = _sel(sel, n)
    out = np.zeros((m, ns), dtype=np.float64, order="F")
    _load().oracle_sgemm(_c(transa), _c(transb), _i64(m), _i64(n), _i64(k), _dbl(alpha),
                         _p(A), _i64(_ld(A)), _p(B), _i64(_ld(B)), _dbl(beta), _p(C),
                         _i64(_ld(C)), _p(out), _i64(max(1, m)), sp, _i64(ns))
    return out


def ssymm(side, uplo, alpha, A, B, beta, C, sel=None):
    """side=L: C <- alpha*A*B + beta*C; side=R: C <- alpha*B*A + beta*C."""
    A, B, C = _f32(A), _f32(B), _f32(C)
    m, n = C.shape
    s, ns, sp = _sel(sel, n)
    out = np.zeros((m, ns), dtype=np.float64, order="F")
    _load().oracle_ssymm(_c(side), _c(uplo), _i64(m), _i64(n), _dbl(alpha), _p(A),
                         _i64(_ld(A)), _p(B), _i64(_ld(B)), _dbl(beta), _p(C), _i64(_ld(C)),
                         _p(out), _i64(max(1, m)), sp, _i64(ns))
    return out


def ssyrk(uplo, trans, alpha, A, beta, C, sel=None):
    """C <- alpha*op(A)*op(A)^T + beta*C on the uplo triangle; rest copied."""
    A, C = _f32(A), _f32(C)
    n = C.shape[0]
    k = A.shape[1] if trans.upper() == "N" else A.shape[0]
    s, ns, sp = _sel(sel, n)
    out = np.zeros((n, ns), dtype=np.float64, order="F")
    _load().oracle_ssyrk(_c(uplo), _c(trans), _i64(n), _i64(k), _dbl(alpha), _p(A),
                         _i64(_ld(A)), _dbl(beta), _p(C), _i64(_ld(C)), _p(out),
                         _i64(max(1, n)), sp, _i64(ns))
    return out


def ssyr2k(uplo, trans, alpha, A, B, beta, C, sel=None):
    """C <- alpha*(op(A)op(B)^T + op(B)op(A)^T) + beta*C on the uplo triangle."""
    A, B, C = _f32(A), _f32(B), _f32(C)
    n = C.shape[0]
    k = A.shape[1] if trans.upper() == "N" else A.shape[0]
    s, ns, sp = _sel(sel, n)
    out = np.zeros((n, ns), dtype=np.float64, order="F")
    _load().oracle_ssyr2k(_c(uplo), _c(trans), _i64(n), _i64(k), _dbl(alpha), _p(A),
                          _i64(_ld(A)), _p(B), _i64(_ld(B)), _dbl(beta), _p(C),
                          _i64(_ld(C)), _p(out), _i64(max(1, n)), sp, _i64(ns))
    return out


def strmm(side, uplo, transa, diag, alpha, A, B, sel=None):
    """side=L: alpha*op(T)*B; side=R: alpha*B*op(T)."""
    A, B = _f32(A), _f32(B)
    m, n = B.shape
    s, ns, sp = _sel(sel, n)
    out = np.zeros((m, ns), dtype=np.float64, order="F")
    _load().oracle_strmm(_c(side), _c(uplo), _c(transa), _c(diag), _i64(m), _i64(n),
                         _dbl(alpha), _p(A), _i64(_ld(A)), _p(B), _i64(_ld(B)), _p(out),
                         _i64(max(1, m)), sp, _i64(ns))
    return out


def strsm(side, uplo, transa, diag, alpha, A, B, sel=None):
    """Solve op(T)X = alpha*B (L) or X op(T) = alpha*B (R).

    side=L: ``sel`` lists columns, result is m x nsel.
    side=R: ``sel`` lists ROWS, result is nsel x n.
    """
    A, B = _f32(A), _f32(B)
    m, n = B.shape
    left = side.upper() == "L"
    s, ns, sp = _sel(sel, n if left else m)
    shape = (m, ns) if left else (ns, n)
    out = np.zeros(shape, dtype=np.float64, order="F")
    _load().oracle_strsm(_c(side), _c(uplo), _c(transa), _c(diag), _i64(m), _i64(n),
                         _dbl(alpha), _p(A), _i64(_ld(A)), _p(B), _i64(_ld(B)), _p(out),
                         _i64(max(1, shape[0])), sp, _i64(ns))
    return out
