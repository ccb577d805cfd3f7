"""Seeded synthetic inputs shared by tests/, bench.py and the oracle checks.

This module holds NO arithmetic of the method (no products, no solves); it
only draws numbers.  It is the one module both the oracle side and the CUDA
side may use ("Input recipe").

Recipe (the paper is silent on distributions, reading Q20):
  * values U(-1, 1) fp32 (zero mean, no benign cancellation);
  * integer-valued matrices in [-4, 4] for the bit-exact pins;
  * symmetric operands: the referenced triangle random, the other strict
    triangle filled with a NaN sentinel (it must never be read, reading Q7);
  * triangular operands "diagonally dominant" (reading Q22): off-diagonal
    U(-1,1) in the referenced triangle, diag='N' -> a_ii = 1 + max(row, col)
    abs-sum of the off-diagonal part; diag='U' -> off-diagonal U(-1,1)/n and
    a NaN sentinel on the stored diagonal; the blank triangle is NaN;
  * padding rows (ld > rows) are NaN sentinels.
Seeds are counter-based: Philox keyed by a hash of (BASE_SEED, tags...), so
every matrix is reproducible from its name alone, independent of call order
and of how many GPUs/ranks participate.
"""
from __future__ import annotations

import hashlib

import numpy as np

BASE_SEED = 20111


def rng(*tags) -> np.random.Generator:
    h = hashlib.sha256(repr((BASE_SEED,) + tuple(tags)).encode()).digest()
    key = int.from_bytes(h[:16], "little")
    return np.random.Generator(np.random.Philox(key=key))


def _fortran(m: int, n: int, ld: int | None, fill=np.nan) -> np.ndarray:
    ld = max(1, m) if ld is None else ld
    if ld < max(1, m):
        raise ValueError("ld < rows")
    buf = np.full((n, ld), fill, dtype=np.float32).T  # F-order (ld x n)
    return buf


def uniform(m: int, n: int, *tags, ld: int | None = None, lo=-1.0, hi=1.0) -> np.ndarray:
    """U(lo, hi) fp32, column-major.  Returns the (ld x n) buffer; rows >= m are NaN."""
    buf = _fortran(m, n, ld)
    g = rng("uniform", m, n, *tags)
    Y = g.random((n, m), dtype=np.float32)
    Y *= np.float32(hi - lo)                # in place: the same fp32 ops, no 2nd temporary
    Y += np.float32(lo)
    buf[:m, :] = Y.T
    return buf


def integers(m: int, n: int, *tags, ld: int | None = None, lo=-4, hi=4) -> np.ndarray:
    """Integer-valued fp32 in [lo, hi], column-major (bit-exact pins)."""
    buf = _fortran(m, n, ld)
    g = rng("integers", m, n, *tags)
    buf[:m, :] = g.integers(lo, hi + 1, size=(n, m)).astype(np.float32).T
    return buf


def nan_outside(X: np.ndarray, uplo: str, keep_diag: bool = True) -> np.ndarray:
    """Fill the strict triangle NOT named by uplo (and optionally the
    diagonal) of the leading square block with NaN sentinels, in place."""
    n = min(X.shape[0], X.shape[1])
    lower = uplo.upper() == "L"
    d = 0 if keep_diag else 1
    for j in range(n):                      # column by column: no n x n index temporaries
        if lower:
            X[:j + d, j] = np.nan           # rows above the diagonal (and it, if not kept)
        else:
            X[j + 1 - d:n, j] = np.nan      # rows below the diagonal (and it, if not kept)
    return X


def symmetric_stored(n: int, uplo: str, *tags, ld: int | None = None, integer=False) -> np.ndarray:
    """Symmetric operand: only the `uplo` triangle is meaningful, the other
    strict triangle is NaN (P:144-148 real/shadow areas)."""
    X = integers(n, n, "sym", *tags, ld=ld) if integer else uniform(n, n, "sym", *tags, ld=ld)
    return nan_outside(X, uplo)


def triangular_dd(n: int, uplo: str, diag: str, *tags, ld: int | None = None) -> np.ndarray:
    """Diagonally dominant triangular operand (reading Q22)."""
    X = uniform(n, n, "tri", uplo, diag, *tags, ld=ld)
    sub = X[:n, :n]
    lower = uplo.upper() == "L"
    # strict triangle kept, the rest (diagonal included) set below; the
    # absolute row / column sums of the strict triangle are accumulated in
    # fp64 over column chunks (no n x n fp64 temporaries at large n)
    ch = 1024
    colsum = np.zeros(n)
    rowsum = np.zeros(n)
    for c0 in range(0, n, ch):
        blk = sub[:, c0:c0 + ch]
        strict = np.tril(blk, -1 - c0) if lower else np.triu(blk, 1 - c0)
        if diag.upper() == "U":
            blk[:, :] = strict / np.float32(max(n, 1))
        else:
            a = np.abs(strict.astype(np.float64))
            colsum[c0:c0 + ch] = a.sum(axis=0)
            rowsum += a.sum(axis=1)
            blk[:, :] = strict
    if diag.upper() == "U":
        nan_outside(X, uplo, keep_diag=False)
    else:
        dom = 1.0 + np.maximum(colsum, rowsum)
        np.fill_diagonal(sub, dom.astype(np.float32))
        nan_outside(X, uplo, keep_diag=True)
    return X


def triangular_integer(n: int, uplo: str, diag: str, *tags, ld: int | None = None,
                       lo=-2, hi=2) -> np.ndarray:
    """Integer-valued triangular operand for bit-exact TRMM pins (diag=N
    diagonal in [1, 2]; blank triangle NaN; diag=U stored diagonal NaN)."""
    X = integers(n, n, "trii", uplo, diag, *tags, ld=ld, lo=lo, hi=hi)
    sub = X[:n, :n]
    d = rng("trii-diag", n, uplo, diag, *tags).integers(1, 3, size=n).astype(np.float32)
    np.fill_diagonal(sub, d)
    nan_outside(X, uplo, keep_diag=diag.upper() != "U")
    return X


def sample_indices(count: int, nsample: int, *tags) -> np.ndarray:
    """Sorted distinct sample of output columns/rows for large-N parity."""
    if nsample >= count:
        return np.arange(count, dtype=np.int64)
    g = rng("sample", count, nsample, *tags)
    s = np.sort(g.choice(count, size=nsample, replace=False)).astype(np.int64)
    # always include both edges (first and ragged last tile)
    s[0], s[-1] = 0, count - 1
    return np.unique(s)
