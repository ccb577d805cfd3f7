// validate.h -- reference-BLAS argument checks (XERBLA numbering), shared by
// the fp32 (abi.cu) and fp64 (d_abi.cu) entry points.  Each returns 0 or the
// 1-based position of the first invalid argument; the stream is appended
// after the BLAS arguments, so the positions are the reference ones
// (include/blas3.h lists them per routine).
#pragma once
#include <ctype.h>
#include <stdint.h>

namespace blas3 {

static inline int up(char c) { return toupper((unsigned char)c); }
static inline bool is_trans(char c) { int u = up(c); return u == 'N' || u == 'T' || u == 'C'; }
static inline bool is_side(char c) { int u = up(c); return u == 'L' || u == 'R'; }
static inline bool is_uplo(char c) { int u = up(c); return u == 'L' || u == 'U'; }
static inline bool is_diag(char c) { int u = up(c); return u == 'N' || u == 'U'; }
static inline int64_t mx1(int64_t v) { return v > 1 ? v : 1; }

static inline int v_gemm(char transa, char transb, int64_t m, int64_t n, int64_t k, int64_t lda, int64_t ldb,
                         int64_t ldc) {
  const bool ta = up(transa) != 'N', tb = up(transb) != 'N';
  if (!is_trans(transa)) return 1;
  if (!is_trans(transb)) return 2;
  if (m < 0) return 3;
  if (n < 0) return 4;
  if (k < 0) return 5;
  if (lda < mx1(ta ? k : m)) return 8;
  if (ldb < mx1(tb ? n : k)) return 10;
  if (ldc < mx1(m)) return 13;
  return 0;
}
static inline int v_symm(char side, char uplo, int64_t m, int64_t n, int64_t lda, int64_t ldb, int64_t ldc) {
  if (!is_side(side)) return 1;
  if (!is_uplo(uplo)) return 2;
  if (m < 0) return 3;
  if (n < 0) return 4;
  if (lda < mx1(up(side) == 'L' ? m : n)) return 7;
  if (ldb < mx1(m)) return 9;
  if (ldc < mx1(m)) return 12;
  return 0;
}
// SYRK (two = false: ldb unused) and SYR2K
static inline int v_syrk(bool two, char uplo, char trans, int64_t n, int64_t k, int64_t lda, int64_t ldb,
                         int64_t ldc) {
  const bool ta = up(trans) != 'N';
  if (!is_uplo(uplo)) return 1;
  if (!is_trans(trans)) return 2;
  if (n < 0) return 3;
  if (k < 0) return 4;
  if (lda < mx1(ta ? k : n)) return 7;
  if (two && ldb < mx1(ta ? k : n)) return 9;
  if (ldc < mx1(n)) return two ? 12 : 10;
  return 0;
}
// STRMM / STRSM
static inline int v_tr(char side, char uplo, char transa, char diag, int64_t m, int64_t n, int64_t lda,
                       int64_t ldb) {
  if (!is_side(side)) return 1;
  if (!is_uplo(uplo)) return 2;
  if (!is_trans(transa)) return 3;
  if (!is_diag(diag)) return 4;
  if (m < 0) return 5;
  if (n < 0) return 6;
  if (lda < mx1(up(side) == 'L' ? m : n)) return 9;
  if (ldb < mx1(m)) return 11;
  return 0;
}

}  // namespace blas3
