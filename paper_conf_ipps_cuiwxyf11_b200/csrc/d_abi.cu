// d_abi.cu -- C ABI of the fp64 family: blas3_d{gemm,symm,syrk,syr2k,trmm,trsm}
// (SURVEY.md §8(f) F4).  Same argument lists, XERBLA codes, quick returns,
// alpha/beta special cases and stream semantics as the fp32 routines
// (include/blas3.h), double scalars and matrices.  Every routine is one (or,
// for TRSM, a sequence of) structured FP64 GEMM launch(es) of d_kernel.cu:
//   DGEMM  C = alpha op(A) op(B) + beta C
//   DSYMM  C = alpha sym(A) B + beta C  /  alpha B sym(A) + beta C   (A mirrored while staged)
//   DSYRK  C = alpha op(A) op(A)^T + beta C, uplo triangle only
//   DSYR2K C = alpha (op(A) op(B)^T + op(B) op(A)^T) + beta C, uplo triangle only
//   DTRMM  B = alpha op(tri(A)) B  /  alpha B op(tri(A))  (blank zero-filled while
//          staged; the product goes to stream-ordered scratch, then back to B)
//   DTRSM  op(tri(A)) X = alpha B  /  X op(tri(A)) = alpha B: B scaled by alpha,
//          then recursive halving in dependency order (Fig. 7):
//          solve the first half, ONE GEMM update of the second half by it,
//          solve the second half; leaves of <= 512 rows in ONE launch each
//          (dtrsm_panel: the panel's rows of 32 right-hand sides per CTA in
//          shared memory, 64-blocks in dependency order with the inverses of
//          all 64-blocks computed up front by substitution, dtri_inv64).
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/blas3.h"
#include "d_kernels.h"
#include "validate.h"

namespace blas3 {
namespace {

DOpnd dn(const double *p, int64_t ld, bool trans) {
  DOpnd o{};
  o.p = p; o.ld = ld; o.kind = DOP_DENSE; o.trans = trans ? 1 : 0;
  return o;
}
DOpnd dsym(const double *p, int64_t ld, bool lower) {
  DOpnd o{};
  o.p = p; o.ld = ld; o.kind = DOP_SYM; o.lower = lower ? 1 : 0;
  return o;
}
DOpnd dtri(const double *p, int64_t ld, bool lower, bool trans, bool unit, int64_t ro = 0, int64_t ko = 0) {
  DOpnd o{};
  o.p = p; o.ld = ld; o.kind = DOP_TRI; o.lower = lower ? 1 : 0; o.trans = trans ? 1 : 0;
  o.unit = unit ? 1 : 0; o.ro = ro; o.ko = ko;
  return o;
}
DProblem dprob(int64_t M, int64_t N, double alpha, double beta, const double *C, int64_t ldc, double *D,
               int64_t ldd) {
  DProblem P{};
  P.M = M; P.N = N; P.alpha = alpha; P.beta = beta; P.C = C; P.ldc = ldc; P.D = D; P.ldd = ldd;
  P.nseg = 1;
  return P;
}
int dfinish(int rc) {
  if (rc) return rc;
  return cudaGetLastError() == cudaSuccess ? 0 : BLAS3_ERR_CUDA;
}
int drun(const DProblem &P, cudaStream_t s) { return launch_dgemm(P, s) ? BLAS3_ERR_CUDA : 0; }

struct DScratch {
  double *p = nullptr;
  cudaStream_t s = nullptr;
  ~DScratch() { if (p) cudaFreeAsync(p, s); }
  int get(size_t bytes, cudaStream_t st) {
    s = st;
    if (cudaMallocAsync((void **)&p, bytes, st) != cudaSuccess) { cudaGetLastError(); p = nullptr; return BLAS3_ERR_ALLOC; }
    return 0;
  }
};

constexpr int64_t DNB = 64;          // diagonal blocks (inverted by dtri_inv64)
constexpr int64_t DPANEL = 512;      // recursion leaves (dtrsm_panel)

}  // namespace
}  // namespace blas3

using namespace blas3;

extern "C" {

int blas3_dgemm(char transa, char transb, int64_t m, int64_t n, int64_t k, double alpha, const double *A,
                int64_t lda, const double *B, int64_t ldb, double beta, double *C, int64_t ldc,
                blas3_stream_t stream) {
  if (const int v = v_gemm(transa, transb, m, n, k, lda, ldb, ldc)) return v;
  if (m == 0 || n == 0 || ((alpha == 0.0 || k == 0) && beta == 1.0)) return 0;
  if (!C) return 12;
  const bool reads = alpha != 0.0 && k > 0;
  if (reads && !A) return 7;
  if (reads && !B) return 9;
  int sms, rc = abi_device_check(sms);
  if (rc) return rc;
  cudaStream_t s = (cudaStream_t)stream;
  if (!reads) return dfinish(launch_dscale(C, ldc, m, n, beta, 0, s) ? BLAS3_ERR_CUDA : 0);
  DProblem P = dprob(m, n, alpha, beta, C, ldc, C, ldc);
  P.seg[0].a = dn(A, lda, up(transa) != 'N');         // Xa(r,k) = op(A)(r,k)
  P.seg[0].b = dn(B, ldb, up(transb) == 'N');         // Xb(c,k) = op(B)(k,c)
  P.seg[0].K = k;
  return dfinish(drun(P, s));
}

int blas3_dsymm(char side, char uplo, int64_t m, int64_t n, double alpha, const double *A, int64_t lda,
                const double *B, int64_t ldb, double beta, double *C, int64_t ldc, blas3_stream_t stream) {
  if (const int v = v_symm(side, uplo, m, n, lda, ldb, ldc)) return v;
  if (m == 0 || n == 0 || (alpha == 0.0 && beta == 1.0)) return 0;
  if (!C) return 11;
  if (alpha != 0.0 && !A) return 6;
  if (alpha != 0.0 && !B) return 8;
  int sms, rc = abi_device_check(sms);
  if (rc) return rc;
  cudaStream_t s = (cudaStream_t)stream;
  if (alpha == 0.0) return dfinish(launch_dscale(C, ldc, m, n, beta, 0, s) ? BLAS3_ERR_CUDA : 0);
  const bool left = up(side) == 'L', lower = up(uplo) == 'L';
  DProblem P = dprob(m, n, alpha, beta, C, ldc, C, ldc);
  if (left) {                 // Xa = sym(A) (m x m), Xb(c,k) = B(k,c)
    P.seg[0].a = dsym(A, lda, lower);
    P.seg[0].b = dn(B, ldb, true);
    P.seg[0].K = m;
  } else {                    // Xa = B, Xb(c,k) = sym(A)(k,c) = sym(A)(c,k)
    P.seg[0].a = dn(B, ldb, false);
    P.seg[0].b = dsym(A, lda, lower);
    P.seg[0].K = n;
  }
  return dfinish(drun(P, s));
}

static int dsyrk_common(bool two, char uplo, char trans, int64_t n, int64_t k, double alpha, const double *A,
                        int64_t lda, const double *B, int64_t ldb, double beta, double *C, int64_t ldc,
                        cudaStream_t s) {
  const bool lower = up(uplo) == 'L', ta = up(trans) != 'N';
  const int tri = lower ? 1 : 2;
  if (n == 0 || ((alpha == 0.0 || k == 0) && beta == 1.0)) return 0;
  if (!C) return two ? 11 : 9;
  const bool reads = alpha != 0.0 && k > 0;
  if (reads && !A) return 6;
  if (two && reads && !B) return 8;
  int sms, rc = abi_device_check(sms);
  if (rc) return rc;
  if (!reads) return dfinish(launch_dscale(C, ldc, n, n, beta, tri, s) ? BLAS3_ERR_CUDA : 0);
  DProblem P = dprob(n, n, alpha, beta, C, ldc, C, ldc);
  P.ctri = tri;
  // trans=N: op(A) = A (n x k): X(r,k) = A(r,k); trans=T: X(r,k) = A(k,r)
  P.seg[0].a = dn(A, lda, ta);
  P.seg[0].b = dn(two ? B : A, two ? ldb : lda, ta);
  P.seg[0].K = k;
  if (two) {
    P.nseg = 2;
    P.seg[1].a = dn(B, ldb, ta);
    P.seg[1].b = dn(A, lda, ta);
    P.seg[1].K = k;
  }
  return dfinish(drun(P, s));
}

int blas3_dsyrk(char uplo, char trans, int64_t n, int64_t k, double alpha, const double *A, int64_t lda,
                double beta, double *C, int64_t ldc, blas3_stream_t stream) {
  if (const int v = v_syrk(false, uplo, trans, n, k, lda, 0, ldc)) return v;
  return dsyrk_common(false, uplo, trans, n, k, alpha, A, lda, nullptr, 0, beta, C, ldc, (cudaStream_t)stream);
}

int blas3_dsyr2k(char uplo, char trans, int64_t n, int64_t k, double alpha, const double *A, int64_t lda,
                 const double *B, int64_t ldb, double beta, double *C, int64_t ldc, blas3_stream_t stream) {
  if (const int v = v_syrk(true, uplo, trans, n, k, lda, ldb, ldc)) return v;
  return dsyrk_common(true, uplo, trans, n, k, alpha, A, lda, B, ldb, beta, C, ldc, (cudaStream_t)stream);
}

int blas3_dtrmm(char side, char uplo, char transa, char diag, int64_t m, int64_t n, double alpha,
                const double *A, int64_t lda, double *B, int64_t ldb, blas3_stream_t stream) {
  if (const int v = v_tr(side, uplo, transa, diag, m, n, lda, ldb)) return v;
  if (m == 0 || n == 0) return 0;
  if (!B) return 10;
  if (alpha != 0.0 && !A) return 8;
  int sms, rc = abi_device_check(sms);
  if (rc) return rc;
  cudaStream_t s = (cudaStream_t)stream;
  if (alpha == 0.0) return dfinish(launch_dscale(B, ldb, m, n, 0.0, 0, s) ? BLAS3_ERR_CUDA : 0);
  const bool left = up(side) == 'L', lower = up(uplo) == 'L', ta = up(transa) != 'N', unit = up(diag) == 'U';
  DScratch W;
  if ((rc = W.get((size_t)m * n * sizeof(double), s))) return rc;
  DProblem P = dprob(m, n, alpha, 0.0, nullptr, 0, W.p, m);
  if (left) {                 // W = alpha op(T) B: Xa(r,k) = op(T)(r,k), Xb(c,k) = B(k,c)
    P.seg[0].a = dtri(A, lda, lower, ta, unit);
    P.seg[0].b = dn(B, ldb, true);
    P.seg[0].K = m;
  } else {                    // W = alpha B op(T): Xa = B, Xb(c,k) = op(T)(k,c) = op(T)^T(c,k)
    P.seg[0].a = dn(B, ldb, false);
    P.seg[0].b = dtri(A, lda, lower, !ta, unit);
    P.seg[0].K = n;
  }
  if ((rc = drun(P, s))) return rc;
  if (cudaMemcpy2DAsync(B, ldb * sizeof(double), W.p, m * sizeof(double), m * sizeof(double), n,
                        cudaMemcpyDeviceToDevice, s) != cudaSuccess)
    return BLAS3_ERR_CUDA;
  return dfinish(0);
}

int blas3_dtrsm(char side, char uplo, char transa, char diag, int64_t m, int64_t n, double alpha,
                const double *A, int64_t lda, double *B, int64_t ldb, blas3_stream_t stream) {
  if (const int v = v_tr(side, uplo, transa, diag, m, n, lda, ldb)) return v;
  if (m == 0 || n == 0) return 0;
  if (!B) return 10;
  if (alpha != 0.0 && !A) return 8;
  int sms, rc = abi_device_check(sms);
  if (rc) return rc;
  cudaStream_t s = (cudaStream_t)stream;
  if (alpha != 1.0 && launch_dscale(B, ldb, m, n, alpha, 0, s)) return BLAS3_ERR_CUDA;
  if (alpha == 0.0) return dfinish(0);
  const bool left = up(side) == 'L', lower = up(uplo) == 'L', ta = up(transa) != 'N', unit = up(diag) == 'U';
  // The system per right-hand side: S y = b.  Left: S = op(T) over B's rows,
  // one right-hand side per column.  Right (X op(T) = B, i.e. op(T)^T x_c = b_c
  // for every row c): S = op(T)^T over B's columns.  S lower -> forward order.
  const bool strans = left ? ta : !ta;
  const bool s_lower = lower != strans;
  const int64_t nt = left ? m : n, nrhs = left ? n : m;
  const int64_t sx = left ? 1 : ldb, sc = left ? ldb : 1;   // element i of right-hand side c
  // the inverses of all 64-blocks of S in one launch, then the recursion
  // down to panels of <= DPANEL rows, each solved by one launch
  DScratch Dinv;
  if ((rc = Dinv.get((size_t)((nt + DNB - 1) / DNB) * DNB * DNB * sizeof(double), s))) return rc;
  if (launch_dtri_inv64(dtri(A, lda, lower, strans, unit), nt, Dinv.p, s)) return BLAS3_ERR_CUDA;
  // rows [lo, hi) of the system, in dependency order by recursive halving
  int err = 0;
  auto solve = [&](auto &&self, int64_t lo, int64_t hi) -> void {
    if (err) return;
    const int64_t w = hi - lo;
    if (w <= DPANEL) {                                // lo is a multiple of 64
      if (launch_dtrsm_panel(dtri(A, lda, lower, strans, unit, lo, lo), Dinv.p + (lo / DNB) * DNB * DNB, (int)w,
                             B + lo * sx, sx, sc, nrhs, s))
        err = BLAS3_ERR_CUDA;
      return;
    }
    const int64_t h = ((w / 2 + DNB - 1) / DNB) * DNB, mid = lo + h;     // first half: whole 64-blocks
    const int64_t f_lo = s_lower ? lo : mid, f_hi = s_lower ? mid : hi;   // solved first
    const int64_t s_lo = s_lower ? mid : lo, s_hi = s_lower ? hi : mid;   // updated, then solved
    self(self, f_lo, f_hi);
    if (err) return;
    // y_s -= S(s, f) y_f
    if (left) {   // B(s, :) -= S(s, f) X(f, :): Xa(r,k) = S(s_lo + r, f_lo + k), Xb(c,k) = B(f_lo + k, c)
      DProblem P = dprob(s_hi - s_lo, n, -1.0, 1.0, B + s_lo, ldb, B + s_lo, ldb);
      P.seg[0].a = dtri(A, lda, lower, strans, unit, s_lo, f_lo);
      P.seg[0].b = dn(B + f_lo, ldb, true);
      P.seg[0].K = f_hi - f_lo;
      if (drun(P, s)) err = BLAS3_ERR_CUDA;
    } else {      // B(:, s) -= X(:, f) S(s, f)^T: Xa(r,k) = B(r, f_lo + k), Xb(c,k) = S(s_lo + c, f_lo + k)
      DProblem P = dprob(m, s_hi - s_lo, -1.0, 1.0, B + s_lo * ldb, ldb, B + s_lo * ldb, ldb);
      P.seg[0].a = dn(B + f_lo * ldb, ldb, false);
      P.seg[0].b = dtri(A, lda, lower, strans, unit, s_lo, f_lo);
      P.seg[0].K = f_hi - f_lo;
      if (drun(P, s)) err = BLAS3_ERR_CUDA;
    }
    self(self, s_lo, s_hi);
  };
  solve(solve, 0, nt);
  return dfinish(err);
}

}  // extern "C"
