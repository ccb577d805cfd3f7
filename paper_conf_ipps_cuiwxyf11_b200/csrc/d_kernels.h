// d_kernels.h -- internal interface of the fp64 family (d_kernel.cu <-> d_abi.cu).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace blas3 {

enum DOpKind : int32_t { DOP_DENSE = 0, DOP_SYM = 1, DOP_TRI = 2 };
// An operand X(r, k) of C = alpha * sum_seg Xa(r, k) Xb(c, k) + beta * C:
// X(r, k) = L(i, j) with (i, j) = trans ? (k + ko, r + ro) : (r + ro, k + ko), L
// the stored matrix (DENSE), sym(stored `lower` triangle) (SYM) or the
// triangle (`lower`, `unit` diagonal, blank = 0) (TRI); column-major, ld.
struct DOpnd {
  const double *p;
  int64_t ld;
  int32_t kind, trans, lower, unit;
  int64_t ro, ko;
};
struct DSeg { DOpnd a, b; int64_t K; };
struct DProblem {
  int64_t M, N;
  double alpha, beta;
  const double *C;            // read when beta != 0
  int64_t ldc;
  double *D;                  // written (may equal C)
  int64_t ldd;
  int32_t nseg, ctri;         // ctri: 0 all of C, 1 lower (r >= c), 2 upper (r <= c)
  DSeg seg[2];
};

int launch_dgemm(const DProblem &P, cudaStream_t s);
// inv(S_bb) of every 64-block on the diagonal of the order-nt TRI operand S
// (offsets 0): Dinv + 4096 b, 64 x 64 column-major (identity-padded)
int launch_dtri_inv64(const DOpnd &S, int64_t nt, double *Dinv, cudaStream_t s);
// a diagonal panel of R <= 512 rows in one launch (64-blocks in dependency
// order, their inverses at Dp), in place: rhs element i of right-hand side c
// at X[i*sx + c*sc]; S's offsets point at the panel's corner
int launch_dtrsm_panel(const DOpnd &S, const double *Dp, int R, double *X, int64_t sx, int64_t sc, int64_t nrhs,
                       cudaStream_t s);
// C <- beta * C (tri 0 all / 1 lower / 2 upper), beta == 0 -> exact zeros
int launch_dscale(double *C, int64_t ldc, int64_t m, int64_t n, double beta, int tri, cudaStream_t s);

// abi.cu: device check (sm_100, SM count) shared with the fp64 entry points
int abi_device_check(int &sms);

}  // namespace blas3
