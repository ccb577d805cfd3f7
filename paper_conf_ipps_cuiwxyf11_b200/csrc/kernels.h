// kernels.h -- internal launcher interface between the routine drivers
// (abi.cu) and the device kernels.  Not part of the public C ABI.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include "problem.h"

namespace blas3 {

void note_launch(int path = 2);      // host-side launch counter (blas3_launch_count[_by_path])

// Structured GEMM kernels (all routines canonicalise to a Problem).
int launch_simt(const Problem &P, cudaStream_t s, int num_sms);
// tcgen05 3xTF32 path; returns 0, -1 (CUDA error) or -4 (TMA encode failure).
int launch_tc(const Problem &P, cudaStream_t s, int num_sms);
// TMA eligibility of one operand / the output (16-B pointer alignment, ld%4).
bool tc_eligible(const Problem &P);

// O(N^2) helpers.
int launch_scale(float *C, int64_t ldc, int64_t m, int64_t n, float beta, int tri,
                 cudaStream_t s);                       // C <- beta*C (beta=0 -> 0), tri: 0/1 lower/2 upper
int launch_copy(float *dst, int64_t ldd, const float *src, int64_t lds, int64_t m, int64_t n,
                cudaStream_t s);

// TRSM diagonal blocks: Dinv[b] = inv(op(A)_bb) for every nb x nb diagonal
// block b of op(A) (last block ragged, zero-padded to nb), column-major with
// leading dimension nb, stored consecutively.  lower_op: op(A) is lower.
int launch_trsm_diag_inv(const float *A, int64_t lda, int64_t n, int trans, int lower,
                         int unit, int nb, float *Dinv, cudaStream_t s);

}  // namespace blas3
