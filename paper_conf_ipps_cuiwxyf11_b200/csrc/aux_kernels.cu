// aux_kernels.cu -- O(N^2) helpers (beta-scaling, copy-back) and the TRSM
// diagonal-block inversion (row A7).
//
// The paper's Adaptor_Solver binds the triangular part of each block's work
// to ONE thread ("binding_triangular(X, 0)", threadIdx.x==0 && threadIdx.y==0,
// P:236-244) because of the B[i] <- B[k], k<i dependence.  On B200
// that sequential step is moved off the critical path: every nb x nb
// diagonal block of op(A) is inverted up front, all blocks in parallel, and
// the sweep applies the inverses with tensor-core GEMMs (abi.cu).  Inside a
// block the inversion uses warp-level primitives: each warp inverts a 32x32
// diagonal sub-block by forward substitution with the row of L held by lane i
// and broadcast by __shfl_sync, then the off-diagonal 32x32 blocks follow by
// block forward substitution, one warp per block column.
#include <cuda_runtime.h>
#include "kernels.h"

namespace blas3 {

// ---------------------------------------------------------------- scale / copy
__global__ void scale_kernel(float *C, int64_t ldc, int64_t m, int64_t n, float beta, int tri) {
  int64_t total = m * n;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    int64_t r = e % m, c = e / m;
    if (tri == 1 && r < c) continue;
    if (tri == 2 && r > c) continue;
    float *p = C + r + c * ldc;
    *p = (beta == 0.f) ? 0.f : beta * *p;     // beta = 0: C not read (Q11)
  }
}

int launch_scale(float *C, int64_t ldc, int64_t m, int64_t n, float beta, int tri, cudaStream_t s) {
  if (m <= 0 || n <= 0) return 0;
  int64_t total = m * n;
  int64_t blocks = imin(cdiv(total, 256), 148 * 16);
  scale_kernel<<<(unsigned)blocks, 256, 0, s>>>(C, ldc, m, n, beta, tri);
  note_launch();
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

__global__ void copy_kernel(float *dst, int64_t ldd, const float *src, int64_t lds, int64_t m, int64_t n) {
  int64_t total = m * n;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    int64_t r = e % m, c = e / m;
    dst[r + c * ldd] = src[r + c * lds];
  }
}

int launch_copy(float *dst, int64_t ldd, const float *src, int64_t lds, int64_t m, int64_t n,
                cudaStream_t s) {
  if (m <= 0 || n <= 0) return 0;
  int64_t blocks = imin(cdiv(m * n, 256), 148 * 16);
  copy_kernel<<<(unsigned)blocks, 256, 0, s>>>(dst, ldd, src, lds, m, n);
  note_launch();
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

// ---------------------------------------------------------------- TRSM diag inverse
namespace {
constexpr int DNB = 128;          // diagonal block size (4 warps x 32)
constexpr int DLD = DNB + 1;      // padded smem row (bank-conflict free)
}

// One CTA (128 threads) per 128-block of L (the stored triangle of A in
// lower form); X = inv(L_bb) written into the panel-inverse workspace.
__global__ void __launch_bounds__(128)
trsm_diag_inv_kernel(const float *A, int64_t lda, int64_t n, int stored_lower, int unit,
                     float *Dinv, int64_t ldD) {
  extern __shared__ float sm[];
  float *L = sm;                  // [DNB][DLD]
  float *X = sm + DNB * DLD;      // [DNB][DLD]
  const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
  const int64_t i0 = (int64_t)blockIdx.x * DNB;
  const int nr = (int)imin(DNB, n - i0);

  // stage L (lower) and clear X; the blank triangle of A is never read (Q8)
  for (int c = 0; c < DNB; ++c) {
    const int r = tid;
    float v = 0.f;
    if (r < nr && c < nr) {
      if (r == c) v = unit ? 1.f : A[(i0 + r) + (i0 + r) * lda];
      else if (r > c) v = stored_lower ? A[(i0 + r) + (i0 + c) * lda] : A[(i0 + c) + (i0 + r) * lda];
    } else if (r == c) {
      v = 1.f;                     // identity padding of a ragged last block
    }
    L[r * DLD + c] = v;
    X[r * DLD + c] = 0.f;
  }
  __syncthreads();

  // phase 1: warp w inverts L_ww (32x32) -- lane i holds row i of L_ww,
  // lane j solves for column j of the inverse; rows broadcast by shuffles.
  {
    const int b = warp * 32;
    float lrow[32], x[32];
#pragma unroll
    for (int k = 0; k < 32; ++k) lrow[k] = L[(b + lane) * DLD + b + k];
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      float acc = (i == lane) ? 1.f : 0.f;
#pragma unroll
      for (int k = 0; k < i; ++k) acc = fmaf(-__shfl_sync(0xffffffffu, lrow[k], i), x[k], acc);
      x[i] = acc / __shfl_sync(0xffffffffu, lrow[i], i);
    }
#pragma unroll
    for (int i = 0; i < 32; ++i) X[(b + i) * DLD + b + lane] = x[i];
  }
  __syncthreads();

  // phase 2: block forward substitution, warp J owns block column J:
  //   X(I,J) = -inv(L_II) * sum_{K=J}^{I-1} L(I,K) X(K,J)
  {
    const int J = warp, c = J * 32 + lane;
    for (int I = J + 1; I < 4; ++I) {
      float t[32];
#pragma unroll
      for (int ii = 0; ii < 32; ++ii) t[ii] = 0.f;
      for (int K = J; K < I; ++K) {
        for (int kk = 0; kk < 32; ++kk) {
          float xk = X[(K * 32 + kk) * DLD + c];
#pragma unroll
          for (int ii = 0; ii < 32; ++ii) t[ii] = fmaf(L[(I * 32 + ii) * DLD + K * 32 + kk], xk, t[ii]);
        }
      }
#pragma unroll 4
      for (int ii = 0; ii < 32; ++ii) {
        float v = 0.f;
#pragma unroll
        for (int q = 0; q < 32; ++q) v = fmaf(X[(I * 32 + ii) * DLD + I * 32 + q], t[q], v);
        X[(I * 32 + ii) * DLD + c] = -v;
      }
      __syncwarp();
    }
  }
  __syncthreads();

  // write inv(L_bb) (lower, column-major) into its panel slot; padded rows/cols zero
  const int64_t bpp = ldD / DNB;                     // 128-blocks per panel
  float *D = Dinv + (blockIdx.x / bpp) * ldD * ldD + (blockIdx.x % bpp) * DNB * (1 + ldD);
  for (int c = 0; c < DNB; ++c) {
    const int r = tid;
    D[r + (int64_t)c * ldD] = (r < nr && c < nr) ? X[r * DLD + c] : 0.f;
  }
}

int launch_trsm_diag_inv(const float *A, int64_t lda, int64_t n, int stored_lower, int unit,
                         float *Dinv, int64_t ldD, cudaStream_t s) {
  if (ldD % DNB) return -1;
  const size_t smem = 2 * DNB * DLD * sizeof(float);
  static bool attr = false;
  if (!attr) {
    if (cudaFuncSetAttribute(trsm_diag_inv_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)smem) != cudaSuccess) return -1;
    attr = true;
  }
  int64_t blocks = cdiv(n, DNB);
  trsm_diag_inv_kernel<<<(unsigned)blocks, 128, smem, s>>>(A, lda, n, stored_lower, unit, Dinv, ldD);
  note_launch();
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

}  // namespace blas3
