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
#include <atomic>
#include "kernels.h"

namespace blas3 {

// ---------------------------------------------------------------- scale / copy
// Column-major 2-D grids: blockIdx.x covers rows (4 per thread when the
// columns are 16-byte aligned), blockIdx.y strides over columns, CU unrolled
// so each thread keeps several independent accesses in flight.  HBM-bound:
// 4 (scale, beta != 0: 8) bytes per element.
namespace {
constexpr int AUX_T = 256, CU = 4;
inline dim3 aux_grid(int64_t m, int64_t n, bool vec) {
  const int64_t rows_per_cta = AUX_T * (vec ? 4 : 1);
  const int64_t gx = cdiv(m, rows_per_cta);
  const int64_t gy = imin(cdiv(n, CU), imax(1, (148 * 32) / imax(1, gx)));
  return dim3((unsigned)gx, (unsigned)imin(gy, 65535));
}
inline bool aligned16(const void *p, int64_t ld, int64_t m) {
  return ((uintptr_t)p % 16 == 0) && ld % 4 == 0 && m % 4 == 0;
}
}  // namespace

template <bool VEC>
__global__ void __launch_bounds__(AUX_T)
scale_kernel(float *C, int64_t ldc, int64_t m, int64_t n, float beta, int tri) {
  const int64_t r = ((int64_t)blockIdx.x * AUX_T + threadIdx.x) * (VEC ? 4 : 1);
  if (r >= m) return;
  for (int64_t c0 = (int64_t)blockIdx.y * CU; c0 < n; c0 += (int64_t)gridDim.y * CU) {
#pragma unroll
    for (int u = 0; u < CU; ++u) {
      const int64_t c = c0 + u;
      if (c >= n) break;
      float *p = C + r + c * ldc;
      if (VEC && tri == 0) {
        float4 v = beta == 0.f ? make_float4(0.f, 0.f, 0.f, 0.f) : *reinterpret_cast<float4 *>(p);
        if (beta != 0.f) { v.x *= beta; v.y *= beta; v.z *= beta; v.w *= beta; }
        *reinterpret_cast<float4 *>(p) = v;
      } else {
#pragma unroll
        for (int e = 0; e < (VEC ? 4 : 1); ++e) {
          const int64_t rr = r + e;
          if (rr >= m || (tri == 1 && rr < c) || (tri == 2 && rr > c)) continue;
          p[e] = (beta == 0.f) ? 0.f : beta * p[e];     // beta = 0: C not read (Q11)
        }
      }
    }
  }
}

int launch_scale(float *C, int64_t ldc, int64_t m, int64_t n, float beta, int tri, cudaStream_t s) {
  if (m <= 0 || n <= 0) return 0;
  const bool vec = aligned16(C, ldc, m);
  const dim3 g = aux_grid(m, n, vec);
  if (vec) scale_kernel<true><<<g, AUX_T, 0, s>>>(C, ldc, m, n, beta, tri);
  else scale_kernel<false><<<g, AUX_T, 0, s>>>(C, ldc, m, n, beta, tri);
  note_launch();
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

template <bool VEC>
__global__ void __launch_bounds__(AUX_T)
copy_kernel(float *dst, int64_t ldd, const float *src, int64_t lds, int64_t m, int64_t n) {
  const int64_t r = ((int64_t)blockIdx.x * AUX_T + threadIdx.x) * (VEC ? 4 : 1);
  if (r >= m) return;
  for (int64_t c0 = (int64_t)blockIdx.y * CU; c0 < n; c0 += (int64_t)gridDim.y * CU) {
    if (VEC) {
      float4 v[CU];
#pragma unroll
      for (int u = 0; u < CU; ++u)
        if (c0 + u < n) v[u] = __ldcs(reinterpret_cast<const float4 *>(src + r + (c0 + u) * lds));
#pragma unroll
      for (int u = 0; u < CU; ++u)
        if (c0 + u < n) __stcs(reinterpret_cast<float4 *>(dst + r + (c0 + u) * ldd), v[u]);
    } else {
#pragma unroll
      for (int u = 0; u < CU; ++u)
        if (c0 + u < n) dst[r + (c0 + u) * ldd] = src[r + (c0 + u) * lds];
    }
  }
}

int launch_copy(float *dst, int64_t ldd, const float *src, int64_t lds, int64_t m, int64_t n,
                cudaStream_t s) {
  if (m <= 0 || n <= 0) return 0;
  const bool vec = aligned16(dst, ldd, m) && aligned16(src, lds, m);
  const dim3 g = aux_grid(m, n, vec);
  if (vec) copy_kernel<true><<<g, AUX_T, 0, s>>>(dst, ldd, src, lds, m, n);
  else copy_kernel<false><<<g, AUX_T, 0, s>>>(dst, ldd, src, lds, m, n);
  note_launch();
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

// ---------------------------------------------------------------- GM_map materialisation
// The paper's Adaptor rule 2 ("GM_map"): the structured operand is
// rewritten once in global memory in the orientation the GEMM kernel stages
// best (MN-major, i.e. plain column-major), so the hot kernel runs its dense
// / zero-blank path.  dst(r, c), 0 <= r < rows, 0 <= c < cols, is
//   MAT_TRANS : src(c, r)
//   MAT_SYM   : the stored triangle (lower: r >= c) selected, else its mirror
//               (selection, never src + src^T - diag, reading Q7)
//   MAT_TRI   : op(T)(r, c) with T the stored triangle, 0 in the blank part,
//               1 on the diagonal when unit (the stored diagonal is not read)
// 64 x 64 output tiles through shared memory: the direct and the mirrored
// source tiles are each read with coalesced column accesses (16-byte vectors
// when the source allows), and only the one(s) the tile needs (both only on
// diagonal tiles); 16 loads per thread are in flight before the exchange.
// HBM-bound: <= 4 B read + 4 B written per element.
namespace {
constexpr int MT = 64, MTH = 256, MPAD = MT + 4, MPADM = MT + 1;   // float4 rows / conflict-free transpose
}
template <bool VEC>
__global__ void __launch_bounds__(MTH)
materialize_kernel(float *dst, int64_t ldd, const float *src, int64_t lds, int64_t rows,
                   int64_t cols, int mode, int lower, int trans, int unit) {
  __shared__ __align__(16) float dir[MT][MPAD];   // dir[c][r] = src(r0 + r, c0 + c)
  __shared__ float mir[MT][MPADM];                // mir[c][r] = src(c0 + c, r0 + r)
  const int64_t r0 = (int64_t)blockIdx.x * MT, c0 = (int64_t)blockIdx.y * MT;
  const int t = threadIdx.x;
  bool need_dir, need_mir;
  if (mode == MAT_TRANS) { need_dir = false; need_mir = true; }
  else {
    // a tile strictly below (r > c everywhere) or above the diagonal needs one side only
    const bool below = r0 >= c0 + MT, above = c0 >= r0 + MT;
    if (mode == MAT_SYM) {
      need_dir = !(below ? !lower : above ? lower : false);
      need_mir = !(below ? lower : above ? !lower : false);
    } else {
      // op(T)(r,c) = trans ? T(c,r) : T(r,c), nonzero iff (r >= c) == (lower != trans)
      const bool blank = (lower != trans) ? above : below;
      need_dir = !trans && !blank;
      need_mir = trans && !blank;
    }
  }
  // thread t covers 4 consecutive elements (e4 .. e4+3) of "line" ln, 4 times
  if (need_dir) {
#pragma unroll
    for (int it = 0; it < 4; ++it) {
      const int idx = t + it * MTH, ln = idx / 16, e4 = (idx % 16) * 4;   // column c0+ln, rows r0+e4..
      const int64_t r = r0 + e4, c = c0 + ln;
      float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
      if (c < cols) {
        const float *p = src + r + c * lds;
        if (VEC && r + 3 < rows) v = __ldg(reinterpret_cast<const float4 *>(p));
        else {
          if (r < rows) v.x = __ldg(p);
          if (r + 1 < rows) v.y = __ldg(p + 1);
          if (r + 2 < rows) v.z = __ldg(p + 2);
          if (r + 3 < rows) v.w = __ldg(p + 3);
        }
      }
      *reinterpret_cast<float4 *>(&dir[ln][e4]) = v;
    }
  }
  if (need_mir) {
#pragma unroll
    for (int it = 0; it < 4; ++it) {
      const int idx = t + it * MTH, ln = idx / 16, e4 = (idx % 16) * 4;   // src column r0+ln, rows c0+e4..
      const int64_t j = r0 + ln, i = c0 + e4;
      float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
      if (j < rows) {
        const float *p = src + i + j * lds;
        if (VEC && i + 3 < cols) v = __ldg(reinterpret_cast<const float4 *>(p));
        else {
          if (i < cols) v.x = __ldg(p);
          if (i + 1 < cols) v.y = __ldg(p + 1);
          if (i + 2 < cols) v.z = __ldg(p + 2);
          if (i + 3 < cols) v.w = __ldg(p + 3);
        }
      }
      mir[e4][ln] = v.x; mir[e4 + 1][ln] = v.y; mir[e4 + 2][ln] = v.z; mir[e4 + 3][ln] = v.w;
    }
  }
  __syncthreads();
#pragma unroll
  for (int it = 0; it < 4; ++it) {
    const int idx = t + it * MTH, ln = idx / 16, e4 = (idx % 16) * 4;       // column c0+ln, rows r0+e4..
    const int64_t c = c0 + ln;
    if (c >= cols) continue;
    float v[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int64_t r = r0 + e4 + q;
      if (mode == MAT_TRANS) v[q] = mir[ln][e4 + q];
      else if (mode == MAT_SYM) {
        const bool direct = lower ? (r >= c) : (r <= c);
        v[q] = direct ? dir[ln][e4 + q] : mir[ln][e4 + q];
      } else {
        const int64_t ti = trans ? c : r, tj = trans ? r : c;     // T(ti, tj)
        const bool nz = lower ? (ti >= tj) : (ti <= tj);
        v[q] = !nz ? 0.f : (unit && ti == tj) ? 1.f : (trans ? mir[ln][e4 + q] : dir[ln][e4 + q]);
      }
    }
    const int64_t r = r0 + e4;
    float *p = dst + r + c * ldd;
    if (VEC && r + 3 < rows) *reinterpret_cast<float4 *>(p) = make_float4(v[0], v[1], v[2], v[3]);
    else {
#pragma unroll
      for (int q = 0; q < 4; ++q)
        if (r + q < rows) p[q] = v[q];
    }
  }
}

int launch_materialize(float *dst, int64_t ldd, const float *src, int64_t lds, int64_t rows,
                       int64_t cols, int mode, int lower, int trans, int unit, cudaStream_t s) {
  if (rows <= 0 || cols <= 0) return 0;
  const dim3 g((unsigned)cdiv(rows, MT), (unsigned)cdiv(cols, MT));
  if (g.y > 65535) return -1;
  const bool vec = ((uintptr_t)dst % 16 == 0) && ((uintptr_t)src % 16 == 0) && ldd % 4 == 0 && lds % 4 == 0;
  if (vec) materialize_kernel<true><<<g, MTH, 0, s>>>(dst, ldd, src, lds, rows, cols, mode, lower, trans, unit);
  else materialize_kernel<false><<<g, MTH, 0, s>>>(dst, ldd, src, lds, rows, cols, mode, lower, trans, unit);
  note_launch();
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

// ---------------------------------------------------------------- TRSM diag inverse
namespace {
constexpr int DNB = 128;          // diagonal block size (4 x 32)
constexpr int DLD = DNB + 4;      // padded smem row (16-B aligned rows for float4 broadcasts)
constexpr int DT = 256;           // threads: 8 warps
}

// One CTA per 128-block of L (the stored triangle of A in lower form);
// X = inv(L_bb) is written into the panel-inverse workspace.
//   staging : the raw 128 x 128 block of A, loaded column by column (coalesced,
//             16 loads in flight per thread), then L built in shared memory
//             (transposed when the stored triangle is the upper one; the blank
//             triangle of A is never read, Q8)
//   phase 1 : warp w < 4 inverts L_ww (32 x 32) by forward substitution --
//             lane j solves column j, the rows of L broadcast by shuffles
//   phase 2 : block forward substitution X(I,J) = -inv(L_II) sum_{K=J}^{I-1}
//             L(I,K) X(K,J); block column J is a chain over I, its 32 rows of
//             the running sum are split between two warps (8 warps, 4 columns)
__global__ void __launch_bounds__(DT)
trsm_diag_inv_kernel(const float *A, int64_t lda, int64_t n, int stored_lower, int unit,
                     float *Dinv, int64_t ldD) {
  extern __shared__ __align__(16) float sm[];
  float *L = sm;                  // [DNB][DLD]  row-major L
  float *X = sm + DNB * DLD;      // [DNB][DLD]  row-major inverse (staging first)
  float *T = X + DNB * DLD;       // [4][32][33] partial sums of phase 2
  const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
  const int64_t i0 = (int64_t)blockIdx.x * DNB;
  const int nr = (int)imin(DNB, n - i0);

  // staging: thread (r = tid % 128) loads columns c = tid/128 + 2u of the raw
  // block (only the stored triangle), 16 independent loads at a time
  {
    const int r = tid % DNB, c0 = tid / DNB;
    const float *col = A + i0 + r + i0 * lda;
    for (int u0 = 0; u0 < DNB / 2; u0 += 16) {
      float v[16];
#pragma unroll
      for (int u = 0; u < 16; ++u) {
        const int c = c0 + 2 * (u0 + u);
        const bool stored = stored_lower ? (r >= c) : (r <= c);
        v[u] = (r < nr && c < nr && stored) ? __ldg(col + (int64_t)c * lda) : 0.f;
      }
#pragma unroll
      for (int u = 0; u < 16; ++u) X[r * DLD + c0 + 2 * (u0 + u)] = v[u];
    }
  }
  __syncthreads();
  for (int e = tid; e < DNB * DNB; e += DT) {
    const int r = e / DNB, c = e % DNB;
    float v = 0.f;
    if (r == c) v = (unit || r >= nr) ? 1.f : X[r * DLD + r];     // identity padding when ragged
    else if (r > c) v = stored_lower ? X[r * DLD + c] : X[c * DLD + r];
    L[r * DLD + c] = v;
  }
  __syncthreads();
  for (int e = tid; e < DNB * DNB; e += DT) X[(e / DNB) * DLD + e % DNB] = 0.f;
  __syncthreads();

  // phase 1
  if (warp < 4) {
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

  // phase 2: warps (2J, 2J+1) own block column J < 3; each sums 16 of the 32
  // rows of t = sum_K L(I,K) X(K,J) (L rows as float4 broadcasts, X(K,J)
  // column in registers), then both apply -inv(L_II) to 16 rows each.
  {
    const int J = warp / 2, h = warp % 2, c = J * 32 + lane;
    float *Tj = T + J * 32 * 33;
    const uint32_t bar = 1 + J;                    // named barrier per column pair
    for (int I = J + 1; I < 4 && J < 3; ++I) {
      float t[16];
#pragma unroll
      for (int ii = 0; ii < 16; ++ii) t[ii] = 0.f;
      for (int K = J; K < I; ++K) {
        float xk[32];
#pragma unroll
        for (int kk = 0; kk < 32; ++kk) xk[kk] = X[(K * 32 + kk) * DLD + c];
#pragma unroll
        for (int ii = 0; ii < 16; ++ii) {
          const float4 *lr = reinterpret_cast<const float4 *>(&L[(I * 32 + h * 16 + ii) * DLD + K * 32]);
#pragma unroll
          for (int q = 0; q < 8; ++q) {
            const float4 l4 = lr[q];
            t[ii] = fmaf(l4.x, xk[4 * q], t[ii]);
            t[ii] = fmaf(l4.y, xk[4 * q + 1], t[ii]);
            t[ii] = fmaf(l4.z, xk[4 * q + 2], t[ii]);
            t[ii] = fmaf(l4.w, xk[4 * q + 3], t[ii]);
          }
        }
      }
#pragma unroll
      for (int ii = 0; ii < 16; ++ii) Tj[(h * 16 + ii) * 33 + lane] = t[ii];
      asm volatile("bar.sync %0, 64;" ::"r"(bar) : "memory");
      float tt[32];
#pragma unroll
      for (int q = 0; q < 32; ++q) tt[q] = Tj[q * 33 + lane];
#pragma unroll
      for (int ii = 0; ii < 16; ++ii) {
        const float4 *xr = reinterpret_cast<const float4 *>(&X[(I * 32 + h * 16 + ii) * DLD + I * 32]);
        float v = 0.f;
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          const float4 x4 = xr[q];
          v = fmaf(x4.x, tt[4 * q], v);
          v = fmaf(x4.y, tt[4 * q + 1], v);
          v = fmaf(x4.z, tt[4 * q + 2], v);
          v = fmaf(x4.w, tt[4 * q + 3], v);
        }
        X[(I * 32 + h * 16 + ii) * DLD + c] = -v;
      }
      asm volatile("bar.sync %0, 64;" ::"r"(bar) : "memory");
    }
  }
  __syncthreads();

  // write inv(L_bb) (lower, column-major) into its panel slot; padded rows/cols zero
  const int64_t bpp = ldD / DNB;                     // 128-blocks per panel
  float *D = Dinv + (blockIdx.x / bpp) * ldD * ldD + (blockIdx.x % bpp) * DNB * (1 + ldD);
  {
    const int r = tid % DNB, c0 = tid / DNB;
#pragma unroll 8
    for (int c = c0; c < DNB; c += 2)
      D[r + (int64_t)c * ldD] = (r < nr && c < nr && r >= c) ? X[r * DLD + c] : 0.f;
    // the blank (upper) triangle of the panel inverse is read as zeros by the
    // structured GEMMs, but only within 256 of the diagonal (tile height): zero
    // the two 128-blocks to the right of this diagonal block (inside the panel)
    // so the workspace needs no memset
    const int64_t bi = blockIdx.x % bpp;
    for (int j = 1; j <= 2 && bi + j < bpp; ++j) {
      float *U = D + (int64_t)j * DNB * ldD;
#pragma unroll 8
      for (int c = c0; c < DNB; c += 2) U[r + (int64_t)c * ldD] = 0.f;
    }
  }
}

// Level 0 of the panel-inverse doubling on CUDA cores (exact fp32 FMAs): for
// every pair [[L11, 0], [L21, L22]] of 128-blocks of L (rows [256p, 256p + 256)),
// the off-diagonal block of its inverse,
//     X21 = -inv(L22) (L21 inv(L11)),
// written into the panel-inverse workspace beside inv(L11) and inv(L22)
// (trsm_diag_inv_kernel, which must have run).  Columns of X21 are
// independent: grid (pairs, 128 / L0C), one CTA per L0C columns.  A ragged last
// pair (L22 of nr2 < 128 rows) reads zeros beyond n and writes zero rows there.
// It replaces two dependent tcgen05 launches of 128-blocks (the first level of
// trsm_doubling_problems) with one launch (profiles/r02_strsm_panel.md).
namespace {
constexpr int L0C = 8;             // columns of X21 per CTA
constexpr int L0R = DNB * L0C / DT; // rows of X21 per thread (4)
constexpr int L0S = DNB + 4;       // smem row stride (16-B aligned rows)
}
__global__ void __launch_bounds__(DT)
trsm_level0_kernel(const float *A, int64_t lda, int64_t n, int stored_lower, float *Dinv, int64_t ldD) {
  extern __shared__ __align__(16) float sm[];
  float *Lr = sm;                          // [128][L0S] row-major: L21, then inv(L22)
  float *Xc = sm + DNB * L0S;              // [128][L0C + 1]: inv(L11)(:, cols), then T(:, cols)
  const int tid = threadIdx.x;
  const int64_t o = (int64_t)blockIdx.x * 2 * DNB;
  const int cs = blockIdx.y * L0C;
  const int nr2 = (int)imin(DNB, n - o - DNB);
  const int64_t bpp = ldD / DNB, b1 = o / DNB;          // 128-blocks per panel; block of L11
  float *D11 = Dinv + (b1 / bpp) * ldD * ldD + (b1 % bpp) * DNB * (1 + ldD);
  const float *D22 = D11 + DNB * (1 + ldD);             // a pair never straddles a panel (ldD >= 256)
  float *D21 = D11 + DNB;
  // the loads are latency-bound: 16 independent ones in flight per thread
  constexpr int LB = 16;
  for (int e0 = tid; e0 < DNB * DNB; e0 += DT * LB) {   // L21(r, c) = L(o + 128 + r, o + c)
    float v[LB];
#pragma unroll
    for (int u = 0; u < LB; ++u) {
      const int e = e0 + u * DT, r = e % DNB, c = e / DNB;
      v[u] = r < nr2 ? (stored_lower ? __ldg(A + (o + DNB + r) + (o + c) * lda)
                                     : __ldg(A + (o + c) + (o + DNB + r) * lda)) : 0.f;
    }
#pragma unroll
    for (int u = 0; u < LB; ++u) { const int e = e0 + u * DT; Lr[(e % DNB) * L0S + e / DNB] = v[u]; }
  }
  {
    float v[DNB * L0C / DT];
#pragma unroll
    for (int u = 0; u < DNB * L0C / DT; ++u) {
      const int e = tid + u * DT, k = e % DNB, c = e / DNB;
      v[u] = __ldg(D11 + k + (int64_t)(cs + c) * ldD);
    }
#pragma unroll
    for (int u = 0; u < DNB * L0C / DT; ++u) { const int e = tid + u * DT; Xc[(e % DNB) * (L0C + 1) + e / DNB] = v[u]; }
  }
  __syncthreads();
  const int c = tid % L0C, rg = tid / L0C;              // thread: rows rg*L0R .. +L0R-1 of column c
  // rows of (Lr x Xc)(:, c); Lr rows read as float4
  auto rows_times = [&](float (&t)[L0R]) {
#pragma unroll
    for (int i = 0; i < L0R; ++i) t[i] = 0.f;
    for (int k = 0; k < DNB; k += 4) {
      const float x0 = Xc[k * (L0C + 1) + c], x1 = Xc[(k + 1) * (L0C + 1) + c];
      const float x2 = Xc[(k + 2) * (L0C + 1) + c], x3 = Xc[(k + 3) * (L0C + 1) + c];
#pragma unroll
      for (int i = 0; i < L0R; ++i) {
        const float4 l = *reinterpret_cast<const float4 *>(&Lr[(rg * L0R + i) * L0S + k]);
        t[i] = fmaf(l.x, x0, t[i]);
        t[i] = fmaf(l.y, x1, t[i]);
        t[i] = fmaf(l.z, x2, t[i]);
        t[i] = fmaf(l.w, x3, t[i]);
      }
    }
  };
  float t[L0R];
  rows_times(t);                                        // T = L21 inv(L11)
  __syncthreads();
#pragma unroll
  for (int i = 0; i < L0R; ++i) Xc[(rg * L0R + i) * (L0C + 1) + c] = t[i];
  for (int e0 = tid; e0 < DNB * DNB; e0 += DT * LB) {
    float v[LB];
#pragma unroll
    for (int u = 0; u < LB; ++u) { const int e = e0 + u * DT; v[u] = __ldg(D22 + e % DNB + (int64_t)(e / DNB) * ldD); }
#pragma unroll
    for (int u = 0; u < LB; ++u) { const int e = e0 + u * DT; Lr[(e % DNB) * L0S + e / DNB] = v[u]; }
  }
  __syncthreads();
  rows_times(t);                                        // inv(L22) T
#pragma unroll
  for (int i = 0; i < L0R; ++i) {
    const int r = rg * L0R + i;
    D21[r + (int64_t)(cs + c) * ldD] = r < nr2 ? -t[i] : 0.f;
  }
}

int launch_trsm_level0(const float *A, int64_t lda, int64_t n, int stored_lower, float *Dinv, int64_t ldD,
                       cudaStream_t s) {
  if (ldD % (2 * DNB)) return -1;
  const int64_t pairs = n > DNB ? (n - DNB + 2 * DNB - 1) / (2 * DNB) : 0;   // pairs with an L21
  if (pairs == 0) return 0;
  const size_t smem = (DNB * L0S + DNB * (L0C + 1)) * sizeof(float);
  static std::atomic<bool> attr[64];
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return -1;
  if (!attr[dev].load(std::memory_order_acquire)) {
    if (cudaFuncSetAttribute(trsm_level0_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) !=
        cudaSuccess) return -1;
    attr[dev].store(true, std::memory_order_release);
  }
  trsm_level0_kernel<<<dim3((unsigned)pairs, DNB / L0C), DT, smem, s>>>(A, lda, n, stored_lower, Dinv, ldD);
  note_launch();
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

// blas3_signal: a stream-ordered release write of a flag
__global__ void signal_kernel(uint32_t *flag, uint32_t value) {
  __threadfence();
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(flag), "r"(value) : "memory");
}
int launch_signal(uint32_t *flag, uint32_t value, cudaStream_t s) {
  signal_kernel<<<1, 1, 0, s>>>(flag, value);
  note_launch();
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

int launch_trsm_diag_inv(const float *A, int64_t lda, int64_t n, int stored_lower, int unit,
                         float *Dinv, int64_t ldD, cudaStream_t s) {
  if (ldD % DNB) return -1;
  const size_t smem = (2 * DNB * DLD + 4 * 32 * 33) * sizeof(float);
  static std::atomic<bool> attr[64];              // per device context
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return -1;
  if (!attr[dev].load(std::memory_order_acquire)) {
    if (cudaFuncSetAttribute(trsm_diag_inv_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)smem) != cudaSuccess) return -1;
    attr[dev].store(true, std::memory_order_release);
  }
  int64_t blocks = cdiv(n, DNB);
  trsm_diag_inv_kernel<<<(unsigned)blocks, DT, smem, s>>>(A, lda, n, stored_lower, unit, Dinv, ldD);
  note_launch();
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

}  // namespace blas3
