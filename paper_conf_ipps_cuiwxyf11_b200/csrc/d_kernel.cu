// d_kernel.cu -- the fp64 family ("DGEMM family"): one
// structured fp64 GEMM kernel that every D routine derives from, plus the
// triangular-solve kernels (64-block inverses, panel leaves).
//
// The paper's method carried over unchanged to double precision
// (PAPER.md P:93-99 SM_alloc(X, Symmetry), P:197-210 padding/peel_triangular,
// P:225-244 Adaptor_Solver): symmetric operands are MIRRORED and triangular
// ones ZERO-FILLED (unit diagonal written) while a tile is staged to shared
// memory, blank triangular k-blocks are skipped through the tile's k-range,
// only the uplo triangle of C is written for SYRK/SYR2K, and TRSM is a blocked
// diagonal-block solve followed by GEMM updates (d_abi.cu).
//
// Which unit: on B200 the FP64 tensor path (DMMA, mma.sync m8n8k4 f64) and the
// FMA pipe (DFMA) top out at the same ~37 TF/s (tools/probes/dmma_rate.cu:
// 37.1 vs 36.4).  DMMA does 256 FMAs per instruction against DFMA's 32, so the
// default instantiation issues DMMA from register fragments; DFMA stays as
// the BLAS3_D_MMA=0 alternative.  Products and sums are fp64 either way.
//
// Kernel: C tile 128 x 128, BK = 16 k-blocks staged through registers into
// double-buffered shared memory (the structure select happens on the way);
// DMMA: 512 threads, each warp a 32 x 32 block of 4 x 4 fragments; DFMA: 256
// threads, 8 x 8 outputs per thread (rows tr + 16 i, columns 4 tc + 64 g + j).
#include <cuda_runtime.h>
#include <stdint.h>
#include <atomic>
#include <stdlib.h>

#include "kernels.h"
#include "d_kernels.h"

namespace blas3 {
namespace {

constexpr int DTM = 128, DTN = 128, DBK = 16;
// shared-row padding: 132 doubles = 32 B mod 128 keeps the DMMA fragment
// loads (4 k-rows x 64 B) at 2 wavefronts and the k-fastest staging stores at
// 4-way; measured against 2 and 8 (tools/lib_ab_fp64.py: DGEMM TN 24.0 vs
// 23.4 / 21.5 TF/s, DSYMM 21.7 vs 21.3 / 20.2)
#ifndef BLAS3_DPAD
#define BLAS3_DPAD 4
#endif
constexpr int DPAD = BLAS3_DPAD;
constexpr int DAP = DTM + DPAD, DBP = DTN + DPAD;
constexpr int DJ = 8;                                // columns per thread (two groups of 4)
constexpr int DNB = 64;                              // TRSM diagonal block

// X(r, k) of an operand: the logical matrix L = stored (dense), sym(stored
// triangle) or tri(stored triangle, unit diagonal, blank = 0), viewed
// transposed when trans, at offsets (ro, ko) of the X index space.
__device__ __forceinline__ double dfetch(const DOpnd &o, int64_t r, int64_t k) {
  const int64_t i = o.trans ? k + o.ko : r + o.ro;
  const int64_t j = o.trans ? r + o.ro : k + o.ko;
  if (o.kind == DOP_DENSE) return __ldg(o.p + i + j * o.ld);
  const bool stored = o.lower ? (i >= j) : (i <= j);
  if (o.kind == DOP_SYM) return stored ? __ldg(o.p + i + j * o.ld) : __ldg(o.p + j + i * o.ld);
  if (!stored) return 0.0;                           // the blank triangle is never read
  if (i == j && o.unit) return 1.0;                  // unit diagonal: the stored value is not read
  return __ldg(o.p + i + j * o.ld);
}

// Is the (rows [r0, r1) x k [k0, k1)) block of X read contiguously along r?
// Dense / tri: the stored orientation (i = r unless trans).  Sym: the stored
// orientation where the block lies in the stored triangle, the mirrored one
// where it lies in the other (diagonal-crossing blocks: either).
__device__ __forceinline__ bool rfast(const DOpnd &o, int64_t r0, int64_t r1, int64_t k0, int64_t k1) {
  if (o.kind != DOP_SYM) return !o.trans;
  // i-range and j-range of the block in L
  const int64_t i0 = o.trans ? k0 + o.ko : r0 + o.ro, i1 = o.trans ? k1 + o.ko : r1 + o.ro;
  const int64_t j0 = o.trans ? r0 + o.ro : k0 + o.ko, j1 = o.trans ? r1 + o.ro : k1 + o.ko;
  const bool all_stored = o.lower ? (i0 >= j1 - 1) : (i1 - 1 <= j0);
  const bool all_mirror = o.lower ? (i1 - 1 < j0) : (i0 > j1 - 1);
  // stored: address i + j ld, contiguous in i; mirrored: j + i ld, contiguous in j
  const bool contig_i = all_stored || !all_mirror;
  return contig_i ? !o.trans : o.trans;
}

// k-range of X's nonzeros for the rows [r0, r1) (blank triangle skipped)
__device__ __forceinline__ void krange(const DOpnd &o, int64_t r0, int64_t r1, int64_t K, int64_t &klo,
                                       int64_t &khi) {
  if (o.kind != DOP_TRI) return;
  const int64_t d = o.ro - o.ko;
  // nonzero iff (lower != trans) ? k <= r + d : k >= r + d
  if (o.lower != (o.trans != 0)) khi = khi < r1 + d ? khi : r1 + d;
  else klo = klo > r0 + d ? klo : r0 + d;
  if (khi > K) khi = K;
  if (klo < 0) klo = 0;
}

// One operand tile (ROWS x DBK) of X into registers: element e = tid + 256 q,
// (r, k) = r-fastest or k-fastest by the block's contiguous direction.
template <int ROWS, int NT>
struct TileLoad {
  static constexpr int PER = ROWS * DBK / NT;
  double v[PER];
  // strided block X(r, k) = base[r * si + k * sk]
  __device__ __forceinline__ void load_strided(const double *base, int64_t si, int64_t sk, int64_t r0, int64_t rmax,
                                               int64_t k0, int64_t kmax, bool rf) {
#pragma unroll
    for (int q = 0; q < PER; ++q) {
      const int e = threadIdx.x + NT * q;
      const int r = rf ? e % ROWS : e / DBK, k = rf ? e / ROWS : e % DBK;
      v[q] = (r0 + r < rmax && k0 + k < kmax) ? __ldg(base + r * si + k * sk) : 0.0;
    }
  }
  // The block's region class decides the access (Adaptor_Symmetry /
  // Adaptor_Triangular): REAL (inside the stored
  // triangle: plain strided loads), SHADOW (SYM, the other triangle: the
  // mirrored strided loads), BLANK (TRI outside the triangle: zeros, nothing
  // read), DIAGONAL-CROSSING (per-element select, dfetch).
  __device__ __forceinline__ void load(const DOpnd &o, int64_t r0, int64_t rmax, int64_t k0, int64_t kmax,
                                       bool rf) {
    // X(r, k) = p[i + j ld], (i, j) = trans ? (k + ko, r + ro) : (r + ro, k + ko)
    const int64_t si = o.trans ? o.ld : 1, sk = o.trans ? 1 : o.ld;
    if (o.kind == DOP_DENSE) {
      load_strided(o.p + r0 * si + k0 * sk, si, sk, r0, rmax, k0, kmax, rf);
      return;
    }
    const int64_t i0 = o.trans ? k0 + o.ko : r0 + o.ro, i1 = i0 + (o.trans ? DBK : ROWS) - 1;
    const int64_t j0 = o.trans ? r0 + o.ro : k0 + o.ko, j1 = j0 + (o.trans ? ROWS : DBK) - 1;
    const bool real = o.lower ? (i0 > j1) : (i1 < j0);            // strictly inside: no diagonal
    const bool other = o.lower ? (i1 < j0) : (i0 > j1);
    if (real) {
      load_strided(o.p + (r0 + o.ro) * si + (k0 + o.ko) * sk, si, sk, r0, rmax, k0, kmax, rf);
      return;
    }
    if (other && o.kind == DOP_TRI) {
#pragma unroll
      for (int q = 0; q < PER; ++q) v[q] = 0.0;
      return;
    }
    if (other) {                                                   // SYM shadow: L(i, j) = p[j + i ld]
      load_strided(o.p + (r0 + o.ro) * sk + (k0 + o.ko) * si, sk, si, r0, rmax, k0, kmax, rf);
      return;
    }
#pragma unroll
    for (int q = 0; q < PER; ++q) {
      const int e = threadIdx.x + NT * q;
      const int r = rf ? e % ROWS : e / DBK, k = rf ? e / ROWS : e % DBK;
      v[q] = (r0 + r < rmax && k0 + k < kmax) ? dfetch(o, r0 + r, k0 + k) : 0.0;
    }
  }
  template <int LD>
  __device__ __forceinline__ void store(double *s, bool rf) const {
#pragma unroll
    for (int q = 0; q < PER; ++q) {
      const int e = threadIdx.x + NT * q;
      const int r = rf ? e % ROWS : e / DBK, k = rf ? e / ROWS : e % DBK;
      s[k * LD + r] = v[q];
    }
  }
};

constexpr size_t DSMEM = 2 * DBK * (DAP + DBP) * sizeof(double);   // 69632 B (dynamic)

// one DMMA (m8n8k4, f64): d += a (8x4 row-major fragment) * b (4x8 col-major)
__device__ __forceinline__ void dmma(double &d0, double &d1, double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0, %1}, {%2}, {%3}, {%0, %1};"
               : "+d"(d0), "+d"(d1) : "d"(a), "d"(b));
}

// MMA = false: DFMA, 8 x 8 outputs per thread.  MMA = true: DMMA m8n8k4 on
// register fragments, each warp a 64 x 32 block (8 x 4 fragments), the same
// staging and epilogue semantics.
// threads per CTA: DMMA 512 (16 warps, each a 32 x 32 block of 4 x 4
// fragments: <= 128 registers), DFMA 256 (8 x 8 outputs per thread)
template <bool MMA> __host__ __device__ constexpr int dthreads() { return MMA ? 512 : 256; }
template <bool MMA>
__global__ void __launch_bounds__(dthreads<MMA>(), 1) dgemm_structured(const __grid_constant__ DProblem P) {
  constexpr int NT = dthreads<MMA>();
  extern __shared__ double dsm[];
  // buffers by integer offset from the __shared__ array (not through a
  // pointer table, which would turn every access into a generic LD/ST)
  constexpr int AOFF = DBK * DAP, BOFF0 = 2 * DBK * DAP, BOFF = DBK * DBP;
  const int64_t tiles_n = (P.N + DTN - 1) / DTN;
  const int64_t tm = blockIdx.x / tiles_n, tn = blockIdx.x % tiles_n;
  const int64_t m0 = tm * DTM, n0 = tn * DTN;
  // SYRK / SYR2K: tiles wholly outside the uplo triangle of C do nothing
  if (P.ctri == 1 && m0 + DTM - 1 < n0) return;
  if (P.ctri == 2 && m0 > n0 + DTN - 1) return;
  const int tr = threadIdx.x % 16, tc = threadIdx.x / 16;
  double acc[8][DJ];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < DJ; ++j) acc[i][j] = 0.0;

  for (int sg = 0; sg < P.nseg; ++sg) {
    const DSeg &S = P.seg[sg];
    int64_t klo = 0, khi = S.K;
    krange(S.a, m0, m0 + DTM, S.K, klo, khi);
    krange(S.b, n0, n0 + DTN, S.K, klo, khi);
    if (klo >= khi) continue;
    klo = klo / DBK * DBK;                            // k-blocks aligned to BK
    const int64_t nkb = (khi - klo + DBK - 1) / DBK;
    TileLoad<DTM, NT> la;
    TileLoad<DTN, NT> lb;
    bool rfa = rfast(S.a, m0, m0 + DTM, klo, klo + DBK), rfb = rfast(S.b, n0, n0 + DTN, klo, klo + DBK);
    la.load(S.a, m0, P.M, klo, khi, rfa);
    lb.load(S.b, n0, P.N, klo, khi, rfb);
    __syncthreads();                                   // previous segment's reads of the buffers
    la.store<DAP>(dsm, rfa);
    lb.store<DBP>(dsm + BOFF0, rfb);
    __syncthreads();
    for (int64_t t = 0; t < nkb; ++t) {
      const int cur = (int)(t & 1);
      const int64_t kn = klo + (t + 1) * DBK;
      if (t + 1 < nkb) {                               // next k-block into registers
        rfa = rfast(S.a, m0, m0 + DTM, kn, kn + DBK);
        rfb = rfast(S.b, n0, n0 + DTN, kn, kn + DBK);
        la.load(S.a, m0, P.M, kn, khi, rfa);
        lb.load(S.b, n0, P.N, kn, khi, rfb);
      }
      const double *as = dsm + cur * AOFF, *bs = dsm + BOFF0 + cur * BOFF;
      if constexpr (MMA) {
        const int lane = threadIdx.x % 32, wid = threadIdx.x / 32;
        const int am = 32 * (wid % 4) + lane / 4, bn = 32 * (wid / 4) + lane / 4, kq = lane % 4;
#pragma unroll
        for (int kk = 0; kk < DBK / 4; ++kk) {
          double a[4], b[4];
#pragma unroll
          for (int i = 0; i < 4; ++i) a[i] = as[(kk * 4 + kq) * DAP + am + 8 * i];
#pragma unroll
          for (int j = 0; j < 4; ++j) b[j] = bs[(kk * 4 + kq) * DBP + bn + 8 * j];
#pragma unroll
          for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int j = 0; j < 4; ++j) dmma(acc[i][2 * j], acc[i][2 * j + 1], a[i], b[j]);
        }
      } else {
#pragma unroll
      for (int k = 0; k < DBK; ++k) {
        double a[8], b[DJ];
#pragma unroll
        for (int i = 0; i < 8; ++i) a[i] = as[k * DAP + tr + 16 * i];
#pragma unroll
        for (int g = 0; g < DJ / 4; ++g) {             // columns 4 tc + 64 g + 0..3
          const double2 b01 = *reinterpret_cast<const double2 *>(bs + k * DBP + 4 * tc + 64 * g);
          const double2 b23 = *reinterpret_cast<const double2 *>(bs + k * DBP + 4 * tc + 64 * g + 2);
          b[4 * g] = b01.x; b[4 * g + 1] = b01.y; b[4 * g + 2] = b23.x; b[4 * g + 3] = b23.y;
        }
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
          for (int j = 0; j < DJ; ++j) acc[i][j] = fma(a[i], b[j], acc[i][j]);
      }
      }
      if (t + 1 < nkb) {
        la.store<DAP>(dsm + (cur ^ 1) * AOFF, rfa);
        lb.store<DBP>(dsm + BOFF0 + (cur ^ 1) * BOFF, rfb);
      }
      __syncthreads();
    }
  }
  // epilogue: D = alpha * acc + beta * C (C not read when beta == 0), uplo mask
#pragma unroll
  for (int j = 0; j < DJ; ++j) {
    // DMMA: acc[i][2 jf + e] is C row 32 (w % 4) + 8 i + lane / 4, column
    // 32 (w / 4) + 8 jf + 2 (lane % 4) + e  (i < 4)
    const int64_t c = MMA ? n0 + 32 * ((threadIdx.x / 32) / 4) + 8 * (j / 2) + 2 * ((threadIdx.x % 32) % 4) + j % 2
                          : n0 + 4 * tc + 64 * (j / 4) + j % 4;
    if (c >= P.N) continue;
#pragma unroll
    for (int i = 0; i < (MMA ? 4 : 8); ++i) {
      const int64_t r = MMA ? m0 + 32 * ((threadIdx.x / 32) % 4) + 8 * i + (threadIdx.x % 32) / 4 : m0 + tr + 16 * i;
      if (r >= P.M) continue;
      if (P.ctri == 1 && r < c) continue;
      if (P.ctri == 2 && r > c) continue;
      double v = P.alpha * acc[i][j];
      if (P.beta != 0.0) v = fma(P.beta, P.C[r + c * P.ldc], v);
      P.D[r + c * P.ldd] = v;
    }
  }
}

// In-register substitution S y = y for one 64-block S (shared, ld DNB + 1),
// forward (S lower) or backward, a division per row as in the oracle
__device__ __forceinline__ void subst64(const double *Ss, double (&y)[DNB], bool lower) {
  if (lower) {
#pragma unroll
    for (int i = 0; i < DNB; ++i) {
      double v = y[i];
#pragma unroll
      for (int j = 0; j < i; ++j) v = fma(-Ss[i + j * (DNB + 1)], y[j], v);
      y[i] = v / Ss[i + i * (DNB + 1)];
    }
  } else {
#pragma unroll
    for (int i = DNB - 1; i >= 0; --i) {
      double v = y[i];
#pragma unroll
      for (int j = i + 1; j < DNB; ++j) v = fma(-Ss[i + j * (DNB + 1)], y[j], v);
      y[i] = v / Ss[i + i * (DNB + 1)];
    }
  }
}
// one 64-block of S into shared memory, padded with the identity beyond nb
__device__ __forceinline__ void load_block64(const DOpnd &S, int64_t o, int nb, double *Ss) {
  for (int e = threadIdx.x; e < DNB * DNB; e += blockDim.x) {
    const int i = e % DNB, j = e / DNB;
    Ss[i + j * (DNB + 1)] = (i < nb && j < nb) ? dfetch(S, o + i, o + j) : (i == j ? 1.0 : 0.0);
  }
}

// inv(S_bb) of every 64-block b on the diagonal of the order-nt triangle S
// (one CTA per block, thread c solves S_bb y = e_c): Dinv + 4096 b, 64 x 64
// column-major, the identity where a ragged last block is padded
__global__ void __launch_bounds__(64) dtri_inv64(const __grid_constant__ DOpnd S, int64_t nt, double *Dinv) {
  __shared__ double Ss[DNB * (DNB + 1)];
  const int64_t o = (int64_t)blockIdx.x * DNB;
  const int nb = (int)(nt - o < DNB ? nt - o : DNB);
  load_block64(S, o, nb, Ss);
  __syncthreads();
  const int c = threadIdx.x;
  double y[DNB];
#pragma unroll
  for (int i = 0; i < DNB; ++i) y[i] = i == c ? 1.0 : 0.0;
  subst64(Ss, y, S.lower != (S.trans != 0));
  double *d = Dinv + (size_t)blockIdx.x * DNB * DNB + (size_t)c * DNB;
#pragma unroll
  for (int i = 0; i < DNB; ++i) d[i] = y[i];
}

// A diagonal panel of R <= DPR rows (64-blocks, processing order forward if S
// is lower) for DRC right-hand sides per CTA, the panel's rows of those
// right-hand sides resident in shared memory:
//   y_i <- inv(S_ii) (y_i - sum_{j before i} S_ij y_j)
// with the 64-block inverses from dtri_inv64 (Dp: this panel's first block).
// One launch replaces the 64-row recursion's small launches at the bottom of
// the DTRSM sweep.
constexpr int DPR = 512, DRC = 32, DPT = 256;
constexpr int DSL = DNB + 1;                          // shared 64-block leading dimension
constexpr size_t DPANEL_SMEM = (size_t)(DPR * DRC + 2 * DNB * DSL) * sizeof(double);   // 193 KB
constexpr int DPE = DNB * DNB / DPT;                  // block elements per thread (16)

// The work list of one panel, in order: for every processing step st, the
// coupling blocks (bi, bj) of the st blocks solved before it, then the
// inverse of block bi (bj = -1): st + 1 items, st(st+1)/2 items before it.
__device__ __forceinline__ void panel_item(int it, int nb, bool lower, int &bi, int &bj) {
  int st = 0;
  while ((st + 1) * (st + 2) / 2 <= it) ++st;
  const int tt = it - st * (st + 1) / 2;              // 0..st; tt == st: the inverse
  bi = lower ? st : nb - 1 - st;
  bj = tt == st ? -1 : (lower ? tt : nb - 1 - tt);
}

__global__ void __launch_bounds__(DPT, 1) dtrsm_panel(const __grid_constant__ DOpnd S, const double *Dp, int R,
                                                      double *X, int64_t sx, int64_t sc, int64_t nrhs) {
  extern __shared__ double dps[];
  double *Y = dps;                                    // Y[i * DRC + c]
  double *Sb = dps + DPR * DRC;                       // two 64-blocks, ld DSL
  const int64_t c0 = (int64_t)blockIdx.x * DRC;
  const int ncol = (int)(nrhs - c0 < DRC ? nrhs - c0 : DRC);
  const int nb = (R + DNB - 1) / DNB;
  const bool lower = S.lower != (S.trans != 0);
  // the panel's rows of this CTA's right-hand sides (i fastest when the rows
  // are contiguous, sx == 1)
  for (int e = threadIdx.x; e < nb * DNB * DRC; e += DPT) {
    const int i = sx == 1 ? e % (nb * DNB) : e / DRC, c = sx == 1 ? e / (nb * DNB) : e % DRC;
    Y[i * DRC + c] = (i < R && c < ncol) ? X[i * sx + (c0 + c) * sc] : 0.0;
  }
  // A coupling block (bi, bj) lies strictly inside the triangle (bj is solved
  // before bi), so it is read as stored: S(r, k) = L(i, j) = p[i + j ld] with
  // (i, j) = trans ? (k + ko, r + ro) : (r + ro, k + ko), without the TRI
  // select; the element order follows the contiguous direction.
  const bool tr = S.trans != 0;
  auto fetch_block = [&](int bi, int bj, double (&v)[DPE]) {
    if (bj < 0) {                                     // inv(S_ii): contiguous 64 x 64
      const double *d = Dp + (size_t)bi * DNB * DNB;
#pragma unroll
      for (int q = 0; q < DPE; ++q) v[q] = __ldg(d + threadIdx.x + DPT * q);
      return;
    }
#pragma unroll
    for (int q = 0; q < DPE; ++q) {
      const int e = threadIdx.x + DPT * q;
      const int rr = tr ? e / DNB : e % DNB, kk = tr ? e % DNB : e / DNB;
      const int64_t gi = (int64_t)bi * DNB + rr, gj = (int64_t)bj * DNB + kk;
      const int64_t li = tr ? gj + S.ko : gi + S.ro, lj = tr ? gi + S.ro : gj + S.ko;
      v[q] = (gi < R && gj < R) ? __ldg(S.p + li + lj * S.ld) : 0.0;
    }
  };
  auto store_block = [&](int bj, const double (&v)[DPE], double *dst) {
#pragma unroll
    for (int q = 0; q < DPE; ++q) {
      const int e = threadIdx.x + DPT * q;
      const int rr = (bj >= 0 && tr) ? e / DNB : e % DNB, kk = (bj >= 0 && tr) ? e % DNB : e / DNB;
      dst[rr + kk * DSL] = v[q];
    }
  };
  // this thread's outputs: row r = tid % 64 of the block, columns cb + 4 q
  // (a warp reads 32 consecutive S rows -- conflict-free -- and broadcast Y;
  // a 4 x 2 register block with 16-B loads measured slower: 245 vs 183 us)
  const int r = threadIdx.x % DNB, cb = threadIdx.x / DNB;
  const int nitems = nb * (nb + 1) / 2;
  double pre[DPE];
  int bi, bj;
  panel_item(0, nb, lower, bi, bj);
  fetch_block(bi, bj, pre);
  double acc[DRC / 4];
#pragma unroll
  for (int q = 0; q < DRC / 4; ++q) acc[q] = 0.0;
  for (int it = 0; it < nitems; ++it) {
    const int cur = it & 1;
    double *Ss = Sb + cur * DNB * DSL;
    store_block(bj, pre, Ss);                         // (its buffer was last read two items ago)
    const int ci = bi, cj = bj;
    if (it + 1 < nitems) {                            // the next block into registers
      panel_item(it + 1, nb, lower, bi, bj);
      fetch_block(bi, bj, pre);
    }
    __syncthreads();
    if (cj >= 0) {                                    // acc += S(ci, cj) y_cj
#pragma unroll 8
      for (int k = 0; k < DNB; ++k) {
        const double sv = Ss[r + k * DSL];
#pragma unroll
        for (int q = 0; q < DRC / 4; ++q) acc[q] = fma(sv, Y[(cj * DNB + k) * DRC + cb + 4 * q], acc[q]);
      }
    } else {                                          // y_ci <- inv(S_ii) (y_ci - acc)
#pragma unroll
      for (int q = 0; q < DRC / 4; ++q) Y[(ci * DNB + r) * DRC + cb + 4 * q] -= acc[q];
      __syncthreads();
#pragma unroll
      for (int q = 0; q < DRC / 4; ++q) acc[q] = 0.0;
#pragma unroll 8
      for (int k = 0; k < DNB; ++k) {
        const double sv = Ss[r + k * DSL];
#pragma unroll
        for (int q = 0; q < DRC / 4; ++q) acc[q] = fma(sv, Y[(ci * DNB + k) * DRC + cb + 4 * q], acc[q]);
      }
      __syncthreads();
#pragma unroll
      for (int q = 0; q < DRC / 4; ++q) {
        Y[(ci * DNB + r) * DRC + cb + 4 * q] = acc[q];
        acc[q] = 0.0;
      }
    }
  }
  __syncthreads();
  for (int e = threadIdx.x; e < nb * DNB * DRC; e += DPT) {
    const int i = sx == 1 ? e % (nb * DNB) : e / DRC, c = sx == 1 ? e / (nb * DNB) : e % DRC;
    if (i < R && c < ncol) X[i * sx + (c0 + c) * sc] = Y[i * DRC + c];
  }
}

// C <- beta * C on the m x n block (tri: 0 all, 1 lower, 2 upper triangle);
// beta == 0 writes exact zeros without reading C
__global__ void dscale_kernel(double *C, int64_t ldc, int64_t m, int64_t c0, double beta, int tri) {
  const int64_t c = c0 + blockIdx.y;
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < m; r += (int64_t)gridDim.x * blockDim.x) {
    if ((tri == 1 && r < c) || (tri == 2 && r > c)) continue;
    double *p = C + r + c * ldc;
    *p = beta == 0.0 ? 0.0 : beta * *p;
  }
}

}  // namespace

int launch_dgemm(const DProblem &P, cudaStream_t s) {
  if (P.M <= 0 || P.N <= 0) return 0;
  const int64_t tiles = ((P.M + DTM - 1) / DTM) * ((P.N + DTN - 1) / DTN);
  if (tiles > 0x7fffffffLL) return -1;
  // BLAS3_D_MMA: 1 (default) DMMA fragments, 0 DFMA (A/B)
  static const bool use_mma = [] { const char *e = getenv("BLAS3_D_MMA"); return e ? atoi(e) != 0 : true; }();
  void (*kfn)(const DProblem) = use_mma ? dgemm_structured<true> : dgemm_structured<false>;
  static std::atomic<bool> attr[64][2];
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return -1;
  if (!attr[dev][use_mma].load(std::memory_order_acquire)) {
    if (cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)DSMEM) != cudaSuccess)
      return -1;
    attr[dev][use_mma].store(true, std::memory_order_release);
  }
  kfn<<<(unsigned)tiles, use_mma ? dthreads<true>() : dthreads<false>(), DSMEM, s>>>(P);
  note_launch(1);
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

int launch_dtri_inv64(const DOpnd &S, int64_t nt, double *Dinv, cudaStream_t s) {
  if (nt <= 0) return 0;
  dtri_inv64<<<(unsigned)((nt + DNB - 1) / DNB), DNB, 0, s>>>(S, nt, Dinv);
  note_launch(1);
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

int launch_dtrsm_panel(const DOpnd &S, const double *Dp, int R, double *X, int64_t sx, int64_t sc, int64_t nrhs,
                       cudaStream_t s) {
  if (R <= 0 || nrhs <= 0) return 0;
  if (R > DPR) return -1;
  static std::atomic<bool> attr[64];
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return -1;
  if (!attr[dev].load(std::memory_order_acquire)) {
    if (cudaFuncSetAttribute(dtrsm_panel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)DPANEL_SMEM) !=
        cudaSuccess)
      return -1;
    attr[dev].store(true, std::memory_order_release);
  }
  dtrsm_panel<<<(unsigned)((nrhs + DRC - 1) / DRC), DPT, DPANEL_SMEM, s>>>(S, Dp, R, X, sx, sc, nrhs);
  note_launch(1);
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

int launch_dscale(double *C, int64_t ldc, int64_t m, int64_t n, double beta, int tri, cudaStream_t s) {
  if (m <= 0 || n <= 0) return 0;
  const unsigned gx = (unsigned)((m + 255) / 256 < 64 ? (m + 255) / 256 : 64);
  for (int64_t c0 = 0; c0 < n; c0 += 65535) {
    const int64_t nc = n - c0 < 65535 ? n - c0 : 65535;
    dscale_kernel<<<dim3(gx, (unsigned)nc), 256, 0, s>>>(C, ldc, m, c0, beta, tri);
    note_launch(2);
    if (cudaGetLastError() != cudaSuccess) return -1;
  }
  return 0;
}

}  // namespace blas3
