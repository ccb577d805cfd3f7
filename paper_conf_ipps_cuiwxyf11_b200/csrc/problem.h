// problem.h -- the one "GEMM with structured operands" problem every routine
// is canonicalised into, and the tile program (thread_grouping / loop_tiling /
// peel_triangular of the paper) shared by the tcgen05
// and SIMT kernels.
//
// Every routine is  C[M x N] = alpha * sum_seg  Xa_seg * Xb_seg^T  + beta * C
// where Xa is an M x K operand and Xb an N x K operand ("rows x k").  An
// operand knows how its element X(r,k) is fetched from a stored matrix G:
//   DENSE  X(r,k) = G(r,k) ("rk": r contiguous)  or  G(k,r) ("kr")
//   SYM    X(r,k) = S(r,k) if (r,k) is in the stored triangle, else S(k,r)
//          (real / shadow area; selection, never addition, Q7)
//   TRI    X(r,k) = T(r,k) or T(k,r) (swap), 0 in the blank triangle,
//          1 on the diagonal when unit (blank never read, Q8)
// SYR2K uses two segments (A*B^T then B*A^T).  SYRK/SYR2K restrict the tile
// schedule and the epilogue to one triangle of C.
#pragma once
#include <stdint.h>

#ifdef __CUDACC__
#define HD __host__ __device__ __forceinline__
#else
#define HD inline
#endif

namespace blas3 {

enum OpKind : int32_t { OP_DENSE = 0, OP_SYM = 1, OP_TRI = 2 };

struct OpDesc {
  const float *ptr;
  int64_t ld;
  int32_t kind;
  int32_t kr;      // DENSE: X(r,k) = G[k + r*ld] (1) or G[r + k*ld] (0)
  int32_t lower;   // SYM/TRI: stored triangle is the lower one
  int32_t swap;    // TRI: X(r,k) = T(k,r)
  int32_t unit;    // TRI: unit diagonal (stored diagonal not read)
  int32_t map_rk;  // tcgen05 path: tensor-map slot of the rk view (-1: none)
  int32_t map_kr;  // tcgen05 path: tensor-map slot of the kr view (-1: none)
  int32_t zero_blank;  // TRI (not unit): the blank triangle is stored as zeros (library
                       // workspace, e.g. the TRSM inverse panels) -> the k-range is still
                       // clipped, but diagonal blocks load as plain blocks (no zero-select)
};

struct Segment {
  OpDesc a;   // M x K
  OpDesc b;   // N x K
  int64_t K;
};

// Two-level batch stride: element offset of batch b is
//   (b / per) * outer + (b % per) * inner
// (used by the TRSM panel-inverse doubling, whose pairs sit at a uniform
// stride along the diagonal of A but at a two-level stride in the compact
// panel-inverse workspace).
struct BatchStride {
  int64_t outer, inner;
};

struct Problem {
  int64_t M, N;
  Segment seg[2];
  int32_t nseg;
  int32_t c_tri;    // 0: full C; 1: lower triangle only; 2: upper only
  int32_t rev_m;    // schedule m-tiles in reverse (longest K first)
  int32_t rev_n;
  int32_t outer;    // full grid order: 0 grouped raster, 1 m-tiles outer, 2 n-tiles outer
  float alpha, beta;
  const float *Cin; int64_t ldcin;   // read only when beta != 0
  float *Cout; int64_t ldcout;
  // batched problems (SIMT route only): nbatch >= 1 independent problems of
  // the same shape; seg[0] operands and C advance by the strides below.
  int64_t nbatch, per;
  BatchStride bs_a, bs_b, bs_c;
  // performance-experiment knobs (env BLAS3_DEBUG_TC; results are WRONG when
  // set, never used by tests or the bench): bit0 skip the split pass,
  // bit1 issue only hi*hi (1xTF32), bit2 skip the epilogue stores,
  // bit3 issue no MMAs (commits only), bit4 issue no TMA loads,
  // bit5 skip the triangular zero-select/unit-diagonal fix-up,
  // bit6 skip the TMEM loads of the epilogue's chunk drains
  int32_t dbg;
  // launch at most this many SMs' worth of CTAs (0: all).  The STRSM driver
  // leaves SMs free for its latency-bound side-stream kernels this way.
  int32_t max_sms;
  // tcgen05 path: 3 = 3xTF32 (lo*hi + hi*lo + hi*hi, fp32-accurate, default),
  // 1 = 1xTF32 (hi*hi only: the BLAS3_MATH_1XTF32 fast mode, TF32 accuracy)
  int32_t passes;
  // full-grid raster: m-tiles per group (0: Tiles::GM); BLAS3_OPT_TC_RASTER
  int32_t raster_gm;
  // tcgen05 path: k-blocks per TMEM partial (power of 2; BLAS3_OPT_TC_KC)
  int32_t kc;
  // tcgen05 path, set at launch: 1 = the epilogue may use 16-B vector
  // accesses of C (Cout, and Cin when beta != 0, 16-B aligned, ld % 4 == 0);
  // tensor-map slot of Cin for the L2 prefetch of C tiles, or -1
  int32_t c_vec;
  int32_t c_pf_map;
  // streamed A (blas3_sgemm_streamed, segment 0): k-block kb of A may be
  // loaded once a_ready[kb / a_panel_kb] >= a_ready_val (null: A resident)
  const uint32_t *a_ready;
  int32_t a_panel_kb;
  uint32_t a_ready_val;
};

HD int64_t batch_off(const BatchStride &s, int64_t b, int64_t per) {
  return (b / per) * s.outer + (b % per) * s.inner;
}

HD int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }
HD int64_t imin(int64_t a, int64_t b) { return a < b ? a : b; }
HD int64_t imax(int64_t a, int64_t b) { return a > b ? a : b; }

// TRI operand: X(r,k) is in the nonzero region iff k <= r ("kle") or k >= r.
HD bool tri_kle(const OpDesc &o) { return o.lower != o.swap; }

// ---------------------------------------------------------------- tile schedule
// Full grid: grouped raster (GM m-tiles per group) for L2 reuse of the B panel.
// Triangular (SYRK/SYR2K): only tiles intersecting the referenced triangle.
template <int BM, int BN>
struct Tiles {
  // m-tiles per group: 8 pair tiles (2048 rows) -- a wave of 74 pair tiles then
  // spans ~8 x 9 tiles (near square), which cut SGEMM N=8192 DRAM reads from
  // 3.34 to 2.60 GB vs 16 (ncu; time unchanged within noise, tools/raster_probe.py)
  static constexpr int GM = 8;

  HD static int64_t tri_first_m(int64_t j) { return (j * BN) / BM; }          // lower
  HD static int64_t tri_end_m(int64_t j, int64_t mt) {                        // upper
    return imin(mt, (j * BN + BN - 1) / BM + 1);
  }

  HD static int64_t count(const Problem &P) {
    int64_t mt = cdiv(P.M, BM), nt = cdiv(P.N, BN);
    if (P.c_tri == 0) return mt * nt;
    int64_t c = 0;
    for (int64_t j = 0; j < nt; ++j)
      c += (P.c_tri == 1) ? imax(0, mt - tri_first_m(j)) : tri_end_m(j, mt);
    return c;
  }

  // tile index -> (m-tile, n-tile)
  HD static void coords(const Problem &P, int64_t t, int64_t &mi, int64_t &nj) {
    int64_t mt = cdiv(P.M, BM), nt = cdiv(P.N, BN);
    if (P.c_tri == 0 && P.outer == 1) {          // whole m-rows in turn (with rev_m:
      mi = t / nt; nj = t - mi * nt;             // longest-processing-time first)
    } else if (P.c_tri == 0 && P.outer == 2) {
      nj = t / mt; mi = t - nj * mt;
    } else if (P.c_tri == 0) {
      const int64_t G = P.raster_gm > 0 ? P.raster_gm : GM;
      int64_t per_group = G * nt;
      int64_t g = t / per_group, local = t - g * per_group;
      int64_t gm = imin(G, mt - g * G);
      mi = g * G + local % gm;
      nj = local / gm;
    } else {
      // longest columns of the triangle first
      for (int64_t jj = 0; jj < nt; ++jj) {
        int64_t j = (P.c_tri == 1) ? jj : nt - 1 - jj;
        int64_t i0 = (P.c_tri == 1) ? tri_first_m(j) : 0;
        int64_t i1 = (P.c_tri == 1) ? mt : tri_end_m(j, mt);
        int64_t cnt = imax(0, i1 - i0);
        if (t < cnt) { mi = i0 + t; nj = j; return; }
        t -= cnt;
      }
      mi = 0; nj = 0;
    }
    if (P.rev_m) mi = mt - 1 - mi;
    if (P.rev_n) nj = nt - 1 - nj;
  }
};

// ---------------------------------------------------------------- K range (peel)
// Blank k-blocks of a triangular operand are skipped for the whole tile
// (peel_triangular): the tile's k-range is clipped at the diagonal.
HD void k_range_op(const OpDesc &o, int64_t r0, int64_t r1, int64_t K,
                   int64_t &k0, int64_t &k1) {
  if (o.kind != OP_TRI) return;
  if (tri_kle(o)) k1 = imin(k1, r1);       // k <= r  -> k < r1
  else            k0 = imax(k0, r0);       // k >= r
  (void)K;
}

// k-range [k0,k1) (element units) of segment s for the tile rows
// [m0,m1) x cols [n0,n1); rounded outward to BK by the caller.
HD void k_range(const Segment &s, int64_t m0, int64_t m1, int64_t n0, int64_t n1,
                int64_t &k0, int64_t &k1) {
  k0 = 0; k1 = s.K;
  k_range_op(s.a, m0, m1, s.K, k0, k1);
  k_range_op(s.b, n0, n1, s.K, k0, k1);
  if (k1 < k0) k1 = k0;
}

// ---------------------------------------------------------------- block classes
// Which stored view(s) a (rows [r0,r1)) x (k [k0,k1)) block of an operand needs.
enum BlockClass : int32_t {
  BLK_RK = 0,      // whole block from the rk view, no fix-up
  BLK_KR = 1,      // whole block from the kr view, no fix-up
  BLK_SYM_DIAG = 2,// symmetric block crossing the diagonal: rk + kr merged
  BLK_TRI_DIAG = 3,// triangular block touching the diagonal: zero-select/unit
  BLK_ZERO = 4     // entirely blank (never loaded)
};

HD int32_t block_class(const OpDesc &o, int64_t r0, int64_t r1, int64_t k0, int64_t k1) {
  // r1, k1 exclusive and > r0, k0.
  if (o.kind == OP_DENSE) return o.kr ? BLK_KR : BLK_RK;
  if (o.kind == OP_SYM) {
    // rk source iff (lower ? r >= k : r <= k)
    bool all_rk = o.lower ? (r0 >= k1 - 1) : (r1 - 1 <= k0);
    bool all_kr = o.lower ? (r1 - 1 <= k0) : (r0 >= k1 - 1);
    if (all_rk) return BLK_RK;
    if (all_kr) return BLK_KR;
    return BLK_SYM_DIAG;
  }
  // TRI: strictly-nonzero block, blank block, or diagonal-touching block
  bool kle = tri_kle(o);
  bool full = kle ? (k1 - 1 < r0) : (k0 > r1 - 1);
  bool blank = kle ? (k0 > r1 - 1) : (k1 - 1 < r0);
  if (blank) return BLK_ZERO;
  if (full || (o.zero_blank && !o.unit)) return o.swap ? BLK_KR : BLK_RK;
  return BLK_TRI_DIAG;
}

// Element fetch with all structure applied (bounds -> 0).  Used by the SIMT
// kernel for every element and by the tcgen05 transform on diagonal blocks.
#ifdef __CUDACC__
__device__ __forceinline__ float load_op(const OpDesc &o, int64_t r, int64_t k,
                                         int64_t R, int64_t K) {
  if (r >= R || k >= K) return 0.f;
  const float *g = o.ptr;
  if (o.kind == OP_DENSE) return o.kr ? __ldg(g + k + r * o.ld) : __ldg(g + r + k * o.ld);
  if (o.kind == OP_SYM) {
    bool rk = o.lower ? (r >= k) : (r <= k);
    return rk ? __ldg(g + r + k * o.ld) : __ldg(g + k + r * o.ld);
  }
  bool nz = tri_kle(o) ? (k <= r) : (k >= r);
  if (!nz) return 0.f;
  if (k == r && o.unit) return 1.f;
  return o.swap ? __ldg(g + k + r * o.ld) : __ldg(g + r + k * o.ld);
}
#endif

}  // namespace blas3
