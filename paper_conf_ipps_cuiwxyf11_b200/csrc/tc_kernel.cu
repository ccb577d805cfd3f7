// tc_kernel.cu -- the one tuned GEMM every routine derives from, B200-native:
// TMA -> shared memory -> staging transform -> tcgen05.mma (3xTF32) -> TMEM
// -> epilogue.  Rows A2-A6 of the hot-path table.
//
// Paper mapping:
//   thread_grouping / loop_tiling  -> persistent CTAs (or CTA
//       pairs, tcgen05 cta_group::2) over a 128x256 (256x256) tile schedule
//       (Tiles<> in problem.h), BK = 32 k-blocks;
//   SM_alloc(X, Transpose|Symmetry)   -> TMA loads each k-block in
//       the orientation it is stored in (K-major or MN-major 128B-swizzled
//       tiles; the UMMA descriptor's major bit absorbs the transpose), and
//       symmetric blocks crossing the diagonal are MERGED from both stored
//       orientations while staging (selection, never src+src^T-diag, Q7);
//   padding/peel_triangular         -> blank k-blocks skipped via
//       the tile's k-range, diagonal blocks zero-SELECTED (+unit diagonal)
//       in shared memory (the blank triangle is never multiplied, Q8);
//   Reg_alloc(C)                        -> fp32 accumulator in TMEM
//       (two 256-column accumulators: epilogue of tile i overlaps tile i+1).
// fp32 accuracy on TF32 tensor cores (north star): every staged value x is
// split into hi = trunc_tf32(x) -- what the tensor core reads from the raw
// TMA-staged word (kind::tf32 ignores the low 13 mantissa bits, DESIGN.md
// Q23) -- and lo = x - hi (exact in fp32, written by the transform warps);
// each k8-step issues lo*hi + hi*lo + hi*hi (small terms first) into one fp32
// TMEM partial that is restarted every Problem::kc k-blocks (Q24).
//
// Warp roles (640 threads, 1 CTA/SM, aligned to warpgroups for setmaxnreg;
// in a pair every CTA runs all roles on its own halves except the MMA issuer,
// which only the leader CTA runs):
//   warp 0        TMA producer (one lane)
//   warp 1        TMEM allocator + MMA issuer (one lane)
//   warps 2..3    idle (pad the first warpgroup)
//   warps 4..11   transform: structure fix-ups + lo split (256 threads)
//   warps 12..19  epilogue: tcgen05.ld -> running sum -> alpha*S + beta*C ->
//                 global (two warps per TMEM lane quarter, 128 columns each)
#include <cuda.h>
#include <cuda_runtime.h>
#include <atomic>
#include <mutex>
#include <vector>
#include <cstdio>
#include <stdlib.h>
#include <string.h>

#include "../../include/blas3.h"
#include "kernels.h"
#include "tc_ptx.h"
#include "tc_stage.h"
#include <cuda_bf16.h>

namespace blas3 {

namespace {
// Tile geometry.  CG = CTA group: CG=1 -> one CTA computes a 128x256 tile;
// CG=2 -> a CTA pair (cluster of 2, tcgen05 cta_group::2) computes a 256x256
// tile, each CTA staging its 128 rows of A and 128 of the 256 B rows: per SM
// the tensor core reads half as many B bytes per flop, and shared-memory
// bandwidth is what bounds this kernel (profiles/r01_sgemm_ncu.md).
constexpr int BK = stage::BK;
constexpr int HA = 128;                    // A rows staged per CTA
constexpr int BN = 256;                    // tile columns (UMMA N)
// Roles are aligned to warpgroups so setmaxnreg can move registers to the
// epilogue, which holds a 128-column fp32 running sum per thread.
constexpr int WARP_TMA = 0, WARP_MMA = 1, WARP_TR0 = 4, NUM_TR_WARPS = 8;
constexpr int WARP_EPI0 = WARP_TR0 + NUM_TR_WARPS, NUM_EPI_WARPS = 8;
constexpr int NTHREADS = (WARP_EPI0 + NUM_EPI_WARPS) * 32;       // 640
// setmaxnreg moves registers inside the CTA's own pool (the launch allocation,
// 96 x 640 = 61440), so 256*EPI_REGS + 384*OTHER_REGS must not exceed it.
constexpr int EPI_REGS = 144, OTHER_REGS = 64;   // 36864 + 24576 = 61440
// Chunked accumulation: the tensor core's fp32 accumulator truncates on every
// UMMA add (Q24), so a TMEM partial only ever sums Problem::kc
// k-blocks (BLAS3_OPT_TC_KC, default 3: K = 96) before the epilogue folds it
// into a register running sum with round-to-nearest adds; the two TMEM
// buffers ping-pong per chunk.
constexpr int EC = 16;                            // epilogue column group
// Tile queue: the producer warp claims tiles (atomic counter, or the static
// round-robin sequence for CTA pairs) and hands them to the MMA, transform
// and epilogue roles through a TQ-deep shared-memory queue.
constexpr int TQ = 4;
constexpr int TR_THREADS = NUM_TR_WARPS * 32;
constexpr int EPI_THREADS = NUM_EPI_WARPS * 32;
constexpr int TMEM_COLS = 512;             // 2 accumulators x BN columns
constexpr int MAX_MAPS = 10;                 // 2 segments x 2 operands x 2 views + C
// epilogue: per epilogue warp one 32-row x 8-column fp32 shared box, the
// transpose between the TMEM layout (thread = row) and 16-B vector accesses
// of column-major C (thread = 4 consecutive rows of one column)
constexpr int EPI_GW = 8, EPI_BOX = 32 * EPI_GW;
using stage::LAYOUT_K;
using stage::LAYOUT_MN;
using stage::op_desc;
using stage::spin_until;

// A work item: the tile (batch member b, tile t at m0, n0) and the range
// [g0, g1) of its k-blocks, counted over the concatenated segments.
struct Work {
  int64_t tb, b, t, m0, n0, g0, g1;
  int32_t slice;          // k-slice of a split tile, or -1 for a whole tile
  int32_t ph;             // phase of a fused launch (0 otherwise)
};

// Two shared-memory rings: a deep RAW ring (TMA destination, read by UMMA as
// hi) lets TMA run RS k-blocks ahead to hide load latency, and a shallow LO
// ring (written by the transform) only has to cover transform/MMA overlap.
template <int CG>
struct Geo {
  static constexpr int TM = HA * CG;                 // tile rows
  static constexpr int HB = BN / CG;                 // B rows staged per CTA
  static constexpr uint32_t A_BYTES = HA * BK * 4;
  static constexpr uint32_t B_BYTES = HB * BK * 4;
  static constexpr int RS = CG == 1 ? 2 : 4;         // raw stages
  static constexpr int LS = 2;                       // lo stages
  struct alignas(1024) RawBuf {
    uint8_t A[A_BYTES];      // TMA destination; read by UMMA as hi (low 13 bits ignored)
    uint8_t B[B_BYTES];
  };
  struct alignas(1024) LoBuf {
    uint8_t A[A_BYTES];      // lo = x - hi (exact in fp32), written by the transform
    uint8_t B[B_BYTES];
  };
  struct Barriers {
    uint64_t full[RS];       // TMA -> transform (expect_tx), local
    uint64_t empty[RS];      // MMA -> TMA: raw slot free (tcgen05.commit, multicast)
    uint64_t ready[LS];      // transform -> MMA (one arrival per CTA of the pair, leader)
    uint64_t lo_empty[LS];   // MMA -> transform: lo slot free (tcgen05.commit, multicast)
    uint64_t tq_full[TQ];    // leader producer -> peer producer: item index published
    uint64_t tq_empty[TQ];   // roles -> leader producer: slot read (3 per CTA; +1 peer producer)
    int64_t tq[TQ];
    uint64_t wk_full[TQ];    // local producer -> local roles: decoded work item published
    Work wk[TQ];
    uint64_t tfull[2];       // MMA -> epilogue: TMEM partial ready (multicast to the pair)
    uint64_t mirror;         // transform: the mirrored view of a symmetric diagonal block landed
    uint64_t tempty[2];      // epilogue -> MMA: partial drained (one arrival per CTA, leader)
    uint32_t tmem_base;
    uint32_t split_last;     // epilogue: this CTA's slice of a split tile is the last one
  };
  struct alignas(1024) EpiStage {
    float box[NUM_EPI_WARPS][3][EPI_BOX];   // epilogue: transpose box + 2 C boxes per warp
  };
  static constexpr size_t SMEM =
      sizeof(RawBuf) * RS + sizeof(LoBuf) * LS + sizeof(EpiStage) + sizeof(Barriers) + 1024;
};

// One phase of a launch: a Problem, the work items it owns and, in a FUSED
// launch (several dependent problems in one persistent grid, e.g. the STRSM
// sweep), the phases it waits for.  Dependencies are tile counters in global
// memory: a tile of phase p starts once every phase in dep_full is complete
// and every phase in dep_slab is complete on the same SLAB (column block of
// the right-hand side for side=L, row block for side=R): the right-hand-side
// columns of a triangular solve are independent, so the sweep advances as a
// wavefront instead of phase by phase.  Items are numbered phase by phase in
// dependency order and claimed in that order, so every dependency of a
// claimed tile belongs to an earlier claim of a running CTA (no deadlock).
struct PhaseDesc {
  Problem P;
  int64_t item0;           // first work item of this phase
  int64_t tiles_per;       // tiles of one batch member (Tiles<TM,BN>::count)
  int64_t ntiles;          // tiles of the phase (all batch members)
  int32_t dep_full;        // bitmask of phases that must be complete
  int32_t dep_slab;        // bitmask of phases that must be complete on this tile's slab
  int32_t slab_m;          // slab = m-tile (1) or n-tile (0)
  int32_t slab_cnt;        // tiles of this phase per slab
};
constexpr int MAX_SLAB = 128;            // slab counters per phase (32768 / 256)

template <int NPH, int NMAPS>
struct TcParamsT {
  CUtensorMap maps[NMAPS];
  PhaseDesc ph[NPH];
  int32_t nphase;
  uint32_t *tile_ctr;      // dynamic tile scheduler counter, or null (static schedule);
                           // 0 when the launch starts and left at 0 by its last claim
  uint32_t tile_claims;    // atomic claims this launch makes in total
  // Split tail (wave quantisation, single-phase launches): work items [0, khead)
  // are whole tiles; the last (ntiles - khead) tiles are cut into ksplit
  // k-slices each, item khead + j -> tile khead + j / ksplit, slice j % ksplit.
  // Slices write fp32 partials to ws; the last arriving slice (ws_cnt) reduces
  // them in slice order and runs the epilogue.
  int64_t nitems, khead;
  int32_t ksplit;
  float *ws;
  uint32_t *ws_cnt;
  uint32_t *dep_ctr;       // fused: [NPH] phase counters, then [NPH][MAX_SLAB] slab counters
  unsigned long long *trace;   // phase timestamps of CTA 0 (env BLAS3_TRACE), or null
  unsigned long long *ph_trace;  // fused, BLAS3_TRACE=2: per phase [first dep-ready, last done] (ns)
  unsigned long long *st_trace;  // fused, BLAS3_TRACE_PH=p: per stage [min, max] over phase p's tiles
  int32_t st_phase;
};
using TcParams = TcParamsT<1, MAX_MAPS>;
constexpr int FUSED_PH = 24, FUSED_MAPS = 72;
using TcFusedParams = TcParamsT<FUSED_PH, FUSED_MAPS>;
static_assert(sizeof(TcFusedParams) <= 32764, "kernel parameter block exceeds 32764 bytes");

// %globaltimer (ns) of the first occurrence of a phase in CTA 0 (diagnostics)
#define BLAS3_TRACE(i)                                                              \
  do {                                                                              \
    if (prm.trace != nullptr && blockIdx.x == 0 && prm.trace[i] == 0ull) {          \
      unsigned long long t_;                                                        \
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));                        \
      prm.trace[i] = t_;                                                            \
    }                                                                               \
  } while (0)


// fused launches, BLAS3_TRACE_PH=p: earliest and latest %globaltimer at which
// any CTA reached stage i for a tile of phase p (diagnostics)
#define BLAS3_STRACE(i, ph_)                                                        \
  do {                                                                              \
    if (FUSED && prm.st_trace != nullptr && (ph_) == prm.st_phase) {               \
      unsigned long long t_;                                                        \
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));                        \
      atomicMin(prm.st_trace + 2 * (i), t_);                                        \
      atomicMax(prm.st_trace + 2 * (i) + 1, t_);                                    \
    }                                                                               \
  } while (0)

// byte offset of element (r, k) inside a staged operand tile
__device__ __forceinline__ uint32_t off_k(int r, int k) {       // K-major, 128 B per row r
  return (uint32_t)(r * 128 + ((((k >> 2) ^ (r & 7)) & 7) << 4) + (k & 3) * 4);
}
// MN-major, 32-row chunks of BK 128-B rows; 128B swizzle with 32-B atomicity
// (TMA SWIZZLE_128B_ATOM_32B == UMMA SWIZZLE_128B_BASE32B == Swizzle<2,5,2>)
__device__ __forceinline__ uint32_t off_mn(int r, int k) {
  return (uint32_t)((r >> 5) * (BK * 128) + k * 128 + (((((r & 31) >> 3) ^ (k & 3)) & 3) << 5) +
                    (r & 7) * 4);
}

__host__ __device__ __forceinline__ int layout_of(const OpDesc &o, int cls) {
  if (o.kind == OP_DENSE) return o.kr ? LAYOUT_K : LAYOUT_MN;
  if (cls == BLK_KR) return LAYOUT_K;
  if (cls == BLK_TRI_DIAG) return o.swap ? LAYOUT_K : LAYOUT_MN;
  return LAYOUT_MN;   // BLK_RK, BLK_SYM_DIAG (merged into the rk orientation)
}

struct StageInfo {
  int clsA, clsB, layA, layB;
};

// Block classes are decided on the WHOLE tile (both CTAs of a pair), so the
// UMMA major bits agree for the two halves; a half whose own block would be
// plain real/shadow is then merged per element, which selects the same values.
template <int CG>
__device__ __forceinline__ StageInfo stage_info(const Problem &P, const Segment &sg, int64_t m0,
                                                int64_t n0, int64_t k0) {
  StageInfo si;
  const int64_t k1 = imin(sg.K, k0 + BK);
  si.clsA = block_class(sg.a, m0, imin(P.M, m0 + Geo<CG>::TM), k0, k1);
  si.clsB = block_class(sg.b, n0, imin(P.N, n0 + BN), k0, k1);
  si.layA = layout_of(sg.a, si.clsA);
  si.layB = layout_of(sg.b, si.clsB);
  return si;
}

// An operand's block class can only change on the k-blocks that intersect
// its rows [r0, r1) (the diagonal band); below and above the band it is
// constant (SYM: rk / kr view; TRI: nonzero / blank).  So per segment the
// band (hull over both operands) and the two outer StageInfos are computed
// once, and stage_info runs per k-block only inside the band (dense
// operands have no band at all).
struct StageBand {
  int64_t b0, b1;
  StageInfo lo, hi;
};
template <int CG>
__device__ __forceinline__ StageBand make_band(const Problem &P, const Segment &sg, int64_t m0,
                                               int64_t n0) {
  StageBand bd;
  bd.b0 = INT64_MAX;
  bd.b1 = INT64_MIN;
  if (sg.a.kind != OP_DENSE) {
    bd.b0 = imin(bd.b0, m0 / BK);
    bd.b1 = imax(bd.b1, cdiv(imin(P.M, m0 + Geo<CG>::TM), BK));
  }
  if (sg.b.kind != OP_DENSE) {
    bd.b0 = imin(bd.b0, n0 / BK);
    bd.b1 = imax(bd.b1, cdiv(imin(P.N, n0 + BN), BK));
  }
  if (bd.b1 < bd.b0) bd.b0 = bd.b1 = 0;           // both dense: one class everywhere
  bd.lo = stage_info<CG>(P, sg, m0, n0, imax(0, bd.b0 - 1) * BK);
  bd.hi = stage_info<CG>(P, sg, m0, n0, imin(imax(0, cdiv(sg.K, BK) - 1), bd.b1) * BK);
  return bd;
}
template <int CG>
__device__ __forceinline__ StageInfo stage_at(const StageBand &bd, const Problem &P, const Segment &sg,
                                              int64_t m0, int64_t n0, int64_t kb) {
  if (kb < bd.b0) return bd.lo;
  if (kb >= bd.b1) return bd.hi;
  return stage_info<CG>(P, sg, m0, n0, kb * BK);
}

template <int CG>
HD void seg_kblocks(const Problem &P, const Segment &sg, int64_t m0,
                                            int64_t n0, int64_t &kb0, int64_t &kb1) {
  int64_t k0, k1;
  k_range(sg, m0, imin(P.M, m0 + Geo<CG>::TM), n0, imin(P.N, n0 + BN), k0, k1);
  kb0 = k0 / BK;
  kb1 = (k1 > k0) ? cdiv(k1, BK) : kb0;
}

template <int CG>
HD int64_t tile_kblocks(const Problem &P, int64_t m0, int64_t n0) {
  int64_t tot = 0;
  for (int s = 0; s < P.nseg; ++s) {
    int64_t a, b;
    seg_kblocks<CG>(P, P.seg[s], m0, n0, a, b);
    tot += b - a;
  }
  return tot;
}

template <int CG, class PRM>
__device__ __forceinline__ Work work_of(const PRM &prm, int64_t item) {
  Work w;
  w.slice = -1;
  w.ph = 0;
  if constexpr (sizeof(prm.ph) / sizeof(prm.ph[0]) > 1) {
    for (int q = 1; q < prm.nphase; ++q)
      if (item >= prm.ph[q].item0) w.ph = q;
    item -= prm.ph[w.ph].item0;
  }
  const Problem &P = prm.ph[w.ph].P;
  const int64_t tiles_per = prm.ph[w.ph].tiles_per;
  w.tb = item;
  if (item >= prm.khead && prm.ksplit > 1) {
    const int64_t j = item - prm.khead;
    w.tb = prm.khead + j / prm.ksplit;
    w.slice = (int32_t)(j % prm.ksplit);
  }
  w.b = w.tb / tiles_per;
  w.t = w.tb - w.b * tiles_per;
  int64_t mi, nj;
  Tiles<Geo<CG>::TM, BN>::coords(P, w.t, mi, nj);
  w.m0 = mi * Geo<CG>::TM;
  w.n0 = nj * BN;
  const int64_t nkb = tile_kblocks<CG>(P, w.m0, w.n0);
  w.g0 = 0;
  w.g1 = nkb;
  if (w.slice >= 0) {
    w.g0 = nkb * w.slice / prm.ksplit;
    w.g1 = nkb * (w.slice + 1) / prm.ksplit;
  }
  return w;
}
// clip a segment's k-blocks [kb0, kb1) to the item's range; gi counts the
// k-blocks of the earlier segments
__device__ __forceinline__ void clip_kblocks(const Work &w, int64_t &gi, int64_t &kb0, int64_t &kb1) {
  const int64_t n = kb1 - kb0;
  const int64_t lo = imax(0, w.g0 - gi), hi = imin(n, w.g1 - gi);
  gi += n;
  kb1 = kb0 + imax(lo, hi);
  kb0 = kb0 + lo;
}

// ---------------------------------------------------------------- producer
// Every operand map is 4-D: (element dims) x (batch-inner, batch-outer);
// (bj, bg) select the batch member (0, 0 for an ordinary problem).
template <class PRM>
__device__ __forceinline__ void load_operand(const PRM &prm, const OpDesc &o, int lay,
                                             uint8_t *raw, int64_t r0, int64_t k0, int rows,
                                             uint64_t *bar, int32_t bj, int32_t bg) {
  if (lay == LAYOUT_MN) {
    const CUtensorMap *m = &prm.maps[o.map_rk];
    for (int c = 0; c < rows / 32; ++c) {
      ptx::tma_load_4d(m, bar, raw + c * (BK * 128), (int32_t)(r0 + 32 * c), (int32_t)k0, bj, bg);
    }
  } else {
    ptx::tma_load_4d(&prm.maps[o.map_kr], bar, raw, (int32_t)k0, (int32_t)r0, bj, bg);
  }
}

// ---------------------------------------------------------------- transform
// Symmetric block crossing the diagonal (staged from the rk view, MN-major):
// the elements whose stored position is the mirrored one (the "shadow area",
// P:144-148) are SELECTED from the block's kr view, S(r,k) := S(k,r), which
// the transform has TMA-loaded (K-major) into the stage's lo slot (`kr`):
// both orientations come from the stored triangle by TMA, no per-element
// global loads (selection, never src + src^T - diag, reading Q7).  Elements
// outside the matrix are zero in both views (TMA zero fill).
__device__ __forceinline__ void sym_merge(const OpDesc &o, uint8_t *raw, const uint8_t *kr, int64_t r0,
                                          int64_t k0, int rows, int t) {
  const int64_t d = r0 - k0;                       // gr - gk = d + r - k
  for (int e = t; e < rows * BK; e += TR_THREADS) {
    const int r = e / BK, k = e % BK;
    const bool mirrored = o.lower ? (d + r - k < 0) : (d + r - k > 0);
    if (mirrored)
      *reinterpret_cast<float *>(raw + off_mn(r, k)) = *reinterpret_cast<const float *>(kr + off_k(r, k));
  }
}

// Triangular block touching the diagonal: zero-select the blank part, force
// the unit diagonal (the stored values there are never used).
// Vectorised: both staged layouts keep 4 consecutive elements along the
// contiguous dimension (r for MN-major, k for K-major) in one 16-B word, so
// each thread handles float4s and rewrites one only when it crosses the
// blank triangle or the diagonal.
__device__ __forceinline__ void tri_fix(const OpDesc &o, int lay, uint8_t *raw, int64_t r0,
                                        int64_t k0, int rows, int64_t R, int64_t K, int t) {
  const bool kle = tri_kle(o);
  const bool unit = o.unit;
  const int nvec = rows * BK / 4;
  for (int e = t; e < nvec; e += TR_THREADS) {
    int r, k, dr, dk;          // first element and the step between the 4 lanes
    uint32_t off;
    if (lay == LAYOUT_MN) { r = (e % (rows / 4)) * 4; k = e / (rows / 4); dr = 1; dk = 0; off = off_mn(r, k); }
    else                  { k = (e % (BK / 4)) * 4; r = e / (BK / 4); dr = 0; dk = 1; off = off_k(r, k); }
    const int64_t d0 = (r0 + r) - (k0 + k);          // gr - gk of lane 0; lane j: d0 + j*(dr - dk)
    const int64_t d3 = d0 + 3 * (dr - dk);
    const int64_t dmin = d0 < d3 ? d0 : d3, dmax = d0 < d3 ? d3 : d0;
    // nonzero iff gr - gk >= 0 (kle) or <= 0; untouched if all 4 lanes are
    // strictly inside the nonzero region (no diagonal element either)
    if (kle ? dmin > 0 : dmax < 0) continue;
    float4 *p = reinterpret_cast<float4 *>(raw + off);
    if (kle ? dmax < 0 : dmin > 0) { *p = make_float4(0.f, 0.f, 0.f, 0.f); continue; }
    float v[4];
    *reinterpret_cast<float4 *>(v) = *p;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int64_t d = d0 + j * (dr - dk);
      const int64_t gr = r0 + r + j * dr, gk = k0 + k + j * dk;
      if (kle ? d < 0 : d > 0) v[j] = 0.f;
      else if (unit && d == 0 && gr < R && gk < K) v[j] = 1.f;
    }
    *p = *reinterpret_cast<float4 *>(v);
  }
}

__device__ __forceinline__ void zero_fill(uint8_t *buf, uint32_t bytes, int t) {
  float4 *b4 = reinterpret_cast<float4 *>(buf);
  for (uint32_t c = t; c < bytes / 16; c += TR_THREADS) b4[c] = make_float4(0.f, 0.f, 0.f, 0.f);
}

// BLAS3_MATH_TF32_BF16X: the two cross terms of the split packed into ONE bf16
// operand pair per k8 step.  For a staged tile (raw, either layout) with
// x = hi + lo (hi = trunc_tf32(x)), the K-major bf16 tile `dst` holds, per
// row and k8 chunk c, two 16-B chunks: A side [lo(8c..8c+7) | hi(8c..8c+7)],
// B side [hi | lo], so one K = 16 bf16 UMMA sums lo_A*hi_B + hi_A*lo_B.
// 128-B rows, SWIZZLE_128B (16-B chunk j of row r at (j ^ (r & 7)) << 4).
__device__ __forceinline__ uint32_t pack_bf16x2(float a, float b) {
  const __nv_bfloat162 v = __floats2bfloat162_rn(a, b);     // a -> low half (lower address)
  return *reinterpret_cast<const uint32_t *>(&v);
}
__device__ __forceinline__ void pack8(const float (&x)[8], uint8_t *row, int r, int c, bool a_side) {
  uint4 hi, lo;
  uint32_t *hp = &hi.x, *lp = &lo.x;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const float h0 = __uint_as_float(__float_as_uint(x[2 * i]) & 0xFFFFE000u);
    const float h1 = __uint_as_float(__float_as_uint(x[2 * i + 1]) & 0xFFFFE000u);
    hp[i] = pack_bf16x2(h0, h1);
    lp[i] = pack_bf16x2(x[2 * i] - h0, x[2 * i + 1] - h1);
  }
  *reinterpret_cast<uint4 *>(row + (((2 * c) ^ (r & 7)) << 4)) = a_side ? lo : hi;
  *reinterpret_cast<uint4 *>(row + (((2 * c + 1) ^ (r & 7)) << 4)) = a_side ? hi : lo;
}
// pack8 in two halves: the packed 16-B chunks into registers (no shared-memory
// writes), and their stores -- so the packing can run before the lo stage is free
struct Packed { uint4 first, second; };
__device__ __forceinline__ Packed pack8_regs(const float (&x)[8], bool a_side) {
  uint4 hi, lo;
  uint32_t *hp = &hi.x, *lp = &lo.x;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const float h0 = __uint_as_float(__float_as_uint(x[2 * i]) & 0xFFFFE000u);
    const float h1 = __uint_as_float(__float_as_uint(x[2 * i + 1]) & 0xFFFFE000u);
    hp[i] = pack_bf16x2(h0, h1);
    lp[i] = pack_bf16x2(x[2 * i] - h0, x[2 * i + 1] - h1);
  }
  return Packed{a_side ? lo : hi, a_side ? hi : lo};
}
__device__ __forceinline__ void store_packed(const Packed &v, uint8_t *row, int r, int c) {
  *reinterpret_cast<uint4 *>(row + (((2 * c) ^ (r & 7)) << 4)) = v.first;
  *reinterpret_cast<uint4 *>(row + (((2 * c + 1) ^ (r & 7)) << 4)) = v.second;
}
__device__ __forceinline__ void load8(const uint8_t *raw, int lay, int r, int c, float (&x)[8]) {
  if (lay == LAYOUT_K) {            // a row's 8 k-values: two swizzled 16-B chunks
    const float4 v0 = *reinterpret_cast<const float4 *>(raw + off_k(r, 8 * c));
    const float4 v1 = *reinterpret_cast<const float4 *>(raw + off_k(r, 8 * c + 4));
    x[0] = v0.x; x[1] = v0.y; x[2] = v0.z; x[3] = v0.w;
    x[4] = v1.x; x[5] = v1.y; x[6] = v1.z; x[7] = v1.w;
  } else {                          // MN-major: a warp's rows are contiguous per k
#pragma unroll
    for (int i = 0; i < 8; ++i) x[i] = *reinterpret_cast<const float *>(raw + off_mn(r, 8 * c + i));
  }
}
__device__ __forceinline__ void pack_cross(const uint8_t *raw, int lay, uint8_t *dst, int rows, int t,
                                           bool a_side) {
  // units (row r, k8 chunk c); two per thread at a time, loads issued first (ILP)
  const int units = rows * 4;
  for (int u = t; u < units; u += 2 * TR_THREADS) {
    const int u2 = u + TR_THREADS;
    const int r0 = u % rows, c0 = u / rows;
    const int r1 = u2 % rows, c1 = u2 / rows;
    float x0[8], x1[8];
    load8(raw, lay, r0, c0, x0);
    if (u2 < units) load8(raw, lay, r1, c1, x1);
    pack8(x0, dst + r0 * 128, r0, c0, a_side);
    if (u2 < units) pack8(x1, dst + r1 * 128, r1, c1, a_side);
  }
}

// ---------------------------------------------------------------- MMA
// A role's warps (nthreads, named barrier `id`) have finished with a stage:
// sync them CTA-locally, then ONE thread arrives on the barrier owned by the
// pair's leader (a cluster-scope release per thread would cost a GPU-scope
// membar + L1 invalidate each).
// ---------------------------------------------------------------- fused-launch dependencies
template <int CG>
__device__ __forceinline__ int64_t slab_of(const PhaseDesc &ph, const Work &w) {
  const int64_t s = ph.slab_m ? w.m0 / Geo<CG>::TM : w.n0 / BN;
  return s < MAX_SLAB ? s : MAX_SLAB - 1;
}
// Wait (one thread) until the tile's dependencies are complete; the acquire
// makes the producing CTAs' stores visible, and the proxy fence orders them
// before this CTA's later TMA (async-proxy) reads.
template <int CG, class PRM>
__device__ __forceinline__ void wait_deps(const PRM &prm, const Work &w, bool async_proxy = true) {
  if constexpr (sizeof(prm.ph) / sizeof(prm.ph[0]) > 1) {
    const PhaseDesc &ph = prm.ph[w.ph];
    if ((ph.dep_full | ph.dep_slab) == 0) return;
    const int64_t slab = slab_of<CG>(ph, w);
    for (int q = 0; q < prm.nphase; ++q) {
      if (ph.dep_full >> q & 1) spin_until(prm.dep_ctr + q, (uint32_t)(prm.ph[q].ntiles * CG));
      if (ph.dep_slab >> q & 1)
        spin_until(prm.dep_ctr + FUSED_PH + q * MAX_SLAB + slab, (uint32_t)(prm.ph[q].slab_cnt * CG));
    }
    if (prm.st_trace != nullptr && w.ph == prm.st_phase && async_proxy) {
      unsigned long long t_;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));
      atomicMin(prm.st_trace + 2 * 10, t_);
      atomicMax(prm.st_trace + 2 * 10 + 1, t_);
    }
    // the producer's TMA (async proxy) reads what other CTAs stored through
    // the generic proxy; the epilogue's plain loads need only the acquire
    if (async_proxy) asm volatile("fence.proxy.async.global;" ::: "memory");
  }
}
// After this CTA's stores of a tile (one thread, after the epilogue barrier).
template <int CG, class PRM>
__device__ __forceinline__ void signal_done(const PRM &prm, const Work &w) {
  if constexpr (sizeof(prm.ph) / sizeof(prm.ph[0]) > 1) {
    const PhaseDesc &ph = prm.ph[w.ph];
    __threadfence();
    atomicAdd(prm.dep_ctr + w.ph, 1u);
    atomicAdd(prm.dep_ctr + FUSED_PH + w.ph * MAX_SLAB + slab_of<CG>(ph, w), 1u);
  }
}

template <int CG>
__device__ __forceinline__ void arrive_leader(uint64_t *bar, uint32_t rank, uint32_t id,
                                              uint32_t nthreads, bool first) {
  ptx::named_bar_sync(id, nthreads);
  if (first) {
    if (CG == 1 || rank == 0) ptx::mbar_arrive(bar);
    else ptx::mbar_arrive_cluster(bar, 0);
  }
}

}  // namespace

// BX: the BLAS3_MATH_TF32_BF16X instantiation (packed bf16 cross terms); a
// compile-time switch so the default 3xTF32 kernel carries none of its code.
template <int CG, class PRM, bool BX = false>
__global__ void __launch_bounds__(NTHREADS, 1)
tc_structured_gemm(const __grid_constant__ PRM prm) {
  constexpr bool FUSED = sizeof(prm.ph) / sizeof(prm.ph[0]) > 1;
  constexpr int NMAPS = sizeof(prm.maps) / sizeof(prm.maps[0]);
  using G = Geo<CG>;
  using RawBuf = typename G::RawBuf;
  using LoBuf = typename G::LoBuf;
  using Barriers = typename G::Barriers;
  constexpr int RS = G::RS, LS = G::LS, TM = G::TM, HB = G::HB;
  extern __shared__ uint8_t smem_raw[];
  // 1024-B aligned base by pointer arithmetic on the __shared__ array (not via
  // an integer round trip), so the compiler keeps the shared address space and
  // emits LDS/STS instead of generic loads/stores in the transform
  uint8_t *smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  RawBuf *raw = reinterpret_cast<RawBuf *>(smem);
  LoBuf *lo = reinterpret_cast<LoBuf *>(smem + sizeof(RawBuf) * RS);
  float *epi_stage = reinterpret_cast<float *>(smem + sizeof(RawBuf) * RS + sizeof(LoBuf) * LS);
  Barriers *bars = reinterpret_cast<Barriers *>(smem + sizeof(RawBuf) * RS + sizeof(LoBuf) * LS +
                                                sizeof(typename G::EpiStage));
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const uint32_t rank = (CG == 2) ? ptx::cluster_ctarank() : 0;
  const int64_t cid = blockIdx.x / CG, ncl = gridDim.x / CG;

  if (threadIdx.x == 0) {
    BLAS3_TRACE(0);
    for (int s = 0; s < RS; ++s) {
      ptx::mbar_init(&bars->full[s], 1);
      ptx::mbar_init(&bars->empty[s], 1);
    }
    for (int s = 0; s < LS; ++s) {
      ptx::mbar_init(&bars->ready[s], CG);
      ptx::mbar_init(&bars->lo_empty[s], 1);
    }
    for (int q = 0; q < TQ; ++q) {
      ptx::mbar_init(&bars->wk_full[q], 1);
      ptx::mbar_init(&bars->tq_full[q], 1);
      ptx::mbar_init(&bars->tq_empty[q], CG == 1 ? 3 : 7);
    }
    for (int a = 0; a < 2; ++a) {
      ptx::mbar_init(&bars->tfull[a], 1);
      ptx::mbar_init(&bars->tempty[a], CG);
    }
    ptx::mbar_init(&bars->mirror, 1);
    ptx::fence_mbar_init();
  }
  if (warp == WARP_MMA) ptx::tmem_alloc<CG>(&bars->tmem_base, TMEM_COLS);
  ptx::tc_fence_before();
  if (CG == 2) ptx::cluster_sync(); else __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = bars->tmem_base;
  // Everything above (barrier init, TMEM allocation, tensor-map prefetch)
  // overlaps the tail of the previous kernel of the stream when launched with
  // PDL; no global memory is touched before the previous grid is complete.
  ptx::griddep_wait();
  if (threadIdx.x == 0) BLAS3_TRACE(1);

  // Tile queue.  The (leader) producer claims work items and publishes them
  // (to the peer producer too, for a CTA pair); every CTA's producer decodes
  // its item once (work_of) into wk[slot] for the local roles.  Consumer
  // side: every thread of a role reads the slot, then one thread releases it
  // at the leader (all roles of both CTAs, plus the peer producer).
  auto next_work = [&](uint32_t &qi, uint32_t bar_id, uint32_t nthreads, bool first) -> Work {
    const int slot = qi % TQ;
    ptx::mbar_wait(&bars->wk_full[slot], (qi / TQ) & 1);
    const Work w = *const_cast<const Work *>(&bars->wk[slot]);
    if (nthreads > 32) ptx::named_bar_sync(bar_id, nthreads);
    else if (nthreads == 32) __syncwarp();
    if (first) {
      if (CG == 1 || rank == 0) ptx::mbar_arrive(&bars->tq_empty[slot]);
      else ptx::mbar_arrive_cluster(&bars->tq_empty[slot], 0);
    }
    ++qi;
    return w;
  };

  // register rebalancing per warpgroup role (setmaxnreg dominates each role's code)
#define BLAS3_DEC_REGS() asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(OTHER_REGS))
#define BLAS3_INC_REGS() asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(EPI_REGS))
  if (warp < WARP_TR0) {
    // first warpgroup: TMA producer (warp 0), MMA issuer (warp 1), 2 spares.
    // setmaxnreg is warpgroup-collective: one instruction, one PC.
    BLAS3_DEC_REGS();
   if (warp == WARP_TMA) {
    // ============================ TMA producer (each CTA stages its own halves)
    if (lane == 0) {
      for (int i = 0; i < NMAPS; ++i) ptx::tma_prefetch(&prm.maps[i]);
      uint32_t it = 0;
      int64_t a_ready_upto = 0;              // streamed A: panels [0, this) seen ready
      for (uint32_t qi = 0;;) {
        int64_t tb;
        const int slot = qi % TQ;
        const uint32_t par = (qi / TQ) & 1;
        if (CG == 1 || rank == 0) {
          // claim an item (dynamic) or take the static round-robin one
          // (the first item of every producer is its own id: no claim round
          // trip -- except in a fused launch, whose items are claimed strictly
          // in dependency order by running CTAs)
          if ((FUSED || qi > 0) && prm.tile_ctr != nullptr) {
            const uint32_t v = atomicAdd(prm.tile_ctr, 1u);
            // the launch's last claim (claims are totally ordered, and no
            // producer claims again after a failing one) resets the counter,
            // so every launch -- and every replay of a captured CUDA graph --
            // starts from 0
            if (v == prm.tile_claims - 1) atomicExch(prm.tile_ctr, 0u);
            tb = FUSED ? (int64_t)v : ncl + (int64_t)v;
          } else {
            tb = cid + (int64_t)qi * ncl;
          }
          if (tb >= prm.nitems) tb = -1;
          BLAS3_TRACE(2);
          ptx::mbar_wait(&bars->tq_empty[slot], par ^ 1);
          if (CG == 2) ptx::st_remote_and_arrive(&bars->tq[slot], tb, &bars->tq_full[slot], 1);
        } else {                                      // the pair's peer follows the leader
          ptx::mbar_wait(&bars->tq_full[slot], par);
          tb = *reinterpret_cast<volatile int64_t *>(&bars->tq[slot]);
          ptx::mbar_arrive_cluster(&bars->tq_empty[slot], 0);
        }
        Work w;
        if (tb >= 0) w = work_of<CG>(prm, tb);
        else w.tb = -1;
        // fused launches: the producing tiles are complete (gpu-scope acquire)
        // BEFORE the item is published, so every local role that takes it
        // through wk_full (release / acquire at CTA scope) also observes the
        // producing CTAs' stores -- the epilogue needs no acquire of its own
        if (tb >= 0) wait_deps<CG>(prm, w);
        bars->wk[slot] = w;
        ptx::mbar_arrive(&bars->wk_full[slot]);       // release: local roles see wk[slot]
        ++qi;
        if (tb < 0) {
          // this CTA has claimed its last tile: the next kernel of the stream
          // may be scheduled onto SMs as they drain (PDL)
          ptx::griddep_launch_dependents();
          break;
        }
        const Problem &P = prm.ph[FUSED ? w.ph : 0].P;
        const int64_t per = P.per > 0 ? P.per : 1;
        const int32_t bj = (int32_t)(w.b % per), bg = (int32_t)(w.b / per);
        const int64_t m0 = w.m0, n0 = w.n0;
        const int64_t ma = m0 + HA * rank, nb = n0 + HB * rank;
        BLAS3_STRACE(0, w.ph);
        if (FUSED && prm.ph_trace != nullptr) {
          unsigned long long t_;
          asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));
          atomicMin(prm.ph_trace + 2 * w.ph, t_);
        }
        // C (beta != 0) into L2 while the tile's last k-blocks are loaded: the
        // epilogue's loads then hit L2, which keeps its store phase (during
        // which the next tile's TMEM partials wait to be drained) short
        int64_t pf_left = (P.c_pf_map >= 0 && w.slice < 0) ? imax(0, (w.g1 - w.g0) - 6) : -1;
        int64_t gi = 0;
        for (int s = 0; s < P.nseg; ++s) {
          const Segment &sg = P.seg[s];
          int64_t kb0, kb1;
          seg_kblocks<CG>(P, sg, m0, n0, kb0, kb1);
          clip_kblocks(w, gi, kb0, kb1);
          const StageBand bd = make_band<CG>(P, sg, m0, n0);
          for (int64_t kb = kb0; kb < kb1; ++kb, ++it) {
            if (pf_left-- == 0) {
              ptx::tma_prefetch_l2_4d(&prm.maps[P.c_pf_map], (int32_t)ma, (int32_t)n0, bj, bg);
              ptx::tma_prefetch_l2_4d(&prm.maps[P.c_pf_map], (int32_t)ma, (int32_t)(n0 + BN / 2), bj, bg);
            }
            const int rs = it % RS;
            const uint32_t ph = (it / RS) & 1;
            const int64_t k0 = kb * BK;
            const StageInfo si = stage_at<CG>(bd, P, sg, m0, n0, kb);
            if (P.a_ready != nullptr && s == 0 && kb / P.a_panel_kb >= a_ready_upto) {
              // streamed A: its panel has landed (acquire), then the TMA reads it
              spin_until(P.a_ready + kb / P.a_panel_kb, P.a_ready_val);
              asm volatile("fence.proxy.async.global;" ::: "memory");
              a_ready_upto = kb / P.a_panel_kb + 1;
            }
            ptx::mbar_wait(&bars->empty[rs], ph ^ 1);
            if (P.dbg & 16) { ptx::mbar_arrive(&bars->full[rs]); continue; }   // diag: no loads
            ptx::mbar_arrive_expect_tx(&bars->full[rs], (HA + HB) * BK * 4);
            load_operand(prm, sg.a, si.layA, raw[rs].A, ma, k0, HA, &bars->full[rs], bj, bg);
            load_operand(prm, sg.b, si.layB, raw[rs].B, nb, k0, HB, &bars->full[rs], bj, bg);
            BLAS3_TRACE(3);
            if (kb == kb0) BLAS3_STRACE(1, w.ph);
          }
        }
      }
      // producer tail: every raw slot released by the MMA before the CTA retires
      for (int i = 0; i < RS; ++i, ++it)
        ptx::mbar_wait(&bars->empty[it % RS], ((it / RS) & 1) ^ 1);
    }
   } else if (warp == WARP_MMA) {
    // ============================ MMA issuer (leader CTA of the pair only)
    if (rank != 0) {                          // peer CTA: only drain the tile queue
      uint32_t qi = 0;
      while (next_work(qi, 0, 32, lane == 0).tb >= 0) {}
    } else {
      uint32_t it = 0, cc = 0, qi = 0;          // k-block, TMEM-chunk, tile-queue counters
      for (;;) {
        const Work w = next_work(qi, 0, 32, lane == 0);
        if (w.tb < 0) break;
        const Problem &P = prm.ph[FUSED ? w.ph : 0].P;
        const int64_t m0 = w.m0, n0 = w.n0;
        const int64_t nkb = w.g1 - w.g0;
        int64_t done = 0;
        int32_t chunk_left = 0;                     // k-blocks left in the open TMEM chunk
        uint32_t accumulate = 0, buf = 0;
        auto open_chunk = [&]() {
          buf = cc & 1;
          const uint32_t aph = (cc >> 1) & 1;
          if (CG == 2) ptx::mbar_wait_cluster(&bars->tempty[buf], aph ^ 1);
          else ptx::mbar_wait(&bars->tempty[buf], aph ^ 1);
          ptx::tc_fence_after();
          accumulate = 0;
        };
        auto close_chunk = [&](bool issued) {
          if (lane == 0) {
            if (issued) {
              if constexpr (CG == 1) ptx::mma_commit(&bars->tfull[buf]);
              else ptx::mma_commit_pair(&bars->tfull[buf], 0x3);
            } else {                                 // empty k-range: partial = 0
              ptx::mbar_arrive(&bars->tfull[buf]);
              if (CG == 2) ptx::mbar_arrive_cluster(&bars->tfull[buf], 1);
            }
          }
          __syncwarp();
          ++cc;
        };
        if (nkb == 0) { open_chunk(); close_chunk(false); continue; }
        int64_t gi = 0;
        for (int s = 0; s < P.nseg; ++s) {
          const Segment &sg = P.seg[s];
          int64_t kb0, kb1;
          seg_kblocks<CG>(P, sg, m0, n0, kb0, kb1);
          clip_kblocks(w, gi, kb0, kb1);
          const StageBand bd = make_band<CG>(P, sg, m0, n0);
          for (int64_t kb = kb0; kb < kb1; ++kb, ++it) {
            if (chunk_left == 0) { open_chunk(); chunk_left = P.kc; }
            const uint32_t d_tmem = tmem + buf * BN;
            const int rs = it % RS, ls = it % LS;
            const uint32_t lph = (it / LS) & 1;
            const StageInfo si = stage_at<CG>(bd, P, sg, m0, n0, kb);
            if (CG == 2) ptx::mbar_wait_cluster(&bars->ready[ls], lph);
            else ptx::mbar_wait(&bars->ready[ls], lph);
            ptx::tc_fence_after();
            if (lane == 0 && kb == kb0) BLAS3_STRACE(4, w.ph);
            if (lane == 0) {
              const uint32_t hiA = ptx::smem_u32(raw[rs].A), hiB = ptx::smem_u32(raw[rs].B);
              const uint32_t loA = ptx::smem_u32(lo[ls].A), loB = ptx::smem_u32(lo[ls].B);
              const uint32_t idesc = ptx::idesc_tf32(TM, BN, si.layA == LAYOUT_MN, si.layB == LAYOUT_MN);
              const bool one = (P.dbg & 2) || P.passes == 1;
              auto mma = [&](uint64_t a, uint64_t b, uint32_t id, uint32_t acc) {
                if constexpr (CG == 1) ptx::mma_tf32_ss(d_tmem, a, b, id, acc);
                else ptx::mma_tf32_ss_pair(d_tmem, a, b, id, acc);
              };
              auto commit = [&](uint64_t *bar) {
                if constexpr (CG == 1) ptx::mma_commit(bar);
                else ptx::mma_commit_pair(bar, 0x3);
              };
              if (!BX && !one && !(P.dbg & 8)) {
                // 3xTF32: the block's 8 cross-term UMMAs first, then its 4
                // hi*hi UMMAs.  In the first block of a TMEM partial the
                // cross terms land in a fresh accumulator still ~2^-11 of its
                // final size, where the accumulator's truncation costs nothing
                // (Q24): a partial of c k-blocks takes 12c - 8
                // full-size truncating adds instead of 12c.
#pragma unroll
                for (int k8 = 0; k8 < BK / 8; ++k8) {
                  mma(op_desc(loA, si.layA, k8), op_desc(hiB, si.layB, k8), idesc, accumulate);
                  mma(op_desc(hiA, si.layA, k8), op_desc(loB, si.layB, k8), idesc, 1);
                  accumulate = 1;
                }
#pragma unroll
                for (int k8 = 0; k8 < BK / 8; ++k8)
                  mma(op_desc(hiA, si.layA, k8), op_desc(hiB, si.layB, k8), idesc, 1);
                BLAS3_TRACE(6);
                commit(&bars->empty[rs]);
                commit(&bars->lo_empty[ls]);
              } else {
#pragma unroll
              for (int k8 = 0; k8 < BK / 8; ++k8) {
                const uint64_t ah = op_desc(hiA, si.layA, k8), al = op_desc(loA, si.layA, k8);
                const uint64_t bh = op_desc(hiB, si.layB, k8), bl = op_desc(loB, si.layB, k8);
                if (P.dbg & 8) continue;                       // diag: no MMAs
                if constexpr (BX) {
                  // packed cross terms (one bf16 UMMA, K = 16, K-major) + hi*hi (tf32)
                  const uint64_t ax = ptx::smem_desc(loA + k8 * 32, 16, 1024, 2);
                  const uint64_t bx = ptx::smem_desc(loB + k8 * 32, 16, 1024, 2);
                  constexpr uint32_t idx = ptx::idesc_bf16(TM, BN, 0, 0);
                  if constexpr (CG == 1) {
                    ptx::mma_bf16_ss(d_tmem, ax, bx, idx, accumulate);
                    ptx::mma_tf32_ss(d_tmem, ah, bh, idesc, 1);
                  } else {
                    ptx::mma_bf16_ss_pair(d_tmem, ax, bx, idx, accumulate);
                    ptx::mma_tf32_ss_pair(d_tmem, ah, bh, idesc, 1);
                  }
                  accumulate = 1;
                  continue;
                }
                if (!one) mma(al, bh, idesc, accumulate);
                if (!one) mma(ah, bl, idesc, 1);
                mma(ah, bh, idesc, one ? accumulate : 1);
                accumulate = 1;
              }
              BLAS3_TRACE(6);
              commit(&bars->empty[rs]);
              commit(&bars->lo_empty[ls]);
              }
            }
            accumulate = 1;
            __syncwarp();
            ++done;
            if (lane == 0 && done == nkb) BLAS3_STRACE(5, w.ph);
            if (--chunk_left == 0 || done == nkb) close_chunk(true);
          }
        }
      }
    }
   }
  } else if (warp < WARP_EPI0) {
    // ============================ transform warps (own halves; arrive at the leader)
    BLAS3_DEC_REGS();
    const int tt = threadIdx.x - WARP_TR0 * 32;
    uint32_t it = 0, qi = 0, mirror_ph = 0;
    for (;;) {
      const Work w = next_work(qi, 4, TR_THREADS, tt == 0);
      if (w.tb < 0) break;
      const Problem &P = prm.ph[FUSED ? w.ph : 0].P;
      const int64_t m0 = w.m0, n0 = w.n0;
      const int64_t ma = m0 + HA * rank, nb = n0 + HB * rank;
      int64_t gi = 0;
      for (int s = 0; s < P.nseg; ++s) {
        const Segment &sg = P.seg[s];
        int64_t kb0, kb1;
        seg_kblocks<CG>(P, sg, m0, n0, kb0, kb1);
        clip_kblocks(w, gi, kb0, kb1);
        const StageBand bd = make_band<CG>(P, sg, m0, n0);
        for (int64_t kb = kb0; kb < kb1; ++kb, ++it) {
          const int rs = it % RS, ls = it % LS;
          const uint32_t ph = (it / RS) & 1, lph = (it / LS) & 1;
          const int64_t k0 = kb * BK;
          const StageInfo si = stage_at<CG>(bd, P, sg, m0, n0, kb);
          // symmetric diagonal block: its mirrored (kr) view goes to this
          // stage's lo slot first (free once the MMA released it), loaded by
          // TMA beside the raw (rk) view, and is merged from shared memory
          const bool symA = si.clsA == BLK_SYM_DIAG, symB = si.clsB == BLK_SYM_DIAG;
          if (symA || symB) {
            ptx::mbar_wait(&bars->lo_empty[ls], lph ^ 1);
            if (tt == 0) {
              const int64_t per = P.per > 0 ? P.per : 1;
              const int32_t bj = (int32_t)(w.b % per), bg = (int32_t)(w.b / per);
              ptx::mbar_arrive_expect_tx(&bars->mirror, (symA ? HA * BK * 4 : 0) + (symB ? HB * BK * 4 : 0));
              if (symA) load_operand(prm, sg.a, LAYOUT_K, lo[ls].A, ma, k0, HA, &bars->mirror, bj, bg);
              if (symB) load_operand(prm, sg.b, LAYOUT_K, lo[ls].B, nb, k0, HB, &bars->mirror, bj, bg);
            }
          }
          ptx::mbar_wait(&bars->full[rs], ph);
          if (tt == 0) BLAS3_TRACE(4);
          if (tt == 0 && kb == kb0) BLAS3_STRACE(2, w.ph);
          RawBuf &rb = raw[rs];
          bool fix = false;
          // fix-ups are decided on this CTA's own half: a half that is entirely
          // in the nonzero region needs none, an entirely blank half is a
          // vectorised zero-fill, only halves touching the diagonal go per element
          const int64_t k1 = imin(sg.K, k0 + BK);
          if (symA || symB) {
            ptx::mbar_wait(&bars->mirror, mirror_ph);
            mirror_ph ^= 1;
            if (symA) sym_merge(sg.a, rb.A, lo[ls].A, ma, k0, HA, tt);
            if (symB) sym_merge(sg.b, rb.B, lo[ls].B, nb, k0, HB, tt);
            ptx::named_bar_sync(1, TR_THREADS);       // merged; the lo slot is free again for the split
          }
          if (si.clsA == BLK_TRI_DIAG) {
            const int own = block_class(sg.a, ma, imin(P.M, ma + HA), k0, k1);
            if (own == BLK_ZERO) { zero_fill(rb.A, G::A_BYTES, tt); fix = true; }
            else if (own == BLK_TRI_DIAG && !(P.dbg & 32)) { tri_fix(sg.a, si.layA, rb.A, ma, k0, HA, P.M, sg.K, tt); fix = true; }
          }
          if (si.clsB == BLK_TRI_DIAG) {
            const int own = block_class(sg.b, nb, imin(P.N, nb + HB), k0, k1);
            if (own == BLK_ZERO) { zero_fill(rb.B, G::B_BYTES, tt); fix = true; }
            else if (own == BLK_TRI_DIAG && !(P.dbg & 32)) { tri_fix(sg.b, si.layB, rb.B, nb, k0, HB, P.N, sg.K, tt); fix = true; }
          }
          if (fix) ptx::named_bar_sync(1, TR_THREADS);
          if constexpr (BX) {                               // packed bf16 cross terms
            if (HA == HB && !(P.dbg & 4096)) {
              // pair tiles: A and B have 128 rows = 2 units per thread each --
              // all four units loaded and packed into registers BEFORE waiting
              // for the lo stage (overlaps the MMA still reading it), then stored
              const int ua = tt, ub = tt + TR_THREADS;
              float xa0[8], xa1[8], xb0[8], xb1[8];
              load8(rb.A, si.layA, ua % HA, ua / HA, xa0);
              load8(rb.A, si.layA, ub % HA, ub / HA, xa1);
              load8(rb.B, si.layB, ua % HB, ua / HB, xb0);
              load8(rb.B, si.layB, ub % HB, ub / HB, xb1);
              const Packed pa0 = pack8_regs(xa0, true), pa1 = pack8_regs(xa1, true);
              const Packed pb0 = pack8_regs(xb0, false), pb1 = pack8_regs(xb1, false);
              ptx::mbar_wait(&bars->lo_empty[ls], lph ^ 1);
              store_packed(pa0, lo[ls].A + (ua % HA) * 128, ua % HA, ua / HA);
              store_packed(pa1, lo[ls].A + (ub % HA) * 128, ub % HA, ub / HA);
              store_packed(pb0, lo[ls].B + (ua % HB) * 128, ua % HB, ua / HB);
              store_packed(pb1, lo[ls].B + (ub % HB) * 128, ub % HB, ub / HB);
            } else {
              ptx::mbar_wait(&bars->lo_empty[ls], lph ^ 1);
              pack_cross(rb.A, si.layA, lo[ls].A, HA, tt, true);
              pack_cross(rb.B, si.layB, lo[ls].B, HB, tt, false);
            }
          } else {
            ptx::mbar_wait(&bars->lo_empty[ls], lph ^ 1);
            if (!(P.dbg & 1) && P.passes != 1) {
              stage::split_pass<TR_THREADS>(rb.A, lo[ls].A, G::A_BYTES, tt);
              stage::split_pass<TR_THREADS>(rb.B, lo[ls].B, G::B_BYTES, tt);
            }
          }
          ptx::fence_proxy_async_smem();
          arrive_leader<CG>(&bars->ready[ls], rank, 2, TR_THREADS, tt == 0);
          if (tt == 0) BLAS3_TRACE(5);
          if (tt == 0 && kb == kb0) BLAS3_STRACE(3, w.ph);
        }
      }
    }
  } else {
    // ============================ epilogue warps (own 128 rows, 128 of the BN columns)
    BLAS3_INC_REGS();
    // Each thread owns one row r and 128 columns: S[] is the fp32 running sum
    // of the kc-chunk partials (round-to-nearest adds), then
    // D = alpha*S + beta*C is stored with coalesced 128-B warp accesses.
    const int q = warp & 3;                     // TMEM lane quarter of this warp
    const int half = (warp - WARP_EPI0) >> 2;   // which 128 of the 256 columns
    constexpr int NG = BN / 2 / EC;             // column groups per thread (8)
    uint32_t cc = 0, qi = 0;
    const uint32_t box_s = ptx::smem_u32(epi_stage + (warp - WARP_EPI0) * 3 * EPI_BOX);
    for (;;) {
      const Work w = next_work(qi, 5, EPI_THREADS, threadIdx.x == WARP_EPI0 * 32);
      if (w.tb < 0) break;
      const Problem &P = prm.ph[FUSED ? w.ph : 0].P;
      const int64_t per = P.per > 0 ? P.per : 1;
      const int64_t coff = (P.nbatch > 1) ? batch_off(P.bs_c, w.b, per) : 0;
      const int64_t m0 = w.m0, n0 = w.n0;
      const int64_t nkb = w.g1 - w.g0;
      const int64_t nchunks = nkb > 0 ? cdiv(nkb, P.kc) : 1;
      float S[NG * EC];
#pragma unroll
      for (int i = 0; i < NG * EC; ++i) S[i] = 0.f;
      for (int64_t c = 0; c < nchunks; ++c, ++cc) {
        const uint32_t buf = cc & 1, ph = (cc >> 1) & 1;
        ptx::mbar_wait(&bars->tfull[buf], ph);
        ptx::tc_fence_after();
        if (threadIdx.x == WARP_EPI0 * 32) BLAS3_TRACE(7);
        if (threadIdx.x == WARP_EPI0 * 32 && c == nchunks - 1) BLAS3_STRACE(6, w.ph);
        if (nkb > 0 && !(P.dbg & 64)) {        // (diag knob 64: no drain loads, results wrong)
          // two 16-column loads in flight per wait: half the TMEM round trips
          // of the drain, which bounds how short a chunk can be without
          // stalling the MMA issuer on the accumulator hand-back
          const uint32_t ta = tmem + buf * BN + half * (BN / 2) + ((uint32_t)(q * 32) << 16);
#pragma unroll
          for (int g = 0; g < NG; g += 2) {
            uint32_t v[EC], u[EC];
            ptx::tmem_ld_32x32b_x16(ta + g * EC, v);
            ptx::tmem_ld_32x32b_x16(ta + (g + 1) * EC, u);
            ptx::tmem_ld_wait();
#pragma unroll
            for (int j = 0; j < EC; ++j) S[g * EC + j] += __uint_as_float(v[j]);
#pragma unroll
            for (int j = 0; j < EC; ++j) S[(g + 1) * EC + j] += __uint_as_float(u[j]);
          }
        }
        ptx::tc_fence_before();
        arrive_leader<CG>(&bars->tempty[buf], rank, 3, EPI_THREADS, threadIdx.x == WARP_EPI0 * 32);
      }
      if (w.slice >= 0) {
        // k-slice of a split tile: publish the partial (this CTA's 128 rows,
        // column-major, coalesced), count the arrival; the last slice sums all
        // partials in slice order (deterministic) and continues to the stores
        const int64_t tt = w.tb - prm.khead;
        const int64_t slab = (int64_t)HA * BN;                       // floats per CTA slice
        const int64_t row = q * 32 + lane, col0 = half * (BN / 2);
        float *mine = prm.ws + ((tt * prm.ksplit + w.slice) * CG + rank) * slab + col0 * HA + row;
#pragma unroll
        for (int i = 0; i < NG * EC; ++i) __stcg(mine + i * HA, S[i]);
        __threadfence();
        ptx::named_bar_sync(5, EPI_THREADS);
        if (threadIdx.x == WARP_EPI0 * 32) {
          uint32_t *cnt = prm.ws_cnt + tt * CG + rank;
          const uint32_t old = atomicAdd(cnt, 1u);
          const uint32_t last = (old == (uint32_t)prm.ksplit - 1) ? 1u : 0u;
          if (last) *cnt = 0u;                                     // self-cleaning for the next launch
          bars->split_last = last;
        }
        ptx::named_bar_sync(5, EPI_THREADS);
        if (!bars->split_last) continue;
        __threadfence();
        const float *part = prm.ws + (tt * prm.ksplit * CG + rank) * slab + col0 * HA + row;
#pragma unroll
        for (int i = 0; i < NG * EC; ++i) S[i] = 0.f;
        for (int sl = 0; sl < prm.ksplit; ++sl) {
          const float *ps = part + (int64_t)sl * CG * slab;
#pragma unroll
          for (int i = 0; i < NG * EC; ++i) S[i] += __ldcg(ps + i * HA);
        }
      }
      if (FUSED) {
        // C may have been written by earlier phases on other SMs: this CTA's
        // producer acquired the dependency counters before publishing the
        // item, and the epilogue took the item through wk_full (CTA-scope
        // release / acquire), so those stores are visible here
        if (threadIdx.x == WARP_EPI0 * 32) BLAS3_STRACE(7, w.ph);
      }
      // ---- store phase: D = alpha*S + beta*C for row r, columns cbase + [0,128).
      // The valid columns of the row form one range [jlo, jhi) (column bound
      // N, uplo mask c_tri); each warp access is a coalesced 128-B line.
      // Column pointers advance by ld (no per-element index math) and edge
      // elements use single predicated ld/st instructions: the epilogue shares
      // issue slots (and the instruction cache) with the transform warps.
      const int64_t r = m0 + HA * rank + q * 32 + lane;
      const int64_t cbase = n0 + half * (BN / 2);
      const int64_t ldi = P.ldcin, ldo = P.ldcout;
      const float *cp = P.Cin + coff + r + cbase * ldi;
      float *op = P.Cout + coff + r + cbase * ldo;
      const float al = P.alpha, be = P.beta;
      const bool st_on = !(P.dbg & 4);
      int jlo = 0, jhi = r < P.M ? (int)imin(BN / 2, P.N - cbase) : 0;
      if (P.c_tri == 1) jhi = (int)imin(jhi, imax(0, r - cbase + 1));   // lower: c <= r
      if (P.c_tri == 2) jlo = (int)imin(BN / 2, imax(0, r - cbase));    // upper: c >= r
      const uint32_t jn = jhi > jlo ? (uint32_t)(jhi - jlo) : 0u;
      const bool full = __all_sync(0xffffffffu, jlo == 0 && jhi == BN / 2);
      const bool none = __all_sync(0xffffffffu, jn == 0u);
      constexpr int SG = 8;
      if (none) {
        // nothing of this warp's 32 x 128 block is referenced (ragged edge)
      } else if (full && P.c_vec == 2 && be != 0.f) {
        // ---- as below, but C arrives by cp.async in the warp's two C boxes,
        // two groups ahead and without registers: the store phase (during
        // which the next tile's TMEM partials wait to be drained) is bound by
        // the L2 latency of C, and the running sum leaves no registers for a
        // deeper register prefetch.  Each lane copies, and later reads back,
        // exactly the float4s it combines (no cross-lane sync on the C boxes).
        const int vr = (lane & 7) * 4, vc = lane >> 3;
        const float *cq = P.Cin + coff + (m0 + HA * rank + q * 32 + vr) + (cbase + vc) * ldi;
        float *oq = P.Cout + coff + (m0 + HA * rank + q * 32 + vr) + (cbase + vc) * ldo;
        const uint32_t own = (uint32_t)(vc * 32 + vr) * 4;
        const uint32_t rd = box_s + own;                                  // transpose box
        const uint32_t cb = box_s + EPI_BOX * 4 + own;                    // C box 0 (box 1: + 1 KiB)
        constexpr int NGW = BN / 2 / EPI_GW;
        auto fetch = [&](int g) {
          const float *src = cq + (int64_t)g * EPI_GW * ldi;
          const uint32_t dst = cb + (uint32_t)(g & 1) * (EPI_BOX * 4);
          ptx::cp_async16(dst, src);
          ptx::cp_async16(dst + 4 * 128, src + 4 * ldi);
        };
        fetch(0); ptx::cp_async_commit();
        fetch(1); ptx::cp_async_commit();
#pragma unroll
        for (int g = 0; g < NGW; ++g) {
#pragma unroll
          for (int j = 0; j < EPI_GW; ++j) ptx::st_shared_f32(box_s + (j * 32 + lane) * 4, al * S[g * EPI_GW + j]);
          __syncwarp();
          float4 d0 = ptx::ld_shared_v4(rd), d1 = ptx::ld_shared_v4(rd + 4 * 128);
          __syncwarp();                                   // transpose box free for the next group
          ptx::cp_async_wait<1>();                        // group g landed (g + 1 may be in flight)
          const uint32_t cg = cb + (uint32_t)(g & 1) * (EPI_BOX * 4);
          const float4 c0v = ptx::ld_shared_v4(cg), c1v = ptx::ld_shared_v4(cg + 4 * 128);
          if (g + 2 < NGW) fetch(g + 2);                  // into the box just read
          ptx::cp_async_commit();                         // (empty groups keep the count uniform)
          d0.x = fmaf(be, c0v.x, d0.x); d0.y = fmaf(be, c0v.y, d0.y);
          d0.z = fmaf(be, c0v.z, d0.z); d0.w = fmaf(be, c0v.w, d0.w);
          d1.x = fmaf(be, c1v.x, d1.x); d1.y = fmaf(be, c1v.y, d1.y);
          d1.z = fmaf(be, c1v.z, d1.z); d1.w = fmaf(be, c1v.w, d1.w);
          if (st_on) { ptx::st_cs_v4(oq, d0); ptx::st_cs_v4(oq + 4 * ldo, d1); }
          oq += EPI_GW * ldo;
        }
      } else if (full && P.c_vec) {
        // ---- 16-B vector accesses of C (NS "coalesced 128-bit epilogue
        // stores"; DESIGN A6), for warps whose whole 32 x 128 block is valid
        // (ragged-edge and uplo-cut warps take the predicated paths below).
        // Per group of 8 columns: alpha*S goes to the warp's shared box
        // column-major (thread = row: conflict-free), is read back as float4s
        // of 4 consecutive rows of one column (lane -> column lane/8 and
        // lane/8 + 4, rows 4*(lane%8)..+3), combined with beta*C read the
        // same way, and stored with st.global.v4: each warp instruction moves
        // 4 columns x 128 B.  C is read one group ahead.
        const int vr = (lane & 7) * 4, vc = lane >> 3;
        const float *cq = P.Cin + coff + (m0 + HA * rank + q * 32 + vr) + (cbase + vc) * ldi;
        float *oq = P.Cout + coff + (m0 + HA * rank + q * 32 + vr) + (cbase + vc) * ldo;
        const uint32_t rd = box_s + (uint32_t)(vc * 32 + vr) * 4;       // float4 of column vc
        constexpr int NGW = BN / 2 / EPI_GW;
        const bool ld_on = be != 0.f;
        float4 c0v = make_float4(0.f, 0.f, 0.f, 0.f), c1v = c0v;
        if (ld_on) { c0v = ptx::ld_cs_v4(cq); c1v = ptx::ld_cs_v4(cq + 4 * ldi); }
#pragma unroll
        for (int g = 0; g < NGW; ++g) {
#pragma unroll
          for (int j = 0; j < EPI_GW; ++j) ptx::st_shared_f32(box_s + (j * 32 + lane) * 4, al * S[g * EPI_GW + j]);
          __syncwarp();
          float4 d0 = ptx::ld_shared_v4(rd), d1 = ptx::ld_shared_v4(rd + 4 * 128);
          __syncwarp();                                   // box free for the next group
          if (ld_on) {
            d0.x = fmaf(be, c0v.x, d0.x); d0.y = fmaf(be, c0v.y, d0.y);
            d0.z = fmaf(be, c0v.z, d0.z); d0.w = fmaf(be, c0v.w, d0.w);
            d1.x = fmaf(be, c1v.x, d1.x); d1.y = fmaf(be, c1v.y, d1.y);
            d1.z = fmaf(be, c1v.z, d1.z); d1.w = fmaf(be, c1v.w, d1.w);
            if (g + 1 < NGW) {
              cq += EPI_GW * ldi;
              c0v = ptx::ld_cs_v4(cq); c1v = ptx::ld_cs_v4(cq + 4 * ldi);
            }
          }
          if (st_on) { ptx::st_cs_v4(oq, d0); ptx::st_cs_v4(oq + 4 * ldo, d1); }
          oq += EPI_GW * ldo;
        }
      } else if (full && be == 0.f) {
        if (st_on) {
#pragma unroll
          for (int i = 0; i < NG * EC; ++i) { ptx::st_cs(op, al * S[i]); op += ldo; }
        }
      } else if (full) {
        // group g+1's C loads are issued before group g's stores (different
        // columns; D is formed in place in S's registers)
        float cv[SG];
#pragma unroll
        for (int j = 0; j < SG; ++j) { cv[j] = ptx::ld_cs(cp); cp += ldi; }
#pragma unroll
        for (int g = 0; g < NG * EC / SG; ++g) {
#pragma unroll
          for (int j = 0; j < SG; ++j) S[g * SG + j] = fmaf(be, cv[j], al * S[g * SG + j]);
          if (g + 1 < NG * EC / SG) {
#pragma unroll
            for (int j = 0; j < SG; ++j) { cv[j] = ptx::ld_cs(cp); cp += ldi; }
          }
          if (st_on) {
#pragma unroll
            for (int j = 0; j < SG; ++j) { ptx::st_cs(op, S[g * SG + j]); op += ldo; }
          }
        }
      } else {
        const bool ld_on = be != 0.f;
#pragma unroll
        for (int g = 0; g < NG * EC / SG; ++g) {
          float cv[SG];
#pragma unroll
          for (int j = 0; j < SG; ++j) {
            cv[j] = ptx::ld_cs_pred(cp, ld_on && (uint32_t)(g * SG + j - jlo) < jn);
            cp += ldi;
          }
#pragma unroll
          for (int j = 0; j < SG; ++j) {
            ptx::st_cs_pred(op, fmaf(be, cv[j], al * S[g * SG + j]),
                            st_on && (uint32_t)(g * SG + j - jlo) < jn);
            op += ldo;
          }
        }
      }
      if (FUSED) {                                 // this CTA's half of the tile is stored
        ptx::named_bar_sync(5, EPI_THREADS);
        if (threadIdx.x == WARP_EPI0 * 32) {
          BLAS3_STRACE(8, w.ph);
          signal_done<CG>(prm, w);
          BLAS3_STRACE(9, w.ph);
          if (prm.ph_trace != nullptr) {
            unsigned long long t_;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));
            atomicMax(prm.ph_trace + 2 * w.ph + 1, t_);
          }
        }
      }
      if (threadIdx.x == WARP_EPI0 * 32) BLAS3_TRACE(8);
    }
    if (threadIdx.x == WARP_EPI0 * 32) BLAS3_TRACE(9);
  }

  ptx::tc_fence_before();
  if (CG == 2) ptx::cluster_sync(); else __syncthreads();
  if (threadIdx.x == 0) BLAS3_TRACE(10);
  if (warp == WARP_MMA) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<CG>(tmem, TMEM_COLS);
    if (lane == 0) BLAS3_TRACE(11);
  }
}

// ====================================================================== host side
typedef CUresult (*EncodeTiledFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                                  const cuuint64_t *, const cuuint64_t *, const cuuint32_t *,
                                  const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFn>(p);
  });
  return fn;
}

// 4-D fp32 tensor map: dim0 contiguous (extent d0), dim1 stride ld floats,
// dims 2/3 = batch (inner, outer) with element strides bs.inner / bs.outer.
// Extents are the sub-problem's, so TMA zero-fills every out-of-range element
// of a tile (including those of a batch member's neighbours).
static bool make_map(CUtensorMap *m, const float *ptr, int64_t d0, int64_t d1, int64_t ld,
                     uint32_t box0, uint32_t box1, CUtensorMapSwizzle swz, int64_t per,
                     int64_t groups, BatchStride bs) {
  EncodeTiledFn fn = encode_fn();
  if (!fn) return false;
  const int64_t plain = ld * d1;               // stride for unit batch dims
  cuuint64_t dims[4] = {(cuuint64_t)d0, (cuuint64_t)d1, (cuuint64_t)per, (cuuint64_t)groups};
  cuuint64_t strides[3] = {(cuuint64_t)ld * 4, (cuuint64_t)(per > 1 ? bs.inner : plain) * 4,
                           (cuuint64_t)(groups > 1 ? bs.outer : plain) * 4};
  cuuint32_t box[4] = {box0, box1, 1, 1};
  cuuint32_t es[4] = {1, 1, 1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, const_cast<float *>(ptr), dims, strides, box, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, swz,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// plain 2-D fp32 map (other kernels of the library): mn32 -> the MN-major
// staging swizzle (SWIZZLE_128B_ATOM_32B), else the K-major one (SWIZZLE_128B)
bool tma_map_f32(CUtensorMap *m, const float *ptr, int64_t d0, int64_t d1, int64_t ld, uint32_t box0,
                 uint32_t box1, bool mn32) {
  return make_map(m, ptr, d0, d1, ld, box0, box1,
                  mn32 ? CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B : CU_TENSOR_MAP_SWIZZLE_128B, 1, 1, BatchStride{0, 0});
}

// maps for one operand with R rows, K columns, staged `rows` at a time
template <class PRM>
static bool op_maps(PRM &prm, int &slot, OpDesc &o, int64_t R, int64_t K, int rows,
                    int64_t per, int64_t groups, BatchStride bs) {
  o.map_rk = o.map_kr = -1;
  const bool need_rk = (o.kind == OP_DENSE && !o.kr) || o.kind == OP_SYM || (o.kind == OP_TRI && !o.swap);
  const bool need_kr = (o.kind == OP_DENSE && o.kr) || o.kind == OP_SYM || (o.kind == OP_TRI && o.swap);
  if (need_rk) {       // X(r,k) = G[r + k*ld]: dim0 = r (R), dim1 = k (K)
    if (slot >= (int)(sizeof(prm.maps) / sizeof(prm.maps[0])) || !make_map(&prm.maps[slot], o.ptr, R, K, o.ld, 32, BK,
                                                CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B, per, groups, bs)) return false;
    o.map_rk = slot++;
  }
  if (need_kr) {       // X(r,k) = G[k + r*ld]: dim0 = k (K), dim1 = r (R)
    if (slot >= (int)(sizeof(prm.maps) / sizeof(prm.maps[0])) || !make_map(&prm.maps[slot], o.ptr, K, R, o.ld, BK, rows,
                                                CU_TENSOR_MAP_SWIZZLE_128B, per, groups, bs)) return false;
    o.map_kr = slot++;
  }
  return true;
}

static bool aligned_op(const OpDesc &o) {
  return (reinterpret_cast<uintptr_t>(o.ptr) % 16 == 0) && (o.ld % 4 == 0);
}

bool tc_eligible(const Problem &P) {
  if (P.nbatch > 1) {                    // batch strides become TMA strides (16-B multiples)
    if (P.nseg != 1 || P.per < 1) return false;
    for (const BatchStride *b : {&P.bs_a, &P.bs_b})
      if (b->inner % 4 || b->outer % 4) return false;
  }
  for (int s = 0; s < P.nseg; ++s)
    if (!aligned_op(P.seg[s].a) || !aligned_op(P.seg[s].b)) return false;
  return true;
}

// CTA-group choice.  The pair kernel (CG=2: 256x256 tiles, tcgen05
// cta_group::2, each CTA staging half of B) needs half the per-SM operand
// traffic and has a 4-deep raw ring: it is faster per SM even when its tiles
// do not fill the machine (measured: SGEMM 2048^3 82.8 vs 106 us, 1024^3 46.0
// vs 48.6 us, profiles/r02_sizes.md).  The single-CTA kernel (128x256 tiles)
// is kept for problems of fewer than 256 rows, where a 256-row pair tile
// would compute mostly padding (the TRSM doubling's 128-blocks, skinny
// updates).  BLAS3_TC_CTA=1|2 forces one (tests).
static int choose_cg(const Problem &P, int num_sms) {
  const int forced = (int)opt(BLAS3_OPT_TC_CTA);
  if (forced) return forced;
  const int64_t nb = P.nbatch > 1 ? P.nbatch : 1;
  return (P.M >= 256 || Tiles<Geo<2>::TM, BN>::count(P) * nb >= num_sms / 2) ? 2 : 1;
}

template <int CG, class PRM>
static int launch_cg(PRM &prm, cudaStream_t stream, int num_sms, bool allow_pdl = true) {
  using G = Geo<CG>;
  int slot = 0;
  for (int p = 0; p < prm.nphase; ++p) {
    Problem &P = prm.ph[p].P;
    for (int s = 0; s < P.nseg; ++s) {
      Segment &sg = P.seg[s];
      if (sg.K <= 0) continue;
      const int64_t nb = P.nbatch > 1 ? P.nbatch : 1;
      const int64_t per = nb > 1 ? P.per : 1, groups = cdiv(nb, per);
      if (!op_maps(prm, slot, sg.a, P.M, sg.K, HA, per, groups, P.bs_a)) return -4;
      if (!op_maps(prm, slot, sg.b, P.N, sg.K, G::HB, per, groups, P.bs_b)) return -4;
    }
  }
  // epilogue access of C: 16-B vectors when aligned; Cin (beta != 0) as an
  // L2-prefetch tensor map (128-row x 128-column boxes, one per CTA half)
  for (int p = 0; p < prm.nphase; ++p) {
    Problem &P = prm.ph[p].P;
    const int64_t nb = P.nbatch > 1 ? P.nbatch : 1;
    auto vec_ok = [&](const float *ptr, int64_t ld, const BatchStride &bs) {
      return reinterpret_cast<uintptr_t>(ptr) % 16 == 0 && ld % 4 == 0 &&
             (nb == 1 || (bs.inner % 4 == 0 && bs.outer % 4 == 0));
    };
    const bool rd = P.beta != 0.f;
    P.c_vec = opt(BLAS3_OPT_TC_VEC_STORE) != 0 && vec_ok(P.Cout, P.ldcout, P.bs_c) &&
              (!rd || vec_ok(P.Cin, P.ldcin, P.bs_c)) ? 1 : 0;
    if (P.c_vec && rd && opt(BLAS3_OPT_TC_C_ASYNC)) P.c_vec = 2;     // C by cp.async into shared boxes
    P.c_pf_map = -1;
    if (!rd || !opt(BLAS3_OPT_TC_C_PREFETCH) || !vec_ok(P.Cin, P.ldcin, P.bs_c) ||
        slot >= (int)(sizeof(prm.maps) / sizeof(prm.maps[0]))) continue;
    const int64_t per = nb > 1 ? P.per : 1, groups = cdiv(nb, per);
    if (!make_map(&prm.maps[slot], P.Cin, P.M, P.N, P.ldcin, HA, BN / 2, CU_TENSOR_MAP_SWIZZLE_NONE, per,
                  groups, P.bs_c)) return -4;
    P.c_pf_map = slot++;
  }
  // the TF32+BF16X instantiation in that mode (every phase of a fused launch
  // carries the same mode)
  const bool bx = prm.ph[0].P.passes == 2;
  void (*kfn)(PRM) = bx ? tc_structured_gemm<CG, PRM, true> : tc_structured_gemm<CG, PRM, false>;
  // the attribute is per device context: remembered per (device, instantiation)
  static std::atomic<bool> attr[64][2];
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return -1;
  if (!attr[dev][bx].load(std::memory_order_acquire)) {
    if (cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)G::SMEM) != cudaSuccess)
      return -1;
    attr[dev][bx].store(true, std::memory_order_release);
  }
  const int64_t items = prm.nitems;        // tiles, or tiles + split-tail slices
  if (items == 0) return 0;
  const int64_t units = imin(items, (int64_t)(num_sms / CG));      // CTAs (CG=1) or pairs
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(units * CG));
  cfg.blockDim = dim3(NTHREADS);
  cfg.dynamicSmemBytes = G::SMEM;
  cfg.stream = stream;
  cudaLaunchAttribute attrs[2];
  attrs[0].id = cudaLaunchAttributeClusterDimension;
  attrs[0].val.clusterDim.x = CG;
  attrs[0].val.clusterDim.y = 1;
  attrs[0].val.clusterDim.z = 1;
  // programmatic dependent launch: this grid's prologue may overlap the tail
  // of the previous kernel on the stream (the kernel waits before touching
  // global memory).  BLAS3_OPT_PDL=0 disables it (experiments).
  const bool pdl = allow_pdl && opt(BLAS3_OPT_PDL) != 0;
  attrs[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attrs[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attrs;
  cfg.numAttrs = pdl ? 2 : 1;
  const cudaError_t e = cudaLaunchKernelEx(&cfg, kfn, prm);
  note_launch(0);
  return (e == cudaSuccess && cudaGetLastError() == cudaSuccess) ? 0 : -1;
}

// Per-launch device state: the dynamic scheduler's claim counter, the split
// tail's partial workspace and arrival counters, and a fused launch's
// dependency counters.
//  * Eager launches: one block per (device, stream).  Launches on one stream
//    never overlap in global memory (each grid waits for the previous one
//    before its first global access, PDL included) and every launch leaves
//    the counters at zero (the last claim resets the claim counter, the last
//    slice of a split tile its arrival counter; fused counters are zeroed by a
//    memset before the launch), so the next launch on the stream starts clean.
//    Launches on different streams never share a block.
//  * Launches captured into a CUDA graph (cudaStreamIsCapturing): a private
//    block allocated, zeroed and freed INSIDE the graph (stream-ordered
//    alloc / memset / free nodes), so every replay of the graph -- on any
//    stream, beside eager calls or other graphs -- owns its counters.
// (the earlier device-wide ring could hand one slot to two
// concurrent launches, and graphs kept per-capture-stream slots.)
struct LaunchState {
  uint32_t *ctr = nullptr;      // claim counter (128 B)
  uint32_t *dep = nullptr;      // fused: [FUSED_PH] phase + [FUSED_PH][MAX_SLAB] slab counters
  float *ws = nullptr;          // split tail partials: dev_sms x HA x BN floats
  uint32_t *ws_cnt = nullptr;   // split tail arrival counters (1024)
  void *graph_block = nullptr;  // captured launch: the private block to free after the kernel
};
constexpr size_t CTR_BYTES = 128, DEP_BYTES = (size_t)FUSED_PH * (1 + MAX_SLAB) * sizeof(uint32_t),
                 WSCNT_BYTES = 1024 * sizeof(uint32_t);
static size_t ws_bytes_for(int dev) {
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  return (size_t)sms * HA * BN * sizeof(float);
}
static bool capturing(cudaStream_t s) {
  cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
  if (cudaStreamIsCapturing(s, &st) != cudaSuccess) { cudaGetLastError(); return false; }
  return st == cudaStreamCaptureStatusActive;
}
// need_ws: the launch splits its tail; need_dep: a fused launch.  Returns false
// on an allocation failure (nothing enqueued).
static bool launch_state(cudaStream_t stream, bool need_ws, bool need_dep, LaunchState &ls) {
  int d = 0;
  if (cudaGetDevice(&d) != cudaSuccess) return false;
  if (capturing(stream)) {
    const size_t wsb = need_ws ? ws_bytes_for(d) : 0;
    const size_t bytes = CTR_BYTES + DEP_BYTES + WSCNT_BYTES + wsb;
    void *blk = nullptr;
    if (cudaMallocAsync(&blk, bytes, stream) != cudaSuccess) { cudaGetLastError(); return false; }
    // (the partials need no zeroing: every slice writes its own before the count)
    if (cudaMemsetAsync(blk, 0, CTR_BYTES + DEP_BYTES + WSCNT_BYTES, stream) != cudaSuccess) {
      cudaGetLastError(); cudaFreeAsync(blk, stream); return false;
    }
    uint8_t *p = static_cast<uint8_t *>(blk);
    ls.ctr = reinterpret_cast<uint32_t *>(p);
    ls.dep = reinterpret_cast<uint32_t *>(p + CTR_BYTES);
    ls.ws_cnt = reinterpret_cast<uint32_t *>(p + CTR_BYTES + DEP_BYTES);
    ls.ws = need_ws ? reinterpret_cast<float *>(p + CTR_BYTES + DEP_BYTES + WSCNT_BYTES) : nullptr;
    ls.graph_block = blk;
    return true;
  }
  struct Key { int dev; cudaStream_t st; };
  struct Entry { Key k; LaunchState s; };
  static std::vector<Entry> tab;
  static std::mutex mu;
  std::lock_guard<std::mutex> lk(mu);
  Entry *e = nullptr;
  for (Entry &x : tab)
    if (x.k.dev == d && x.k.st == stream) { e = &x; break; }
  if (!e) { tab.push_back(Entry{Key{d, stream}, LaunchState{}}); e = &tab.back(); }
  LaunchState &st = e->s;
  auto zalloc = [](void **p, size_t bytes, bool zero) {
    if (cudaMalloc(p, bytes) != cudaSuccess) { cudaGetLastError(); *p = nullptr; return false; }
    if (zero && cudaMemset(*p, 0, bytes) != cudaSuccess) { cudaGetLastError(); cudaFree(*p); *p = nullptr; return false; }
    return true;
  };
  if (!st.ctr && !zalloc(reinterpret_cast<void **>(&st.ctr), CTR_BYTES, true)) return false;
  if (need_dep && !st.dep && !zalloc(reinterpret_cast<void **>(&st.dep), DEP_BYTES, true)) return false;
  if (need_ws && !st.ws) {
    if (!zalloc(reinterpret_cast<void **>(&st.ws_cnt), WSCNT_BYTES, true)) return false;
    if (!zalloc(reinterpret_cast<void **>(&st.ws), ws_bytes_for(d), false)) {
      cudaFree(st.ws_cnt); st.ws_cnt = nullptr; return false;
    }
  }
  ls = st;
  ls.graph_block = nullptr;
  return true;
}
static void release_state(cudaStream_t stream, const LaunchState &ls) {
  if (ls.graph_block) cudaFreeAsync(ls.graph_block, stream);
}

// Wave quantisation: with T tiles on U producers the last wave holds
// R = T mod U tiles (all T when T < U) and leaves U - R producers idle.
// Those R tiles are cut into S = U / R k-slices.  Only worth it while the
// tail is a sizeable share of the launch (fewer than 8 waves) and each slice
// keeps >= 8 k-blocks (its partial write-back costs about what ~3 k-blocks
// of MMA do).
template <int CG>
static void plan_split(TcParams &prm, int num_sms) {
  const Problem &P = prm.ph[0].P;
  const int64_t nb = P.nbatch > 1 ? P.nbatch : 1;
  const int64_t tiles_per = Tiles<Geo<CG>::TM, BN>::count(P), T = tiles_per * nb;
  prm.ph[0].tiles_per = tiles_per;
  prm.ph[0].ntiles = T;
  prm.nitems = T; prm.khead = T; prm.ksplit = 1;
  if (!opt(BLAS3_OPT_TC_SPLIT) || T == 0) return;
  const int64_t U = imin(T, (int64_t)(num_sms / CG));
  const int64_t R = T < (int64_t)(num_sms / CG) ? T : T % U;
  if (R == 0 || T >= 8 * U) return;
  int64_t S = imin((int64_t)(num_sms / CG) / R, 16);
  if (S < 2) return;
  const int64_t head = T - R;
  int64_t min_kb = INT64_MAX;
  for (int64_t tb = head; tb < T; ++tb) {
    const int64_t t = tb % tiles_per;
    int64_t mi, nj;
    Tiles<Geo<CG>::TM, BN>::coords(P, t, mi, nj);
    min_kb = imin(min_kb, tile_kblocks<CG>(P, mi * Geo<CG>::TM, nj * BN));
  }
  S = imin(S, min_kb / 8);
  if (S < 2) return;
  prm.khead = head;
  prm.ksplit = (int32_t)S;
  prm.nitems = head + R * S;
}

static int debug_bits() {
  static int dbg = -1;
  if (dbg < 0) { const char *e = getenv("BLAS3_DEBUG_TC"); dbg = e ? atoi(e) : 0; }
  return dbg;
}

int launch_tc(const Problem &P0, cudaStream_t stream, int num_sms) {
  static TcParams prm;                    // host staging (the launch copies it)
  static std::mutex mu;
  std::lock_guard<std::mutex> lk(mu);
  memset(&prm, 0, sizeof(prm));
  prm.nphase = 1;
  prm.ph[0].P = P0;
  prm.ph[0].P.dbg = debug_bits();
  if (prm.ph[0].P.kc <= 0) prm.ph[0].P.kc = 3;
  const int cg = choose_cg(prm.ph[0].P, num_sms);
  const bool dyn = opt(BLAS3_OPT_TC_STATIC) == 0;
  if (cg == 2) plan_split<2>(prm, num_sms); else plan_split<1>(prm, num_sms);
  const bool split = prm.ksplit > 1;
  LaunchState ls;
  if ((dyn || split) && prm.nitems > 0) {
    if (!launch_state(stream, split, false, ls)) {
      if (!split) return -1;
      prm.nitems = prm.khead = prm.ph[0].ntiles; prm.ksplit = 1;      // no workspace: no split
      if (dyn && !launch_state(stream, false, false, ls)) return -1;
    }
    if (prm.ksplit > 1) { prm.ws = ls.ws; prm.ws_cnt = ls.ws_cnt; }
    // claims: (items - producers) beyond the first wave + one failing claim per producer
    if (dyn) { prm.tile_ctr = ls.ctr; prm.tile_claims = (uint32_t)prm.nitems; }
  }
  // diagnostics: BLAS3_TRACE=1 prints CTA 0's phase timeline (synchronises)
  static int trace = -1;
  static unsigned long long *tbuf = nullptr;
  if (trace < 0) { const char *e = getenv("BLAS3_TRACE"); trace = (e && e[0] == '1') ? 1 : 0; }
  if (trace) {
    if (!tbuf && cudaMalloc(&tbuf, 16 * sizeof(unsigned long long)) != cudaSuccess) return -1;
    cudaMemsetAsync(tbuf, 0, 16 * sizeof(unsigned long long), stream);
    prm.trace = tbuf;
  }
  const int rc = cg == 2 ? launch_cg<2>(prm, stream, num_sms, ls.graph_block == nullptr)
                         : launch_cg<1>(prm, stream, num_sms, ls.graph_block == nullptr);
  release_state(stream, ls);
  if (trace && rc == 0) {
    unsigned long long h[16];
    cudaStreamSynchronize(stream);
    cudaMemcpy(h, tbuf, sizeof(h), cudaMemcpyDeviceToHost);
    static const char *names[12] = {"entry", "prologue", "claim", "tma", "full", "ready",
                                    "mma", "tfull", "stored", "epi_exit", "final_sync", "dealloc"};
    fprintf(stderr, "[blas3 trace] cg=%d M=%lld N=%lld K=%lld:", cg, (long long)P0.M,
            (long long)P0.N, (long long)P0.seg[0].K);
    for (int i = 1; i < 12; ++i)
      fprintf(stderr, " %s=%.2f", names[i], h[i] ? (double)(h[i] - h[0]) / 1e3 : -1.0);
    fprintf(stderr, " us\n");
  }
  return rc;
}

int launch_tc_fused(const FusedPhase *phases, int nph, cudaStream_t stream, int num_sms) {
  if (nph < 1 || nph > FUSED_PH) return -1;
  static TcFusedParams prm;               // host staging (the launch copies it)
  static std::mutex mu;
  std::lock_guard<std::mutex> lk(mu);
  memset(&prm, 0, sizeof(prm));
  constexpr int CG = 2;                   // one tile geometry for every phase (slabs align)
  using TL = Tiles<Geo<CG>::TM, BN>;
  int64_t item = 0;
  for (int p = 0; p < nph; ++p) {
    PhaseDesc &ph = prm.ph[p];
    ph.P = phases[p].P;
    ph.P.dbg = debug_bits();
    if (ph.P.kc <= 0) ph.P.kc = 3;
    if (!tc_eligible(ph.P) || ph.P.max_sms) return -1;
    const int64_t nb = ph.P.nbatch > 1 ? ph.P.nbatch : 1;
    ph.tiles_per = TL::count(ph.P);
    ph.ntiles = ph.tiles_per * nb;
    ph.item0 = item;
    item += ph.ntiles;
    ph.dep_full = phases[p].dep_full;
    ph.dep_slab = phases[p].dep_slab;
    ph.slab_m = phases[p].slab_m;
    ph.slab_cnt = (int32_t)(phases[p].slab_m ? cdiv(ph.P.N, BN) : cdiv(ph.P.M, Geo<CG>::TM));
    if ((ph.dep_full | ph.dep_slab) >> p) return -1;        // dependencies point backwards only
    for (int s = 0; s < ph.P.nseg; ++s)                      // SYM diagonal merges read global memory
      if (ph.P.seg[s].a.kind == OP_SYM || ph.P.seg[s].b.kind == OP_SYM) return -1;
    const int64_t nslab = phases[p].slab_m ? cdiv(ph.P.M, Geo<CG>::TM) : cdiv(ph.P.N, BN);
    if (nslab > MAX_SLAB) return -1;
  }
  prm.nphase = nph;
  prm.nitems = item;
  prm.khead = item;
  prm.ksplit = 1;
  if (item == 0) return 0;
  LaunchState ls;
  if (!launch_state(stream, false, true, ls)) return -1;
  prm.dep_ctr = ls.dep;
  if (cudaMemsetAsync(prm.dep_ctr, 0, DEP_BYTES, stream) != cudaSuccess) { release_state(stream, ls); return -1; }
  const int64_t units = imin(item, (int64_t)(num_sms / CG));
  prm.tile_ctr = ls.ctr;
  prm.tile_claims = (uint32_t)(item + units);
  // diagnostics: BLAS3_TRACE=2 prints each phase's [first start, last end] (synchronises)
  static int trace = -1;
  static unsigned long long *tbuf = nullptr;
  if (trace < 0) { const char *e = getenv("BLAS3_TRACE"); trace = (e && e[0] == '2') ? 1 : 0; }
  if (trace) {
    if (!tbuf && cudaMalloc(&tbuf, 2 * FUSED_PH * sizeof(unsigned long long)) != cudaSuccess) return -1;
    unsigned long long init[2 * FUSED_PH];
    for (int i = 0; i < FUSED_PH; ++i) { init[2 * i] = ~0ull; init[2 * i + 1] = 0ull; }
    cudaMemcpyAsync(tbuf, init, sizeof(init), cudaMemcpyHostToDevice, stream);
    cudaStreamSynchronize(stream);
    prm.ph_trace = tbuf;
  }
  // BLAS3_TRACE_PH=p: per-stage [earliest, latest] over the tiles of phase p
  static int st_phase = -2;
  static unsigned long long *sbuf = nullptr;
  constexpr int NST = 12;
  if (st_phase == -2) { const char *e = getenv("BLAS3_TRACE_PH"); st_phase = e ? atoi(e) : -1; }
  if (st_phase >= 0 && st_phase < nph) {
    if (!sbuf && cudaMalloc(&sbuf, 2 * NST * sizeof(unsigned long long)) != cudaSuccess) return -1;
    unsigned long long init[2 * NST];
    for (int i = 0; i < NST; ++i) { init[2 * i] = ~0ull; init[2 * i + 1] = 0ull; }
    cudaMemcpyAsync(sbuf, init, sizeof(init), cudaMemcpyHostToDevice, stream);
    cudaStreamSynchronize(stream);
    prm.st_trace = sbuf;
    prm.st_phase = st_phase;
  }
  // no PDL: the counters' memset node precedes this grid on the stream
  const int rc = launch_cg<CG>(prm, stream, num_sms, false);
  release_state(stream, ls);
  if (trace && rc == 0) {
    unsigned long long h[2 * FUSED_PH];
    cudaStreamSynchronize(stream);
    cudaMemcpy(h, tbuf, sizeof(h), cudaMemcpyDeviceToHost);
    unsigned long long t0 = ~0ull;
    for (int p = 0; p < nph; ++p) t0 = h[2 * p] < t0 ? h[2 * p] : t0;
    for (int p = 0; p < nph; ++p)
      fprintf(stderr, "[blas3 fused] phase %2d M=%6lld N=%6lld K=%6lld tiles=%5lld: %8.1f .. %8.1f us\n", p,
              (long long)prm.ph[p].P.M, (long long)prm.ph[p].P.N, (long long)prm.ph[p].P.seg[0].K,
              (long long)prm.ph[p].ntiles, (h[2 * p] - t0) / 1e3, (h[2 * p + 1] - t0) / 1e3);
  }
  if (prm.st_trace && rc == 0) {
    static const char *names[NST] = {"deps_ready", "tma_issued", "raw_full", "split_done", "mma_start",
                                     "mma_last_issued", "tmem_full", "epi_deps", "stored", "signaled",
                                     "prod_acquired", "tmem_drained"};
    unsigned long long h[2 * NST];
    cudaStreamSynchronize(stream);
    cudaMemcpy(h, sbuf, sizeof(h), cudaMemcpyDeviceToHost);
    const unsigned long long t0 = h[0];
    fprintf(stderr, "[blas3 stages] phase %d (%lld tiles):", st_phase, (long long)prm.ph[st_phase].ntiles);
    for (int i = 0; i < NST; ++i)
      if (h[2 * i + 1]) fprintf(stderr, " %s=%.2f/%.2f", names[i], (h[2 * i] - t0) / 1e3, (h[2 * i + 1] - t0) / 1e3);
    fprintf(stderr, " us (earliest/latest tile)\n");
  }
  return rc;
}

}  // namespace blas3
