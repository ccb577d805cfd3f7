// panel_kernel.cu -- STRSM diagonal-panel solve (rows A7/A8 of the hot-path
// table): every right-hand-side slab of 256 columns (rows for side=R) is
// forward-substituted through the whole R x R diagonal panel by ONE team of
// two CTA pairs, so the panel's dependency chain (Fig. 14
// / Adaptor_Solver: X_i needs X_k, k < i) never becomes a grid-wide step.
//
// With the panel split into 256-row blocks (processing order i = 0..nblk-1;
// block i at rows blk_row(i): 256 i forward, 256 (nblk-1-i) backward) and
//     M(i, i) = alpha * inv(op(A)_ii)                     (diagonal blocks)
//     M(i, j) = -inv(op(A)_ii) op(A)_ij, j solved before  (left; side=R transposed)
// precomputed from A alone, block i of the solution is ONE sum of i + 1
// "groups" of K = 256:
//     X_i = M(i, i) B_i  +  sum_{j<i} M(i, j) X_j        (group 0, groups j + 1)
// The team (2-4 CTA pairs, as many as the machine holds) splits the groups of
// every block between its members (host-side greedy balance, gmask): member 0
// always takes the newest group (j = i - 1, the only one that waits for the
// block just solved), sums its partial with the helpers' (members 1.., fp32
// partials through L2) and stores X_i in place over B_i; the helpers' groups
// are older, so their partials run ahead.  A pair
// computes 256 x 256 tiles, the tcgen05 shape at which the 3xTF32 UMMAs run
// at full rate (a 128-wide N takes as long per instruction as 256).
//
// Kernel structure (640 threads per CTA, the tc_kernel.cu roles):
//   warp 0      TMA producer: M rows (its 128) x 32 k, X/B rows k x its 128 RHS
//   warp 1      MMA issuer (leader CTA): 3xTF32 tcgen05.mma cta_group::2,
//               M = N = 256, TMEM partials restarted every kc k-blocks
//   warps 4-11  transform: lo = x - trunc_tf32(x) (hi is the raw TMA tile)
//   warps 12-19 epilogue: partials -> register sum (+ the helper's partial) ->
//               X_i stored -> release counter (member 0) / partial -> L2 (member 1)
#include <cuda.h>
#include <cuda_runtime.h>
#include <atomic>
#include <cstring>
#include <mutex>
#include <stdlib.h>
#include <cstdio>

#include "../../include/blas3.h"
#include "kernels.h"
#include "tc_ptx.h"
#include "tc_stage.h"

namespace blas3 {
namespace {

constexpr int BK = stage::BK;              // k-block (elements)
constexpr int HA = 128;                    // M rows staged per CTA (block = 256 per pair)
constexpr int BLK = 256;                   // rows of X per block (UMMA M of the pair)
constexpr int KB_BLK = BLK / BK;           // k-blocks per group (8)
constexpr int PN = 256;                    // right-hand sides per team (UMMA N)
constexpr int HB = PN / 2;                 // right-hand sides staged per CTA
constexpr int RS = 4, LS = 2;              // raw / lo stages
constexpr int NACC = 2;                    // TMEM partials (2 x 256 columns)
constexpr int MAX_BLK = 32;                // blocks per panel (R <= 8192)
constexpr int MAX_MEM = 4;                 // CTA pairs per team
constexpr int WARP_TMA = 0, WARP_MMA = 1, WARP_TR0 = 4, NUM_TR_WARPS = 8;
constexpr int WARP_EPI0 = WARP_TR0 + NUM_TR_WARPS, NUM_EPI_WARPS = 8;
constexpr int NTHREADS = (WARP_EPI0 + NUM_EPI_WARPS) * 32;       // 640
constexpr int TR_THREADS = NUM_TR_WARPS * 32, EPI_THREADS = NUM_EPI_WARPS * 32;
constexpr int EPI_REGS = 144, OTHER_REGS = 64;
constexpr int NCOL = PN / 2;               // columns per epilogue thread (two warps per lane quarter)
using stage::LAYOUT_K;
using stage::LAYOUT_MN;
using stage::op_desc;
constexpr size_t PART_FLOATS = (size_t)HA * PN;   // one CTA's partial (128 rows x 256)

struct alignas(1024) Stage {
  uint8_t A[HA * BK * 4];                  // 16 KiB
  uint8_t B[HB * BK * 4];                  // 16 KiB
};
struct Bars {
  uint64_t full[RS], empty[RS], ready[LS], lo_empty[LS];
  uint64_t tfull[NACC], tempty[NACC];
  uint32_t tmem_base;
};
constexpr size_t SMEM = sizeof(Stage) * (RS + LS) + sizeof(Bars) + 1024;

struct PanelParams {
  CUtensorMap mapA;                        // M: rk (left) / kr (right) view
  CUtensorMap mapB;                        // X over B: kr (left) / rk (right) view
  float *X;                                // panel origin: left X(k,n) = X[k + n ldx], right X[n + k ldx]
  float *ws;                               // helper partials: [team][helper][slot 2][rank 2][col 256][row 128]
  uint32_t *ctr;                           // [team][MAX_MEM]: X blocks stored, then each helper's
                                           // partials written (x2 CTAs each)
  int64_t ldx, R, nrhs;
  int32_t nblk, layA, layB, right, forward, kc, nslab, nteams, nmem;
  // extra members (one CTA pair serving several teams, see role_of): the
  // device-level split -- T_dev teams, E_dev extras, extra e = slab % E_dev --
  // fixes every slab's group masks (and with them the rounding); a launch
  // that cannot place the extras (fold = 1) has each team's last core member
  // compute the extra's partial as a second item per block
  int32_t tdev, edev, nextra, fold;
  int32_t dbg;                             // BLAS3_DEBUG_PANEL knock-outs (timing experiments only)
  unsigned long long *trace;               // BLAS3_TRACE_PANEL: per-block stage times of team 0 (diagnostics)
  uint32_t gmask[2][MAX_BLK][MAX_MEM];     // [class][block i][member h]: groups summed by h (h = nmem: the extra)
};

// first row of processing block i
__device__ __forceinline__ int64_t blk_row(const PanelParams &p, int i) {
  return (int64_t)(p.forward ? i : p.nblk - 1 - i) * BLK;
}
// group-mask class of a slab: 0 if its extra serves the most teams, else 1
__host__ __device__ __forceinline__ int slab_class(int tdev, int edev, int slab) {
  return (edev == 0 || tdev % edev == 0 || slab % edev < tdev % edev) ? 0 : 1;
}
// groups of block i summed by member h for slab (bit g: group g; g = 0 the
// block's own right-hand side, g >= 1 the solved block g - 1)
__device__ __forceinline__ uint32_t groups_of(const PanelParams &p, int slab, int i, int h) {
  return p.gmask[slab_class(p.tdev, p.edev, slab)][i][h];
}
constexpr int MAX_SERVE = 8;               // teams per extra pair at most
// The work items of one CTA pair, in the order all four roles visit them.
//   core pair (team, member hc): for every slab of the team (slab = team +
//     r * nteams), for every block i: member hc's partial (hc = 0: the owner,
//     which also stores X_i); with fold, member nmem - 1 follows each of its
//     items with the extra's (member nmem) partial of the same block;
//   extra pair e (every team owns exactly one slab): for every block i, for
//     every team it serves (slab = e + j * nextra): member nmem's partial.
struct Role {
  int team0, hc, extra, nserved, nper, nitems;
};
__device__ __forceinline__ Role role_of(const PanelParams &p, int pair) {
  Role r;
  const int ncore = p.nteams * p.nmem;
  r.extra = pair >= ncore;
  if (r.extra) {
    r.team0 = pair - ncore;
    r.hc = p.nmem;
    r.nserved = (p.nteams - r.team0 + p.nextra - 1) / p.nextra;
    r.nper = 1;
    r.nitems = p.nblk * r.nserved;
  } else {
    r.team0 = pair / p.nmem;
    r.hc = pair % p.nmem;
    r.nserved = 1;
    r.nper = (p.fold && r.hc == p.nmem - 1) ? 2 : 1;
    r.nitems = (p.nslab - r.team0 + p.nteams - 1) / p.nteams * p.nblk * r.nper;
  }
  return r;
}
struct Item {
  int slab, team, i, h, j;                 // j: served-team index (extras), else 0
  uint32_t gblk, gbase;                    // block counter of the slab's team, its value at block 0
};
__device__ __forceinline__ Item item_of(const PanelParams &p, const Role &r, int idx) {
  Item it;
  if (r.extra) {
    it.i = idx / r.nserved;
    it.j = idx % r.nserved;
    it.slab = r.team0 + it.j * p.nextra;
    it.team = it.slab;
    it.h = p.nmem;
    it.gblk = (uint32_t)it.i;
    it.gbase = 0;
  } else {
    const int per_slab = p.nblk * r.nper, rr = idx / per_slab, rem = idx % per_slab;
    it.i = rem / r.nper;
    it.h = r.hc + rem % r.nper;
    it.j = 0;
    it.slab = r.team0 + rr * p.nteams;
    it.team = r.team0;
    it.gbase = (uint32_t)(rr * p.nblk);
    it.gblk = it.gbase + (uint32_t)it.i;
  }
  return it;
}

__device__ __forceinline__ void load_op(const CUtensorMap *m, int lay, uint8_t *dst, int64_t r0,
                                        int64_t k0, int rows, uint64_t *bar) {
  if (lay == LAYOUT_MN) {
    for (int c = 0; c < rows / 32; ++c)
      ptx::tma_load_4d(m, bar, dst + c * (BK * 128), (int32_t)(r0 + 32 * c), (int32_t)k0, 0, 0);
  } else {
    ptx::tma_load_4d(m, bar, dst, (int32_t)k0, (int32_t)r0, 0, 0);
  }
}
__device__ __forceinline__ void arrive_leader(uint64_t *bar, uint32_t rank, uint32_t id, uint32_t n,
                                              bool first) {
  ptx::named_bar_sync(id, n);
  if (first) {
    if (rank == 0) ptx::mbar_arrive(bar);
    else ptx::mbar_arrive_cluster(bar, 0);
  }
}
// Team hand-offs go through global counters (the two pairs of a team are
// different clusters): release = __threadfence + atomicAdd after a CTA's
// stores; acquire = ld.acquire.gpu poll, plus a proxy fence before TMA reads.
__device__ __forceinline__ void wait_count(const uint32_t *ctr, uint32_t target) {
  stage::spin_until(ctr, target, 64);
}

// diagnostics: %globaltimer of stage st of block i, team 0, CTA rank 0 of member h
__device__ __forceinline__ void ptrace(const PanelParams &p, int h, int i, int st) {
  if (p.trace != nullptr && blockIdx.x == 2 * h && h < 2 && i < MAX_BLK) {
    unsigned long long v;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(v));
    p.trace[(h * MAX_BLK + i) * 4 + st] = v;
  }
}

__global__ void __launch_bounds__(NTHREADS, 1) trsm_panel_kernel(const __grid_constant__ PanelParams prm) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  Stage *raw = reinterpret_cast<Stage *>(smem);
  Stage *lo = raw + RS;
  Bars *bars = reinterpret_cast<Bars *>(smem + sizeof(Stage) * (RS + LS));
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const uint32_t rank = ptx::cluster_ctarank();
  const int pair = blockIdx.x / 2;
  const Role role = role_of(prm, pair);
  const int h = role.hc;                                   // 0: owner of its team's X, else a helper
  const int nblk = prm.nblk;
  // members whose partial the owner adds: the core helpers, then the extra
  const int mlast = prm.nmem - 1 + (prm.edev > 0 ? 1 : 0);

  if (threadIdx.x == 0) {
    for (int s = 0; s < RS; ++s) { ptx::mbar_init(&bars->full[s], 1); ptx::mbar_init(&bars->empty[s], 1); }
    for (int s = 0; s < LS; ++s) { ptx::mbar_init(&bars->ready[s], 2); ptx::mbar_init(&bars->lo_empty[s], 1); }
    for (int a = 0; a < NACC; ++a) { ptx::mbar_init(&bars->tfull[a], 1); ptx::mbar_init(&bars->tempty[a], 2); }
    ptx::fence_mbar_init();
  }
  if (warp == WARP_MMA) ptx::tmem_alloc<2>(&bars->tmem_base, NACC * PN);
  ptx::tc_fence_before();
  ptx::cluster_sync();
  ptx::tc_fence_after();
  const uint32_t tmem = bars->tmem_base;
  ptx::griddep_wait();

#define BLAS3_DEC_REGS() asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(OTHER_REGS))
#define BLAS3_INC_REGS() asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(EPI_REGS))
  if (warp < WARP_TR0) {
    BLAS3_DEC_REGS();
    if (warp == WARP_TMA && lane == 0) {
      // ============================ producer (each CTA stages its own halves)
      ptx::tma_prefetch(&prm.mapA);
      ptx::tma_prefetch(&prm.mapB);
      uint32_t it = 0, x_seen[MAX_SERVE] = {};
      for (int idx = 0; idx < role.nitems; ++idx) {
        const Item e = item_of(prm, role, idx);
        const uint32_t *ctr_x = prm.ctr + MAX_MEM * e.team;
        if (e.i == 0) x_seen[e.j] = 0;
        const int64_t n0 = (int64_t)e.slab * PN + HB * rank;
        const int64_t r0 = blk_row(prm, e.i) + HA * rank;
        for (uint32_t m = groups_of(prm, e.slab, e.i, e.h); m; m &= m - 1) {
          const int g = __ffs(m) - 1;
          if (g > 0 && !(prm.dbg & 1)) {              // X of solved block g - 1 stored (both CTAs of the owner)
            const uint32_t need = 2 * (e.gbase + g);
            if (need > x_seen[e.j]) {
              wait_count(ctr_x, need);
              asm volatile("fence.proxy.async.global;" ::: "memory");
              x_seen[e.j] = need;
            }
          }
          const int64_t kg = blk_row(prm, g == 0 ? e.i : g - 1);
          for (int w = 0; w < KB_BLK; ++w, ++it) {
            const int rs = it % RS;
            ptx::mbar_wait(&bars->empty[rs], ((it / RS) & 1) ^ 1);
            ptx::mbar_arrive_expect_tx(&bars->full[rs], (HA + HB) * BK * 4);
            load_op(&prm.mapA, prm.layA, raw[rs].A, r0, kg + w * BK, HA, &bars->full[rs]);
            load_op(&prm.mapB, prm.layB, raw[rs].B, n0, kg + w * BK, HB, &bars->full[rs]);
          }
        }
      }
      for (int i = 0; i < RS; ++i, ++it) ptx::mbar_wait(&bars->empty[it % RS], ((it / RS) & 1) ^ 1);
    } else if (warp == WARP_MMA && rank == 0) {
      // ============================ MMA issuer (leader CTA)
      const uint32_t idesc = ptx::idesc_tf32(BLK, PN, prm.layA == LAYOUT_MN, prm.layB == LAYOUT_MN);
      uint32_t it = 0, cc = 0;
      for (int idx = 0; idx < role.nitems; ++idx) {
        {
          const Item e = item_of(prm, role, idx);
          const int i = e.i;
          const int nkb = KB_BLK * __popc(groups_of(prm, e.slab, i, e.h));
          int left = 0;
          uint32_t acc = 0, buf = 0;
          for (int t = 0; t < nkb; ++t, ++it) {
            if (left == 0) {
              buf = cc % NACC;
              ptx::mbar_wait_cluster(&bars->tempty[buf], ((cc / NACC) & 1) ^ 1);
              ptx::tc_fence_after();
              acc = 0;
              left = prm.kc;
            }
            const int rs = it % RS, ls = it % LS;
            ptx::mbar_wait_cluster(&bars->ready[ls], (it / LS) & 1);
            ptx::tc_fence_after();
            if (lane == 0 && t == 0 && !role.extra) ptrace(prm, e.h, i, 0);
            if (lane == 0 && t == nkb - KB_BLK && !role.extra) ptrace(prm, e.h, i, 1);
            if (lane == 0) {
              const uint32_t d = tmem + buf * PN;
              const uint32_t hiA = ptx::smem_u32(raw[rs].A), hiB = ptx::smem_u32(raw[rs].B);
              const uint32_t loA = ptx::smem_u32(lo[ls].A), loB = ptx::smem_u32(lo[ls].B);
              if (!(prm.dbg & 8)) {
                // cross terms first (small, into a fresh partial), then hi*hi (Q24)
#pragma unroll
                for (int k8 = 0; k8 < BK / 8; ++k8) {
                  ptx::mma_tf32_ss_pair(d, op_desc(loA, prm.layA, k8), op_desc(hiB, prm.layB, k8), idesc, acc);
                  ptx::mma_tf32_ss_pair(d, op_desc(hiA, prm.layA, k8), op_desc(loB, prm.layB, k8), idesc, 1);
                  acc = 1;
                }
#pragma unroll
                for (int k8 = 0; k8 < BK / 8; ++k8)
                  ptx::mma_tf32_ss_pair(d, op_desc(hiA, prm.layA, k8), op_desc(hiB, prm.layB, k8), idesc, 1);
              }
              ptx::mma_commit_pair(&bars->empty[rs], 0x3);
              ptx::mma_commit_pair(&bars->lo_empty[ls], 0x3);
            }
            acc = 1;
            __syncwarp();
            if (--left == 0 || t == nkb - 1) {
              if (lane == 0) ptx::mma_commit_pair(&bars->tfull[buf], 0x3);
              __syncwarp();
              ++cc;
              left = 0;
            }
          }
        }
      }
    }
  } else if (warp < WARP_EPI0) {
    // ============================ transform (own halves)
    BLAS3_DEC_REGS();
    const int tt = threadIdx.x - WARP_TR0 * 32;
    uint32_t it = 0;
    for (int idx = 0; idx < role.nitems; ++idx) {
      {
        const Item e = item_of(prm, role, idx);
        const int nkb = KB_BLK * __popc(groups_of(prm, e.slab, e.i, e.h));
        for (int t = 0; t < nkb; ++t, ++it) {
          const int rs = it % RS, ls = it % LS;
          ptx::mbar_wait(&bars->full[rs], (it / RS) & 1);
          ptx::mbar_wait(&bars->lo_empty[ls], ((it / LS) & 1) ^ 1);
          if (!(prm.dbg & 2)) {
            stage::split_pass<TR_THREADS>(raw[rs].A, lo[ls].A, HA * BK * 4, tt);
            stage::split_pass<TR_THREADS>(raw[rs].B, lo[ls].B, HB * BK * 4, tt);
          }
          ptx::fence_proxy_async_smem();
          arrive_leader(&bars->ready[ls], rank, 2, TR_THREADS, tt == 0);
        }
      }
    }
  } else {
    // ============================ epilogue (own 128 rows; two warps per lane quarter)
    BLAS3_INC_REGS();
    const int q = warp & 3, half = (warp - WARP_EPI0) >> 2;
    const bool lead = threadIdx.x == WARP_EPI0 * 32;
    const int rloc = q * 32 + lane;                           // row within this CTA's 128
    uint32_t cc = 0;
    for (int idx = 0; idx < role.nitems; ++idx) {
      {
        const Item e = item_of(prm, role, idx);
        const int i = e.i, hh = e.h;
        const uint32_t gblk = e.gblk;
        uint32_t *ctr_x = prm.ctr + MAX_MEM * e.team;
        const int64_t c0 = (int64_t)e.slab * PN + half * NCOL;   // first right-hand side of this thread
        const int nkb = KB_BLK * __popc(groups_of(prm, e.slab, i, hh));
        const int nch = nkb > 0 ? (nkb + prm.kc - 1) / prm.kc : 0;
        // helper m's slot for this block: [col][row] (a warp's accesses per column are one 128-B line)
        auto slot = [&](int m) {
          return prm.ws + (((((size_t)e.team * (MAX_MEM - 1) + (m - 1)) * 2 + (gblk & 1)) * 2 + rank) * PART_FLOATS) +
                 (size_t)(half * NCOL) * HA + rloc;
        };
        float S[NCOL];
#pragma unroll
        for (int j = 0; j < NCOL; ++j) S[j] = 0.f;
        // member 0 adds the helper's partial (which runs ahead) while its MMA
        // works on the newest group: before waiting for that group's first chunk
        const int cpart = hh == 0 ? (nkb - KB_BLK) / prm.kc : -1;
        for (int c = 0; c < nch; ++c, ++cc) {
          if (c == cpart) {
            for (int m = 1; m <= mlast; ++m) {
              if (lead) wait_count(ctr_x + m, 2 * (gblk + 1));
              ptx::named_bar_sync(5, EPI_THREADS);
              const float *part = slot(m);
#pragma unroll
              for (int j = 0; j < NCOL; ++j) S[j] += __ldcg(part + (size_t)j * HA);
            }
          }
          const uint32_t buf = cc % NACC;
          ptx::mbar_wait(&bars->tfull[buf], (cc / NACC) & 1);
          ptx::tc_fence_after();
          const uint32_t ta = tmem + buf * PN + half * NCOL + ((uint32_t)(q * 32) << 16);
#pragma unroll
          for (int g = 0; g < NCOL / 16; g += 2) {
            uint32_t v[16], u[16];
            ptx::tmem_ld_32x32b_x16(ta + g * 16, v);
            ptx::tmem_ld_32x32b_x16(ta + (g + 1) * 16, u);
            ptx::tmem_ld_wait();
#pragma unroll
            for (int j = 0; j < 16; ++j) S[g * 16 + j] += __uint_as_float(v[j]);
#pragma unroll
            for (int j = 0; j < 16; ++j) S[(g + 1) * 16 + j] += __uint_as_float(u[j]);
          }
          ptx::tc_fence_before();
          arrive_leader(&bars->tempty[buf], rank, 3, EPI_THREADS, lead);
        }
        if (lead && !role.extra) ptrace(prm, hh, i, 2);
        if (hh > 0) {
          // helper: the slot was last read for block gblk - 2 (X of it stored)
          if (lead && gblk >= 2) wait_count(ctr_x, 2 * (gblk - 1));
          ptx::named_bar_sync(5, EPI_THREADS);
          float *part = slot(hh);
#pragma unroll
          for (int j = 0; j < NCOL; ++j) __stcg(part + (size_t)j * HA, S[j]);
          ptx::named_bar_sync(5, EPI_THREADS);
          if (lead) { __threadfence(); atomicAdd(ctr_x + hh, 1u); if (!role.extra) ptrace(prm, hh, i, 3); }
          continue;
        }
        // member 0: X_i
        // X_i rows [blk_row + 128 rank, +128) x right-hand sides [c0, c0 + 128)
        const int64_t row = blk_row(prm, i) + HA * rank + rloc;
        const int64_t nval = prm.nrhs - c0;                  // valid columns (warp-uniform)
        if (!prm.right) {
          float *p = prm.X + row + c0 * prm.ldx;
#pragma unroll
          for (int j = 0; j < NCOL; ++j) {
            if (j < nval) *p = S[j];
            p += prm.ldx;
          }
        } else {
          float *p = prm.X + c0 + row * prm.ldx;
          const bool vec = nval >= NCOL && (prm.ldx % 4) == 0 && (reinterpret_cast<uintptr_t>(p) % 16) == 0;
          if (vec) {
#pragma unroll
            for (int j = 0; j < NCOL; j += 4)
              *reinterpret_cast<float4 *>(p + j) = make_float4(S[j], S[j + 1], S[j + 2], S[j + 3]);
          } else {
#pragma unroll
            for (int j = 0; j < NCOL; ++j)
              if (j < nval) p[j] = S[j];
          }
        }
        ptx::named_bar_sync(5, EPI_THREADS);
        if (lead) { __threadfence(); atomicAdd(ctr_x, 1u); ptrace(prm, h, i, 3); }
      }
    }
  }

  ptx::tc_fence_before();
  ptx::cluster_sync();
  if (warp == WARP_MMA) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<2>(tmem, NACC * PN);
  }
#undef BLAS3_DEC_REGS
#undef BLAS3_INC_REGS
}

// M's diagonal blocks: alpha * inv(op(A)_bb), natural column-major, zeros in
// the blank triangle, from the lower-form inverses in the panel-inverse
// workspace (inv(L_bb); op(A)_bb = L_bb if lower_op, else L_bb^T).
__global__ void panel_diag_kernel(const float *Dp, int64_t ldD, float *M, int64_t ldm, int lower_op,
                                  float alpha) {
  const int64_t o = (int64_t)blockIdx.y * BLK;
  const int c = blockIdx.x, r = threadIdx.x;
  float v = 0.f;
  if (lower_op) { if (r >= c) v = Dp[(o + r) + (o + c) * ldD]; }
  else          { if (c >= r) v = Dp[(o + c) + (o + r) * ldD]; }
  M[(o + r) + (o + c) * ldm] = alpha * v;
}

}  // namespace

int launch_trsm_panel_diag(const float *Dp, int64_t ldD, float *M, int64_t ldm, int64_t R, bool lower_op,
                           float alpha, cudaStream_t s) {
  if (R % BLK) return -1;
  panel_diag_kernel<<<dim3(BLK, (unsigned)(R / BLK)), BLK, 0, s>>>(Dp, ldD, M, ldm, lower_op ? 1 : 0, alpha);
  note_launch();
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

// member 0's serial hand-off per block in tenths of a group (BLAS3_PANEL_HANDOFF, experiments)
static int64_t prm_handoff() {
  static const int64_t v = [] { const char *e = getenv("BLAS3_PANEL_HANDOFF"); return e ? atoll(e) : 3; }();
  return v;
}
// members per team at most (BLAS3_PANEL_MEMBERS, 1..MAX_MEM; default 3, when
// the machine holds them: N = 4096, 16 teams, kernel 167 us with three
// members against 187 with two and 200 with four -- with four, member 0 only
// keeps the newest group and its per-block chain, which now includes reading
// three partials, bounds the solve; profiles/r02_strsm_panel.md)
static int panel_members() {
  static const int v = [] { const char *e = getenv("BLAS3_PANEL_MEMBERS"); const int m = e ? atoi(e) : 3;
                            return m < 1 ? 1 : (m > MAX_MEM ? MAX_MEM : m); }();
  return v;
}
// teams: one per 256 right-hand sides (at most num_sms / 4); members: the
// CTA pairs the machine holds per team, up to panel_members()
// The member count -- and with it each block's split into partial sums, i.e.
// the rounding -- follows the DEVICE's SM count, not the launch limit
// (BLAS3_OPT_MAX_SMS): a solve on fewer SMs runs fewer teams, each looping over
// more slabs, and gives the same bits (tests/test_trsm_panel_gpu.py).
static int device_sms() {
  static std::atomic<int> cache[64];
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return 148;
  int v = cache[dev].load(std::memory_order_relaxed);
  if (v == 0) {
    if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || v < 2) v = 148;
    cache[dev].store(v, std::memory_order_relaxed);
  }
  return v;
}
// extra members (BLAS3_PANEL_EXTRA=1; off by default: measured slower, see profiles/r02_strsm_panel.md): with one slab per team and
// CTA pairs left over (N = 8192: 32 teams x 2 members = 64 of 74 pairs), each
// leftover pair helps up to MAX_SERVE teams (extra e: slabs e, e + E, ...)
static int panel_extra_on() {
  static const int v = [] { const char *e = getenv("BLAS3_PANEL_EXTRA"); return e ? atoi(e) : 0; }();
  return v;
}
struct PanelShape {
  int64_t teams;                 // teams of this launch
  int nmem;                      // core members per team
  int tdev, edev;                // device-level teams and extras (fix the group split)
  int nextra, fold;              // extras placed in this launch / folded into the last core member
};
static PanelShape panel_shape(int64_t nrhs, int num_sms) {
  PanelShape sh{};
  const int64_t nslab = (nrhs + PN - 1) / PN, pairs = num_sms / 2, full = device_sms() / 2;
  const int nmem_dev = (int)imax(1, imin(panel_members(), full / imin(nslab, imax(1, full / 2))));
  sh.nmem = nmem_dev;
  if (sh.nmem > pairs) sh.nmem = (int)imax(1, pairs);  // (a launch limit below one team)
  sh.teams = imin(nslab, imax(1, pairs / sh.nmem));
  const int64_t tdev = imin(nslab, imax(1, full / nmem_dev));
  int64_t edev = 0;
  // (only where the machine could not give every team the preferred member
  // count: a whole extra per team is a 4th member, measured slower at N = 4096)
  if (panel_extra_on() && nslab == tdev && nmem_dev < panel_members() && nmem_dev + 1 <= MAX_MEM) {
    edev = imin(tdev, full - tdev * nmem_dev);
    if (edev > 0 && (tdev + edev - 1) / edev > MAX_SERVE) edev = 0;
  }
  sh.tdev = (int)tdev;
  sh.edev = (int)edev;
  const bool place = edev > 0 && sh.nmem == nmem_dev && sh.teams == tdev && pairs >= tdev * nmem_dev + edev;
  sh.nextra = place ? (int)edev : 0;
  sh.fold = edev > 0 && !place ? 1 : 0;
  return sh;
}
size_t trsm_panel_ws_bytes(int64_t nrhs, int num_sms) {
  const int64_t t = panel_shape(nrhs, num_sms).teams;
  return (size_t)t * (MAX_MEM - 1) * 4 * PART_FLOATS * sizeof(float) + (size_t)t * MAX_MEM * sizeof(uint32_t);
}

int launch_trsm_panel(const float *M, int64_t ldm, float *X, int64_t ldx, bool right, int64_t R,
                      int64_t nrhs, bool forward, int kc, void *ws, cudaStream_t s, int num_sms) {
  if (R <= 0 || R % BLK || R / BLK > MAX_BLK || nrhs <= 0 || kc < 1 || !ws) return -1;
  const PanelShape sh = panel_shape(nrhs, num_sms);
  const int64_t nteams = sh.teams;
  const int nmem = sh.nmem;
  if (nteams < 1) return -1;
  static PanelParams prm;
  static std::mutex mu;
  std::lock_guard<std::mutex> lk(mu);
  memset(&prm, 0, sizeof(prm));
  // M: left rk (Xa(r,k) = M[r + k ldm]) / right kr (Xa(r,k) = M[k + r ldm]);
  // X: left kr (Xb(n,k) = X[k + n ldx]) / right rk (Xb(n,k) = X[n + k ldx])
  prm.layA = right ? LAYOUT_K : LAYOUT_MN;
  prm.layB = right ? LAYOUT_MN : LAYOUT_K;
  bool ok = right ? tma_map_f32(&prm.mapA, M, R, R, ldm, BK, HA, false)
                  : tma_map_f32(&prm.mapA, M, R, R, ldm, 32, BK, true);
  ok = ok && (right ? tma_map_f32(&prm.mapB, X, nrhs, R, ldx, 32, BK, true)
                    : tma_map_f32(&prm.mapB, X, R, nrhs, ldx, BK, HB, false));
  if (!ok) return -4;
  prm.X = X;
  prm.ws = static_cast<float *>(ws);
  prm.ctr = reinterpret_cast<uint32_t *>(static_cast<uint8_t *>(ws) +
                                         (size_t)nteams * (MAX_MEM - 1) * 4 * PART_FLOATS * sizeof(float));
  prm.ldx = ldx;
  prm.R = R;
  prm.nrhs = nrhs;
  prm.nblk = (int32_t)(R / BLK);
  prm.right = right ? 1 : 0;
  prm.forward = forward ? 1 : 0;
  prm.kc = kc;
  prm.nslab = (int32_t)((nrhs + PN - 1) / PN);
  prm.nteams = (int32_t)nteams;
  prm.nmem = nmem;
  // group split of every block: member 0 takes the newest group (it alone
  // waits for the block just solved), every other group goes to the member
  // with the least work so far (ties to a helper, whose partial runs ahead).
  // Member 0 is also charged its serial per-block hand-off (store, release,
  // reload of X_i), 0.3 of a group: kernel 187 / 189 us at N = 4096 / 8192
  // against 194 / 196 at 0.6 and 188 / 190 at 0 (profiles/r02_strsm_panel.md)
  prm.tdev = sh.tdev;
  prm.edev = sh.edev;
  prm.nextra = sh.nextra;
  prm.fold = sh.fold;
  const int64_t grp = 10, handoff = prm_handoff();
  for (int cls = 0; cls < 2; ++cls) {
    // the extra (member nmem) serves w teams: a group costs it w times as much
    static const int64_t xw = [] { const char *e = getenv("BLAS3_PANEL_XW"); return e ? atoll(e) : 0; }();
    const int64_t w = sh.edev == 0 ? 0 : (cls == 0 ? (sh.tdev + sh.edev - 1) / sh.edev : sh.tdev / sh.edev) + xw;
    const int mlast = nmem - 1 + (sh.edev > 0 ? 1 : 0);
    int64_t load[MAX_MEM] = {0, 0, 0, 0};
    for (int i = 0; i < prm.nblk; ++i) {
      uint32_t gm[MAX_MEM] = {0, 0, 0, 0};
      gm[0] = 1u << i;
      load[0] += grp + handoff;
      for (int g = 0; g < i; ++g) {
        int best = 0;
        if (sh.edev == 0) {
          for (int m = nmem - 1; m >= 0; --m)
            if (load[m] < load[best]) best = m;
          if (nmem > 1 && best == 0 && load[nmem - 1] == load[0]) best = nmem - 1;
        } else {
          // least load after taking the group (ties to the later member: the
          // extra takes the oldest groups, whose partials can run furthest ahead)
          auto after = [&](int m) { return load[m] + grp * (m == nmem ? w : 1); };
          best = mlast;
          for (int m = mlast - 1; m >= 0; --m)
            if (after(m) < after(best)) best = m;
        }
        gm[best] |= 1u << g;
        load[best] += grp * (best == nmem && sh.edev > 0 ? w : 1);
      }
      for (int m = 0; m < MAX_MEM; ++m) prm.gmask[cls][i][m] = gm[m];
    }
  }
  static const int dbg = [] { const char *e = getenv("BLAS3_DEBUG_PANEL"); return e ? atoi(e) : 0; }();
  prm.dbg = dbg;
  static const bool trace = getenv("BLAS3_TRACE_PANEL") != nullptr;
  static unsigned long long *tbuf = nullptr;
  if (trace) {
    if (!tbuf && cudaMalloc(&tbuf, 2 * MAX_BLK * 4 * sizeof(unsigned long long)) != cudaSuccess) return -1;
    cudaMemsetAsync(tbuf, 0, 2 * MAX_BLK * 4 * sizeof(unsigned long long), s);
    prm.trace = tbuf;
  }
  static std::atomic<bool> attr[64];
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return -1;
  if (!attr[dev].load(std::memory_order_acquire)) {
    if (cudaFuncSetAttribute(trsm_panel_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SMEM) !=
        cudaSuccess)
      return -1;
    attr[dev].store(true, std::memory_order_release);
  }
  if (cudaMemsetAsync(prm.ctr, 0, (size_t)nteams * MAX_MEM * sizeof(uint32_t), s) != cudaSuccess) return -1;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(2 * (nmem * nteams + sh.nextra)));
  cfg.blockDim = dim3(NTHREADS);
  cfg.dynamicSmemBytes = SMEM;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = 2;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  const cudaError_t e = cudaLaunchKernelEx(&cfg, trsm_panel_kernel, prm);
  note_launch(3);
  if (trace && e == cudaSuccess) {            // member, block: mma start / newest group / drained / released (us)
    unsigned long long hb[2 * MAX_BLK * 4];
    cudaStreamSynchronize(s);
    cudaMemcpy(hb, tbuf, sizeof(hb), cudaMemcpyDeviceToHost);
    unsigned long long t0 = ~0ull;
    for (int k = 0; k < 2 * MAX_BLK * 4; ++k) if (hb[k] && hb[k] < t0) t0 = hb[k];
    for (int hh = 0; hh < 2; ++hh)
      for (int i = 0; i < prm.nblk && hh < nmem; ++i) {
        const unsigned long long *r = hb + (hh * MAX_BLK + i) * 4;
        auto us = [&](unsigned long long v) { return v ? (double)(v - t0) / 1e3 : -1.0; };
        fprintf(stderr, "[panel] m%d blk %2d groups %2d: mma %7.2f newest %7.2f drained %7.2f released %7.2f\n", hh, i,
                __builtin_popcount(prm.gmask[0][i][hh]), us(r[0]), us(r[1]),
                us(r[2]), us(r[3]));
      }
  }
  return (e == cudaSuccess && cudaGetLastError() == cudaSuccess) ? 0 : -1;
}

}  // namespace blas3
