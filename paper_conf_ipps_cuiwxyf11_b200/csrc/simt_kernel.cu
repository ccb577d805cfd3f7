// simt_kernel.cu -- exact-FP32 SIMT variant of the structured GEMM (row A10).
//
// The paper's own kernel class: shared-memory tiles + register-blocked C
// ("SM_alloc" P:93-99, "Reg_alloc(C)" P:101, Volkov-style scheme P:75) with
// the structure of every routine applied while the tile is staged to shared
// memory (mirror / zero-select / unit diagonal, via load_op) and the uplo
// mask applied in the epilogue.  128x128 CTA tile, BK=8, 256 threads, 8x8
// outputs per thread, register-prefetched double buffer, one CTA per SM
// (251 registers: the 64 accumulators and both operand prefetches stay in
// registers, no spills).  Dense operands of interior tiles -- and the blocks
// of structured operands that lie entirely inside one stored orientation --
// are fetched by per-thread pointers advanced by a constant stride per k-block.  It is the route for
// arguments TMA cannot address (unaligned pointers, ld % 4 != 0) and the FP32
// comparison point for the 3xTF32 path.
//
// The Problem stays in kernel-parameter space (dynamic segment indexing
// becomes constant-bank loads); only the current segment's operand
// descriptors are copied to registers.
#include <cuda_runtime.h>
#include "problem.h"
#include "kernels.h"

namespace blas3 {

namespace {
constexpr int BM = 128, BN = 128, BK = 8, NT = 256, PADS = 4;
constexpr int EPT = BM * BK / NT;         // elements of each operand fetched per thread (4)

struct Stage {
  float a[BK][BM + PADS];
  float b[BK][BN + PADS];
};

// r-contiguous ("rk") or k-contiguous ("kr") element mapping for coalescing
__device__ __forceinline__ void elem_map(bool kr, int tid, int i, int &r, int &k) {
  const int e = tid + i * NT;
  if (kr) { k = e % BK; r = e / BK; } else { r = e % BM; k = e / BM; }
}
__device__ __forceinline__ bool prefers_kr(const OpDesc &o) {
  return o.kind == OP_DENSE ? o.kr != 0 : (o.kind == OP_TRI ? o.swap != 0 : false);
}

// A BM x BK block of a structured operand that the strided-pointer fetch may
// read as stored: TRI blocks strictly inside the nonzero triangle (or any
// block of a zero-filled, non-unit TRI workspace), SYM blocks entirely in the
// stored (rk) triangle.  Diagonal-touching / shadow blocks take fetch().
__device__ __forceinline__ bool plain_block(const OpDesc &o, int64_t r0, int64_t kb) {
  if (o.kind == OP_DENSE) return true;
  if (o.kind == OP_TRI) {
    if (o.zero_blank && !o.unit) return true;
    return tri_kle(o) ? (kb + BK <= r0) : (kb >= r0 + BM);
  }
  return o.lower ? (kb + BK - 1 <= r0) : (kb >= r0 + BM - 1);
}

__device__ __forceinline__ void fetch(const OpDesc &o, bool kr, int64_t R, int64_t K, int64_t r0,
                                      int64_t kb, float (&v)[EPT]) {
#pragma unroll
  for (int i = 0; i < EPT; ++i) {
    int r, k;
    elem_map(kr, threadIdx.x, i, r, k);
    v[i] = load_op(o, r0 + r, kb + k, R, K);
  }
}

__device__ __forceinline__ void stash(float (*dst)[BM + PADS], bool kr, const float (&v)[EPT]) {
#pragma unroll
  for (int i = 0; i < EPT; ++i) {
    int r, k;
    elem_map(kr, threadIdx.x, i, r, k);
    dst[k][r] = v[i];
  }
}
}  // namespace

__global__ void __launch_bounds__(NT, 1)
simt_structured_gemm(const Problem P) {
  __shared__ __align__(16) Stage st[2];
  const int tid = threadIdx.x, tx = tid % 16, ty = tid / 16;
  const int64_t tiles_per = Tiles<BM, BN>::count(P);
  const int64_t nb = P.nbatch > 0 ? P.nbatch : 1;
  const int64_t ntiles = tiles_per * nb;

  for (int64_t tb = blockIdx.x; tb < ntiles; tb += gridDim.x) {
    const int64_t b = tb / tiles_per, t = tb - b * tiles_per;
    int64_t mi, nj;
    Tiles<BM, BN>::coords(P, t, mi, nj);
    const int64_t m0 = mi * BM, n0 = nj * BN;
    const int64_t m1 = imin(P.M, m0 + BM), n1 = imin(P.N, n0 + BN);

    float acc[8][8];
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
      for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;

    for (int s = 0; s < P.nseg; ++s) {
      OpDesc oa = P.seg[s].a, ob = P.seg[s].b;     // registers from here on
      const int64_t K = P.seg[s].K;
      if (nb > 1) {
        oa.ptr += batch_off(P.bs_a, b, P.per);
        ob.ptr += batch_off(P.bs_b, b, P.per);
      }
      Segment sg; sg.a = oa; sg.b = ob; sg.K = K;
      int64_t k0, k1;
      k_range(sg, m0, m1, n0, n1, k0, k1);
      k0 = (k0 / BK) * BK;
      if (k1 <= k0) continue;
      const bool akr = prefers_kr(oa), bkr = prefers_kr(ob);
      // dense operands of interior tiles: per-thread element pointers, advanced
      // by a constant stride per k-block (no per-element structure or bounds
      // logic); the k-tail and structured / edge operands take fetch()
      const bool fa = m0 + BM <= P.M, fb = n0 + BN <= P.N;
      const float *pa[EPT], *pb[EPT];
      const int64_t sa = akr ? BK : BK * oa.ld, sb = bkr ? BK : BK * ob.ld;
#pragma unroll
      for (int i = 0; i < EPT; ++i) {
        int r, k;
        elem_map(akr, tid, i, r, k);
        pa[i] = akr ? oa.ptr + (k0 + k) + (m0 + r) * oa.ld : oa.ptr + (m0 + r) + (k0 + k) * oa.ld;
        elem_map(bkr, tid, i, r, k);
        pb[i] = bkr ? ob.ptr + (k0 + k) + (n0 + r) * ob.ld : ob.ptr + (n0 + r) + (k0 + k) * ob.ld;
      }
      auto fetch_a = [&](int64_t kb, float (&v)[EPT]) {
        if (fa && kb + BK <= K && plain_block(oa, m0, kb)) {
#pragma unroll
          for (int i = 0; i < EPT; ++i) v[i] = __ldg(pa[i] + ((kb - k0) / BK) * sa);
        } else fetch(oa, akr, P.M, K, m0, kb, v);
      };
      auto fetch_b = [&](int64_t kb, float (&v)[EPT]) {
        if (fb && kb + BK <= K && plain_block(ob, n0, kb)) {
#pragma unroll
          for (int i = 0; i < EPT; ++i) v[i] = __ldg(pb[i] + ((kb - k0) / BK) * sb);
        } else fetch(ob, bkr, P.N, K, n0, kb, v);
      };
      float va[EPT], vb[EPT];
      fetch_a(k0, va);
      fetch_b(k0, vb);
      int buf = 0;
      __syncthreads();  // previous tile/segment finished reading smem
      stash(st[0].a, akr, va);
      stash(st[0].b, bkr, vb);
      __syncthreads();
      for (int64_t kb = k0; kb < k1; kb += BK) {
        const bool more = kb + BK < k1;
        if (more) {
          fetch_a(kb + BK, va);
          fetch_b(kb + BK, vb);
        }
        const Stage &S = st[buf];
#pragma unroll
        for (int k = 0; k < BK; ++k) {
          const float4 a0 = *reinterpret_cast<const float4 *>(&S.a[k][tx * 4]);
          const float4 a1 = *reinterpret_cast<const float4 *>(&S.a[k][64 + tx * 4]);
          const float4 b0 = *reinterpret_cast<const float4 *>(&S.b[k][ty * 4]);
          const float4 b1 = *reinterpret_cast<const float4 *>(&S.b[k][64 + ty * 4]);
          const float a[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
          const float bb[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
          for (int i = 0; i < 8; ++i)
#pragma unroll
            for (int j = 0; j < 8; ++j) acc[i][j] = fmaf(a[i], bb[j], acc[i][j]);
        }
        if (more) {
          stash(st[buf ^ 1].a, akr, va);
          stash(st[buf ^ 1].b, bkr, vb);
          __syncthreads();
          buf ^= 1;
        }
      }
    }

    // epilogue: D = alpha*acc + beta*C on the (masked) tile
    const int64_t coff = (nb > 1) ? batch_off(P.bs_c, b, P.per) : 0;
    const float *cin = P.Cin + coff;
    float *cout = P.Cout + coff;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int64_t c = n0 + (j < 4 ? ty * 4 + j : 64 + ty * 4 + (j - 4));
      if (c >= P.N) continue;
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int64_t r = m0 + (i < 4 ? tx * 4 + i : 64 + tx * 4 + (i - 4));
        if (r >= P.M) continue;
        if (P.c_tri == 1 && r < c) continue;
        if (P.c_tri == 2 && r > c) continue;
        float v = P.alpha * acc[i][j];
        if (P.beta != 0.f) v = fmaf(P.beta, cin[r + c * P.ldcin], v);
        cout[r + c * P.ldcout] = v;
      }
    }
  }
}

int launch_simt(const Problem &P, cudaStream_t stream, int num_sms) {
  int64_t tiles = Tiles<BM, BN>::count(P) * (P.nbatch > 0 ? P.nbatch : 1);
  if (tiles == 0) return 0;
  static int occ = 0;
  if (occ == 0 && (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, simt_structured_gemm, NT, 0) !=
                   cudaSuccess || occ < 1)) {
    cudaGetLastError();
    occ = 1;
  }
  int64_t grid = imin(tiles, (int64_t)num_sms * occ);
  simt_structured_gemm<<<(unsigned)grid, NT, 0, stream>>>(P);
  note_launch(1);
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

}  // namespace blas3
