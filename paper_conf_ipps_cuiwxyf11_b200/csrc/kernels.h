// kernels.h -- internal launcher interface between the routine drivers
// (abi.cu) and the device kernels.  Not part of the public C ABI.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include "problem.h"

namespace blas3 {

void note_launch(int path = 2);      // host-side launch counter (blas3_launch_count[_by_path]; 0..3)
int64_t opt(int key);                // tuning option (blas3_set_option / environment)

// Structured GEMM kernels (all routines canonicalise to a Problem).
int launch_simt(const Problem &P, cudaStream_t s, int num_sms);
// tcgen05 3xTF32 path; returns 0, -1 (CUDA error) or -4 (TMA encode failure).
int launch_tc(const Problem &P, cudaStream_t s, int num_sms);
// TMA eligibility of one operand / the output (16-B pointer alignment, ld%4).
bool tc_eligible(const Problem &P);
// Several dependent problems in ONE persistent launch (tcgen05 path, CTA
// pairs): phase p's tiles wait for the phases in dep_full (complete) and
// dep_slab (complete on the same slab: n-tile, or m-tile when slab_m).
// Dependencies must point to earlier phases.  Returns 0, -1 (not fusable /
// CUDA error: the caller falls back to one launch per phase) or -4.
struct FusedPhase {
  Problem P;
  int32_t dep_full, dep_slab, slab_m;
};
constexpr int MAX_FUSED_PHASES = 24;
int launch_tc_fused(const FusedPhase *phases, int nph, cudaStream_t s, int num_sms);

// O(N^2) helpers.
int launch_scale(float *C, int64_t ldc, int64_t m, int64_t n, float beta, int tri,
                 cudaStream_t s);                       // C <- beta*C (beta=0 -> 0), tri: 0/1 lower/2 upper
int launch_copy(float *dst, int64_t ldd, const float *src, int64_t lds, int64_t m, int64_t n,
                cudaStream_t s);
// GM_map (paper Adaptor rule 2): dst (rows x cols, column-major) <- op(src)
enum MatMode : int { MAT_TRANS = 0, MAT_SYM = 1, MAT_TRI = 2 };
int launch_materialize(float *dst, int64_t ldd, const float *src, int64_t lds, int64_t rows,
                       int64_t cols, int mode, int lower, int trans, int unit, cudaStream_t s);

// stream-ordered release write *flag = value (blas3_signal)
int launch_signal(uint32_t *flag, uint32_t value, cudaStream_t s);

// 2-D fp32 TMA map (dim0 contiguous, extent d0; dim1 stride ld floats), box
// box0 x box1, MN-major (mn32) or K-major staging swizzle.
bool tma_map_f32(CUtensorMap *m, const float *ptr, int64_t d0, int64_t d1, int64_t ld, uint32_t box0,
                 uint32_t box1, bool mn32);

// STRSM diagonal-panel solve (panel_kernel.cu).  The R x R panel (R a
// multiple of 256, at most 8192) in 256-row blocks, processing order forward
// (block i at rows 256 i) or backward; M (R x R, column-major, ldm) holds
// alpha * inv(op(A)_bb) on its diagonal blocks and the precomputed couplings
// -inv(op(A)_ss) op(A)_sf (left: M(s,f)) / -op(A)_fs inv(op(A)_ss) (right:
// M(f,s)) of every block s to the blocks f solved before it.  X is the panel
// of B, solved in place: left X(k,n) = X[k + n ldx] (nrhs columns), right
// X[n + k ldx] (nrhs rows).  One team of two CTA pairs per 256 right-hand
// sides; ws: trsm_panel_ws_bytes(nrhs, num_sms) bytes of device workspace
// (16-B aligned; the partials of the teams and their counters).
size_t trsm_panel_ws_bytes(int64_t nrhs, int num_sms);
int launch_trsm_panel(const float *M, int64_t ldm, float *X, int64_t ldx, bool right, int64_t R,
                      int64_t nrhs, bool forward, int kc, void *ws, cudaStream_t s, int num_sms);
// M's diagonal blocks from the lower-form inverses of the panel-inverse
// workspace (Dp: the panel's ldD x ldD inverse, its 256-blocks complete).
int launch_trsm_panel_diag(const float *Dp, int64_t ldD, float *M, int64_t ldm, int64_t R, bool lower_op,
                           float alpha, cudaStream_t s);

// TRSM diagonal blocks: for every 128 x 128 diagonal block b of L, where L
// is the stored triangle of A brought to lower form (L(i,j) = A(i,j) if A is
// stored lower, A(j,i) if stored upper; unit -> L(i,i) = 1), writes inv(L_bb)
// (lower) into the panel-inverse workspace: panel p = b / (panel/128) is an
// ldD x ldD column-major block at Dinv + p*ldD*ldD, block b sits on its
// diagonal.  The last block may be ragged (zero-padded).
int launch_trsm_diag_inv(const float *A, int64_t lda, int64_t n, int stored_lower, int unit,
                         float *Dinv, int64_t ldD, cudaStream_t s);

// Level 0 of that doubling (128 -> 256) on CUDA cores, one launch: for every
// 256-row pair of L, X21 = -inv(L22) L21 inv(L11) beside the 128-block inverses
// (launch_trsm_diag_inv first).  ldD a multiple of 256.
int launch_trsm_level0(const float *A, int64_t lda, int64_t n, int stored_lower, float *Dinv, int64_t ldD,
                       cudaStream_t s);

}  // namespace blas3
