/*
 * blas3.h -- C ABI of the B200-native (sm_100a) single-precision Level-3 BLAS
 * derived from one tuned GEMM, after Cui, Wang, Xue, Yang, Feng, "Automatic
 * Library Generation for BLAS3 on GPUs", IPDPS 2011
 * (/root/reference/PAPER.md, cited P:<line>).
 *
 * The paper generates GEMM, SYMM, TRMM and TRSM variants from the GEMM-NN
 * optimisation scheme (Fig. 3) by adaptors for Transpose,
 * Symmetry, Triangular and Solver structure and states that
 * matrices are column-major "to be consistent with BLAS3".
 * The argument conventions below are therefore the reference-BLAS ones.
 *
 * Common rules for every entry point
 * ----------------------------------
 *  Layout     All matrices are fp32, column-major: X(i,j) = X[i + j*ldx].
 *  Memory     A, B, C are DEVICE pointers (e.g. torch.Tensor.data_ptr() of a
 *             tensor with strides (1, ld)) on the current CUDA device.
 *             alpha/beta are host floats.  The caller owns every buffer; the
 *             library keeps only caches (tensor-map descriptors) and uses
 *             stream-ordered scratch (cudaMallocAsync) where a routine needs
 *             it (STRMM, STRSM).
 *  Streams    Work is enqueued on `stream` (NULL = legacy default stream) and
 *             is asynchronous: no entry point synchronises the host.  Calls
 *             can be captured into a CUDA graph (stream capture) and
 *             replayed; the first call on a given stream allocates that
 *             stream's library state (tile-scheduler and split-tail
 *             buffers), so make one eager call on the capture stream first.
 *  Aliasing   C must not alias A or B (as in BLAS); B is overwritten in place
 *             by STRMM/STRSM.
 *  Sizes      int64_t (N = 32768 needs byte offsets beyond 2^32); otherwise
 *             identical to the BLAS INTEGER arguments.
 *  Characters case-insensitive; trans 'C' == 'T' for real data.
 *  Return     0 on success.
 *             > 0 : 1-based position of the first invalid argument in
 *                   reference-BLAS XERBLA order, checked before anything is
 *                   launched; nothing is modified.  (A NULL matrix pointer
 *                   that would be referenced is reported by its position.)
 *             < 0 : runtime failure: BLAS3_ERR_CUDA (a CUDA launch/runtime
 *                   error), BLAS3_ERR_ARCH (current device is not sm_100),
 *                   BLAS3_ERR_ALLOC (scratch allocation failed),
 *                   BLAS3_ERR_TMA (tensor-map encoding failed),
 *                   BLAS3_ERR_UNSUPPORTED (a configuration the entry point
 *                   does not cover, e.g. a streamed operand in SIMT mode).
 *             The ABI never aborts and never throws.
 *  Special    beta == 0: C is not read (NaN/Inf in C do not propagate).
 *  values     alpha == 0: A and B are not read (C <- beta*C; B <- 0 for
 *             STRMM/STRSM).  Entries outside the referenced triangle of a
 *             symmetric/triangular A, and its diagonal when diag = 'U', are
 *             never read (readings Q7, Q8, Q11, Q12).
 *  Math       BLAS3_MATH_3XTF32 (default): tcgen05 tensor cores with a
 *             3xTF32 split (hi*hi + hi*lo + lo*hi) and fp32 accumulation in
 *             TMEM.  BLAS3_MATH_SIMT_FP32: exact-fp32 FFMA kernels.
 *             BLAS3_MATH_TF32_BF16X: opt-in: hi*hi as one TF32 UMMA and
 *             the two cross terms lo*hi + hi*lo packed into ONE BF16 UMMA (K = 16,
 *             hi and lo rounded to bf16): 2 UMMAs per k-step instead of 3,
 *             output-relative error ~1e-6 above the 3XTF32 split (DESIGN Q28).
 *             BLAS3_MATH_1XTF32: opt-in fast mode, one TF32 pass
 *             (inputs truncated to TF32, 10-bit mantissa; normwise error
 *             ~1e-3, NOT the fp32 accuracy of the other two modes).
 *             Arguments that violate TMA's 16-byte rules (pointer not
 *             16-byte aligned or ld % 4 != 0) run on the SIMT kernels in
 *             either mode.
 */
#ifndef BLAS3_B200_H
#define BLAS3_B200_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st *blas3_stream_t; /* identical to cudaStream_t */

enum {
    BLAS3_OK = 0,
    BLAS3_ERR_CUDA = -1,
    BLAS3_ERR_ARCH = -2,
    BLAS3_ERR_ALLOC = -3,
    BLAS3_ERR_TMA = -4,
    BLAS3_ERR_UNSUPPORTED = -5
};

enum { BLAS3_MATH_3XTF32 = 0, BLAS3_MATH_SIMT_FP32 = 1, BLAS3_MATH_1XTF32 = 2, BLAS3_MATH_TF32_BF16X = 3 };

/* SGEMM: C <- alpha*op(A)*op(B) + beta*C, op(X) = X or X^T.
 * op(A) is m x k, op(B) is k x n, C is m x n.  Paper: GEMM-NN/-TN loop nests
 * (P:77), Adaptor_Transpose.
 * XERBLA: 1 transa, 2 transb, 3 m<0, 4 n<0, 5 k<0,
 *         8 lda < max(1, transa=N ? m : k), 10 ldb < max(1, transb=N ? k : n),
 *         13 ldc < max(1, m). */
int blas3_sgemm(char transa, char transb, int64_t m, int64_t n, int64_t k,
                float alpha, const float *A, int64_t lda, const float *B, int64_t ldb,
                float beta, float *C, int64_t ldc, blas3_stream_t stream);

/* SGEMM with A STREAMED in column panels (transa = 'N'; multi-GPU row F1,
 * the device-side consumption of a panel-pipelined broadcast, P:382 future
 * work).  Same arithmetic and result as blas3_sgemm (bit for bit at the same
 * SM count: one kernel, k-blocks in the same order) -- but it may start before all
 * of A has arrived: A's columns come in panels of `panel_k` columns (a
 * multiple of 32), and panel p (columns [p*panel_k, (p+1)*panel_k)) is read
 * only once panel_ready[p] >= ready_value.  Another stream or device agent
 * (e.g. an NCCL broadcast of the panel followed by blas3_signal on that
 * stream) writes the flags; the kernel polls them with gpu-scope acquires and
 * orders its TMA reads after them.  The flags are caller-owned device memory
 * (ceil(k / panel_k) uint32), never reset by the library: give every call a
 * larger ready_value.  A panel that never arrives traps the kernel after 4 s
 * (a broken pipeline fails loudly instead of hanging).
 * XERBLA: as blas3_sgemm, plus 1 transa != 'N', 14 panel_ready NULL, 15 panel_k
 * not a positive multiple of 32.  BLAS3_ERR_UNSUPPORTED in SIMT mode or when A
 * / B are not TMA-addressable (16-B aligned, ld % 4 == 0). */
int blas3_sgemm_streamed(char transa, char transb, int64_t m, int64_t n, int64_t k,
                         float alpha, const float *A, int64_t lda, const float *B, int64_t ldb,
                         float beta, float *C, int64_t ldc, const uint32_t *panel_ready,
                         int64_t panel_k, uint32_t ready_value, blas3_stream_t stream);

/* Stream-ordered release write: *flag = value once every earlier operation on
 * `stream` has completed (a one-thread kernel: fence, then st.release.gpu).
 * The producer side of blas3_sgemm_streamed's panel flags.  Returns 0 or
 * BLAS3_ERR_CUDA. */
int blas3_signal(uint32_t *flag, uint32_t value, blas3_stream_t stream);

/* SSYMM: side=L: C <- alpha*A*B + beta*C (A m x m);
 *        side=R: C <- alpha*B*A + beta*C (A n x n).
 * A symmetric; only its `uplo` triangle ("real area") is read, the "shadow
 * area" is derived from it (Adaptor_Symmetry).  C, B are m x n.
 * XERBLA: 1 side, 2 uplo, 3 m<0, 4 n<0, 7 lda < max(1, side=L ? m : n),
 *         9 ldb < max(1, m), 12 ldc < max(1, m). */
int blas3_ssymm(char side, char uplo, int64_t m, int64_t n, float alpha,
                const float *A, int64_t lda, const float *B, int64_t ldb,
                float beta, float *C, int64_t ldc, blas3_stream_t stream);

/* SSYRK: trans=N: C <- alpha*A*A^T + beta*C (A n x k);
 *        trans=T: C <- alpha*A^T*A + beta*C (A k x n).
 * Only the `uplo` triangle of the n x n C is read and written; the other
 * triangle is left bit-identical.  (Not evaluated in the paper; required by
 * BASELINE.json's north star.)
 * XERBLA: 1 uplo, 2 trans, 3 n<0, 4 k<0, 7 lda < max(1, trans=N ? n : k),
 *         10 ldc < max(1, n). */
int blas3_ssyrk(char uplo, char trans, int64_t n, int64_t k, float alpha,
                const float *A, int64_t lda, float beta, float *C, int64_t ldc,
                blas3_stream_t stream);

/* SSYR2K: trans=N: C <- alpha*(A*B^T + B*A^T) + beta*C (A, B n x k);
 *         trans=T: C <- alpha*(A^T*B + B^T*A) + beta*C (A, B k x n).
 * Only the `uplo` triangle of C is read and written.
 * XERBLA: 1 uplo, 2 trans, 3 n<0, 4 k<0, 7 lda < max(1, trans=N ? n : k),
 *         9 ldb < max(1, trans=N ? n : k), 12 ldc < max(1, n). */
int blas3_ssyr2k(char uplo, char trans, int64_t n, int64_t k, float alpha,
                 const float *A, int64_t lda, const float *B, int64_t ldb,
                 float beta, float *C, int64_t ldc, blas3_stream_t stream);

/* STRMM: side=L: B <- alpha*op(A)*B (A m x m); side=R: B <- alpha*B*op(A)
 * (A n x n).  A triangular (`uplo`), unit diagonal when diag='U'; the blank
 * triangle is never read (Adaptor_Triangular; TRMM-LL-N P:395-398).
 * B (m x n) is overwritten in place without clobbering rows still to be read.
 * XERBLA: 1 side, 2 uplo, 3 transa, 4 diag, 5 m<0, 6 n<0,
 *         9 lda < max(1, side=L ? m : n), 11 ldb < max(1, m). */
int blas3_strmm(char side, char uplo, char transa, char diag, int64_t m, int64_t n,
                float alpha, const float *A, int64_t lda, float *B, int64_t ldb,
                blas3_stream_t stream);

/* STRSM: side=L: solve op(A)*X = alpha*B; side=R: solve X*op(A) = alpha*B.
 * X overwrites B (m x n).  Blocked: diagonal blocks inverted with warp-level
 * primitives, then block sweep with tensor-core GEMM updates (Adaptor_Solver,
 * P:225-244, TRSM-LL-N P:397-398).  A must be non-singular (diag='N'); no
 * pivoting or singularity check, as in BLAS.
 * XERBLA: as STRMM. */
int blas3_strsm(char side, char uplo, char transa, char diag, int64_t m, int64_t n,
                float alpha, const float *A, int64_t lda, float *B, int64_t ldb,
                blas3_stream_t stream);

/* ---- fp64 family (the paper is fp32-only).
 * blas3_d{gemm,symm,syrk,syr2k,trmm,trsm}: the same semantics, argument
 * lists, XERBLA codes, quick returns, alpha/beta special cases, ownership
 * and stream rules as the s-routines above, on column-major fp64 matrices in
 * device memory with host double scalars.  Arithmetic: fp64 products and sums
 * throughout (one structured fp64 GEMM kernel, d_kernel.cu, on DMMA m8n8k4
 * fragments; B200's DMMA and DFMA share one 37 TF/s roofline, DMMA needs 8x
 * fewer instructions); symmetric operands are mirrored and triangular ones zero-filled
 * while staged to shared memory, as in the fp32 kernels.  DTRMM uses
 * stream-ordered scratch of m*n doubles.  DTRSM scales B by alpha, then
 * solves by recursive halving (diagonal blocks of 64 by substitution, GEMM
 * updates).  Not affected by the math mode or the tuning options. */
int blas3_dgemm(char transa, char transb, int64_t m, int64_t n, int64_t k,
                double alpha, const double *A, int64_t lda, const double *B, int64_t ldb,
                double beta, double *C, int64_t ldc, blas3_stream_t stream);
int blas3_dsymm(char side, char uplo, int64_t m, int64_t n, double alpha,
                const double *A, int64_t lda, const double *B, int64_t ldb,
                double beta, double *C, int64_t ldc, blas3_stream_t stream);
int blas3_dsyrk(char uplo, char trans, int64_t n, int64_t k, double alpha,
                const double *A, int64_t lda, double beta, double *C, int64_t ldc,
                blas3_stream_t stream);
int blas3_dsyr2k(char uplo, char trans, int64_t n, int64_t k, double alpha,
                 const double *A, int64_t lda, const double *B, int64_t ldb,
                 double beta, double *C, int64_t ldc, blas3_stream_t stream);
int blas3_dtrmm(char side, char uplo, char transa, char diag, int64_t m, int64_t n,
                double alpha, const double *A, int64_t lda, double *B, int64_t ldb,
                blas3_stream_t stream);
int blas3_dtrsm(char side, char uplo, char transa, char diag, int64_t m, int64_t n,
                double alpha, const double *A, int64_t lda, double *B, int64_t ldb,
                blas3_stream_t stream);

/* Process-wide math mode (BLAS3_MATH_3XTF32 default; the environment
 * variable BLAS3_MATH=simt|3xtf32|1xtf32|bf16x overrides the default at load).
 * Returns 0, or 1 if `mode` is not a valid mode (nothing changed). */
int blas3_set_math_mode(int mode);
int blas3_get_math_mode(void);

/* Tuning options: the variant choice of the paper's generator (its search
 * over optimisation schemes) as process-wide
 * integer knobs read by every later call.  Every value selects among
 * implementations that compute the same result (each is parity-tested).
 * Each option starts from its environment variable (named in brackets, read
 * once at the first call) or its default.
 *   BLAS3_OPT_GM_MAP       [BLAS3_GM_MAP]   GM_map adaptor: rewrite a
 *                          transposed / symmetric / triangular operand in global
 *                          memory first.  -1 auto (default: per-routine size
 *                          thresholds below), 0 never, 1 always
 *   BLAS3_OPT_GM_MIN_GEMM  SGEMM transa!='N': auto threshold on n (default 1<<30 = off)
 *   BLAS3_OPT_GM_MIN_SYMM  SSYMM: auto threshold on the non-symmetric extent (1<<30 = off:
 *                          sym(A) is merged while staging, the paper's rule 3, P:144-158;
 *                          within 1-5% of GM_map at N >= 4096, faster for side=L at 2048)
 *   BLAS3_OPT_GM_MIN_TRMM  STRMM: auto threshold on the right-hand-side extent (1<<30)
 *   BLAS3_OPT_GM_MIN_TRSM  STRSM transa!='N': auto threshold on the RHS extent (1<<30)
 *                          (auto also requires the structured order >= 2048)
 *   BLAS3_OPT_TC_CTA       [BLAS3_TC_CTA]   0 auto (default), 1 single-CTA 128x256
 *                          tiles, 2 CTA-pair 256x256 tiles (cta_group::2)
 *   BLAS3_OPT_TC_SPLIT     [BLAS3_TC_SPLIT] 1 split the tail wave along K (default), 0 off
 *   BLAS3_OPT_TC_STATIC    [BLAS3_TC_STATIC] 0 dynamic tile scheduler (default), 1 static
 *   BLAS3_OPT_PDL          [BLAS3_PDL]      1 programmatic dependent launch (default), 0 off
 *   BLAS3_OPT_TRSM_NB      [BLAS3_TRSM_NB]  STRSM panel width: power of 2 in [128, 8192] (2048)
 *   BLAS3_OPT_TRSM_SLABS   [BLAS3_TRSM_SLABS] right-hand-side slabs on own streams, 1..4 (2)
 *   BLAS3_OPT_TRSM_SLAB_MIN [BLAS3_TRSM_SLAB_MIN] minimum slab width, >= 256 (16384:
 *                          one slab up to 32767 right-hand sides -- measured 5.6%
 *                          faster than two at 8192, profiles/r02_trsm_options.md)
 *   BLAS3_OPT_TRSM_RESERVE [BLAS3_TRSM_RESERVE] SMs the first panel's sweep leaves to
 *                          the panel-inverse doubling chain, 0..74, or -1 (default,
 *                          auto: 48 from order 8192, 16 below)
 *   BLAS3_OPT_TRSM_GEO_LEAF [BLAS3_TRSM_GEO_LEAF] the first panel is halved down to
 *                          this width: power of 2 in [128, 8192] (256)
 *   BLAS3_OPT_TRSM_FUSED   [BLAS3_TRSM_FUSED] 1: the whole STRSM (panel-inverse
 *                          doubling + sweep) as one persistent dependency-driven
 *                          launch when it fits; 2: when the diagonal-panel solver
 *                          took the first panel, the sweep over the other panels
 *                          (with their last doubling level) as one such launch;
 *                          0 (default): one launch per step on the caller's and
 *                          the side streams
 *   BLAS3_OPT_TRSM_FIRST_YM [BLAS3_TRSM_FIRST_YM] 1 (default): the first panel's
 *                          blocks are solved as X_s = Y_s - M X_f with Y, M
 *                          precomputed off the critical path; 0: update + solve
 *   BLAS3_OPT_TRSM_FIRST_FUSED [BLAS3_TRSM_FIRST_FUSED] 1 (default): the first
 *                          panel (its doubling, Y, M and the X chain) as ONE
 *                          persistent dependency-driven launch; 0: separate
 *                          launches on side streams
 *   BLAS3_OPT_TRSM_FIRST_SPLIT [BLAS3_TRSM_FIRST_SPLIT] F (power of 2): only
 *                          the first F rows (L) / columns (R) of the first
 *                          panel (processing order) run as the fused chain;
 *                          the rest of the panel is swept right-looking in
 *                          blocks of F, F, 2F, 4F, ...: the block solved last
 *                          updates EVERY later row of the matrix in one bulk
 *                          GEMM, then the next block is one leaf solve (its
 *                          inverse doubled up front on a side stream).
 *                          0 (default): the whole first panel in the chain
 *   BLAS3_OPT_TRSM_FIRST_ALL [BLAS3_TRSM_FIRST_ALL] 1: every panel's inverse
 *                          doubling runs inside the first panel's fused
 *                          launch (the levels its chain needs first, the
 *                          rest after the chain) on all SMs; 0 (default): the
 *                          other panels' doubling on a side stream beside it
 *   BLAS3_OPT_TC_RASTER    [BLAS3_TC_RASTER] tile rows per group of the grouped
 *                          raster order of full grids (L2 reuse), 0..64; 0 =
 *                          the built-in default (8)
 *   BLAS3_OPT_TC_KC        [BLAS3_TC_KC]    tcgen05 path: k-blocks (32 deep) summed in
 *                          one TMEM partial before it is folded into the
 *                          round-to-nearest register sum (Q24): 1..64,
 *                          default 3 (K = 96).  The tensor core's accumulator
 *                          truncates on every UMMA add (~4e-8 relative per add,
 *                          coherent on same-sign data); each k-block issues its
 *                          8 cross-term UMMAs before its 4 hi*hi ones, so a
 *                          partial of c blocks takes 12c - 8 full-size adds.
 *                          Measured (SGEMM, K = 8192): e_rel 7.9e-7 on U(-1,1),
 *                          1.66e-6 on U(0,1) at 3; 3.8e-6 / 9.9e-6 at 16.  Each
 *                          drain stalls the tensor pipe briefly: SGEMM N = 8192
 *                          at 2 / 3 / 4 / 16 = 89 / 98 / 98 / 100 %
 *   BLAS3_OPT_TC_VEC_STORE [BLAS3_TC_VEC_STORE] tcgen05 epilogue: 1 (default) C is
 *                          read and written with 16-B vector accesses (each
 *                          warp's rows transposed through a 1 KiB shared box:
 *                          a thread holds 4 consecutive rows of one column),
 *                          when C is 16-B aligned with ldc % 4 == 0; 0 per-thread
 *                          coalesced 4-B accesses
 *   BLAS3_OPT_MAX_SMS      [BLAS3_MAX_SMS]  launch at most this many SMs' worth of CTAs
 *                          (0 = all, default): leaves SMs to concurrent kernels,
 *                          e.g. NCCL broadcasts overlapped with the products
 *                          (paper_conf_ipps_cuiwxyf11_b200.dist)
 *   BLAS3_OPT_TC_C_PREFETCH [BLAS3_TC_C_PREFETCH] tcgen05 epilogue, beta != 0: 1
 *                          (default) each CTA's C tile is prefetched into L2
 *                          (one TMA prefetch) a few TMEM chunks before it is
 *                          read, so the store phase does not wait on HBM; 0 off
 *   BLAS3_OPT_TC_C_ASYNC   [BLAS3_TC_C_ASYNC] tcgen05 epilogue, beta != 0 with 16-B vector
 *                          access: 1 C goes to shared memory by cp.async two 8-column
 *                          groups ahead of its use; 0 (default) one group ahead in
 *                          registers (measured within noise of each other: SGEMM
 *                          +2%, tall-skinny SSYRK -2%)
 *   BLAS3_OPT_TRSM_PANEL   [BLAS3_TRSM_PANEL] 1 (default): STRSM's first processed
 *                          panel by the diagonal-panel solver -- one CTA pair per
 *                          128 right-hand sides forward-substitutes the whole
 *                          panel (256-row blocks, precomputed couplings
 *                          -inv(op(A)_ss) op(A)_sf), no grid-wide dependency
 *                          steps; 0: the fused doubling + geometric chain; 2: the
 *                          same as 1 (kept for scripts).  Used when the panel's
 *                          order is a multiple of 256 and B is 16-B aligned with
 *                          ldb % 4 == 0
 *   BLAS3_OPT_TRSM_PANEL2  [BLAS3_TRSM_PANEL2] with the first panel by the solver:
 *                          1 the SECOND processed panel by the solver as well (its
 *                          256-block inverses and couplings built on a side stream
 *                          beside the first panel; the update before it in place),
 *                          so no inverse doubling of that panel sits between the
 *                          first update and its solve; 0 (default): the leaf (panel
 *                          inverse by doubling) as for the later panels (measured
 *                          within 1% of each other at N = 8192, 18% slower at 4096)
 * blas3_set_option returns 0, or 1 for an unknown key or an invalid value
 * (nothing changed).  blas3_get_option returns the current value, or
 * INT64_MIN for an unknown key. */
enum {
    BLAS3_OPT_GM_MAP = 0, BLAS3_OPT_GM_MIN_GEMM = 1, BLAS3_OPT_GM_MIN_SYMM = 2,
    BLAS3_OPT_GM_MIN_TRMM = 3, BLAS3_OPT_GM_MIN_TRSM = 4, BLAS3_OPT_TC_CTA = 5,
    BLAS3_OPT_TC_SPLIT = 6, BLAS3_OPT_TC_STATIC = 7, BLAS3_OPT_PDL = 8,
    BLAS3_OPT_TRSM_NB = 9, BLAS3_OPT_TRSM_SLABS = 10, BLAS3_OPT_TRSM_SLAB_MIN = 11,
    BLAS3_OPT_TRSM_RESERVE = 12, BLAS3_OPT_TRSM_GEO_LEAF = 13, BLAS3_OPT_TRSM_FUSED = 14,
    BLAS3_OPT_TRSM_FIRST_YM = 15, BLAS3_OPT_TRSM_FIRST_FUSED = 16, BLAS3_OPT_TRSM_FIRST_SPLIT = 17,
    BLAS3_OPT_TRSM_FIRST_ALL = 18, BLAS3_OPT_TC_RASTER = 19, BLAS3_OPT_TC_KC = 20,
    BLAS3_OPT_TC_VEC_STORE = 21, BLAS3_OPT_MAX_SMS = 22, BLAS3_OPT_TC_C_PREFETCH = 23,
    BLAS3_OPT_TC_C_ASYNC = 24, BLAS3_OPT_TRSM_PANEL = 25, BLAS3_OPT_TRSM_PANEL2 = 26,
    BLAS3_OPT_COUNT = 27
};
int blas3_set_option(int key, int64_t value);
int64_t blas3_get_option(int key);

/* Optional caller-owned device scratch used before falling back to
 * cudaMallocAsync.  The buffer must stay valid while calls that may use it
 * are in flight, and it is process-wide: calls that use it must not run
 * concurrently on different streams (as with one cuBLAS workspace); without
 * it every call takes its own stream-ordered scratch, and calls on different
 * streams / host threads are independent.  (ptr=NULL, bytes=0 removes it.)
 * Returns 0. */
int blas3_set_workspace(void *dptr, size_t bytes);

/* Number of kernels the library launched since load (host-side counter;
 * the bench uses it to report gpu_launches). */
int64_t blas3_launch_count(void);

/* Same counter split by route: BLAS3_PATH_TCGEN05 (tcgen05 tensor-core
 * structured GEMM, any tensor math mode), BLAS3_PATH_SIMT (FP32 SIMT structured GEMM),
 * BLAS3_PATH_AUX (scale / copy / TRSM diagonal-inverse kernels),
 * BLAS3_PATH_TRSM_PANEL (the STRSM diagonal-panel solver, tcgen05).  Returns -1
 * for an unknown path.  Lets tests assert which route a call took. */
enum { BLAS3_PATH_TCGEN05 = 0, BLAS3_PATH_SIMT = 1, BLAS3_PATH_AUX = 2, BLAS3_PATH_TRSM_PANEL = 3 };
int64_t blas3_launch_count_by_path(int path);

/* Static string for a return code. */
const char *blas3_error_string(int code);

/* ABI version (major*100 + minor). */
int blas3_version(void);

#ifdef __cplusplus
}
#endif
#endif /* BLAS3_B200_H */
