// abi.cu -- the extern "C" boundary (include/blas3.h) and the routine
// drivers: argument validation in XERBLA order, quick returns and alpha/beta
// special cases (row A1), canonicalisation of every variant into one
// structured-GEMM Problem (row A2), the in-place STRMM (row A9) and the
// blocked STRSM sweep (rows A7/A8).
#include <cuda_runtime.h>
#include <ctype.h>
#include <stdlib.h>
#include <string.h>
#include <atomic>
#include <functional>
#include <mutex>
#include <vector>

#include "../../include/blas3.h"
#include "kernels.h"
#include "validate.h"

namespace blas3 {

static std::atomic<int64_t> g_launches{0};
static std::atomic<int64_t> g_path_launches[4];
void note_launch(int path) {
  g_launches.fetch_add(1, std::memory_order_relaxed);
  if (path >= 0 && path < 4) g_path_launches[path].fetch_add(1, std::memory_order_relaxed);
}

// ---- tuning options (include/blas3.h): defaults, environment names, ranges
struct OptSpec { const char *env; int64_t def, lo, hi; bool pow2; };
static const OptSpec kOpt[BLAS3_OPT_COUNT] = {
    {"BLAS3_GM_MAP", -1, -1, 1, false},
    {"BLAS3_GM_MIN_GEMM", int64_t(1) << 30, 0, int64_t(1) << 40, false},
    {"BLAS3_GM_MIN_SYMM", int64_t(1) << 30, 0, int64_t(1) << 40, false},
    {"BLAS3_GM_MIN_TRMM", int64_t(1) << 30, 0, int64_t(1) << 40, false},
    {"BLAS3_GM_MIN_TRSM", int64_t(1) << 30, 0, int64_t(1) << 40, false},
    {"BLAS3_TC_CTA", 0, 0, 2, false},
    {"BLAS3_TC_SPLIT", 1, 0, 1, false},
    {"BLAS3_TC_STATIC", 0, 0, 1, false},
    {"BLAS3_PDL", 1, 0, 1, false},
    {"BLAS3_TRSM_NB", 2048, 128, 8192, true},
    {"BLAS3_TRSM_SLABS", 2, 1, 4, false},
    {"BLAS3_TRSM_SLAB_MIN", 16384, 256, int64_t(1) << 40, false},
    {"BLAS3_TRSM_RESERVE", -1, -1, 74, false},
    {"BLAS3_TRSM_GEO_LEAF", 256, 128, 8192, true},
    {"BLAS3_TRSM_FUSED", 0, 0, 2, false},
    {"BLAS3_TRSM_FIRST_YM", 1, 0, 1, false},
    {"BLAS3_TRSM_FIRST_FUSED", 1, 0, 1, false},
    {"BLAS3_TRSM_FIRST_SPLIT", 0, 0, 8192, true},
    {"BLAS3_TRSM_FIRST_ALL", 0, 0, 1, false},
    {"BLAS3_TC_RASTER", 0, 0, 64, false},
    {"BLAS3_TC_KC", 3, 1, 64, false},
    {"BLAS3_TC_VEC_STORE", 1, 0, 1, false},
    {"BLAS3_MAX_SMS", 0, 0, 4096, false},
    {"BLAS3_TC_C_PREFETCH", 1, 0, 1, false},
    {"BLAS3_TC_C_ASYNC", 0, 0, 1, false},
    {"BLAS3_TRSM_PANEL", 1, 0, 2, false},
    {"BLAS3_TRSM_PANEL2", 0, 0, 2, false},
};
static std::atomic<int64_t> g_opt[BLAS3_OPT_COUNT];
static std::once_flag g_opt_once;
static bool opt_valid(int key, int64_t v) {
  const OptSpec &o = kOpt[key];
  if (v < o.lo || v > o.hi) return false;
  if (o.pow2 && (v & (v - 1))) return false;
  return true;
}
static void opt_init() {
  std::call_once(g_opt_once, [] {
    for (int k = 0; k < BLAS3_OPT_COUNT; ++k) {
      int64_t v = kOpt[k].def;
      const char *e = getenv(kOpt[k].env);
      if (e && *e) {
        const int64_t x = atoll(e);
        if (opt_valid(k, x)) v = x;
      }
      g_opt[k].store(v);
    }
  });
}
static std::atomic<int> g_math{-1};   // -1: not initialised
static void *g_ws = nullptr;
static size_t g_ws_bytes = 0;

static int global_math_mode() {
  int m = g_math.load(std::memory_order_acquire);
  if (m < 0) {
    const char *e = getenv("BLAS3_MATH");
    const int env = (e && (e[0] == 's' || e[0] == 'S')) ? BLAS3_MATH_SIMT_FP32
                    : (e && e[0] == '1') ? BLAS3_MATH_1XTF32
                    : (e && (e[0] == 'b' || e[0] == 'B')) ? BLAS3_MATH_TF32_BF16X : BLAS3_MATH_3XTF32;
    int expect = -1;
    g_math.compare_exchange_strong(expect, env);
    m = g_math.load(std::memory_order_acquire);
  }
  return m;
}

// Per-call snapshot of the process-wide options and math mode: every entry
// point takes one (CallOpts) before it reads any, so a blas3_set_option /
// blas3_set_math_mode from another thread mid-call can never give one call
// two different panel widths, tile shapes or modes.
struct OptSnap { int64_t v[BLAS3_OPT_COUNT]; int math; };
static thread_local const OptSnap *t_snap = nullptr;
struct CallOpts {
  OptSnap snap;
  const OptSnap *prev;
  CallOpts() : prev(t_snap) {
    opt_init();
    for (int k = 0; k < BLAS3_OPT_COUNT; ++k) snap.v[k] = g_opt[k].load(std::memory_order_relaxed);
    snap.math = global_math_mode();
    t_snap = &snap;
  }
  ~CallOpts() { t_snap = prev; }
};
int64_t opt(int key) {
  if (key < 0 || key >= BLAS3_OPT_COUNT) return 0;
  if (t_snap) return t_snap->v[key];
  opt_init();
  return g_opt[key].load(std::memory_order_relaxed);
}
static int math_mode() { return t_snap ? t_snap->math : global_math_mode(); }
static bool tensor_mode() { return math_mode() != BLAS3_MATH_SIMT_FP32; }

// per-device facts: SM count, sm_100 check
struct DevInfo { int sms = 0; int ok = -1; };
static DevInfo g_dev[64];
static std::mutex g_dev_mu;

static int device_check(int &sms) {
  int d = 0;
  if (cudaGetDevice(&d) != cudaSuccess || d < 0 || d >= 64) return BLAS3_ERR_CUDA;
  std::lock_guard<std::mutex> lk(g_dev_mu);
  DevInfo &di = g_dev[d];
  if (di.ok < 0) {
    cudaDeviceProp p;
    if (cudaGetDeviceProperties(&p, d) != cudaSuccess) return BLAS3_ERR_CUDA;
    di.ok = (p.major == 10 && p.minor == 0) ? 1 : 0;
    di.sms = p.multiProcessorCount;
    // keep freed scratch cached in the pool (no host sync on reuse)
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, d) == cudaSuccess) {
      uint64_t thr = UINT64_MAX;
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
  }
  sms = di.sms;
  const int64_t cap = opt(BLAS3_OPT_MAX_SMS);          // SMs left to concurrent kernels
  if (cap >= 2 && cap < sms) sms = (int)cap;
  return di.ok ? 0 : BLAS3_ERR_ARCH;
}

int abi_device_check(int &sms) { return device_check(sms); }

// stream-ordered scratch: caller-provided workspace first, else the pool
struct Scratch {
  float *p = nullptr;
  bool owned = false;
  cudaStream_t s = nullptr;
  ~Scratch() { if (owned && p) cudaFreeAsync(p, s); }
};
static int get_scratch(Scratch &sc, size_t bytes, cudaStream_t s, size_t offset = 0) {
  sc.s = s;
  if (g_ws && offset + bytes <= g_ws_bytes) { sc.p = (float *)((char *)g_ws + offset); return 0; }
  if (cudaMallocAsync((void **)&sc.p, bytes, s) != cudaSuccess) { cudaGetLastError(); return BLAS3_ERR_ALLOC; }
  sc.owned = true;
  return 0;
}

static int run_problem(const Problem &P, cudaStream_t s, int sms) {
  if (P.M <= 0 || P.N <= 0) return 0;
  if (P.max_sms > 0 && P.max_sms < sms) sms = P.max_sms;
  if (tensor_mode() && tc_eligible(P)) {
    Problem Q = P;
    Q.passes = math_mode() == BLAS3_MATH_1XTF32 ? 1 : math_mode() == BLAS3_MATH_TF32_BF16X ? 2 : 3;
    return launch_tc(Q, s, sms);
  }
  int rc = launch_simt(P, s, sms);
  return rc ? BLAS3_ERR_CUDA : 0;
}

static OpDesc dense(const float *p, int64_t ld, bool kr) {
  OpDesc o; memset(&o, 0, sizeof(o));
  o.ptr = p; o.ld = ld; o.kind = OP_DENSE; o.kr = kr; o.map_rk = o.map_kr = -1;
  return o;
}
static OpDesc sym(const float *p, int64_t ld, bool lower) {
  OpDesc o = dense(p, ld, false); o.kind = OP_SYM; o.lower = lower; return o;
}
static OpDesc tri(const float *p, int64_t ld, bool lower, bool swap, bool unit) {
  OpDesc o = dense(p, ld, false); o.kind = OP_TRI; o.lower = lower; o.swap = swap; o.unit = unit;
  return o;
}
// a TRI operand in library workspace whose blank triangle holds zeros
static OpDesc tri_zeroed(const float *p, int64_t ld, bool lower, bool swap) {
  OpDesc o = tri(p, ld, lower, swap, false); o.zero_blank = 1; return o;
}
static Problem problem(int64_t M, int64_t N, float alpha, float beta, const float *Cin,
                       int64_t ldcin, float *Cout, int64_t ldcout) {
  Problem P; memset(&P, 0, sizeof(P));
  P.M = M; P.N = N; P.nseg = 1; P.alpha = alpha; P.beta = beta;
  P.Cin = Cin; P.ldcin = ldcin; P.Cout = Cout; P.ldcout = ldcout;
  P.nbatch = 1; P.per = 1;
  P.raster_gm = (int32_t)opt(BLAS3_OPT_TC_RASTER);
  P.kc = (int32_t)opt(BLAS3_OPT_TC_KC);
  P.c_vec = 0;
  P.c_pf_map = -1;
  P.a_ready = nullptr;
  return P;
}

// plain dense GEMM used by the TRSM sweep: C = alpha*Xa*Xb^T + beta*C
static int gemm_dense(int64_t M, int64_t N, int64_t K, float alpha, const float *a, int64_t lda,
                      bool a_kr, const float *b, int64_t ldb, bool b_kr, float beta, float *C,
                      int64_t ldc, cudaStream_t s, int sms) {
  if (M <= 0 || N <= 0) return 0;
  Problem P = problem(M, N, alpha, beta, C, ldc, C, ldc);
  P.seg[0].a = dense(a, lda, a_kr);
  P.seg[0].b = dense(b, ldb, b_kr);
  P.seg[0].K = K;
  return run_problem(P, s, sms);
}


static inline int finish(int rc) {
  if (rc) return rc;
  return cudaGetLastError() == cudaSuccess ? 0 : BLAS3_ERR_CUDA;
}

// GM_map policy (paper Adaptor rule 2): rewrite the
// structured / transposed operand once in global memory (O(n^2) traffic) when
// the O(n^2 * other) product is large enough to amortise it; the GEMM kernel
// then stages a plain MN-major operand.  `order` = order of the rewritten
// operand, `other` = the remaining product dimension.  Env BLAS3_GM_MAP:
// 0 = never, 1 = always (tests), unset = by size.
static bool use_gm_map(int64_t order, int64_t other, int min_key) {
  const int64_t e = opt(BLAS3_OPT_GM_MAP);
  if (e >= 0) return e == 1;
  return order >= 2048 && other >= opt(min_key);
}
static inline int64_t ld4(int64_t rows) { return (imax(rows, 1) + 3) / 4 * 4; }

}  // namespace blas3

using namespace blas3;

extern "C" {

int blas3_version(void) { return 100; }
int64_t blas3_launch_count(void) { return g_launches.load(); }
int64_t blas3_launch_count_by_path(int path) {
  return (path >= 0 && path < 4) ? g_path_launches[path].load() : -1;
}

int blas3_set_option(int key, int64_t value) {
  if (key < 0 || key >= BLAS3_OPT_COUNT) return 1;
  opt_init();
  if (!opt_valid(key, value)) return 1;
  g_opt[key].store(value);
  return 0;
}
int64_t blas3_get_option(int key) {
  if (key < 0 || key >= BLAS3_OPT_COUNT) return INT64_MIN;
  return opt(key);
}

int blas3_set_math_mode(int mode) {
  if (mode != BLAS3_MATH_3XTF32 && mode != BLAS3_MATH_SIMT_FP32 && mode != BLAS3_MATH_1XTF32 &&
      mode != BLAS3_MATH_TF32_BF16X) return 1;
  g_math.store(mode, std::memory_order_release);
  return 0;
}
int blas3_get_math_mode(void) { return global_math_mode(); }

int blas3_set_workspace(void *dptr, size_t bytes) {
  g_ws = bytes ? dptr : nullptr;
  g_ws_bytes = dptr ? bytes : 0;
  return 0;
}

const char *blas3_error_string(int code) {
  switch (code) {
    case BLAS3_OK: return "success";
    case BLAS3_ERR_CUDA: return "CUDA launch or runtime error";
    case BLAS3_ERR_ARCH: return "current device is not sm_100 (B200)";
    case BLAS3_ERR_ALLOC: return "scratch allocation failed";
    case BLAS3_ERR_TMA: return "TMA tensor-map encoding failed";
    case BLAS3_ERR_UNSUPPORTED: return "configuration not supported by this entry point";
    default: return code > 0 ? "invalid argument (value = 1-based XERBLA position)" : "unknown error";
  }
}

// ------------------------------------------------------------------- SGEMM
int blas3_sgemm(char transa, char transb, int64_t m, int64_t n, int64_t k, float alpha,
                const float *A, int64_t lda, const float *B, int64_t ldb, float beta, float *C,
                int64_t ldc, blas3_stream_t stream) {
  CallOpts call_opts;
  const bool ta = up(transa) != 'N', tb = up(transb) != 'N';
  if (const int v = v_gemm(transa, transb, m, n, k, lda, ldb, ldc)) return v;
  if (m == 0 || n == 0 || ((alpha == 0.f || k == 0) && beta == 1.f)) return 0;
  if (!C) return 12;
  const bool reads_ab = alpha != 0.f && k > 0;
  if (reads_ab && !A) return 7;
  if (reads_ab && !B) return 9;
  int sms, rc = device_check(sms);
  if (rc) return rc;
  cudaStream_t s = (cudaStream_t)stream;
  if (!reads_ab) return finish(launch_scale(C, ldc, m, n, beta, 0, s) ? BLAS3_ERR_CUDA : 0);
  Problem P = problem(m, n, alpha, beta, C, ldc, C, ldc);
  P.seg[0].a = dense(A, lda, ta);       // op(A)(r,k) = A(k,r) when transposed -> "kr"
  P.seg[0].b = dense(B, ldb, !tb);      // Xb(c,k) = op(B)(k,c)
  P.seg[0].K = k;
  Scratch Wm;
  if (ta && tensor_mode() && use_gm_map(imax(m, k), n, BLAS3_OPT_GM_MIN_GEMM)) {
    // GM_map: op(A) = A^T materialised m x k (the K-major A operand stages
    // slower than the MN-major one)
    const int64_t ldw = ld4(m);
    if ((rc = get_scratch(Wm, (size_t)ldw * k * sizeof(float), s))) return rc;
    if (launch_materialize(Wm.p, ldw, A, lda, m, k, MAT_TRANS, 0, 0, 0, s)) return BLAS3_ERR_CUDA;
    P.seg[0].a = dense(Wm.p, ldw, false);
  }
  return finish(run_problem(P, s, sms));
}

// ------------------------------------------------------------------- SGEMM, A streamed in panels
int blas3_sgemm_streamed(char transa, char transb, int64_t m, int64_t n, int64_t k, float alpha,
                         const float *A, int64_t lda, const float *B, int64_t ldb, float beta, float *C,
                         int64_t ldc, const uint32_t *panel_ready, int64_t panel_k, uint32_t ready_value,
                         blas3_stream_t stream) {
  CallOpts call_opts;
  const bool tb = up(transb) != 'N';
  if (up(transa) != 'N') return 1;             // A's panels are K-ranges of its columns
  if (!is_trans(transb)) return 2;
  if (m < 0) return 3;
  if (n < 0) return 4;
  if (k < 0) return 5;
  if (lda < mx1(m)) return 8;
  if (ldb < mx1(tb ? n : k)) return 10;
  if (ldc < mx1(m)) return 13;
  if (!panel_ready) return 14;
  if (panel_k <= 0 || panel_k % 32) return 15;
  if (m == 0 || n == 0 || ((alpha == 0.f || k == 0) && beta == 1.f)) return 0;
  if (!C) return 12;
  const bool reads_ab = alpha != 0.f && k > 0;
  if (reads_ab && !A) return 7;
  if (reads_ab && !B) return 9;
  int sms, rc = device_check(sms);
  if (rc) return rc;
  cudaStream_t s = (cudaStream_t)stream;
  if (!reads_ab) return finish(launch_scale(C, ldc, m, n, beta, 0, s) ? BLAS3_ERR_CUDA : 0);
  Problem P = problem(m, n, alpha, beta, C, ldc, C, ldc);
  P.seg[0].a = dense(A, lda, false);
  P.seg[0].b = dense(B, ldb, !tb);
  P.seg[0].K = k;
  P.a_ready = panel_ready;
  P.a_panel_kb = (int32_t)(panel_k / 32);
  P.a_ready_val = ready_value;
  // the panel wait lives in the tcgen05 producer (no host synchronisation anywhere)
  if (!tensor_mode() || !tc_eligible(P)) return BLAS3_ERR_UNSUPPORTED;
  return finish(run_problem(P, s, sms));
}

int blas3_signal(uint32_t *flag, uint32_t value, blas3_stream_t stream) {
  if (!flag) return 1;
  return finish(launch_signal(flag, value, (cudaStream_t)stream) ? BLAS3_ERR_CUDA : 0);
}

// ------------------------------------------------------------------- SSYMM
int blas3_ssymm(char side, char uplo, int64_t m, int64_t n, float alpha, const float *A,
                int64_t lda, const float *B, int64_t ldb, float beta, float *C, int64_t ldc,
                blas3_stream_t stream) {
  CallOpts call_opts;
  const bool left = up(side) == 'L', lower = up(uplo) == 'L';
  if (const int v = v_symm(side, uplo, m, n, lda, ldb, ldc)) return v;
  if (m == 0 || n == 0 || (alpha == 0.f && beta == 1.f)) return 0;
  if (!C) return 11;
  if (alpha != 0.f && !A) return 6;
  if (alpha != 0.f && !B) return 8;
  int sms, rc = device_check(sms);
  if (rc) return rc;
  cudaStream_t s = (cudaStream_t)stream;
  if (alpha == 0.f) return finish(launch_scale(C, ldc, m, n, beta, 0, s) ? BLAS3_ERR_CUDA : 0);
  Problem P = problem(m, n, alpha, beta, C, ldc, C, ldc);
  const int64_t ka = left ? m : n;
  // (SIMT mode: always from order 512 -- the materialisation is ~0.5% of the
  // FFMA GEMM, and the shadow area would otherwise be read uncoalesced)
  // (tcgen05, auto: GM_map below order 4096, where it measured faster at every
  // size -- 512 / 1024 / 1536 / 2048 / 3072: 86-88 / 88 / 89-91 / 91-92 / 95% of
  // SGEMM against 74 / 79 / 84-86 / 90 / 93-94% staged, profiles/r02_gm_map.md --
  // and from 4096 the merge while staging, the paper's rule 3, within 1-5%)
  const int64_t gm = opt(BLAS3_OPT_GM_MAP);
  if (tensor_mode() ? (gm < 0 ? ka < 4096 || use_gm_map(ka, left ? n : m, BLAS3_OPT_GM_MIN_SYMM) : gm == 1)
                    : (gm != 0 && (gm == 1 || ka >= 512))) {
    // GM_map: sym(A) materialised as a full ka x ka matrix, then a plain GEMM
    Scratch Wm;
    const int64_t ldw = ld4(ka);
    if ((rc = get_scratch(Wm, (size_t)ldw * ka * sizeof(float), s))) return rc;
    if (launch_materialize(Wm.p, ldw, A, lda, ka, ka, MAT_SYM, lower, 0, 0, s)) return BLAS3_ERR_CUDA;
    if (left) { P.seg[0].a = dense(Wm.p, ldw, false); P.seg[0].b = dense(B, ldb, true); P.seg[0].K = m; }
    else      { P.seg[0].a = dense(B, ldb, false); P.seg[0].b = dense(Wm.p, ldw, false); P.seg[0].K = n; }
    return finish(run_problem(P, s, sms));
  }
  if (left) {                       // C = Asym * B : Xa = Asym (m x m), Xb(c,k) = B(k,c)
    P.seg[0].a = sym(A, lda, lower);
    P.seg[0].b = dense(B, ldb, true);
    P.seg[0].K = m;
  } else {                          // C = B * Asym : Xa = B, Xb(c,k) = Asym(k,c) = Asym(c,k)
    P.seg[0].a = dense(B, ldb, false);
    P.seg[0].b = sym(A, lda, lower);
    P.seg[0].K = n;
  }
  return finish(run_problem(P, s, sms));
}

// ------------------------------------------------------------------- SSYRK / SSYR2K
static int syrk_common(bool two, char uplo, char trans, int64_t n, int64_t k, float alpha,
                       const float *A, int64_t lda, const float *B, int64_t ldb, float beta,
                       float *C, int64_t ldc, cudaStream_t s) {
  CallOpts call_opts;
  const bool lower = up(uplo) == 'L', ta = up(trans) != 'N';
  const int tri = lower ? 1 : 2;
  if (n == 0 || ((alpha == 0.f || k == 0) && beta == 1.f)) return 0;
  if (!C) return two ? 11 : 9;
  const bool reads = alpha != 0.f && k > 0;
  if (reads && !A) return 6;
  if (two && reads && !B) return 8;
  int sms, rc = device_check(sms);
  if (rc) return rc;
  if (!reads) return finish(launch_scale(C, ldc, n, n, beta, tri, s) ? BLAS3_ERR_CUDA : 0);
  Problem P = problem(n, n, alpha, beta, C, ldc, C, ldc);
  P.c_tri = tri;
  // trans=N: op(A) = A (n x k) -> X(r,k) = A(r,k) "rk"; trans=T: X(r,k) = A(k,r) "kr"
  P.seg[0].a = dense(A, lda, ta);
  P.seg[0].b = dense(two ? B : A, two ? ldb : lda, ta);
  P.seg[0].K = k;
  if (two) {
    P.nseg = 2;
    P.seg[1].a = dense(B, ldb, ta);
    P.seg[1].b = dense(A, lda, ta);
    P.seg[1].K = k;
  }
  return finish(run_problem(P, s, sms));
}

int blas3_ssyrk(char uplo, char trans, int64_t n, int64_t k, float alpha, const float *A,
                int64_t lda, float beta, float *C, int64_t ldc, blas3_stream_t stream) {
  if (const int v = v_syrk(false, uplo, trans, n, k, lda, 0, ldc)) return v;
  return syrk_common(false, uplo, trans, n, k, alpha, A, lda, nullptr, 0, beta, C, ldc,
                     (cudaStream_t)stream);
}

int blas3_ssyr2k(char uplo, char trans, int64_t n, int64_t k, float alpha, const float *A,
                 int64_t lda, const float *B, int64_t ldb, float beta, float *C, int64_t ldc,
                 blas3_stream_t stream) {
  if (const int v = v_syrk(true, uplo, trans, n, k, lda, ldb, ldc)) return v;
  return syrk_common(true, uplo, trans, n, k, alpha, A, lda, B, ldb, beta, C, ldc,
                     (cudaStream_t)stream);
}

// ------------------------------------------------------------------- STRMM / STRSM validation
static int tr_validate(char side, char uplo, char transa, char diag, int64_t m, int64_t n,
                       int64_t lda, int64_t ldb) {
  return v_tr(side, uplo, transa, diag, m, n, lda, ldb);
}

// ------------------------------------------------------------------- STRMM (row A9)

// B <- alpha*op(A)*B (L) or alpha*B*op(A) (R).  The tile-parallel product
// reads rows (L) / columns (R) of B that other tiles overwrite, so the
// product goes to stream-ordered scratch and is copied back (A9).
int blas3_strmm(char side, char uplo, char transa, char diag, int64_t m, int64_t n, float alpha,
                const float *A, int64_t lda, float *B, int64_t ldb, blas3_stream_t stream) {
  CallOpts call_opts;
  int v = tr_validate(side, uplo, transa, diag, m, n, lda, ldb);
  if (v) return v;
  if (m == 0 || n == 0) return 0;
  if (!B) return 10;
  if (alpha != 0.f && !A) return 8;
  int sms, rc = device_check(sms);
  if (rc) return rc;
  cudaStream_t s = (cudaStream_t)stream;
  if (alpha == 0.f) return finish(launch_scale(B, ldb, m, n, 0.f, 0, s) ? BLAS3_ERR_CUDA : 0);
  const bool left = up(side) == 'L', lower = up(uplo) == 'L', ta = up(transa) != 'N',
             unit = up(diag) == 'U';
  Scratch W, Wm;
  if ((rc = get_scratch(W, (size_t)m * n * sizeof(float), s))) return rc;
  Problem P = problem(m, n, alpha, 0.f, nullptr, 0, W.p, m);
  const int64_t ka = left ? m : n;
  if (tensor_mode() && use_gm_map(ka, left ? n : m, BLAS3_OPT_GM_MIN_TRMM)) {
    // GM_map: op(T) materialised MN-major with zeros in the blank triangle and
    // the unit diagonal written: the kernel clips k-ranges but loads every
    // block as a plain block (no zero-select / transpose)
    const int64_t ldw = ld4(ka);
    const bool lop = lower != ta;                  // op(T) is lower
    if ((rc = get_scratch(Wm, (size_t)ldw * ka * sizeof(float), s, (size_t)m * n * sizeof(float))))
      return rc;
    if (launch_materialize(Wm.p, ldw, A, lda, ka, ka, MAT_TRI, lower, ta, unit, s)) return BLAS3_ERR_CUDA;
    if (left) {   // Xa(r,k) = Wop(r,k)
      P.seg[0].a = tri_zeroed(Wm.p, ldw, lop, false);
      P.seg[0].b = dense(B, ldb, true);
      P.seg[0].K = m;
      P.rev_m = tri_kle(P.seg[0].a);
      P.outer = 1;
    } else {      // Xb(c,k) = Wop(k,c)
      P.seg[0].a = dense(B, ldb, false);
      P.seg[0].b = tri_zeroed(Wm.p, ldw, lop, true);
      P.seg[0].K = n;
      P.rev_n = tri_kle(P.seg[0].b);
      P.outer = 2;
    }
    if ((rc = run_problem(P, s, sms))) return rc;
    if (launch_copy(B, ldb, W.p, m, m, n, s)) return BLAS3_ERR_CUDA;
    return finish(0);
  }
  if (left) {     // Xa(r,k) = op(T)(r,k) -> swap = trans ; Xb(c,k) = B(k,c)
    P.seg[0].a = tri(A, lda, lower, ta, unit);
    P.seg[0].b = dense(B, ldb, true);
    P.seg[0].K = m;
    P.rev_m = tri_kle(P.seg[0].a);        // longest k-ranges first:
    P.outer = 1;                          // whole m-rows in turn (LPT)
  } else {        // Xa = B ; Xb(c,k) = op(T)(k,c) -> swap = !trans
    P.seg[0].a = dense(B, ldb, false);
    P.seg[0].b = tri(A, lda, lower, !ta, unit);
    P.seg[0].K = n;
    P.rev_n = tri_kle(P.seg[0].b);
    P.outer = 2;
  }
  if ((rc = run_problem(P, s, sms))) return rc;
  if (launch_copy(B, ldb, W.p, m, m, n, s)) return BLAS3_ERR_CUDA;
  return finish(0);
}

// ------------------------------------------------------------------- STRSM (rows A7, A8)
// Dependency order of the solver: X_i needs X_k, k < i.  The
// paper binds the diagonal step to one thread; here it is taken off
// the critical path.  With L = the stored triangle of A in lower form
// (op(A) = L or L^T):
//   1. every 128-block of L is inverted by the warp-level kernel (row A7);
//   2. 128 -> 256 -> 512 -> NBO doubling builds inv(L_pp) of every NBO-wide
//      diagonal panel: for each diagonal pair [[L11,0],[L21,L22]],
//      X21 = -inv(L22) * (L21 * inv(L11)) as two batched GEMMs per level;
//   3. the sweep (row A8) visits panels in dependency order, recursively
//      halving the panel range: solve the first half, one GEMM update of the
//      second half by the first (K = nt/2, nt/4, ...), solve the second half;
//      a single panel is X_p = alpha_p * inv(op(A)_pp) * B_p (TRI operand).
//      alpha is folded into the first operation that touches each row.
// Every flop of steps 2-3 runs in the structured GEMM kernels.
// panel width (a power of two >= 128, the diagonal block; BLAS3_OPT_TRSM_NB)
static int64_t trsm_nbo() { return opt(BLAS3_OPT_TRSM_NB); }

// Doubling levels 128 -> NBO for the panels of the order-nt triangle whose
// top-left corner is A (and whose panel inverses start at D); the 128-block
// inverses are already on D's diagonal.  Tw: (nt / 2sz) x sz^2 + sz^2 floats.
// Builds the problems in order: per level, T = L21 inv(L11) (step 1) then
// X21 = -inv(L22) T (step 2), for the full pairs and a ragged last pair.
struct LevelProblem { int lvl, step; Problem P; };
static void trsm_doubling_problems(const float *A, int64_t lda, int64_t nt, bool lower, float *D,
                                   float *Tw, std::vector<LevelProblem> &out) {
  const int64_t NBO = trsm_nbo();
  for (int64_t sz = 128, lvl = 0; sz < NBO; sz *= 2, ++lvl) {
    if (sz >= nt) continue;            // no pair reaches this level
    // pair b covers rows/cols [o, o + 2 sz) of L, o = 2 sz b; L21 = L[o+sz.., o..]
    const int64_t per = NBO / (2 * sz);
    const int64_t full = nt / (2 * sz);                    // pairs entirely inside L
    const int64_t rag_rows = nt - full * 2 * sz - sz;        // second half of a ragged pair
    // L21 as an Xa operand: X(r,k) = L(o+sz+r, o+k) = lower ? A(o+sz+r, o+k) : A(o+k, o+sz+r)
    auto l21 = [&](int64_t o) { return lower ? A + (o + sz) + o * lda : A + o + (o + sz) * lda; };
    auto dblk = [&](int64_t o) { return D + (o / NBO) * NBO * NBO + (o % NBO) * (1 + NBO); };
    for (int pass = 0; pass < 2; ++pass) {
      const int64_t cnt = pass == 0 ? full : (rag_rows > 0 ? 1 : 0);
      if (cnt == 0) continue;
      const int64_t o = pass == 0 ? 0 : full * 2 * sz;
      const int64_t m2 = pass == 0 ? sz : rag_rows;          // rows of L21 / order of L22
      float *T = Tw + (pass == 0 ? 0 : full * sz * sz);       // the ragged pair's own slot
      // T = L21 * inv(L11): Xa = L21 (m2 x sz), Xb(c,k) = inv(L11)(k,c) (lower -> TRI swap)
      Problem P1 = problem(m2, sz, 1.f, 0.f, nullptr, 0, T, m2);
      P1.seg[0].a = dense(l21(o), lda, !lower);
      P1.seg[0].b = tri_zeroed(dblk(o), NBO, true, true);
      P1.seg[0].K = sz;
      P1.nbatch = cnt; P1.per = per;
      P1.bs_a = {per * 2 * sz * (1 + lda), 2 * sz * (1 + lda)};
      P1.bs_b = {NBO * NBO, 2 * sz * (1 + NBO)};
      P1.bs_c = {per * sz * sz, sz * sz};
      out.push_back({(int)lvl, 1, P1});
      // X21 = -inv(L22) * T: Xa = inv(L22) (lower TRI), Xb(c,k) = T(k,c) (kr)
      Problem P2 = problem(m2, sz, -1.f, 0.f, nullptr, 0, dblk(o) + sz, NBO);
      P2.seg[0].a = tri_zeroed(dblk(o) + sz * (1 + NBO), NBO, true, false);
      P2.seg[0].b = dense(T, m2, true);
      P2.seg[0].K = m2;
      P2.nbatch = cnt; P2.per = per;
      P2.bs_a = {NBO * NBO, 2 * sz * (1 + NBO)};
      P2.bs_b = {per * sz * sz, sz * sz};
      P2.bs_c = {NBO * NBO, 2 * sz * (1 + NBO)};
      out.push_back({(int)lvl, 2, P2});
    }
  }
}
// Runs the doubling on stream s, recording ev_lvl[l] once the inverses of
// every aligned 2^(l+8)-block are complete.
// Levels [from, to) only (to < 0: all).
static int trsm_panel_doubling(const float *A, int64_t lda, int64_t nt, bool lower, float *D,
                               float *Tw, cudaStream_t s, int sms, cudaEvent_t *ev_lvl, int from = 0,
                               int to = -1) {
  std::vector<LevelProblem> probs;
  trsm_doubling_problems(A, lda, nt, lower, D, Tw, probs);
  size_t i = 0;
  int rc;
  for (int64_t sz = 128, lvl = 0; sz < trsm_nbo(); sz *= 2, ++lvl) {
    if (to >= 0 && lvl >= to) break;
    for (; i < probs.size() && probs[i].lvl == lvl; ++i)
      if (lvl >= from && (rc = run_problem(probs[i].P, s, sms))) return rc;
    if (lvl >= from && cudaEventRecord(ev_lvl[lvl], s) != cudaSuccess) return BLAS3_ERR_CUDA;
  }
  return 0;
}

// Side streams of the STRSM driver, per device, created once: one for the
// panel-inverse doubling of all but the first panel, and up to MAX_SLABS for
// the per-slab sweeps.  Fork/join is event-based, so the call stays
// asynchronous (and graph-capturable) on the caller's stream.
constexpr int MAX_SLABS = 4, MAX_LEVELS = 8;
struct TrsmStreams {
  cudaStream_t side, side2, side3, slab[MAX_SLABS];
  cudaEvent_t ev_fork, ev_fork2, ev_lvl[MAX_LEVELS], ev_lvl2[MAX_LEVELS], ev_ym[MAX_LEVELS],
      ev_join[MAX_SLABS];
};
static std::mutex g_trsm_mu;
static TrsmStreams *trsm_streams() {
  static TrsmStreams tab[64];
  static bool made[64] = {};
  int d = 0;
  if (cudaGetDevice(&d) != cudaSuccess || d < 0 || d >= 64) return nullptr;
  TrsmStreams &t = tab[d];
  if (!made[d]) {
    const unsigned fl = cudaEventDisableTiming;
    // the doubling chain is latency-bound and on the critical path: its
    // kernels get SMs before the sweep's (highest stream priority)
    int lo_pri = 0, hi_pri = 0;
    if (cudaDeviceGetStreamPriorityRange(&lo_pri, &hi_pri) != cudaSuccess) return nullptr;
    if (cudaStreamCreateWithPriority(&t.side, cudaStreamNonBlocking, hi_pri) != cudaSuccess) return nullptr;
    if (cudaStreamCreateWithPriority(&t.side2, cudaStreamNonBlocking, lo_pri) != cudaSuccess) return nullptr;
    if (cudaStreamCreateWithPriority(&t.side3, cudaStreamNonBlocking, hi_pri) != cudaSuccess) return nullptr;
    for (int i = 0; i < MAX_LEVELS; ++i)
      if (cudaEventCreateWithFlags(&t.ev_lvl[i], fl) != cudaSuccess ||
          cudaEventCreateWithFlags(&t.ev_lvl2[i], fl) != cudaSuccess ||
          cudaEventCreateWithFlags(&t.ev_ym[i], fl) != cudaSuccess) return nullptr;
    for (int i = 0; i < MAX_SLABS; ++i) {
      if (cudaStreamCreateWithFlags(&t.slab[i], cudaStreamNonBlocking) != cudaSuccess ||
          cudaEventCreateWithFlags(&t.ev_join[i], fl) != cudaSuccess) return nullptr;
    }
    if (cudaEventCreateWithFlags(&t.ev_fork, fl) != cudaSuccess ||
        cudaEventCreateWithFlags(&t.ev_fork2, fl) != cudaSuccess) return nullptr;
    made[d] = true;
  }
  return &t;
}
// number of right-hand-side slabs (BLAS3_OPT_TRSM_SLABS at most, each at least
// BLAS3_OPT_TRSM_SLAB_MIN columns (rows) wide)
static int64_t trsm_slabs(int64_t other) {
  const int64_t mn = opt(BLAS3_OPT_TRSM_SLAB_MIN) / 256 * 256;
  return imax(1, imin(opt(BLAS3_OPT_TRSM_SLABS), other / mn));
}
static inline int64_t align_down(int64_t v, int64_t a) { return v / a * a; }
// SMs the first panel's sweep kernels leave free for its doubling chain
// (-1 = auto: 48 from order 8192 on, where the other panels' doubling has the
// most work beside the chain; 16 below -- measured, profiles/r02_trsm_options.md)
static int64_t trsm_reserve(int64_t nt) {
  const int64_t v = opt(BLAS3_OPT_TRSM_RESERVE);
  return v >= 0 ? v : (nt >= 8192 ? 48 : 16);
}
// width below which the first panel's geometric halving stops (power of 2)
static int64_t trsm_geo_leaf() { return opt(BLAS3_OPT_TRSM_GEO_LEAF); }

// ---- fused STRSM: the whole solve as ONE persistent launch (after the
// 128-block inverses).  The doubling levels and the sweep are phases of one
// grid; a sweep tile waits only for the previous sweep phase ON ITS OWN SLAB
// (256 right-hand-side columns for side=L, rows for side=R) and a leaf for the
// doubling level that built its inverse, so the solve runs as a wavefront
// over the independent right-hand sides: no kernel boundaries, no launch
// tails, and the latency-bound first panel overlaps the doubling.  Every
// update writes the first panel of its output range to W (fixed leading
// dimension), every later leaf reads W and writes B, and the first leaf (at
// most one 256-row tile per slab) runs in place -- no copy-backs.
// Returns 1 (not fusable: the caller runs the multi-launch path) before
// anything is enqueued, 0 on success, < 0 on a CUDA error.
// A geometric pair of the first panel: first half f (solved before), second
// half s (aligned block of width h), with the precomputed Y_s and M buffers.
struct GeoPair { int64_t f_lo, f_hi, s_lo, s_hi, h; float *Y, *M; int64_t ldy, ldm; };

struct TrsmGeom {
  bool left, lower, ta, unit, lower_op, forward;
  int64_t m, n, nt, NBO, npanel, other;
  float alpha;
  const float *A; int64_t lda;
  float *B; int64_t ldb;
  float *D, *Tw, *W;
};
// first_solved (BLAS3_OPT_TRSM_FUSED = 2): the first processed panel is
// already solved (the diagonal-panel solver, earlier on the stream) and the
// other panels' doubling levels below lvl_from are complete (side stream,
// waited on by the caller): the launch holds the remaining levels of the
// other panels -- claimed first -- and the sweep after the first panel.
static int strsm_fused(const TrsmGeom &g, cudaStream_t s, int sms, bool first_solved = false,
                       int lvl_from = 0) {
  const int64_t NBO = g.NBO, nt = g.nt;
  const int64_t ldw = g.left ? NBO : g.m;              // W(r, c) = W[r + c * ldw]
  std::vector<LevelProblem> lv;
  if (!first_solved) trsm_doubling_problems(g.A, g.lda, nt, g.lower, g.D, g.Tw, lv);
  else if (g.npanel > 1) {                             // the other panels only
    const int64_t o = g.forward ? NBO : 0, len = g.forward ? nt - NBO : (g.npanel - 1) * NBO;
    trsm_doubling_problems(g.A + o * (1 + g.lda), g.lda, len, g.lower, g.D + (o / NBO) * NBO * NBO, g.Tw, lv);
  }
  int nlvl = 0;
  for (int64_t sz = 128; sz < NBO; sz *= 2) ++nlvl;

  std::vector<FusedPhase> ph;
  bool ok = true;
  uint32_t lvl_mask[MAX_LEVELS] = {};                  // phases (step 2) completing level l
  int emitted_lvl = -1;
  // Exact slab dependencies from each sweep phase's accesses: rows (L) /
  // columns (R) of B read and written, and whether it reads / writes W.  A
  // phase waits (on its slab) for every earlier sweep phase it conflicts with
  // (read-after-write, write-after-read, write-after-write).
  struct Acc { int idx; int64_t r_lo[2], r_hi[2], w_lo, w_hi; bool rw, ww; };
  std::vector<Acc> acc;
  auto overlap = [](int64_t a0, int64_t a1, int64_t b0, int64_t b1) { return a0 < b1 && b0 < a1; };
  auto add = [&](const Problem &P, uint32_t full, uint32_t slab) -> int {
    if ((int)ph.size() >= MAX_FUSED_PHASES) { ok = false; return 0; }
    FusedPhase f;
    f.P = P; f.dep_full = (int32_t)full; f.dep_slab = (int32_t)slab; f.slab_m = g.left ? 0 : 1;
    if (math_mode() == BLAS3_MATH_TF32_BF16X) f.P.passes = 2;   // (1xTF32: fused stays 3xTF32)
    ph.push_back(f);
    return (int)ph.size() - 1;
  };
  auto emit_level = [&](int l) {                        // step 1 after level l-1, step 2 after step 1
    uint32_t step1 = 0;
    for (const LevelProblem &q : lv)
      if (q.lvl == l && q.step == 1) step1 |= 1u << add(q.P, l > 0 ? lvl_mask[l - 1] : 0u, 0u);
    for (const LevelProblem &q : lv)
      if (q.lvl == l && q.step == 2) lvl_mask[l] |= 1u << add(q.P, step1, 0u);
  };
  auto levels_upto = [&](int l) {
    for (; emitted_lvl < l && emitted_lvl + 1 < nlvl; ) emit_level(++emitted_lvl);
  };
  auto sweep = [&](const Problem &P, int need, Acc a) {
    levels_upto(need);
    const uint32_t full = need >= 0 ? lvl_mask[need] : 0u;
    uint32_t slab = 0;
    for (const Acc &q : acc) {
      bool c = (q.ww && a.rw) || (q.rw && a.ww) || (q.ww && a.ww);
      for (int i = 0; i < 2 && !c; ++i) {
        c = overlap(q.w_lo, q.w_hi, a.r_lo[i], a.r_hi[i]) || overlap(q.r_lo[i], q.r_hi[i], a.w_lo, a.w_hi);
      }
      c = c || overlap(q.w_lo, q.w_hi, a.w_lo, a.w_hi);
      if (c) slab |= 1u << q.idx;
    }
    a.idx = add(P, full, slab);
    acc.push_back(a);
    levels_upto(need + 1);                              // one level of lookahead
  };
  // in-place parts of split updates, emitted right after the next leaf so the
  // critical leaf is claimed before the bulk update (items run in claim order)
  std::vector<std::function<void()>> pending;
  auto flush_pending = [&]() {
    std::vector<std::function<void()>> p;
    p.swap(pending);
    for (auto &f : p) f();
  };
  auto leaf_acc = [](int64_t e0, int64_t cnt, bool src_w) {
    Acc a{};
    a.r_lo[0] = src_w ? 0 : e0; a.r_hi[0] = src_w ? 0 : e0 + cnt;
    a.w_lo = e0; a.w_hi = e0 + cnt;
    a.rw = src_w;
    return a;
  };
  auto upd_acc = [](int64_t k_lo, int64_t k_hi, int64_t o_lo, int64_t o_hi, bool to_w) {
    Acc a{};
    a.r_lo[0] = k_lo; a.r_hi[0] = k_hi; a.r_lo[1] = o_lo; a.r_hi[1] = o_hi;
    if (!to_w) { a.w_lo = o_lo; a.w_hi = o_hi; }
    a.ww = to_w;
    return a;
  };
  // leaf: X rows (L) / columns (R) [e0, e0 + cnt) of the aligned block of width wblk
  auto leaf = [&](int64_t e0, int64_t cnt, int64_t wblk, bool scaled, bool src_w) {
    if (!src_w && cnt > 256) { ok = false; return; }    // in place only as one tile per slab
    int need = -1;
    for (int64_t w2 = 256; w2 <= wblk; w2 *= 2) ++need;
    const float a1 = scaled ? 1.f : g.alpha;
    const float *Dp = g.D + (e0 / NBO) * NBO * NBO + (e0 % NBO) * (1 + NBO);
    if (g.left) {
      Problem P = problem(cnt, g.n, a1, 0.f, nullptr, 0, g.B + e0, g.ldb);
      P.seg[0].a = tri_zeroed(Dp, NBO, true, !g.lower_op);
      P.seg[0].b = src_w ? dense(g.W, ldw, true) : dense(g.B + e0, g.ldb, true);
      P.seg[0].K = cnt;
      P.rev_m = tri_kle(P.seg[0].a);
      P.outer = 2;                                     // slab (n-tile) outer, LPT rows inside
      sweep(P, need, leaf_acc(e0, cnt, src_w));
      flush_pending();
    } else {
      Problem P = problem(g.m, cnt, a1, 0.f, nullptr, 0, g.B + e0 * g.ldb, g.ldb);
      P.seg[0].a = src_w ? dense(g.W, ldw, false) : dense(g.B + e0 * g.ldb, g.ldb, false);
      P.seg[0].b = tri_zeroed(Dp, NBO, true, g.lower_op);
      P.seg[0].K = cnt;
      P.rev_n = tri_kle(P.seg[0].b);
      P.outer = 1;                                     // slab (m-tile) outer
      sweep(P, need, leaf_acc(e0, cnt, src_w));
      flush_pending();
    }
  };
  // update: [o_lo, o_hi) <- a1 * B_o - op(A)(o, k) X_k, k in [k_lo, k_hi); to W or in place
  auto update = [&](int64_t k_lo, int64_t k_hi, int64_t o_lo, int64_t o_hi, float a1, bool to_w) {
    if (g.left) {
      const float *pa = g.ta ? g.A + k_lo + o_lo * g.lda : g.A + o_lo + k_lo * g.lda;
      Problem P = to_w ? problem(o_hi - o_lo, g.n, -1.f, a1, g.B + o_lo, g.ldb, g.W, ldw)
                       : problem(o_hi - o_lo, g.n, -1.f, a1, g.B + o_lo, g.ldb, g.B + o_lo, g.ldb);
      P.seg[0].a = dense(pa, g.lda, g.ta);
      P.seg[0].b = dense(g.B + k_lo, g.ldb, true);
      P.seg[0].K = k_hi - k_lo;
      P.outer = 2;
      sweep(P, -1, upd_acc(k_lo, k_hi, o_lo, o_hi, to_w));
    } else {
      const float *pb = g.ta ? g.A + o_lo + k_lo * g.lda : g.A + k_lo + o_lo * g.lda;
      Problem P = to_w ? problem(g.m, o_hi - o_lo, -1.f, a1, g.B + o_lo * g.ldb, g.ldb, g.W, ldw)
                       : problem(g.m, o_hi - o_lo, -1.f, a1, g.B + o_lo * g.ldb, g.ldb,
                                 g.B + o_lo * g.ldb, g.ldb);
      P.seg[0].a = dense(g.B + k_lo * g.ldb, g.ldb, false);
      P.seg[0].b = dense(pb, g.lda, !g.ta);
      P.seg[0].K = k_hi - k_lo;
      P.outer = 1;
      sweep(P, -1, upd_acc(k_lo, k_hi, o_lo, o_hi, to_w));
    }
  };
  const int64_t geo_leaf = trsm_geo_leaf();
  std::function<void(int64_t, int64_t, bool)> geo = [&](int64_t lo, int64_t w, bool scaled) {
    const int64_t e1 = imin(nt, lo + w);
    if (w <= geo_leaf) { leaf(lo, e1 - lo, w, scaled, false); return; }
    const int64_t h = w / 2, mid = lo + h;
    if (mid >= e1) { geo(lo, h, scaled); return; }
    const int64_t f_lo = g.forward ? lo : mid, f_hi = g.forward ? mid : e1;
    const int64_t s_lo = g.forward ? mid : lo, s_hi = g.forward ? e1 : mid;
    geo(f_lo, h, scaled);
    update(f_lo, f_hi, s_lo, s_hi, scaled ? 1.f : g.alpha, true);
    leaf(s_lo, s_hi - s_lo, h, true, true);
  };
  auto elem = [&](int64_t qa, int64_t qb, int64_t &lo, int64_t &hi) {
    const int64_t pa = g.forward ? qa : g.npanel - qb, pb = g.forward ? qb : g.npanel - qa;
    lo = pa * NBO;
    hi = imin(nt, pb * NBO);
  };
  std::function<void(int64_t, int64_t, bool, bool)> rec = [&](int64_t q0, int64_t q1, bool scaled,
                                                              bool in_w) {
    if (q1 - q0 == 1) {
      const int64_t p = g.forward ? q0 : g.npanel - 1 - q0;
      const int64_t p0 = p * NBO, pr = imin(NBO, nt - p0);
      if (q0 == 0) { if (!first_solved) geo(p0, NBO, scaled); }
      else leaf(p0, pr, NBO, scaled, in_w);
      return;
    }
    const int64_t mid = q0 + (q1 - q0) / 2;
    rec(q0, mid, scaled, in_w);
    int64_t k_lo, k_hi, o_lo, o_hi;
    elem(q0, mid, k_lo, k_hi);
    elem(mid, q1, o_lo, o_hi);
    const float a1 = scaled ? 1.f : g.alpha;
    if (q1 - mid == 1) update(k_lo, k_hi, o_lo, o_hi, a1, true);
    else {                        // the first panel of [mid, q1) to W, the rest in place
      int64_t f_lo, f_hi;
      elem(mid, mid + 1, f_lo, f_hi);
      update(k_lo, k_hi, f_lo, f_hi, a1, true);
      const int64_t r_lo = g.forward ? f_hi : o_lo, r_hi = g.forward ? o_hi : f_lo;
      pending.push_back([=, &update]() { update(k_lo, k_hi, r_lo, r_hi, a1, false); });
    }
    rec(mid, q1, true, true);
  };
  if (first_solved) {                                  // the remaining levels first, then the sweep
    emitted_lvl = lvl_from - 1;
    levels_upto(nlvl - 1);
  }
  rec(0, g.npanel, false, false);
  flush_pending();
  if (!ok || ph.empty()) return 1;
  for (const FusedPhase &f : ph)
    if (!tc_eligible(f.P)) return 1;
  // 128-block inverses (the fused phases read them), then the one launch
  if (!first_solved && launch_trsm_diag_inv(g.A, g.lda, nt, g.lower, g.unit, g.D, NBO, s)) return BLAS3_ERR_CUDA;
  const int rc = launch_tc_fused(ph.data(), (int)ph.size(), s, sms);
  return rc == 0 ? 0 : (rc == -4 ? BLAS3_ERR_TMA : BLAS3_ERR_CUDA);
}

// The first processed panel as ONE fused launch (BLAS3_OPT_TRSM_FIRST_FUSED).
// Phases, in claim order: the panel's doubling levels (each step waits for
// the previous one), the first leaf (in place: one 256-row tile per slab),
// then per geometric pair j: M_j and Y_j (wait for the level that built
// inv(op(A)_ss)) and X_j = Y_j - M_j X_f (waits for M_j, and on its slab for
// Y_j and every earlier chain phase).  Returns 1 if not fusable (nothing
// enqueued), 0 on success, < 0 on a CUDA error.  The 128-block inverses must
// already be on the stream.  [r_lo, r_hi): the aligned block whose doubling
// levels the launch builds (default: the whole panel).
static int strsm_first_fused(const TrsmGeom &g, const std::vector<GeoPair> &gp, int64_t pfirst,
                             cudaStream_t s, int sms, int64_t r_lo = -1, int64_t r_hi = -1,
                             bool all = false) {
  const int64_t NBO = g.NBO, nt = g.nt;
  if (all) { r_lo = 0; r_hi = nt; pfirst = 0; }        // every panel's doubling, whole grid
  else if (r_lo < 0) { r_lo = pfirst * NBO; r_hi = imin(nt, r_lo + NBO); }   // doubling range: the panel
  std::vector<LevelProblem> lv;
  trsm_doubling_problems(g.A + r_lo * (1 + g.lda), g.lda, r_hi - r_lo, g.lower,
                         g.D + pfirst * NBO * NBO + (r_lo - pfirst * NBO) * (1 + NBO), g.Tw, lv);
  auto level_of = [](int64_t w) { int l = -1; for (int64_t w2 = 256; w2 <= w; w2 *= 2) ++l; return l; };
  int need = 0;                                         // levels used: inv of every s block
  for (const GeoPair &p : gp) need = imax(need, level_of(p.h) + 1);
  std::vector<FusedPhase> ph;
  auto add = [&](const Problem &P, uint32_t full, uint32_t slab) -> int {
    FusedPhase f;
    f.P = P; f.dep_full = (int32_t)full; f.dep_slab = (int32_t)slab; f.slab_m = g.left ? 0 : 1;
    if (math_mode() == BLAS3_MATH_TF32_BF16X) f.P.passes = 2;   // (1xTF32: fused stays 3xTF32)
    ph.push_back(f);
    return (int)ph.size() - 1;
  };
  uint32_t lvl_mask[MAX_LEVELS] = {};
  auto emit_level = [&](int l) {
    uint32_t step1 = 0;
    for (const LevelProblem &q : lv)
      if (q.lvl == l && q.step == 1) step1 |= 1u << add(q.P, l > 0 ? lvl_mask[l - 1] : 0u, 0u);
    for (const LevelProblem &q : lv)
      if (q.lvl == l && q.step == 2) lvl_mask[l] |= 1u << add(q.P, step1, 0u);
  };
  for (int l = 0; l < need; ++l) emit_level(l);
  // first leaf: the block solved before every pair's f
  const int64_t l_lo = gp[0].f_lo, l_cnt = gp[0].f_hi - gp[0].f_lo;
  if (l_cnt > 256) return 1;
  const int l_lv = level_of(gp[0].h);
  const float *Dl = g.D + (l_lo / NBO) * NBO * NBO + (l_lo % NBO) * (1 + NBO);
  uint32_t chain = 0;
  {
    Problem P;
    if (g.left) {
      P = problem(l_cnt, g.n, g.alpha, 0.f, nullptr, 0, g.B + l_lo, g.ldb);
      P.seg[0].a = tri_zeroed(Dl, NBO, true, !g.lower_op);
      P.seg[0].b = dense(g.B + l_lo, g.ldb, true);
      P.rev_m = tri_kle(P.seg[0].a);
      P.outer = 2;
    } else {
      P = problem(g.m, l_cnt, g.alpha, 0.f, nullptr, 0, g.B + l_lo * g.ldb, g.ldb);
      P.seg[0].a = dense(g.B + l_lo * g.ldb, g.ldb, false);
      P.seg[0].b = tri_zeroed(Dl, NBO, true, g.lower_op);
      P.rev_n = tri_kle(P.seg[0].b);
      P.outer = 1;
    }
    P.seg[0].K = l_cnt;
    chain |= 1u << add(P, l_lv >= 0 ? lvl_mask[l_lv] : 0u, 0u);
  }
  for (const GeoPair &p : gp) {
    const int64_t ns = p.s_hi - p.s_lo, nf = p.f_hi - p.f_lo;
    const int lvp = level_of(p.h);
    const uint32_t lmask = lvp >= 0 ? lvl_mask[lvp] : 0u;
    const float *Ds = g.D + (p.s_lo / NBO) * NBO * NBO + (p.s_lo % NBO) * (1 + NBO);
    Problem PM, PY, PX;
    if (g.left) {
      PM = problem(ns, nf, 1.f, 0.f, nullptr, 0, p.M, p.ldm);
      PM.seg[0].a = tri_zeroed(Ds, NBO, true, !g.lower_op);
      PM.seg[0].b = g.ta ? dense(g.A + p.f_lo + p.s_lo * g.lda, g.lda, false)
                         : dense(g.A + p.s_lo + p.f_lo * g.lda, g.lda, true);
      PM.seg[0].K = ns;
      PM.rev_m = tri_kle(PM.seg[0].a);
      PY = problem(ns, g.n, g.alpha, 0.f, nullptr, 0, p.Y, p.ldy);
      PY.seg[0].a = tri_zeroed(Ds, NBO, true, !g.lower_op);
      PY.seg[0].b = dense(g.B + p.s_lo, g.ldb, true);
      PY.seg[0].K = ns;
      PY.rev_m = tri_kle(PY.seg[0].a);
      PY.outer = 2;
      PX = problem(ns, g.n, -1.f, 1.f, p.Y, p.ldy, g.B + p.s_lo, g.ldb);
      PX.seg[0].a = dense(p.M, p.ldm, false);
      PX.seg[0].b = dense(g.B + p.f_lo, g.ldb, true);
      PX.seg[0].K = nf;
      PX.outer = 2;
    } else {
      PM = problem(nf, ns, 1.f, 0.f, nullptr, 0, p.M, p.ldm);
      PM.seg[0].a = g.ta ? dense(g.A + p.s_lo + p.f_lo * g.lda, g.lda, true)
                         : dense(g.A + p.f_lo + p.s_lo * g.lda, g.lda, false);
      PM.seg[0].b = tri_zeroed(Ds, NBO, true, g.lower_op);
      PM.seg[0].K = ns;
      PM.rev_n = tri_kle(PM.seg[0].b);
      PY = problem(g.m, ns, g.alpha, 0.f, nullptr, 0, p.Y, p.ldy);
      PY.seg[0].a = dense(g.B + p.s_lo * g.ldb, g.ldb, false);
      PY.seg[0].b = tri_zeroed(Ds, NBO, true, g.lower_op);
      PY.seg[0].K = ns;
      PY.rev_n = tri_kle(PY.seg[0].b);
      PY.outer = 1;
      PX = problem(g.m, ns, -1.f, 1.f, p.Y, p.ldy, g.B + p.s_lo * g.ldb, g.ldb);
      PX.seg[0].a = dense(g.B + p.f_lo * g.ldb, g.ldb, false);
      PX.seg[0].b = dense(p.M, p.ldm, true);
      PX.seg[0].K = nf;
      PX.outer = 1;
    }
    const int im = add(PM, lmask, 0u);
    const int iy = add(PY, lmask, 0u);
    chain |= 1u << add(PX, 1u << im, chain | (1u << iy));
  }
  if (all) {                                            // the other panels' last levels, claimed last
    int nl = 0;
    for (int64_t sz = 128; sz < NBO; sz *= 2) ++nl;
    for (int l = need; l < nl; ++l) emit_level(l);
  }
  if ((int)ph.size() > MAX_FUSED_PHASES) return 1;
  for (const FusedPhase &f : ph)
    if (!tc_eligible(f.P)) return 1;
  // the chain is latency-bound: leave SMs to the other panels' doubling,
  // which runs concurrently on a side stream
  const int rc = launch_tc_fused(ph.data(), (int)ph.size(), s,
                                 all ? sms : (int)imax(sms / 2, sms - trsm_reserve(nt)));
  return rc == 0 ? 0 : (rc == -4 ? BLAS3_ERR_TMA : BLAS3_ERR_CUDA);
}

// The diagonal-panel solver (panel_kernel.cu) for panel pidx: level 0 of the
// panel's doubling (its 256-block inverses), the couplings
// M = -inv(op(A)_ss) op(A)_sf of every 256-block s (one batched GEMM over the
// whole panel row -- the kernel reads only the solved part) and
// a_diag * inv(op(A)_ss) on M's diagonal (strsm_panel_prep), then ONE launch
// in which every team of CTA pairs forward-substitutes its 256 right-hand
// sides through the panel, in place over B (strsm_panel_run).
// panel_ok: whether the solver applies (order a multiple of 256, B aligned).
static bool panel_ok(const TrsmGeom &g, int64_t pidx) {
  const int64_t R = imin(g.NBO, g.nt - pidx * g.NBO);
  return R > 0 && R % 256 == 0 && R <= 8192 && (reinterpret_cast<uintptr_t>(g.B) % 16) == 0 && g.ldb % 4 == 0;
}
static int strsm_panel_prep(const TrsmGeom &g, int64_t pidx, float a_diag, float *Mw, cudaStream_t s, int sms) {
  const int64_t NBO = g.NBO, p0 = pidx * NBO, R = imin(NBO, g.nt - p0), ldm = R;
  const int64_t nb = R / 256;
  float *Dp = g.D + pidx * NBO * NBO;
  const float *Ap = g.A + p0 * (1 + g.lda);
  Problem P;
  if (g.left) {        // M(s, c) = -sum_k inv(op(A)_ss)(r, k) op(A)(s_lo + k, p0 + c), batch over s
    P = problem(256, R, -1.f, 0.f, nullptr, 0, Mw, ldm);
    P.seg[0].a = tri_zeroed(Dp, NBO, true, !g.lower_op);
    P.seg[0].b = dense(Ap, g.lda, !g.ta);
    P.rev_m = tri_kle(P.seg[0].a);
    P.bs_a = {0, 256 * (1 + NBO)};
    P.bs_b = {0, g.ta ? 256 * g.lda : 256};
    P.bs_c = {0, 256};
  } else {             // M(f, s) = -sum_k op(A)(p0 + f, s_lo + k) inv(op(A)_ss)(k, c)
    P = problem(R, 256, -1.f, 0.f, nullptr, 0, Mw, ldm);
    P.seg[0].a = dense(Ap, g.lda, g.ta);
    P.seg[0].b = tri_zeroed(Dp, NBO, true, g.lower_op);
    P.rev_n = tri_kle(P.seg[0].b);
    P.bs_a = {0, g.ta ? 256 : 256 * g.lda};
    P.bs_b = {0, 256 * (1 + NBO)};
    P.bs_c = {0, 256 * ldm};
  }
  P.seg[0].K = 256;
  P.nbatch = nb;
  P.per = nb;
  if (nb > 1 && !tc_eligible(P)) return 1;
  int rc;
  // level 0 of the panel's doubling (its 256-block inverses) on CUDA cores,
  // one launch, then the couplings
  if (launch_trsm_level0(Ap, g.lda, R, g.lower, Dp, NBO, s)) return BLAS3_ERR_CUDA;
  if (nb > 1 && (rc = run_problem(P, s, sms))) return rc;
  if (launch_trsm_panel_diag(Dp, NBO, Mw, ldm, R, g.lower_op, a_diag, s)) return BLAS3_ERR_CUDA;
  return 0;
}
static int strsm_panel_run(const TrsmGeom &g, int64_t pidx, const float *Mw, void *pws, cudaStream_t s, int sms) {
  const int64_t p0 = pidx * g.NBO, R = imin(g.NBO, g.nt - p0);
  float *X = g.left ? g.B + p0 : g.B + p0 * g.ldb;
  const int rc = launch_trsm_panel(Mw, R, X, g.ldb, !g.left, R, g.other, g.forward, (int)opt(BLAS3_OPT_TC_KC), pws,
                                   s, sms);
  return rc == 0 ? 0 : (rc == -4 ? BLAS3_ERR_TMA : BLAS3_ERR_CUDA);
}
// The first processed panel (BLAS3_OPT_TRSM_PANEL): returns 1 if not
// applicable (nothing enqueued), 0, or < 0 on an error.
static int strsm_first_panel(const TrsmGeom &g, int64_t pfirst, float *Mw, void *pws, cudaStream_t s, int sms) {
  if (!panel_ok(g, pfirst)) return 1;
  int rc = strsm_panel_prep(g, pfirst, g.alpha, Mw, s, sms);
  if (rc) return rc;
  return strsm_panel_run(g, pfirst, Mw, pws, s, sms);
}

int blas3_strsm(char side, char uplo, char transa, char diag, int64_t m, int64_t n, float alpha,
                const float *A, int64_t lda, float *B, int64_t ldb, blas3_stream_t stream) {
  CallOpts call_opts;
  int v = tr_validate(side, uplo, transa, diag, m, n, lda, ldb);
  if (v) return v;
  if (m == 0 || n == 0) return 0;
  if (!B) return 10;
  if (alpha != 0.f && !A) return 8;
  int sms, rc = device_check(sms);
  if (rc) return rc;
  cudaStream_t s = (cudaStream_t)stream;
  if (alpha == 0.f) return finish(launch_scale(B, ldb, m, n, 0.f, 0, s) ? BLAS3_ERR_CUDA : 0);

  const bool left = up(side) == 'L';
  bool lower = up(uplo) == 'L', ta = up(transa) != 'N', unit = up(diag) == 'U';
  const bool lower_op = lower != ta;               // op(A) = L (true) or L^T (false)
  const int64_t nt = left ? m : n;                 // order of A
  const int64_t NBO = trsm_nbo();
  const int64_t npanel = cdiv(nt, NBO);
  const int64_t other = left ? n : m;              // RHS extent
  const bool forward = left ? lower_op : !lower_op;

  // GM_map canonicalisation for transposed variants: op(A) is materialised
  // (MN-major, zeros in the blank triangle, unit diagonal written), and the
  // solve runs on it as a non-transposed triangle with the same op(A) -- the
  // sweep's update GEMMs then stage op(A) blocks in the MN-major orientation.
  Scratch Aop;
  size_t aop_bytes = 0;
  if (ta && tensor_mode() && use_gm_map(nt, other, BLAS3_OPT_GM_MIN_TRSM)) {
    const int64_t ldw = ld4(nt);
    aop_bytes = (size_t)ldw * nt * sizeof(float);
    if ((rc = get_scratch(Aop, aop_bytes, s))) return rc;
    if (launch_materialize(Aop.p, ldw, A, lda, nt, nt, MAT_TRI, lower, ta, unit, s)) return BLAS3_ERR_CUDA;
    A = Aop.p; lda = ldw; lower = lower_op; ta = false; unit = false;
  }

  const size_t d_bytes = (size_t)npanel * NBO * NBO * sizeof(float);
  // doubling scratch: nt/2sz pairs x sz^2 floats at the widest level
  const size_t t_rest = (size_t)nt * (NBO / 4), t_first = (size_t)NBO * NBO / 4;
  const size_t t_bytes = (t_rest + 2 * t_first) * sizeof(float);   // + first-split s blocks
  const size_t w_bytes = (size_t)NBO * other * sizeof(float);        // one solved panel
  Scratch D, Tw, W;
  if ((rc = get_scratch(D, d_bytes, s, aop_bytes))) return rc;
  if ((rc = get_scratch(Tw, t_bytes, s, aop_bytes + d_bytes))) return rc;
  if ((rc = get_scratch(W, w_bytes, s, aop_bytes + d_bytes + t_bytes))) return rc;

  if (opt(BLAS3_OPT_TRSM_FUSED) == 1 && tensor_mode()) {
    const TrsmGeom g{left, lower, ta, unit, lower_op, forward, m, n, nt, NBO, npanel, other, alpha,
                     A, lda, B, ldb, D.p, Tw.p, W.p};
    rc = strsm_fused(g, s, sms);
    if (rc <= 0) return finish(rc);
  }

  std::lock_guard<std::mutex> lk(g_trsm_mu);          // the per-device side streams
  TrsmStreams *ts = trsm_streams();
  if (!ts) return BLAS3_ERR_CUDA;
  // First-panel precompute (BLAS3_OPT_TRSM_FIRST_YM): each geometric pair
  // (first half f solved, second half s) would be "update s by f, then solve
  // s" on the critical path.  Instead, with Y_s = a * inv(op(A)_ss) B_s and
  // M_sf = inv(op(A)_ss) op(A)_sf -- neither needs X -- a third high-priority
  // stream computes Y and M as soon as inv(op(A)_ss) exists, and the chain is
  // left with ONE GEMM per pair, X_s = Y_s - M_sf X_f (K = |f|): the first
  // panel's sequential k-blocks halve.  (side=R: X_s = Y_s - X_f M_fs with
  // Y_s = a B_s inv(op(A)_ss), M_fs = op(A)_fs inv(op(A)_ss).)
  const int64_t pfirst = forward ? 0 : npanel - 1;
  int nlvl = 0;
  for (int64_t sz = 128; sz < NBO; sz *= 2) ++nlvl;
  // BLAS3_OPT_TRSM_PANEL: the first panel by the diagonal-panel solver (its
  // M workspace after W); the geometric chain's Y/M are then not needed
  const int64_t r_first = imin(NBO, nt - pfirst * NBO);
  // (at every right-hand-side count: STRSM 2048 / 4096 / 8192 x 4096 RHS / 8192
  // measured 2.6 / 7.5 / 3.3 / 3.4% faster than the fused chain, profiles/r02_strsm_panel.md)
  const bool use_panel = opt(BLAS3_OPT_TRSM_PANEL) != 0 && tensor_mode() && r_first % 256 == 0;
  // BLAS3_OPT_TRSM_PANEL2: the second processed panel by the solver too (one
  // right-hand-side slab; the panel's 256-block inverses and couplings on the
  // high-priority side stream beside the first panel's kernel)
  const int64_t psecond = forward ? 1 : npanel - 2;
  const int64_t r_second = npanel >= 2 ? imin(NBO, nt - psecond * NBO) : 0;
  const bool want_panel2 = use_panel && npanel >= 2 && opt(BLAS3_OPT_TRSM_PANEL2) != 0 && r_second % 256 == 0 &&
                           trsm_slabs(other) == 1 && opt(BLAS3_OPT_TRSM_FUSED) != 2;
  Scratch Mw;
  const size_t m_bytes = (size_t)r_first * r_first * sizeof(float);
  const size_t pws_bytes = trsm_panel_ws_bytes(other, sms);
  const size_t m2_bytes = want_panel2 ? (size_t)r_second * r_second * sizeof(float) : 0;
  if (use_panel &&
      (rc = get_scratch(Mw, m_bytes + pws_bytes + m2_bytes, s, aop_bytes + d_bytes + t_bytes + w_bytes)))
    return rc;
  float *Mw2 = want_panel2 ? reinterpret_cast<float *>(reinterpret_cast<uint8_t *>(Mw.p) + m_bytes + pws_bytes)
                           : nullptr;
  std::vector<GeoPair> gp;
  Scratch YM;
  const bool use_ym = !use_panel && (opt(BLAS3_OPT_TRSM_FIRST_YM) != 0 || opt(BLAS3_OPT_TRSM_FIRST_FUSED) != 0);
  if (use_ym) {
    std::function<void(int64_t, int64_t)> pairs = [&](int64_t lo, int64_t w) {
      const int64_t e1 = imin(nt, lo + w);
      if (w <= trsm_geo_leaf()) return;
      const int64_t h = w / 2, mid = lo + h;
      if (mid >= e1) { pairs(lo, h); return; }
      const int64_t f_lo = forward ? lo : mid, f_hi = forward ? mid : e1;
      const int64_t s_lo = forward ? mid : lo, s_hi = forward ? e1 : mid;
      pairs(f_lo, h);
      gp.push_back({f_lo, f_hi, s_lo, s_hi, h, nullptr, nullptr, 0, 0});
    };
    pairs(pfirst * NBO, NBO);
    if ((int)gp.size() > MAX_LEVELS) gp.clear();
    size_t fl = 0;
    for (GeoPair &p : gp) {
      const int64_t ns = p.s_hi - p.s_lo, nf = p.f_hi - p.f_lo;
      p.ldy = left ? ld4(ns) : ld4(m);
      p.ldm = left ? ld4(ns) : ld4(nf);
      fl += (size_t)p.ldy * (left ? n : ns) + (size_t)p.ldm * (left ? nf : ns);
    }
    if (!gp.empty()) {
      if ((rc = get_scratch(YM, fl * sizeof(float), s, aop_bytes + d_bytes + t_bytes + w_bytes))) return rc;
      float *cur = YM.p;
      for (GeoPair &p : gp) {
        const int64_t ns = p.s_hi - p.s_lo, nf = p.f_hi - p.f_lo;
        p.Y = cur; cur += (size_t)p.ldy * (left ? n : ns);
        p.M = cur; cur += (size_t)p.ldm * (left ? nf : ns);
      }
    }
  }

  // 1. every 128-block inverse on the caller's stream; then the doubling
  //    levels of all panels on the high-priority side stream, one event per
  //    level, while the sweep starts on blocks whose inverse already exists.
  if (launch_trsm_diag_inv(A, lda, nt, lower, unit, D.p, NBO, s)) return BLAS3_ERR_CUDA;
  if (cudaEventRecord(ts->ev_fork, s) != cudaSuccess ||
      cudaStreamWaitEvent(ts->side, ts->ev_fork, 0) != cudaSuccess) return BLAS3_ERR_CUDA;
  // BLAS3_OPT_TRSM_FIRST_ALL: every panel's doubling inside the first panel's
  // fused launch (levels the chain needs first, the rest claimed after the
  // chain), on the whole grid -- no side stream competes for SMs
  bool all_done = false, panel_done = false;
  if (use_panel) {
    const TrsmGeom g{left, lower, ta, unit, lower_op, forward, m, n, nt, NBO, npanel, other, alpha,
                     A, lda, B, ldb, D.p, Tw.p + t_rest, W.p};
    rc = strsm_first_panel(g, pfirst, Mw.p, reinterpret_cast<uint8_t *>(Mw.p) + m_bytes, s, sms);
    if (rc < 0) return rc;
    panel_done = rc == 0;
  }
  if (!panel_done && opt(BLAS3_OPT_TRSM_FIRST_ALL) && opt(BLAS3_OPT_TRSM_FIRST_FUSED) &&
      opt(BLAS3_OPT_TRSM_FIRST_SPLIT) == 0 && tensor_mode() && !gp.empty()) {
    const TrsmGeom g{left, lower, ta, unit, lower_op, forward, m, n, nt, NBO, npanel, other, alpha,
                     A, lda, B, ldb, D.p, Tw.p, W.p};
    rc = strsm_first_fused(g, gp, pfirst, s, sms, -1, -1, true);
    if (rc < 0) return rc;
    all_done = rc == 0;
  }
  // the first processed panel: ONE fused persistent launch (its doubling
  // levels, the precomputed Y and M of every geometric pair, and the chain
  // leaf -> X_1 -> X_2 -> ... with per-slab tile-counter dependencies) on the
  // caller's stream; else its levels on the high-priority side stream and
  // the Y/M precompute on a third stream, the chain on the slab streams.
  bool first_done = false, ym_ready = false;
  // BLAS3_OPT_TRSM_FIRST_SPLIT = F: only the first F rows (L) / columns (R)
  // of the first panel (processing order) run as the latency-bound fused
  // chain.  The outer geometric pairs (s blocks of width F, 2F, ...) leave it:
  // after the chain, the block solved last updates EVERY later row of the
  // matrix in one bulk GEMM (full machine), then the next s block is one
  // leaf solve -- a right-looking sweep with geometrically growing blocks.
  // The s blocks' inverses are doubled up front on the high-priority side
  // stream, concurrently with the chain (they do not depend on X).
  std::vector<GeoPair> outer;                         // popped pairs, inner -> outer
  const int64_t fsplit = opt(BLAS3_OPT_TRSM_FIRST_SPLIT);
  first_done = all_done || panel_done;
  // the second panel's precompute on side3 (after the 128-block inverses);
  // alpha is already applied by the update that precedes its solve
  bool panel2 = false;
  if (want_panel2 && panel_done) {
    const TrsmGeom g{left, lower, ta, unit, lower_op, forward, m, n, nt, NBO, npanel, other, alpha,
                     A, lda, B, ldb, D.p, Tw.p, W.p};
    if (panel_ok(g, psecond)) {
      if (cudaStreamWaitEvent(ts->side3, ts->ev_fork, 0) != cudaSuccess) return BLAS3_ERR_CUDA;
      rc = strsm_panel_prep(g, psecond, 1.f, Mw2, ts->side3, sms);
      if (rc < 0) return rc;
      panel2 = rc == 0;
      if (panel2 && cudaEventRecord(ts->ev_ym[0], ts->side3) != cudaSuccess) return BLAS3_ERR_CUDA;
    }
  }
  if (!first_done && opt(BLAS3_OPT_TRSM_FIRST_FUSED) && tensor_mode() && !gp.empty()) {
    if (fsplit > 0)
      while (gp.size() >= 2 && gp.back().h >= fsplit && outer.size() < (size_t)MAX_LEVELS) { outer.insert(outer.begin(), gp.back()); gp.pop_back(); }
    const int64_t c_lo = outer.empty() ? -1 : outer[0].f_lo, c_hi = outer.empty() ? -1 : outer[0].f_hi;
    const TrsmGeom g{left, lower, ta, unit, lower_op, forward, m, n, nt, NBO, npanel, other, alpha,
                     A, lda, B, ldb, D.p, Tw.p + t_rest, W.p};
    rc = strsm_first_fused(g, gp, pfirst, s, sms, c_lo, c_hi);
    if (rc < 0) return rc;
    first_done = rc == 0;
    if (!first_done) {                                // not fusable: no split either
      for (const GeoPair &p : outer) gp.push_back(p);
      outer.clear();
    }
    if (!outer.empty()) {
      // s-block inverses: sub-panel doubling per popped pair on the side stream
      if (cudaStreamWaitEvent(ts->side, ts->ev_fork, 0) != cudaSuccess) return BLAS3_ERR_CUDA;
      for (size_t j = 0; j < outer.size(); ++j) {
        const GeoPair &p = outer[j];
        if ((rc = trsm_panel_doubling(A + p.s_lo * (1 + lda), lda, p.s_hi - p.s_lo, lower,
                                      D.p + pfirst * NBO * NBO + (p.s_lo - pfirst * NBO) * (1 + NBO),
                                      Tw.p + t_rest + t_first, ts->side, sms, ts->ev_ym)))
          return rc;
        if (cudaEventRecord(ts->ev_lvl[j], ts->side) != cudaSuccess) return BLAS3_ERR_CUDA;
      }
    }
  }
  const bool split = !outer.empty();
  if (!first_done) {
    const int64_t o = pfirst * NBO;
    if ((rc = trsm_panel_doubling(A + o * (1 + lda), lda, imin(NBO, nt - o), lower,
                                  D.p + pfirst * NBO * NBO, Tw.p + t_rest, ts->side, sms, ts->ev_lvl)))
      return rc;
  }
  // the other panels' levels (needed one panel sweep later) on a second side
  // stream.  Enqueued AFTER the first panel's launches: the host takes a few
  // microseconds per launch, and the first panel is the critical path (the
  // fused chain started ~125 us late at N = 8192 when these ~8 launches were
  // enqueued before it; profiles/r02_strsm_timeline.md)
  // BLAS3_OPT_TRSM_FUSED = 2 (after the panel solver): the sweep over the
  // other panels as ONE fused launch, holding the last doubling level of
  // those panels (the side stream builds the levels below it)
  const bool fused_sweep = panel_done && opt(BLAS3_OPT_TRSM_FUSED) == 2 && npanel > 1 && nlvl >= 2 &&
                           math_mode() == BLAS3_MATH_3XTF32;
  // the panels the doubling serves: all but the first (and the second when the
  // solver takes it)
  const int64_t prest = forward ? (panel2 ? 2 : 1) : 0, orest = prest * NBO;
  const int64_t nrest = imin(nt, (forward ? npanel : npanel - (panel2 ? 2 : 1)) * NBO) - orest;
  const bool rest_dbl = npanel > 1 && !all_done && nrest > 0;
  if (rest_dbl) {
    if (cudaStreamWaitEvent(ts->side2, ts->ev_fork, 0) != cudaSuccess) return BLAS3_ERR_CUDA;
    // (beside the panel solver, level 0 on CUDA cores in one launch, as for the first panel)
    const int from = panel_done && nlvl >= 1 ? 1 : 0;
    if (from == 1 && (launch_trsm_level0(A + orest * (1 + lda), lda, nrest, lower, D.p + prest * NBO * NBO, NBO,
                                         ts->side2) ||
                      cudaEventRecord(ts->ev_lvl2[0], ts->side2) != cudaSuccess))
      return BLAS3_ERR_CUDA;
    if ((rc = trsm_panel_doubling(A + orest * (1 + lda), lda, nrest, lower, D.p + prest * NBO * NBO, Tw.p,
                                  ts->side2, sms, ts->ev_lvl2, from, fused_sweep ? nlvl - 1 : -1)))
      return rc;
  }
  if (fused_sweep) {
    if (cudaStreamWaitEvent(s, ts->ev_lvl2[nlvl - 2], 0) != cudaSuccess) return BLAS3_ERR_CUDA;
    const TrsmGeom g{left, lower, ta, unit, lower_op, forward, m, n, nt, NBO, npanel, other, alpha,
                     A, lda, B, ldb, D.p, Tw.p, W.p};
    rc = strsm_fused(g, s, sms, true, nlvl - 1);
    if (rc <= 0) return finish(rc);
    // not fusable: the last level on the side stream, then the multi-launch sweep
    if ((rc = trsm_panel_doubling(A + orest * (1 + lda), lda, nrest, lower, D.p + prest * NBO * NBO, Tw.p,
                                  ts->side2, sms, ts->ev_lvl2, nlvl - 1, -1)))
      return rc;
  }
  if (cudaEventRecord(ts->ev_fork2, s) != cudaSuccess) return BLAS3_ERR_CUDA;
  if (!gp.empty() && !first_done && opt(BLAS3_OPT_TRSM_FIRST_YM)) {
    ym_ready = true;
    {
      if (cudaStreamWaitEvent(ts->side3, ts->ev_fork, 0) != cudaSuccess) return BLAS3_ERR_CUDA;
      for (size_t j = 0; j < gp.size(); ++j) {
        const GeoPair &p = gp[j];
        const int64_t ns = p.s_hi - p.s_lo, nf = p.f_hi - p.f_lo;
        int lv = -1;                                    // level that built inv(op(A)_ss)
        for (int64_t w2 = 256; w2 <= p.h; w2 *= 2) ++lv;
        if (lv >= 0 && cudaStreamWaitEvent(ts->side3, ts->ev_lvl[lv], 0) != cudaSuccess) return BLAS3_ERR_CUDA;
        const float *Ds = D.p + (p.s_lo / NBO) * NBO * NBO + (p.s_lo % NBO) * (1 + NBO);
        if (left) {
          // M = inv(op(A)_ss) op(A)_sf : Xb(c,k) = op(A)(s_lo+k, f_lo+c)
          Problem PM = problem(ns, nf, 1.f, 0.f, nullptr, 0, p.M, p.ldm);
          PM.seg[0].a = tri_zeroed(Ds, NBO, true, !lower_op);
          PM.seg[0].b = ta ? dense(A + p.f_lo + p.s_lo * lda, lda, false)
                           : dense(A + p.s_lo + p.f_lo * lda, lda, true);
          PM.seg[0].K = ns;
          PM.rev_m = tri_kle(PM.seg[0].a);
          // Y = alpha inv(op(A)_ss) B_s
          Problem PY = problem(ns, n, alpha, 0.f, nullptr, 0, p.Y, p.ldy);
          PY.seg[0].a = tri_zeroed(Ds, NBO, true, !lower_op);
          PY.seg[0].b = dense(B + p.s_lo, ldb, true);
          PY.seg[0].K = ns;
          PY.rev_m = tri_kle(PY.seg[0].a);
          PY.outer = 1;
          if ((rc = run_problem(PM, ts->side3, sms)) || (rc = run_problem(PY, ts->side3, sms))) return rc;
        } else {
          // M = op(A)_fs inv(op(A)_ss) : Xa(r,k) = op(A)(f_lo+r, s_lo+k), Xb(c,k) = inv(k,c)
          Problem PM = problem(nf, ns, 1.f, 0.f, nullptr, 0, p.M, p.ldm);
          PM.seg[0].a = ta ? dense(A + p.s_lo + p.f_lo * lda, lda, true)
                           : dense(A + p.f_lo + p.s_lo * lda, lda, false);
          PM.seg[0].b = tri_zeroed(Ds, NBO, true, lower_op);
          PM.seg[0].K = ns;
          PM.rev_n = tri_kle(PM.seg[0].b);
          // Y = alpha B_s inv(op(A)_ss)
          Problem PY = problem(m, ns, alpha, 0.f, nullptr, 0, p.Y, p.ldy);
          PY.seg[0].a = dense(B + p.s_lo * ldb, ldb, false);
          PY.seg[0].b = tri_zeroed(Ds, NBO, true, lower_op);
          PY.seg[0].K = ns;
          PY.rev_n = tri_kle(PY.seg[0].b);
          PY.outer = 2;
          if ((rc = run_problem(PM, ts->side3, sms)) || (rc = run_problem(PY, ts->side3, sms))) return rc;
        }
        if (cudaEventRecord(ts->ev_ym[j], ts->side3) != cudaSuccess) return BLAS3_ERR_CUDA;
      }
    }
  }


  // 2. the sweep, independently per slab of the right-hand side (columns of B
  //    for side=L, rows for side=R), each slab on its own stream.
  //    Panels (NBO wide) are visited in dependency order by recursive halving
  //    of the panel range: solve the first half; ONE GEMM update of the second
  //    half by the first (K = nt/2, nt/4, ...); solve the second half.  The
  //    FIRST processed panel is itself halved geometrically down to 256-wide
  //    blocks (its first blocks only need the first doubling levels), so the
  //    sweep starts ~one level after the 128-block inverses instead of after
  //    the whole doubling chain.  A leaf [e0, e0+cnt) -- an aligned block of
  //    width wblk, clipped to the matrix -- is X = a1 * inv(op(A)_blk) * B_blk
  //    with the inverse read from D (the diagonal blocks of a panel inverse
  //    are the inverses of the aligned sub-blocks).  alpha is folded into the
  //    first operation that touches each row (`scaled`).
  const int64_t nslab = trsm_slabs(other);
  for (int64_t q = 0; q < nslab; ++q) {
    const int64_t c0 = align_down(other * q / nslab, 256), c1 = q + 1 == nslab ? other : align_down(other * (q + 1) / nslab, 256);
    cudaStream_t st = nslab == 1 ? s : ts->slab[q];
    if (st != s && cudaStreamWaitEvent(st, ts->ev_fork2, 0) != cudaSuccess) return BLAS3_ERR_CUDA;
    float *Bq = left ? B + c0 * ldb : B + c0;
    float *Wq = left ? W.p + c0 * NBO : W.p + c0;
    const int64_t mq = left ? m : c1 - c0, nq = left ? c1 - c0 : n;
    int waited = first_done ? nlvl : -1;              // highest first-panel level waited on
                                                      // (the fused launch built them all)
    bool waited_rest = all_done;                      // the other panels' inverses waited on

    // leaf: rows (L) / columns (R) [e0, e0 + cnt) of X, aligned block width wblk
    // kernels of the first panel leave SMs to the latency-bound doubling
    // chain of that panel (high-priority side stream)
    const int32_t first_sms = (int32_t)imax(sms / 2, sms - trsm_reserve(nt));
    int64_t app_lo = 0, app_hi = 0;                   // split sweep: updates already applied
    auto leaf = [&](int64_t e0, int64_t cnt, int64_t wblk, bool scaled, bool in_w, bool restrict_sms = true) -> int {
      int rc2;
      int lv = -1;                                    // doubling level that built inv(block)
      for (int64_t w2 = 256; w2 <= wblk; w2 *= 2) ++lv;
      if (e0 / NBO == pfirst) {
        if (lv > waited) {
          if (cudaStreamWaitEvent(st, ts->ev_lvl[lv], 0) != cudaSuccess) return BLAS3_ERR_CUDA;
          waited = lv;
        }
      } else if (lv >= 0 && !waited_rest) {            // full panels: the last level of the rest
        if (cudaStreamWaitEvent(st, ts->ev_lvl2[nlvl - 1], 0) != cudaSuccess) return BLAS3_ERR_CUDA;
        waited_rest = true;
      }
      const float a1 = scaled ? 1.f : alpha;
      const float *Dp = D.p + (e0 / NBO) * NBO * NBO + (e0 % NBO) * (1 + NBO);
      if (left) {
        // X = a1 * inv(op(A)_bb) * B_b: Xa(r,k) = Dop(r,k), Dop = lower_op ? D : D^T
        Problem P = in_w ? problem(cnt, nq, a1, 0.f, nullptr, 0, Bq + e0, ldb)
                         : problem(cnt, nq, a1, 0.f, nullptr, 0, Wq, cnt);
        P.seg[0].a = tri_zeroed(Dp, NBO, true, !lower_op);
        P.seg[0].b = in_w ? dense(Wq, cnt, true) : dense(Bq + e0, ldb, true);
        P.seg[0].K = cnt;
        P.rev_m = tri_kle(P.seg[0].a);
        P.outer = 1;                     // all longest m-rows first (LPT)
        if (e0 / NBO == pfirst && restrict_sms) P.max_sms = first_sms;
        if ((rc2 = run_problem(P, st, sms))) return rc2;
        if (!in_w && launch_copy(Bq + e0, ldb, Wq, cnt, cnt, nq, st)) return BLAS3_ERR_CUDA;
      } else {
        // X = a1 * B_b * inv(op(A)_bb): Xb(c,k) = Dop(k,c) -> TRI swap = lower_op
        Problem P = in_w ? problem(mq, cnt, a1, 0.f, nullptr, 0, Bq + e0 * ldb, ldb)
                         : problem(mq, cnt, a1, 0.f, nullptr, 0, Wq, m);
        P.seg[0].a = in_w ? dense(Wq, m, false) : dense(Bq + e0 * ldb, ldb, false);
        P.seg[0].b = tri_zeroed(Dp, NBO, true, lower_op);
        P.seg[0].K = cnt;
        P.rev_n = tri_kle(P.seg[0].b);
        P.outer = 2;
        if (e0 / NBO == pfirst && restrict_sms) P.max_sms = first_sms;
        if ((rc2 = run_problem(P, st, sms))) return rc2;
        if (!in_w && launch_copy(Bq + e0 * ldb, ldb, Wq, m, mq, cnt, st)) return BLAS3_ERR_CUDA;
      }
      return 0;
    };
    // update: rows (L) / columns (R) [o_lo, o_hi) <- a1 * B_o - op(A)(o, k) X_k, k in [k_lo, k_hi);
    // to_w: the result goes to W (the next operation is the leaf solve of o)
    auto update = [&](int64_t k_lo, int64_t k_hi, int64_t o_lo, int64_t o_hi, float a1, bool to_w,
                      bool restrict_sms = true, int lim = 0) -> int {
      const bool rs = restrict_sms && o_lo / NBO == pfirst && (o_hi - 1) / NBO == pfirst;
      if (left) {   // Xa(r,kk) = op(A)(o_lo+r, k_lo+kk): !ta -> A(o_lo+r, k_lo+kk) rk; ta -> A(k_lo+kk, o_lo+r) kr
        const float *pa = ta ? A + k_lo + o_lo * lda : A + o_lo + k_lo * lda;
        Problem P = to_w ? problem(o_hi - o_lo, nq, -1.f, a1, Bq + o_lo, ldb, Wq, o_hi - o_lo)
                         : problem(o_hi - o_lo, nq, -1.f, a1, Bq + o_lo, ldb, Bq + o_lo, ldb);
        P.seg[0].a = dense(pa, lda, ta);
        P.seg[0].b = dense(Bq + k_lo, ldb, true);
        P.seg[0].K = k_hi - k_lo;
        if (rs) P.max_sms = first_sms;
        if (lim > 0) P.max_sms = lim;
        return run_problem(P, st, sms);
      }
      // B(:,o) <- a1*B(:,o) - X_k * op(A)(k, o):
      // Xb(c,kk) = op(A)(k_lo+kk, o_lo+c): !ta -> A(k_lo+kk, o_lo+c) kr; ta -> A(o_lo+c, k_lo+kk) rk
      const float *pb = ta ? A + o_lo + k_lo * lda : A + k_lo + o_lo * lda;
      Problem P = to_w ? problem(mq, o_hi - o_lo, -1.f, a1, Bq + o_lo * ldb, ldb, Wq, m)
                       : problem(mq, o_hi - o_lo, -1.f, a1, Bq + o_lo * ldb, ldb, Bq + o_lo * ldb, ldb);
      P.seg[0].a = dense(Bq + k_lo * ldb, ldb, false);
      P.seg[0].b = dense(pb, lda, !ta);
      P.seg[0].K = k_hi - k_lo;
      if (rs) P.max_sms = first_sms;
      if (lim > 0) P.max_sms = lim;
      return run_problem(P, st, sms);
    };
    // geometric solve of the aligned block [lo, lo + w) (clipped to nt): the
    // first half (in processing order) recursively, the second as one leaf
    size_t gj = 0;                                    // next geometric pair (processing order)
    std::function<int(int64_t, int64_t, bool)> geo = [&](int64_t lo, int64_t w, bool scaled) -> int {
      int rc2;
      const int64_t e1 = imin(nt, lo + w);
      if (w <= trsm_geo_leaf()) return leaf(lo, e1 - lo, w, scaled, false);
      const int64_t h = w / 2, mid = lo + h;
      if (mid >= e1) return geo(lo, h, scaled);          // upper half empty (ragged end)
      const int64_t f_lo = forward ? lo : mid, f_hi = forward ? mid : e1;   // first half
      const int64_t s_lo = forward ? mid : lo, s_hi = forward ? e1 : mid;   // second half
      if ((rc2 = geo(f_lo, h, scaled))) return rc2;
      if (ym_ready && gj < gp.size() && gp[gj].s_lo == s_lo && gp[gj].f_lo == f_lo && !scaled) {
        // X_s = Y_s - M_sf X_f (Y, M precomputed on the third stream)
        const GeoPair &p = gp[gj];
        if (cudaStreamWaitEvent(st, ts->ev_ym[gj], 0) != cudaSuccess) return BLAS3_ERR_CUDA;
        ++gj;
        const int64_t ns = s_hi - s_lo, nf = f_hi - f_lo;
        if (left) {
          Problem P = problem(ns, nq, -1.f, 1.f, p.Y + c0 * p.ldy, p.ldy, Bq + s_lo, ldb);
          P.seg[0].a = dense(p.M, p.ldm, false);
          P.seg[0].b = dense(Bq + f_lo, ldb, true);
          P.seg[0].K = nf;
          P.max_sms = first_sms;
          return run_problem(P, st, sms);
        }
        Problem P = problem(mq, ns, -1.f, 1.f, p.Y + c0, p.ldy, Bq + s_lo * ldb, ldb);
        P.seg[0].a = dense(Bq + f_lo * ldb, ldb, false);
        P.seg[0].b = dense(p.M, p.ldm, true);
        P.seg[0].K = nf;
        P.max_sms = first_sms;
        return run_problem(P, st, sms);
      }
      if ((rc2 = update(f_lo, f_hi, s_lo, s_hi, scaled ? 1.f : alpha, true))) return rc2;
      return leaf(s_lo, s_hi - s_lo, h, true, true);
    };
    auto elem = [&](int64_t qa, int64_t qb, int64_t &lo, int64_t &hi) {  // processing -> elements
      const int64_t pa = forward ? qa : npanel - qb, pb = forward ? qb : npanel - qa;
      lo = pa * NBO;
      hi = imin(nt, pb * NBO);
    };
    // in_w: the rows (L) / columns (R) of a single-panel range were left in W
    // (already updated) by the preceding update, so the solve reads W and writes
    // B directly -- no copy-back.
    std::function<int(int64_t, int64_t, bool, bool)> rec = [&](int64_t q0, int64_t q1, bool scaled,
                                                               bool in_w) -> int {
      int rc2;
      if (q1 - q0 == 1) {
        const int64_t p = forward ? q0 : npanel - 1 - q0;
        const int64_t p0 = p * NBO, pr = imin(NBO, nt - p0);
        if (q0 == 0) return first_done ? 0 : geo(p0, NBO, scaled);   // the first processed panel
        if (q0 == 1 && panel2) {                       // the second, by the solver, in place
          const TrsmGeom g{left, lower, ta, unit, lower_op, forward, m, n, nt, NBO, npanel, other, alpha,
                           A, lda, B, ldb, D.p, Tw.p, W.p};
          if (cudaStreamWaitEvent(st, ts->ev_ym[0], 0) != cudaSuccess) return BLAS3_ERR_CUDA;
          return strsm_panel_run(g, p, Mw2, reinterpret_cast<uint8_t *>(Mw.p) + m_bytes, st, sms);
        }
        return leaf(p0, pr, NBO, scaled, in_w);
      }
      const int64_t mid = q0 + (q1 - q0) / 2;
      if ((rc2 = rec(q0, mid, scaled, false))) return rc2;
      int64_t k_lo, k_hi, o_lo, o_hi;
      elem(q0, mid, k_lo, k_hi);                       // solved part
      elem(mid, q1, o_lo, o_hi);                       // part to update
      if (split) {                                     // updates applied by the split sweep
        if (forward && k_lo < app_hi) k_lo = imax(k_lo, app_hi);
        if (!forward && k_hi > app_lo) k_hi = imin(k_hi, app_lo);
      }
      // updated panel goes straight to W (not the solver's: it works in place)
      const bool to_w = (q1 - mid == 1) && !(mid == 1 && panel2);
      // (before the second panel's solve, optionally leave SMs to the side
      // streams: BLAS3_PANEL2_FREE SMs, default 0)
      static const int64_t p2_free = [] { const char *e = getenv("BLAS3_PANEL2_FREE"); return e ? atoll(e) : 0; }();
      const int lim = mid == 1 && panel2 && p2_free > 0 ? (int)imax(2, sms - p2_free) : 0;
      if ((rc2 = update(k_lo, k_hi, o_lo, o_hi, scaled ? 1.f : alpha, to_w, true, lim))) return rc2;
      return rec(mid, q1, true, to_w);
    };
    if (split) {
      // right-looking over the popped pairs: the block solved last [a_lo, a_hi)
      // updates every later row (L) / column (R) in one bulk GEMM, then the
      // next s block is one leaf (its inverse from the side stream)
      int64_t a_lo = outer[0].f_lo, a_hi = outer[0].f_hi;
      for (size_t j = 0; j < outer.size(); ++j) {
        const GeoPair &p = outer[j];
        const int64_t r_lo = forward ? a_hi : 0, r_hi = forward ? nt : a_lo;
        // when s is all that is left, the update goes to W and the leaf reads W
        const bool last = r_lo == p.s_lo && r_hi == p.s_hi;
        if ((rc = update(a_lo, a_hi, r_lo, r_hi, j == 0 ? alpha : 1.f, last, false))) return rc;
        if (cudaStreamWaitEvent(st, ts->ev_lvl[j], 0) != cudaSuccess) return BLAS3_ERR_CUDA;
        if ((rc = leaf(p.s_lo, p.s_hi - p.s_lo, p.h, true, last, false))) return rc;
        a_lo = p.s_lo; a_hi = p.s_hi;
      }
      app_lo = forward ? 0 : a_hi;                    // k ranges whose update is applied
      app_hi = forward ? a_lo : nt;
    }
    if ((rc = rec(0, npanel, split, false))) return rc;
    if (st != s && (cudaEventRecord(ts->ev_join[q], st) != cudaSuccess ||
                    cudaStreamWaitEvent(s, ts->ev_join[q], 0) != cudaSuccess)) return BLAS3_ERR_CUDA;
  }
  if (ym_ready && cudaStreamWaitEvent(s, ts->ev_ym[gp.size() - 1], 0) != cudaSuccess)
    return BLAS3_ERR_CUDA;
  if (split && cudaStreamWaitEvent(s, ts->ev_lvl[outer.size() - 1], 0) != cudaSuccess)
    return BLAS3_ERR_CUDA;
  // the side streams' last levels are part of this call (scratch is freed on s)
  if (!first_done && nlvl > 0 && cudaStreamWaitEvent(s, ts->ev_lvl[nlvl - 1], 0) != cudaSuccess)
    return BLAS3_ERR_CUDA;
  if (nlvl > 0 && rest_dbl && cudaStreamWaitEvent(s, ts->ev_lvl2[nlvl - 1], 0) != cudaSuccess)
    return BLAS3_ERR_CUDA;
  if (panel2 && cudaStreamWaitEvent(s, ts->ev_ym[0], 0) != cudaSuccess) return BLAS3_ERR_CUDA;
  return finish(0);
}

}  // extern "C"
