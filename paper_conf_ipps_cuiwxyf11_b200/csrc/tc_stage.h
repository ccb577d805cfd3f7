// tc_stage.h -- staging helpers shared by the tcgen05 kernels (tc_kernel.cu,
// panel_kernel.cu): the 3xTF32 lo split, the UMMA shared-memory descriptors of
// the two staged tile layouts, and the acquire poll of a global counter.
#pragma once
#include <stdint.h>
#include "tc_ptx.h"

namespace blas3 {
namespace stage {

constexpr int BK = 32;                       // k-block (elements)
constexpr int LAYOUT_K = 0, LAYOUT_MN = 1;   // K-major / MN-major staged tile

// 3xTF32 split without rewriting hi: kind::tf32 UMMA reads the raw fp32
// word and ignores its low 13 mantissa bits, i.e. it consumes
// hi = trunc_tf32(x) directly from the TMA-staged tile (pinned by
// tests/test_parity_gpu.py::test_split_is_real).  Only lo = x - hi (exact in
// fp32: the 13 bits below hi) is produced; the tensor core reads its top 11
// bits the same way, so hi + tf32(lo) represents x to within 2^-21 |x|, far
// below the K-linear accumulation error of the fp32 TMEM accumulator
// (Q17, Q24).  Two ops per element (LOP + FADD).
__device__ __forceinline__ float split_lo(float x) {
  const float hi = __uint_as_float(__float_as_uint(x) & 0xFFFFE000u);
  return x - hi;
}
// lo of a whole staged tile (either layout: the split is elementwise), NT threads
template <int NT>
__device__ __forceinline__ void split_pass(const uint8_t *raw, uint8_t *lo, uint32_t bytes, int t) {
  const float4 *r4 = reinterpret_cast<const float4 *>(raw);
  float4 *l4 = reinterpret_cast<float4 *>(lo);
#pragma unroll 4
  for (uint32_t c = t; c < bytes / 16; c += NT) {
    const float4 v = r4[c];
    float4 l;
    l.x = split_lo(v.x);
    l.y = split_lo(v.y);
    l.z = split_lo(v.z);
    l.w = split_lo(v.w);
    l4[c] = l;
  }
}

// UMMA descriptor of k8-step k8 of a staged tile at shared address base:
// MN-major 32-element chunks BK*128 B apart (SWIZZLE_128B_BASE32B), or K-major
// 128-B rows in 8-row atoms (SWIZZLE_128B)
__device__ __forceinline__ uint64_t op_desc(uint32_t base, int lay, int k8) {
  if (lay == LAYOUT_MN) return ptx::smem_desc(base + k8 * 1024, BK * 128, 512, 1);
  return ptx::smem_desc(base + k8 * 32, 16, 1024, 2);
}

// One thread waits until *ctr >= target (gpu-scope acquire: the stores that
// preceded the producers' release are visible afterwards).  A dependency that
// is never satisfied traps after 4 s instead of hanging the device.
__device__ __forceinline__ void spin_until(const uint32_t *ctr, uint32_t target, unsigned sleep_ns = 128) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
  if (v >= target) return;
  unsigned long long t0, t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  for (;;) {
    __nanosleep(sleep_ns);
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
    if (v >= target) return;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t - t0 > 4000000000ull) __trap();
  }
}

}  // namespace stage
}  // namespace blas3
