// Throughput probe: FP64 DFMA (CUDA cores) vs DMMA m8n8k4 (mma.sync f64) on
// one B200, all SMs, register operands only (no memory traffic).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o dmma_rate dmma_rate.cu
#include <cstdio>
#include <cuda_runtime.h>

__global__ void dfma_loop(double *out, int iters) {
  double a[16];
  for (int i = 0; i < 16; ++i) a[i] = threadIdx.x * 1e-3 + i;
  const double b = 1.0000001, c = 1e-9;
  for (int t = 0; t < iters; ++t)
#pragma unroll
    for (int i = 0; i < 16; ++i) a[i] = fma(a[i], b, c);
  double s = 0;
  for (int i = 0; i < 16; ++i) s += a[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void dmma_loop(double *out, int iters) {
  double acc[8][2];
  for (int i = 0; i < 8; ++i) { acc[i][0] = threadIdx.x; acc[i][1] = 1.0; }
  double a = 1.0000001 + threadIdx.x * 1e-9, b = 0.9999999;
  for (int t = 0; t < iters; ++t) {
#pragma unroll
    for (int i = 0; i < 8; ++i)
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0, %1}, {%2}, {%3}, {%0, %1};"
                   : "+d"(acc[i][0]), "+d"(acc[i][1]) : "d"(a), "d"(b));
  }
  double s = 0;
  for (int i = 0; i < 8; ++i) s += acc[i][0] + acc[i][1];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double *out;
  cudaMalloc(&out, sizeof(double) * sms * 8 * 1024);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int iters = 20000;
  for (int warps = 4; warps <= 32; warps *= 2) {
    const int thr = warps * 32;
    dfma_loop<<<sms, thr>>>(out, 10);
    cudaEventRecord(e0);
    dfma_loop<<<sms, thr>>>(out, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    const double fl = 2.0 * 16 * iters * (double)thr * sms;
    printf("DFMA  warps/SM %2d: %.1f TFLOP/s\n", warps, fl / ms / 1e9);
    dmma_loop<<<sms, thr>>>(out, 10);
    cudaEventRecord(e0);
    dmma_loop<<<sms, thr>>>(out, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    const double fl2 = 2.0 * 8 * 8 * 4 * 8 * (double)iters * warps * sms;   // 8 MMAs of 8x8x4 per warp-iteration
    printf("DMMA  warps/SM %2d: %.1f TFLOP/s\n", warps, fl2 / ms / 1e9);
  }
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
