// peak.cu — FP64 FMA throughput microbenchmark (the FP64 roofline denominator, which
// MEASURED_PEAKS.json does not provide): every thread runs 8 independent DFMA chains.
#include "internal.h"

namespace {

__global__ void dfma_kernel(double* out, int iters, double a, double b) {
  double x[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) x[k] = threadIdx.x * 1e-9 + k;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 8; ++k) x[k] = fma(x[k], a, b);
  }
  double s = 0;
#pragma unroll
  for (int k = 0; k < 8; ++k) s += x[k];
  if (s == 1234.5678) out[blockIdx.x] = s;  // keep the chains alive
}

}  // namespace

extern "C" cst_status cst_fp64_peak(int device, double* tflops, double* sm_clock_ghz) {
  if (!tflops) return cst::fail(CST_E_INVALID, "null argument");
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess || n == 0) {
    cudaGetLastError();
    return cst::fail(CST_E_CUDA, "no CUDA device available");
  }
  CST_CUDA(cudaSetDevice(device));
  int sms = 0;
  CST_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device));
  double* out = nullptr;
  CST_CUDA(cudaMalloc(&out, sizeof(double) * 65536));
  const int blocks = sms * 8, threads = 256, iters = 1 << 16;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  dfma_kernel<<<blocks, threads>>>(out, 1024, 0.999999, 1e-7);  // warm-up
  cudaEventRecord(e0);
  dfma_kernel<<<blocks, threads>>>(out, iters, 0.999999, 1e-7);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaFree(out);
  CST_CUDA(cudaGetLastError());
  const double flops = 2.0 * 8.0 * (double)iters * blocks * threads;
  *tflops = flops / (ms * 1e-3) / 1e12;
  if (sm_clock_ghz) {
    int khz = 0;
    cudaDeviceGetAttribute(&khz, cudaDevAttrClockRate, device);
    *sm_clock_ghz = khz * 1e-6;
  }
  return CST_OK;
}
