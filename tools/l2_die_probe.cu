// l2_die_probe.cu — DESIGN.md §4.3: does a line cached for one half of the SMs serve the other half from L2?
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o l2die tools/l2_die_probe.cu; ncu --metrics dram__bytes_read.sum --cache-control none -k regex:rd -s 1 -c 3 ./l2die [eo]
// Does a line cached by one die's SMs serve the other die's SMs from L2?
// Phase kernels read a 48 MB buffer from CTAs on SMs with smid < SPLIT (or >= SPLIT) only.
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ unsigned smid() { unsigned r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }
__global__ void rd(const double2* __restrict__ x, size_t n, int lo, int hi, double* sink, int* cnt,
                   int parity) {
  __shared__ int slot;
  const unsigned s = smid();
  if (parity >= 0) { if ((int)(s & 1) != parity) return; }
  else if (s < (unsigned)lo || s >= (unsigned)hi) return;
  if (threadIdx.x == 0) slot = atomicAdd(cnt, 1);
  __syncthreads();
  const int nct = parity >= 0 ? 74 : hi - lo;  // one CTA per eligible SM does the work (extra CTAs exit)
  if (slot >= nct) return;
  double acc = 0;
  for (size_t i = (size_t)slot * blockDim.x + threadIdx.x; i < n; i += (size_t)nct * blockDim.x) {
    double2 v = x[i]; acc += v.x + v.y;
  }
  if (acc == 12345.678) sink[0] = acc;
}
int main(int argc, char** argv) {
  const size_t bytes = 48ull << 20, n = bytes / 16;
  double2* x; double* sink; int* cnt;
  cudaMalloc(&x, bytes); cudaMalloc(&sink, 8); cudaMalloc(&cnt, 4 * 8);
  cudaMemset(x, 0, bytes); cudaMemset(cnt, 0, 32);
  int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  const int split = nsm / 2;
  // warm-up launch, then: A = [0, split) reads; B = [split, nsm) reads; C = [0, split) again
  const bool eo = argc > 1;
  rd<<<nsm * 8, 512>>>(x, n, 0, nsm, sink, cnt + 0, -1);
  cudaMemset(cnt, 0, 32);
  // flush L2 with a big unrelated buffer
  char* f; cudaMalloc(&f, 512ull << 20); cudaMemset(f, 1, 512ull << 20);
  rd<<<nsm * 8, 512>>>(x, n, 0, split, sink, cnt + 1, eo ? 0 : -1);      // phase A
  rd<<<nsm * 8, 512>>>(x, n, split, nsm, sink, cnt + 2, eo ? 1 : -1);    // phase B: other SMs
  rd<<<nsm * 8, 512>>>(x, n, 0, split, sink, cnt + 3, eo ? 0 : -1);      // phase C: A's SMs
  cudaDeviceSynchronize();
  printf("nsm %d split %d err %s\n", nsm, split, cudaGetErrorString(cudaGetLastError()));
  return 0;
}
