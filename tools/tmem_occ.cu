// tmem_occ.cu — do kernels that use tcgen05.alloc run more than one CTA per SM?
// Launch 148*8 CTAs of 128 threads that each spin ~50 us; compare a plain kernel with one
// that allocates 32 / 128 TMEM columns.  Build + run:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tmem_occ tools/tmem_occ.cu
#include <cstdio>
#include <cuda_runtime.h>
typedef unsigned int u32;

template <int COLS>
__global__ void spin(long long cycles, int* maxconc, int* conc) {
  __shared__ u32 slot;
  if (COLS > 0) {
    if (threadIdx.x < 32) {
      asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                       (u32)__cvta_generic_to_shared(&slot)), "r"(COLS) : "memory");
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
  }
  u32 smid;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
  if (threadIdx.x == 0) {
    int c = atomicAdd(&conc[smid], 1) + 1;
    atomicMax(&maxconc[smid], c);
  }
  long long t0 = clock64();
  while (clock64() - t0 < cycles) {}
  __syncthreads();
  if (threadIdx.x == 0) atomicSub(&conc[smid], 1);
  if (COLS > 0) {
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    if (threadIdx.x < 32)
      asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(slot), "r"(COLS) : "memory");
  }
}

template <int COLS>
void run(const char* name) {
  int *mc, *c;
  cudaMalloc(&mc, 4096);
  cudaMalloc(&c, 4096);
  cudaMemset(mc, 0, 4096);
  cudaMemset(c, 0, 4096);
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, spin<COLS>, 128, 0);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  spin<COLS><<<148, 128>>>(1000, mc, c);
  cudaDeviceSynchronize();
  cudaMemset(mc, 0, 4096);
  cudaEventRecord(a);
  spin<COLS><<<148 * 8, 128>>>(100000, mc, c);
  cudaEventRecord(b);
  cudaError_t e = cudaDeviceSynchronize();
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  int h[1024];
  cudaMemcpy(h, mc, 4096, cudaMemcpyDeviceToHost);
  int mx = 0;
  for (int i = 0; i < 148; ++i) mx = h[i] > mx ? h[i] : mx;
  printf("%-12s occupancy-api %d  time %.3f ms  max concurrent CTAs/SM %d  %s\n", name, occ, ms, mx,
         cudaGetErrorString(e));
}

int main() {
  run<0>("plain");
  run<32>("tmem32");
  run<128>("tmem128");
  run<256>("tmem256");
  return 0;
}
