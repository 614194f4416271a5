// tmem_bench.cu — microbenchmark: tcgen05.ld / tcgen05.st throughput per SM on sm_100a,
// against LDS.64 for comparison.  Decides whether TMEM can hold a stencil's
// streamed-direction queue.  Build + run:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tmem_bench tools/tmem_bench.cu
//   /tmp/tmem_bench
#include <cstdio>
#include <cuda_runtime.h>

typedef unsigned int u32;

__device__ __forceinline__ void tm_alloc(u32* slot, u32 ncols) {
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                   (u32)__cvta_generic_to_shared(slot)),
               "r"(ncols)
               : "memory");
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tm_dealloc(u32 taddr, u32 ncols) {
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols)
               : "memory");
}

#define LD16(taddr, r)                                                                         \
  asm volatile(                                                                                \
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13," \
      "%14,%15}, [%16];"                                                                       \
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),   \
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]),            \
        "=r"(r[13]), "=r"(r[14]), "=r"(r[15])                                                  \
      : "r"(taddr))
#define ST16(taddr, r)                                                                         \
  asm volatile(                                                                                \
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12," \
      "%13,%14,%15,%16};" ::"r"(taddr),                                                        \
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), \
      "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]),       \
      "r"(r[15])                                                                               \
      : "memory")

// mode 0: ld only (wait every NB loads), 1: st only, 2: ld+st, 3: LDS.64 reference,
// 4: LDTM and LDS.64 interleaved (do the two pipes add up?)
template <int MODE, int NB>
__global__ void bench(int iters, unsigned long long* out, u32* sink) {
  __shared__ u32 slot;
  __shared__ double sm[4096];
  const int warp = threadIdx.x / 32;
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) sm[i] = i;
  if (MODE != 3) {
    if (warp == 0) tm_alloc(&slot, 512);
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
  } else {
    __syncthreads();
  }
  const u32 base = MODE != 3 ? slot : 0;
  // warp w -> lanes 32*(w%4); columns by warp group (w/4)
  const u32 lane_off = (u32)((warp % 4) * 32) << 16;
  const int ngroups = blockDim.x / 128 > 0 ? blockDim.x / 128 : 1;
  const u32 colspan = 512 / ngroups;
  const u32 col0 = (warp / 4) * colspan;
  u32 acc = 0;
  u32 r[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) r[i] = threadIdx.x + i;
  double dacc = 0;
  __syncthreads();
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int b = 0; b < NB; ++b) {
      const u32 col = col0 + ((it * NB + b) * 16) % colspan;
      const u32 ta = base + lane_off + col;
      if (MODE == 0 || MODE == 2 || MODE == 4) LD16(ta, r);
      if (MODE == 1 || MODE == 2) {
        if (MODE == 2) asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        ST16(ta, r);
      }
      if (MODE == 3 || MODE == 4) {
        const double* p = sm + ((threadIdx.x + it * 7 + b * 33) & 3583);
        dacc += p[0] + p[64] + p[128] + p[192] + p[256] + p[320] + p[384] + p[448];
      }
    }
    if (MODE == 0 || MODE == 4) {
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
      for (int i = 0; i < 16; ++i) acc += r[i];
    }
    if (MODE == 1 || MODE == 2) asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
  if (acc == 0xdeadbeef || dacc == -1.0) sink[0] = acc;
  if (MODE != 3) {
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    if (warp == 0) tm_dealloc(base, 512);
  }
}

template <int MODE, int NB>
void run(const char* name, int threads) {
  const int blocks = 148, iters = 4000;
  unsigned long long* d;
  u32* sink;
  cudaMalloc(&d, blocks * 8);
  cudaMalloc(&sink, 4);
  bench<MODE, NB><<<blocks, threads>>>(10, d, sink);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a);
  bench<MODE, NB><<<blocks, threads>>>(iters, d, sink);
  cudaEventRecord(b);
  cudaError_t e = cudaDeviceSynchronize();
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  unsigned long long h[148];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  double cyc = 0;
  for (int i = 0; i < blocks; ++i) cyc += h[i];
  cyc /= blocks;
  // bytes per SM moved: threads * iters * NB * 64 B (16 x 32-bit) ; LDS: 8 doubles
  const double bytes = (double)threads * iters * NB * 64.0;
  printf("%-10s threads %4d: %s  %.3f ms  %.0f cyc  %.1f B/clk/SM  %.2f TB/s/SM\n", name, threads,
         e == cudaSuccess ? "ok" : cudaGetErrorString(e), ms, cyc, bytes / cyc,
         bytes / (ms * 1e-3) / 1e12);
  cudaFree(d);
  cudaFree(sink);
}

int main() {
  for (int t : {128, 256, 512}) {
    run<0, 4>("tmem_ld", t);
    run<0, 1>("tmem_ld_w1", t);
    run<4, 4>("ldtm+lds", t);
    run<1, 4>("tmem_st", t);
    run<2, 4>("tmem_ldst", t);
    run<3, 4>("lds64", t);
  }
  return 0;
}
