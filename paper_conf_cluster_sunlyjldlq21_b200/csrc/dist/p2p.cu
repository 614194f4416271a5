// p2p.cu — device-side ordering of the fused peer-memory halo exchange (dist.cpp,
// SURVEY §8(f) NEXT-3): flag words written over CUDA IPC mappings (NVLink / NVSwitch on a
// multi-GPU node) with release stores and polled with acquire loads.
#include "../runtime/internal.h"

namespace {

__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void st_release_sys(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ unsigned long long globaltimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Runs after the stream's previous kernels (whose stores, local and remote, are complete);
// the system-scope fence orders them before the flag for the observer on the peer GPU.
__global__ void signal_kernel(unsigned long long* f0, unsigned long long* f1,
                              unsigned long long value) {
  __threadfence_system();
  if (f0) st_release_sys(f0, value);
  if (f1) st_release_sys(f1, value);
}

__global__ void wait_kernel(const unsigned long long* f0, unsigned long long t0,
                            const unsigned long long* f1, unsigned long long t1) {
  const unsigned long long start = globaltimer();
  const unsigned long long limit = 30ull * 1000 * 1000 * 1000;  // ns
  while ((f0 && ld_acquire_sys(f0) < t0) || (f1 && ld_acquire_sys(f1) < t1)) {
    __nanosleep(256);
    if (globaltimer() - start > limit) __trap();  // a dead or desynchronised peer
  }
}

}  // namespace

namespace cst {

cst_status p2p_signal(cudaStream_t s, unsigned long long* f0, unsigned long long* f1,
                      unsigned long long value) {
  signal_kernel<<<1, 1, 0, s>>>(f0, f1, value);
  CST_CUDA(cudaGetLastError());
  return CST_OK;
}

cst_status p2p_wait(cudaStream_t s, const unsigned long long* f0, unsigned long long t0,
                    const unsigned long long* f1, unsigned long long t1) {
  wait_kernel<<<1, 1, 0, s>>>(f0, t0, f1, t1);
  CST_CUDA(cudaGetLastError());
  return CST_OK;
}

}  // namespace cst
