// cst_ptx.cuh — inline-PTX helpers for sm_100a: mbarrier, TMA (cp.async.bulk.tensor),
// proxy fences.  Compiled by NVRTC as part of every kernel variant.
#ifndef CST_PTX_CUH
#define CST_PTX_CUH

typedef unsigned int u32;
typedef unsigned long long u64;

__device__ __forceinline__ u32 smem_u32(const void* p) {
  return (u32)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ void mbar_init(u64* bar, u32 count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count)
               : "memory");
}

__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(u64* bar, u32 bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void mbar_arrive(u64* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void mbar_wait(u64* bar, u32 parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "LAB_WAIT:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra LAB_DONE;\n\t"
      "bra LAB_WAIT;\n"
      "LAB_DONE:\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

// 3-D TMA tile load global -> shared, completion signalled on `bar` (complete_tx bytes).
__device__ __forceinline__ void tma_load_3d(void* dst, const void* tmap, u64* bar, int c0,
                                            int c1, int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(smem_u32(dst)),
      "l"((u64)tmap), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2)
      : "memory");
}

__device__ __forceinline__ void tma_prefetch_desc(const void* tmap) {
  asm volatile("prefetch.tensormap [%0];" ::"l"((u64)tmap) : "memory");
}

__device__ __forceinline__ double ldg_nc(const double* p) { return __ldg(p); }

// ---- tensor memory (TMEM) as a per-thread queue store (qstore = 2) --------
// 128 lanes x 512 columns x 32 bit per SM; warp w reaches lanes 32*(w%4) .. +31.  Measured
// on B200 (tools/tmem_bench.cu): tcgen05.ld 430-1030 B/clk/SM, tcgen05.st 230-360 B/clk/SM,
// and LDTM runs beside LDS (the shared-memory pipe is not shared).
__device__ __forceinline__ void tmem_alloc(u32* slot, u32 ncols) {  // whole warp
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                   smem_u32(slot)),
               "r"(ncols)
               : "memory");
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_dealloc(u32 taddr, u32 ncols) {  // whole warp
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols)
               : "memory");
}
__device__ __forceinline__ void tmem_fence_before_sync() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tmem_fence_after_sync() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tmem_wait_st() {
  asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ double tmem_d(u32 lo, u32 hi) {
  return __hiloint2double((int)hi, (int)lo);
}
// one double into columns [taddr, taddr + 1] of the thread's lane
__device__ __forceinline__ void tmem_st_d(u32 taddr, double v) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x2.b32 [%0], {%1, %2};" ::"r"(taddr),
               "r"((u32)__double2loint(v)), "r"((u32)__double2hiint(v)));
}
// Split-phase queue load: tmem_ld_issue starts the loads of a point's ring — R doubles
// (in logical plane order, from rotating slots) and the partial output A — into raw
// 32-bit registers;
// tmem_ld_wait completes every outstanding tcgen05.ld of the thread and takes the registers
// as in-out operands, so no use of them can be scheduled above it.
template <int R_>
struct TmQ {
  u32 r[2 * R_ + 2];
};
// ring in logical order: q.r[2m..2m+1] <- columns ta[m] (m < R), A <- column tb
template <int R_>
__device__ __forceinline__ void tmem_ld_issue(const u32 (&ta)[R_], u32 tb, TmQ<R_>& q) {
#define CST_LDTM2(i, a) \
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x2.b32 {%0, %1}, [%2];" \
               : "=r"(q.r[2 * (i)]), "=r"(q.r[2 * (i) + 1]) : "r"(a) : "memory")
#pragma unroll
  for (int m = 0; m < R_; ++m) CST_LDTM2(m, ta[m]);
  CST_LDTM2(R_, tb);
#undef CST_LDTM2
}
template <int R_>
__device__ __forceinline__ void tmem_ld_wait(TmQ<R_>& q) {
  if constexpr (R_ == 1) {
    asm volatile("tcgen05.wait::ld.sync.aligned;"
                 : "+r"(q.r[0]), "+r"(q.r[1]), "+r"(q.r[2]), "+r"(q.r[3]));
  } else if constexpr (R_ == 2) {
    asm volatile("tcgen05.wait::ld.sync.aligned;"
                 : "+r"(q.r[0]), "+r"(q.r[1]), "+r"(q.r[2]), "+r"(q.r[3]), "+r"(q.r[4]),
                   "+r"(q.r[5]));
  } else if constexpr (R_ == 3) {
    asm volatile("tcgen05.wait::ld.sync.aligned;"
                 : "+r"(q.r[0]), "+r"(q.r[1]), "+r"(q.r[2]), "+r"(q.r[3]), "+r"(q.r[4]),
                   "+r"(q.r[5]), "+r"(q.r[6]), "+r"(q.r[7]));
  } else {
    asm volatile("tcgen05.wait::ld.sync.aligned;"
                 : "+r"(q.r[0]), "+r"(q.r[1]), "+r"(q.r[2]), "+r"(q.r[3]), "+r"(q.r[4]),
                   "+r"(q.r[5]), "+r"(q.r[6]), "+r"(q.r[7]), "+r"(q.r[8]), "+r"(q.r[9]));
  }
}
template <int R_>
__device__ __forceinline__ double tmq_u(const TmQ<R_>& q, int s) {  // ring slot s
  return tmem_d(q.r[2 * s], q.r[2 * s + 1]);
}
template <int R_>
__device__ __forceinline__ double tmq_a(const TmQ<R_>& q) {  // the partial output A
  return tmem_d(q.r[2 * R_], q.r[2 * R_ + 1]);
}

// Raw split-phase TMEM access for wider rings (hypterm: 5 doubles per plane slot).  The
// loads carry outputs only; tmem_wait_ld() completes them and tmem_pin() then passes each
// register through an empty volatile asm so that no use is scheduled above the wait.
__device__ __forceinline__ void tmem_ld_x8(u32 a, u32* r) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]),
                 "=r"(r[6]), "=r"(r[7])
               : "r"(a)
               : "memory");
}
__device__ __forceinline__ void tmem_ld_x2(u32 a, u32* r) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x2.b32 {%0, %1}, [%2];"
               : "=r"(r[0]), "=r"(r[1])
               : "r"(a)
               : "memory");
}
__device__ __forceinline__ void tmem_wait_ld() {
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
template <int N>
__device__ __forceinline__ void tmem_pin(u32 (&r)[N]) {
#pragma unroll
  for (int i = 0; i < N; ++i) asm volatile("" : "+r"(r[i]));
}
// five doubles into columns [a, a + 10)
__device__ __forceinline__ void tmem_st_5d(u32 a, const double* v) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"r"(a),
      "r"((u32)__double2loint(v[0])), "r"((u32)__double2hiint(v[0])),
      "r"((u32)__double2loint(v[1])), "r"((u32)__double2hiint(v[1])),
      "r"((u32)__double2loint(v[2])), "r"((u32)__double2hiint(v[2])),
      "r"((u32)__double2loint(v[3])), "r"((u32)__double2hiint(v[3])));
  asm volatile("tcgen05.st.sync.aligned.32x32b.x2.b32 [%0], {%1, %2};" ::"r"(a + 8),
               "r"((u32)__double2loint(v[4])), "r"((u32)__double2hiint(v[4])));
}

#endif
