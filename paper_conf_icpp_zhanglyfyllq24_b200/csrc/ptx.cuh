// ptx.cuh -- thin inline-PTX wrappers for sm_100a: mbarrier, bulk TMA, cp.async,
// tcgen05 (alloc, cp, mma, mma.sp, commit, ld), clusters, programmatic launch.
// Product code (libjigsaw.so).  Layout notes are in DESIGN.md §5.
#pragma once
#include <cstdint>
#include <cuda.h>

namespace jig {

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ---------------------------------------------------------------- mbarrier
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void fence_barrier_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra DONE_%=;\n\t"
      "bra WAIT_%=;\n"
      "DONE_%=:\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

// ---------------------------------------------------------------- TMA
// 1-D bulk copy global -> shared, completes `bytes` on the mbarrier.
// Explicit shared-space accesses (a generic LD/ST on a shared address would take
// the generic path and queue behind global traffic in L1TEX).
__device__ __forceinline__ int32_t ld_shared_s32(uint32_t saddr) {
  int32_t v;
  asm volatile("ld.shared.b32 %0, [%1];" : "=r"(v) : "r"(saddr) : "memory");
  return v;
}
__device__ __forceinline__ void st_shared_s32(uint32_t saddr, int32_t v) {
  asm volatile("st.shared.b32 [%0], %1;" ::"r"(saddr), "r"(v) : "memory");
}
__device__ __forceinline__ uint4 ld_shared_v4u(uint32_t saddr) {
  uint4 v;
  asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(saddr)
               : "memory");
  return v;
}
__device__ __forceinline__ void st_shared_v4u(uint32_t saddr, uint4 v) {
  asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(saddr), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}
// Prefetch `bytes` (multiple of 16, 16-byte aligned) of global memory into L2.
__device__ __forceinline__ void bulk_prefetch_l2(const void* src, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(src), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
// Bulk copy shared::cta -> shared::cluster (a peer CTA's shared memory, or this
// CTA's), completing `bytes` transaction bytes on the mbarrier at shared::cluster
// address `rbar` (in the destination CTA).
__device__ __forceinline__ void bulk_s2cluster(uint32_t rdst, uint32_t src, uint32_t bytes, uint32_t rbar) {
  asm volatile("cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   rdst),
               "r"(src), "r"(bytes), "r"(rbar)
               : "memory");
}
// ---------------------------------------------------------------- tcgen05
template <uint32_t kCols>
__device__ __forceinline__ void tmem_alloc(uint32_t* dst_smem) {  // whole warp
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                   smem_u32(dst_smem)),
               "n"(kCols));
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
}
template <uint32_t kCols>
__device__ __forceinline__ void tmem_dealloc(uint32_t taddr) {  // whole warp
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "n"(kCols));
}
__device__ __forceinline__ void tc_fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
// D[tmem] (+)= A[smem, 2:4 compressed] . B[smem], metadata at [tmem_e].
__device__ __forceinline__ void tc_mma_sp_f16(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc,
                                              uint32_t e_tmem, uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %5, 0;\n\t"
      "tcgen05.mma.sp.cta_group::1.kind::f16 [%0], %1, %2, [%3], %4, p;\n\t}" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(e_tmem), "r"(idesc), "r"(accumulate)
      : "memory");
}
// Dense: D[tmem] (+)= A[smem] . B[smem]  (K = 16 for f16).
__device__ __forceinline__ void tc_mma_f16(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc,
                                           uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}
// 32 lanes (this warp's quarter) x 32 consecutive 32-bit columns.
__device__ __forceinline__ void tc_ld_32x32b_x32(uint32_t taddr, uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
      "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]),
        "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]),
        "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
}
__device__ __forceinline__ void tc_wait_ld() {
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
// TMEM store of 32 columns x 32 lanes (one 32-bit value per lane and column):
// the inverse of tc_ld_32x32b_x32 (CUDA-core entries added to the accumulator, f3)
__device__ __forceinline__ void tc_st_32x32b_x32(uint32_t taddr, const uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], "
      "{%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
      "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};"
      ::"r"(taddr), "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]),
        "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]),
        "r"(r[16]), "r"(r[17]), "r"(r[18]), "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]),
        "r"(r[24]), "r"(r[25]), "r"(r[26]), "r"(r[27]), "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31])
      : "memory");
}
__device__ __forceinline__ void tc_wait_st() {
  asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
}

// ---- CTA-pair forms (cta_group::2; pinned by tools/probe_sp2.cu, profiles/r01_probe_pair.txt).
// The pair's MMA is issued by the even CTA of the cluster; operands at the same
// shared-memory offsets in both CTAs (A: each CTA's 128 rows, B: each CTA's N/2
// columns), accumulators and metadata in each CTA's own TMEM.
template <uint32_t kCols>
__device__ __forceinline__ void tmem_alloc_pair(uint32_t* dst_smem) {  // whole warp, both CTAs
  asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                   smem_u32(dst_smem)),
               "n"(kCols));
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
}
template <uint32_t kCols>
__device__ __forceinline__ void tmem_dealloc_pair(uint32_t taddr) {  // whole warp, both CTAs
  asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(taddr), "n"(kCols));
}
__device__ __forceinline__ void tc_mma_sp_f16_pair(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc,
                                                   uint32_t e_tmem, uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %5, 0;\n\t"
      "tcgen05.mma.sp.cta_group::2.kind::f16 [%0], %1, %2, [%3], %4, p;\n\t}" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(e_tmem), "r"(idesc), "r"(accumulate)
      : "memory");
}
// The four k-steps of a full sparse k-block in one asm block: descriptor s is
// desc0 + s * step (16-byte units in the address field), metadata column
// e + (s & 2), selector id2 = s & 1 (idesc1 = idesc0 | 1).  `acc0` = accumulate
// flag of the first step (the others always accumulate).
// Metadata copy / commit executed by the whole converged warp (one elected lane).
template <bool kPairT>
__device__ __forceinline__ void tc_cp_128x128b_warp(uint32_t taddr, uint64_t sdesc) {
  if constexpr (kPairT)
    asm volatile("{\n\t.reg .pred q;\n\telect.sync _|q, 0xffffffff;\n\t"
                 "@q tcgen05.cp.cta_group::2.128x128b [%0], %1;\n\t}" ::"r"(taddr), "l"(sdesc) : "memory");
  else
    asm volatile("{\n\t.reg .pred q;\n\telect.sync _|q, 0xffffffff;\n\t"
                 "@q tcgen05.cp.cta_group::1.128x128b [%0], %1;\n\t}" ::"r"(taddr), "l"(sdesc) : "memory");
}
template <bool kPairT>
__device__ __forceinline__ void tc_commit_warp(uint64_t* bar) {
  if constexpr (kPairT)
    asm volatile(
        "{\n\t.reg .pred q;\n\telect.sync _|q, 0xffffffff;\n\t"
        "@q tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;\n\t}" ::"r"(
            smem_u32(bar)),
        "h"((uint16_t)3)
        : "memory");
  else
    asm volatile("{\n\t.reg .pred q;\n\telect.sync _|q, 0xffffffff;\n\t"
                 "@q tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(
                     smem_u32(bar))
                 : "memory");
}
// Same, executed by the whole converged warp: one lane is elected inside the
// asm, so the compiler sees warp-uniform code around the tcgen05 ops.
template <bool kPairT>
__device__ __forceinline__ void tc_mma_sp_f16_x4_warp(uint32_t d_tmem, uint64_t adesc0, uint64_t bdesc0,
                                                      uint32_t astep, uint32_t bstep, uint32_t e_tmem,
                                                      uint32_t idesc0, uint32_t acc0) {
  if constexpr (kPairT) {
    asm volatile(
        "{\n\t.reg .pred p, q;\n\t.reg .b64 a1, a2, a3, b1, b2, b3, as, bs;\n\t.reg .b32 e2, i1;\n\t"
        "elect.sync _|q, 0xffffffff;\n\t"
        "cvt.u64.u32 as, %3;\n\tcvt.u64.u32 bs, %4;\n\t"
        "add.s64 a1, %1, as;\n\tadd.s64 a2, a1, as;\n\tadd.s64 a3, a2, as;\n\t"
        "add.s64 b1, %2, bs;\n\tadd.s64 b2, b1, bs;\n\tadd.s64 b3, b2, bs;\n\t"
        "add.u32 e2, %5, 2;\n\tor.b32 i1, %6, 1;\n\t"
        "setp.ne.b32 p, %7, 0;\n\t"
        "@q tcgen05.mma.sp.cta_group::2.kind::f16 [%0], %1, %2, [%5], %6, p;\n\t"
        "@q tcgen05.mma.sp.cta_group::2.kind::f16 [%0], a1, b1, [%5], i1, 1;\n\t"
        "@q tcgen05.mma.sp.cta_group::2.kind::f16 [%0], a2, b2, [e2], %6, 1;\n\t"
        "@q tcgen05.mma.sp.cta_group::2.kind::f16 [%0], a3, b3, [e2], i1, 1;\n\t}" ::"r"(d_tmem),
        "l"(adesc0), "l"(bdesc0), "r"(astep), "r"(bstep), "r"(e_tmem), "r"(idesc0), "r"(acc0)
        : "memory");
  } else {
    asm volatile(
        "{\n\t.reg .pred p, q;\n\t.reg .b64 a1, a2, a3, b1, b2, b3, as, bs;\n\t.reg .b32 e2, i1;\n\t"
        "elect.sync _|q, 0xffffffff;\n\t"
        "cvt.u64.u32 as, %3;\n\tcvt.u64.u32 bs, %4;\n\t"
        "add.s64 a1, %1, as;\n\tadd.s64 a2, a1, as;\n\tadd.s64 a3, a2, as;\n\t"
        "add.s64 b1, %2, bs;\n\tadd.s64 b2, b1, bs;\n\tadd.s64 b3, b2, bs;\n\t"
        "add.u32 e2, %5, 2;\n\tor.b32 i1, %6, 1;\n\t"
        "setp.ne.b32 p, %7, 0;\n\t"
        "@q tcgen05.mma.sp.cta_group::1.kind::f16 [%0], %1, %2, [%5], %6, p;\n\t"
        "@q tcgen05.mma.sp.cta_group::1.kind::f16 [%0], a1, b1, [%5], i1, 1;\n\t"
        "@q tcgen05.mma.sp.cta_group::1.kind::f16 [%0], a2, b2, [e2], %6, 1;\n\t"
        "@q tcgen05.mma.sp.cta_group::1.kind::f16 [%0], a3, b3, [e2], i1, 1;\n\t}" ::"r"(d_tmem),
        "l"(adesc0), "l"(bdesc0), "r"(astep), "r"(bstep), "r"(e_tmem), "r"(idesc0), "r"(acc0)
        : "memory");
  }
}
__device__ __forceinline__ void tc_mma_f16_pair(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc,
                                                uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}

// ---------------------------------------------------------------- descriptors
// Shared-memory matrix descriptor (sm_100 "version 1").  Byte quantities.
//   layout: 0 = no swizzle (core matrices 8 rows x 16 B), 2 = 128B swizzle
__device__ __forceinline__ uint64_t smem_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo,
                                              uint32_t layout) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
  d |= (uint64_t)1 << 46;  // version
  d |= (uint64_t)(layout & 7) << 61;
  return d;
}
// Instruction descriptor, kind::f16, f16 A/B, f32 accumulate.
//   a_mn / b_mn: 1 = MN-major operand; sparse: 2:4 A with metadata selector id2.
__host__ __device__ constexpr uint32_t idesc_f16(int M, int N, int a_mn, int b_mn, int sparse,
                                                 int id2 = 0) {
  return (uint32_t)(id2 & 3) | ((uint32_t)(sparse & 1) << 2) | (1u << 4) /*f32 acc*/ |
         (0u << 7) /*A f16*/ | (0u << 10) /*B f16*/ | ((uint32_t)a_mn << 15) |
         ((uint32_t)b_mn << 16) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

}  // namespace jig

namespace jig {
// ---------------------------------------------------------------- cp.async (LDGSTS)
// 16-byte cp.async to a shared::cta address; `zero` = write zeros, read nothing
// (ignore-src predicate: maps to the LDGSTS ZFILL predicate, no size arithmetic).
__device__ __forceinline__ void cp_async_16_zfill(uint32_t dst, const void* src, bool zero) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %2, 0;\n\t"
      "cp.async.cg.shared.global [%0], [%1], 16, p;\n\t}" ::"r"(dst),
      "l"(src), "r"((uint32_t)zero)
      : "memory");
}
// Arrive on `bar` once all prior cp.async of this thread have completed (no pending++).
__device__ __forceinline__ void cp_async_mbar_arrive_noinc(uint64_t* bar) {
  asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// ---------------------------------------------------------------- clusters / DSMEM
__device__ __forceinline__ uint32_t cluster_ctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
// Exit rendezvous of a cluster: a relaxed arrive does not wait for this thread's
// outstanding global stores to be performed (the release form does).
__device__ __forceinline__ void cluster_sync_relaxed() {
  asm volatile("barrier.cluster.arrive.relaxed.aligned;\n\tbarrier.cluster.wait.aligned;" ::: "memory");
}
// Split cluster barrier: arrive now, wait (acquire) later, only where needed.
__device__ __forceinline__ void cluster_arrive_relaxed() {
  asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");
}
__device__ __forceinline__ void cluster_wait() { asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory"); }
// Named CTA barriers (ids 2..15 free for the kernel's own use; 0 = __syncthreads).
__device__ __forceinline__ void named_bar_sync(int id, int nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}
__device__ __forceinline__ void named_bar_arrive(int id, int nthreads) {
  asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}
// shared::cta address of this CTA -> shared::cluster address of the same offset in CTA `rank`
__device__ __forceinline__ uint32_t mapa_shared(uint32_t saddr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
  return r;
}
// Arrive (release, cluster scope) on the mbarrier at shared::cluster address `rbar`.
__device__ __forceinline__ void mbar_arrive_cluster(uint32_t rbar) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(rbar) : "memory");
}
// Relaxed remote arrive: no release fence (a cluster-scope release waits for the
// SM's outstanding memory operations, ~1000 cycles with the B gathers in flight).
__device__ __forceinline__ void mbar_arrive_cluster_relaxed(uint32_t rbar) {
  asm volatile("mbarrier.arrive.relaxed.cluster.shared::cluster.b64 _, [%0];" ::"r"(rbar) : "memory");
}
// Wait (acquire, cluster scope) for phase `parity` of a local mbarrier that remote CTAs arrive on.
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra DONE_%=;\n\t"
      "bra WAIT_%=;\n"
      "DONE_%=:\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// ---------------------------------------------------------------- programmatic dependent launch
// Block this thread until the grids this launch depends on (the previous kernels
// of the stream) have completed and their memory is visible.  A no-op when the
// launch carries no programmatic dependency.
__device__ __forceinline__ void griddep_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
// Allow the dependent grid (the next kernel of the stream launched with the
// programmatic attribute) to be scheduled once every CTA of this grid has
// issued this or exited.
__device__ __forceinline__ void griddep_launch_dependents() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
}  // namespace jig
