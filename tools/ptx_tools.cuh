// tools/ptx_tools.cuh -- inline-PTX wrappers used only by the developer probes in
// tools/ (tile::gather4 and 2-D tensor TMA, single-thread tcgen05 commit / cp,
// cluster barriers with release/acquire, st.async).  Not part of libjigsaw.so:
// the product kernels use paper_conf_icpp_zhanglyfyllq24_b200/csrc/ptx.cuh.
#pragma once
#include "../paper_conf_icpp_zhanglyfyllq24_b200/csrc/ptx.cuh"

namespace jig {
// Non-blocking parity test of an mbarrier phase.
__device__ __forceinline__ bool mbar_test(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}
// Wait with back-off (mbar_test polling).
__device__ __forceinline__ void mbar_wait_sleep(uint64_t* bar, uint32_t parity, uint32_t ns) {
  while (!mbar_test(bar, parity)) __nanosleep(ns);
}

// Four rows (r0..r3) x one box of columns starting at c0 of a 2-D tensor map.
__device__ __forceinline__ void tma_gather4(void* dst, const CUtensorMap* map, int32_t c0, int32_t r0,
                                            int32_t r1, int32_t r2, int32_t r3, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(smem_u32(dst)),
      "l"(map), "r"(c0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, int32_t c0, int32_t c1,
                                            uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3}], [%4];" ::"r"(smem_u32(dst)),
      "l"(map), "r"(c0), "r"(c1), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void prefetch_tmap(const CUtensorMap* map) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(map) : "memory");
}


// All prior async tcgen05 ops of this thread arrive on `bar` once complete.
__device__ __forceinline__ void tc_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                   smem_u32(bar))
               : "memory");
}
// SMEM (128 rows x 16 B, K-major no-swizzle core matrices) -> TMEM lanes 0..127, 4 columns.
__device__ __forceinline__ void tc_cp_128x128b(uint32_t taddr, uint64_t sdesc) {
  asm volatile("tcgen05.cp.cta_group::1.128x128b [%0], %1;" ::"r"(taddr), "l"(sdesc) : "memory");
}

// Completion of this thread's prior pair MMAs arrives on `bar` (same offset) in both CTAs.
__device__ __forceinline__ void tc_commit_pair(uint64_t* bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"((uint16_t)3)
      : "memory");
}
__device__ __forceinline__ void tc_cp_128x128b_pair(uint32_t taddr, uint64_t sdesc) {
  asm volatile("tcgen05.cp.cta_group::2.128x128b [%0], %1;" ::"r"(taddr), "l"(sdesc) : "memory");
}

template <bool kPairT>
__device__ __forceinline__ void tc_mma_sp_f16_x4(uint32_t d_tmem, uint64_t adesc0, uint64_t bdesc0, uint32_t astep,
                                                 uint32_t bstep, uint32_t e_tmem, uint32_t idesc0, uint32_t acc0) {
  if constexpr (kPairT) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t.reg .b64 a1, a2, a3, b1, b2, b3, as, bs;\n\t.reg .b32 e2, i1;\n\t"
        "cvt.u64.u32 as, %3;\n\tcvt.u64.u32 bs, %4;\n\t"
        "add.s64 a1, %1, as;\n\tadd.s64 a2, a1, as;\n\tadd.s64 a3, a2, as;\n\t"
        "add.s64 b1, %2, bs;\n\tadd.s64 b2, b1, bs;\n\tadd.s64 b3, b2, bs;\n\t"
        "add.u32 e2, %5, 2;\n\tor.b32 i1, %6, 1;\n\t"
        "setp.ne.b32 p, %7, 0;\n\t"
        "tcgen05.mma.sp.cta_group::2.kind::f16 [%0], %1, %2, [%5], %6, p;\n\t"
        "tcgen05.mma.sp.cta_group::2.kind::f16 [%0], a1, b1, [%5], i1, 1;\n\t"
        "tcgen05.mma.sp.cta_group::2.kind::f16 [%0], a2, b2, [e2], %6, 1;\n\t"
        "tcgen05.mma.sp.cta_group::2.kind::f16 [%0], a3, b3, [e2], i1, 1;\n\t}" ::"r"(d_tmem),
        "l"(adesc0), "l"(bdesc0), "r"(astep), "r"(bstep), "r"(e_tmem), "r"(idesc0), "r"(acc0)
        : "memory");
  } else {
    asm volatile(
        "{\n\t.reg .pred p;\n\t.reg .b64 a1, a2, a3, b1, b2, b3, as, bs;\n\t.reg .b32 e2, i1;\n\t"
        "cvt.u64.u32 as, %3;\n\tcvt.u64.u32 bs, %4;\n\t"
        "add.s64 a1, %1, as;\n\tadd.s64 a2, a1, as;\n\tadd.s64 a3, a2, as;\n\t"
        "add.s64 b1, %2, bs;\n\tadd.s64 b2, b1, bs;\n\tadd.s64 b3, b2, bs;\n\t"
        "add.u32 e2, %5, 2;\n\tor.b32 i1, %6, 1;\n\t"
        "setp.ne.b32 p, %7, 0;\n\t"
        "tcgen05.mma.sp.cta_group::1.kind::f16 [%0], %1, %2, [%5], %6, p;\n\t"
        "tcgen05.mma.sp.cta_group::1.kind::f16 [%0], a1, b1, [%5], i1, 1;\n\t"
        "tcgen05.mma.sp.cta_group::1.kind::f16 [%0], a2, b2, [e2], %6, 1;\n\t"
        "tcgen05.mma.sp.cta_group::1.kind::f16 [%0], a3, b3, [e2], i1, 1;\n\t}" ::"r"(d_tmem),
        "l"(adesc0), "l"(bdesc0), "r"(astep), "r"(bstep), "r"(e_tmem), "r"(idesc0), "r"(acc0)
        : "memory");
  }
}

// 16-byte global -> shared copy; src_bytes = 0 writes 16 zero bytes (zero fill).
__device__ __forceinline__ void cp_async_16(void* dst, const void* src, uint32_t src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(dst)), "l"(src),
               "r"(src_bytes)
               : "memory");
}

__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// 16-byte asynchronous store into (possibly remote) shared memory of the cluster,
// completing 16 transaction bytes on the mbarrier at `rbar` (same CTA as `raddr`).
__device__ __forceinline__ void st_async_v4(uint32_t raddr, uint32_t a, uint32_t b, uint32_t c, uint32_t d,
                                            uint32_t rbar) {
  asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.b32 [%0], {%1, %2, %3, %4}, [%5];" ::"r"(
                   raddr),
               "r"(a), "r"(b), "r"(c), "r"(d), "r"(rbar)
               : "memory");
}

}  // namespace jig
