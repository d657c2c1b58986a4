// tools/probe_sp2.cu -- developer probe (not product): pins the semantics of the
// CTA-pair sparse MMA on B200 before the kernel uses it:
//   tcgen05.mma.sp.cta_group::2.kind::f16, M = 256 (128 rows per CTA), N = 128
//   (64 B columns stored per CTA), K = 32 logical; TMEM alloc cta_group::2;
//   metadata copied by the leader with tcgen05.cp.cta_group::2; commit
//   multicast to both CTAs' mbarriers.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -o probe2 tools/probe_sp2.cu
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "ptx_tools.cuh"

using namespace jig;

#define CK(x)                                                                        \
  do {                                                                               \
    cudaError_t e = (x);                                                             \
    if (e != cudaSuccess) {                                                          \
      printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); \
      exit(1);                                                                       \
    }                                                                                \
  } while (0)

constexpr int N = 128;        // full N of the MMA; each CTA stores N/2 = 64 columns
constexpr int KROWS = 40;

__global__ void __cluster_dims__(2, 1, 1) pair_kernel(const uint8_t* A_img /*[2][4096]*/, const uint8_t* E_img /*[2][2048]*/,
                                                      const __half* B, const int* rows, int bsplit, float* D) {
  __shared__ __align__(1024) uint8_t sB[32 * 128];
  __shared__ __align__(128) uint8_t sA[4096];
  __shared__ __align__(128) uint8_t sE[2048];
  __shared__ uint64_t bar_mma;
  __shared__ uint32_t tmem_base;
  const int tid = threadIdx.x, warp = tid / 32;
  const uint32_t rank = cluster_ctarank();
  for (int i = tid; i < 4096; i += blockDim.x) sA[i] = A_img[rank * 4096 + i];
  for (int i = tid; i < 2048; i += blockDim.x) sE[i] = E_img[rank * 2048 + i];
  // B columns of this CTA: bsplit = 1 -> rank r holds columns [64r, 64r+64); 0 -> both hold 0..63
  const int c0 = bsplit ? 64 * rank : 0;
  for (int i = tid; i < 32 * 8; i += blockDim.x) {
    int k = i / 8, c = i % 8;
    int r = rows[k];
    uint4 v = make_uint4(0, 0, 0, 0);
    if (r >= 0) v = *reinterpret_cast<const uint4*>(B + (size_t)r * N + c0 + c * 8);
    *reinterpret_cast<uint4*>(sB + k * 128 + ((c ^ (k % 8)) * 16)) = v;
  }
  if (tid == 0) {
    mbar_init(&bar_mma, 1);
    fence_barrier_init();
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base)),
                 "n"(256));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  fence_proxy_async();
  tc_fence_before();
  cluster_sync_all();
  tc_fence_after();
  const uint32_t tbase = tmem_base;
  if (rank == 0 && tid == 0) {
    const uint64_t edesc = smem_desc(smem_u32(sE), 16, 128, 0);
    asm volatile("tcgen05.cp.cta_group::2.128x128b [%0], %1;" ::"r"(tbase + 128), "l"(edesc) : "memory");
    const uint64_t adesc = smem_desc(smem_u32(sA), 128, 256, 0);
    const uint64_t bdesc = smem_desc(smem_u32(sB), 4096, 1024, 2);
    const uint32_t idesc = idesc_f16(256, N, 0, 1, 1, 0);
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %5, 0;\n\t"
        "tcgen05.mma.sp.cta_group::2.kind::f16 [%0], %1, %2, [%3], %4, p;\n\t}" ::"r"(tbase),
        "l"(adesc), "l"(bdesc), "r"(tbase + 128), "r"(idesc), "r"(0u)
        : "memory");
    asm volatile(
        "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
            smem_u32(&bar_mma)),
        "h"((uint16_t)3)
        : "memory");
  }
  mbar_wait(&bar_mma, 0);
  tc_fence_after();
  if (warp < 4) {
    for (int cc = 0; cc < N; cc += 32) {
      uint32_t r[32];
      tc_ld_32x32b_x32(tbase + ((uint32_t)(warp * 32) << 16) + cc, r);
      tc_wait_ld();
      const int row = rank * 128 + warp * 32 + (tid % 32);
      for (int j = 0; j < 32; ++j) D[row * N + cc + j] = __uint_as_float(r[j]);
    }
  }
  tc_fence_before();
  cluster_sync_all();
  if (warp == 0) {
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tbase), "n"(256));
  }
}

static float h2f(uint16_t h) {
  __half x;
  memcpy(&x, &h, 2);
  return __half2float(x);
}
static uint16_t f2h(float f) {
  __half x = __float2half_rn(f);
  uint16_t h;
  memcpy(&h, &x, 2);
  return h;
}

int main() {
  srand(5);
  const int M = 256, KL = 32;
  std::vector<float> Al(M * KL, 0.f);
  std::vector<uint16_t> vals(M * 16);
  std::vector<uint32_t> meta32(M, 0);
  for (int r = 0; r < M; ++r)
    for (int q = 0; q < 8; ++q) {
      int i0 = rand() % 4, i1 = rand() % 4;
      while (i1 == i0) i1 = rand() % 4;
      if (i0 > i1) { int t = i0; i0 = i1; i1 = t; }
      for (int k = 0; k < 2; ++k) {
        int pos = k ? i1 : i0;
        float v = (float)((rand() % 7) - 3);
        if (v == 0) v = 1;
        uint16_t h = f2h(v);
        vals[r * 16 + 2 * q + k] = h;
        Al[r * KL + 4 * q + pos] = h2f(h);
      }
      meta32[r] |= (uint32_t)(i0 + 4 * i1) << (4 * q);
    }
  std::vector<uint8_t> Aimg(2 * 4096);
  std::vector<uint32_t> E(2 * 512, 0);
  for (int half = 0; half < 2; ++half) {
    for (int rr = 0; rr < 128; ++rr) {
      const int r = half * 128 + rr;
      for (int c = 0; c < 2; ++c)
        memcpy(&Aimg[half * 4096 + (rr / 8) * 256 + c * 128 + (rr % 8) * 16], &vals[r * 16 + c * 8], 16);
    }
    for (int L = 0; L < 128; ++L) {
      int rr = 16 * (L / 16) + (L % 8), k1 = (L / 8) % 2;
      const int r = half * 128 + rr;
      uint32_t lo = (meta32[r] >> (16 * k1)) & 0xFFFF, hi = (meta32[r + 8] >> (16 * k1)) & 0xFFFF;
      E[half * 512 + L * 4] = lo | (hi << 16);
    }
  }
  std::vector<uint16_t> Bh(KROWS * N);
  for (auto& x : Bh) x = f2h((float)((rand() % 9) - 4) * 0.5f);
  int rows[32];
  for (int k = 0; k < 32; ++k) rows[k] = (k * 7 + 3) % KROWS;
  std::vector<float> Dref(M * N, 0.f);
  for (int r = 0; r < M; ++r)
    for (int n = 0; n < N; ++n) {
      double s = 0;
      for (int k = 0; k < KL; ++k) s += (double)Al[r * KL + k] * h2f(Bh[rows[k] * N + n]);
      Dref[r * N + n] = (float)s;
    }
  uint8_t *dA, *dE;
  __half* dB;
  int* dR;
  float* dD;
  CK(cudaMalloc(&dA, 8192));
  CK(cudaMalloc(&dE, 4096));
  CK(cudaMalloc(&dB, Bh.size() * 2));
  CK(cudaMalloc(&dR, 32 * 4));
  CK(cudaMalloc(&dD, M * N * 4));
  CK(cudaMemcpy(dA, Aimg.data(), 8192, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dE, E.data(), 4096, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dB, Bh.data(), Bh.size() * 2, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dR, rows, 128, cudaMemcpyHostToDevice));
  for (int bsplit = 1; bsplit >= 0; --bsplit) {
    CK(cudaMemset(dD, 0, M * N * 4));
    pair_kernel<<<2, 128>>>(dA, dE, dB, dR, bsplit, dD);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("bsplit %d kernel error %s\n", bsplit, cudaGetErrorString(e)); return 1; }
    std::vector<float> D(M * N);
    CK(cudaMemcpy(D.data(), dD, M * N * 4, cudaMemcpyDeviceToHost));
    int bad = 0, badlo = 0;
    for (int i = 0; i < M * N; ++i) {
      if (fabs(D[i] - Dref[i]) > 1e-3) { ++bad; if ((i % N) < 64) ++badlo; }
    }
    printf("pair sparse M256 N128 (B columns split across the CTAs = %d): mismatches %d / %d (in cols<64: %d)  "
           "D[0]=%g ref %g  D[row128]=%g ref %g  D[0][64]=%g ref %g\n",
           bsplit, bad, M * N, badlo, D[0], Dref[0], D[128 * N], Dref[128 * N], D[64], Dref[64]);
  }
  return 0;
}
