// tools/probe_pair_rate.cu -- developer probe (not product): issue rate of
// tcgen05.mma.sp kind::f16 with operands resident in shared memory, single CTA
// (cta_group::1, M = 128) vs CTA pair (cta_group::2, M = 256), N = 64 / 128 / 256,
// all 148 SMs busy.  Values are arbitrary (rate only).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -o probe_pair_rate tools/probe_pair_rate.cu
#include <cuda_runtime.h>

#include <cstdio>

#include "ptx_tools.cuh"

using namespace jig;

constexpr int kIters = 2048;

// mode 0: MMAs only (metadata copied once); 1: every 4 MMAs (one k-block) are
// preceded by a tcgen05.cp of their metadata block; 2: the cp of block i+1 is
// issued before the MMAs of block i (double-buffered metadata columns).
// mode 4: as mode 0, while warps 1-3 stream 16-byte cp.async (LDGSTS) from a
// 64 MB global buffer into a separate 32 KB shared region (the B-producer load).
__device__ uint4 g_src[4 << 20];
__device__ volatile int g_stop[148];
template <int N, bool kPair, int kMode>
__global__ void __launch_bounds__(384, 1) rate_kernel(long long* cycles) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  constexpr int NL = kPair ? N / 2 : N;  // B columns held per CTA
  constexpr int kBBytes = 32 * NL * 2;   // one k-step of B: 32 rows x NL halves
  uint8_t* sB = sm;                       // 4 buffers
  uint8_t* sA = sB + 4 * kBBytes;         // 4 x 4 KB
  uint8_t* sE = sA + 4 * 4096;            // 2 KB
  __shared__ uint64_t bar, bar2;
  __shared__ uint32_t slot;
  const int tid = threadIdx.x;
  for (int i = tid; i < (4 * kBBytes + 4 * 4096) / 4; i += blockDim.x)
    reinterpret_cast<uint32_t*>(sm)[i] = 0x3c003c00u ^ (i * 2654435761u & 0x00ff00ffu);
  for (int i = tid; i < 512; i += blockDim.x) reinterpret_cast<uint32_t*>(sE)[i] = 0x44444444u;  // (0,1) groups
  if (tid == 0) {
    mbar_init(&bar, 1);
    mbar_init(&bar2, 1);
    fence_barrier_init();
  }
  if (tid < 32) {
    if constexpr (kPair)
      tmem_alloc_pair<512>(&slot);
    else
      tmem_alloc<512>(&slot);
  }
  fence_proxy_async();
  tc_fence_before();
  if constexpr (kPair)
    cluster_sync_all();
  else
    __syncthreads();
  tc_fence_after();
  const uint32_t tb = slot;
  const bool issuer = tid == 0 && (!kPair || cluster_ctarank() == 0);
  if (kMode == 4 && tid >= 128) {
    // background LDGSTS (the B-producer load): 8 warps stream 16-byte cp.async
    // from an L2-resident 2 MB window into a 32 KB shared ring, ~4 groups in flight
    uint8_t* bg = sE + 2048;
    const int t = tid - 128;
    const size_t base = (size_t)(blockIdx.x % 16) * 131072;
    int it = 0;
    for (; it < 200000; ++it) {
      const size_t src = (base + (size_t)(it % 256) * 512 + t * 2) & ((4 << 20) - 1);
      cp_async_16(bg + (((it % 8) * 4096 + t * 16) & 32767), &g_src[src], 16);
      cp_async_16(bg + (((it % 8) * 4096 + 4096 * 8 + t * 16) & 32767), &g_src[src + 1], 16);
      asm volatile("cp.async.commit_group;" ::: "memory");
      asm volatile("cp.async.wait_group 4;" ::: "memory");
      if ((it & 63) == 0 && g_stop[blockIdx.x]) break;
    }
    asm volatile("cp.async.wait_all;" ::: "memory");
    if (t == 0) cycles[148 + blockIdx.x] = it;
  }
  if (issuer) {
    const uint32_t e_tmem = tb + 256 + 8;
    const uint64_t edesc = smem_desc(smem_u32(sE), 16, 128, 0);
    if constexpr (kPair) {
      tc_cp_128x128b_pair(e_tmem, edesc);
      tc_cp_128x128b_pair(e_tmem + 4, edesc);
    } else {
      tc_cp_128x128b(e_tmem, edesc);
      tc_cp_128x128b(e_tmem + 4, edesc);
    }
    const uint32_t idesc = idesc_f16(kPair ? 256 : 128, N, 0, 1, 1, 0);
    const long long t0 = clock64();
    for (int i = 0; i < kIters; ++i) {
      const int b = i & 3;
      uint32_t et = e_tmem;
      if (kMode == 5 && b == 0 && i > 0) {  // a commit per 4 MMAs (the per-k-block stage release)
        if constexpr (kPair)
          tc_commit_pair(&bar2);
        else
          tc_commit(&bar2);
      }
      if ((kMode == 1 || kMode == 5) && b == 0) {
        if constexpr (kPair)
          tc_cp_128x128b_pair(e_tmem, edesc);
        else
          tc_cp_128x128b(e_tmem, edesc);
      }
      if (kMode == 2) {
        et = e_tmem + 4 * ((i >> 2) & 1);
        if (b == 0) {
          if constexpr (kPair)
            tc_cp_128x128b_pair(e_tmem + 4 * (((i >> 2) + 1) & 1), edesc);
          else
            tc_cp_128x128b(e_tmem + 4 * (((i >> 2) + 1) & 1), edesc);
        }
      }
      const uint64_t adesc = smem_desc(smem_u32(sA + b * 4096), 128, 256, 0);
      const uint64_t bdesc = smem_desc(smem_u32(sB + b * kBBytes), 4096, 1024, 2);
      // mode 3: consecutive MMAs alternate between two accumulators (tb, tb + 128)
      const uint32_t d = kMode == 3 ? tb + 128 * (i & 1) : tb;
      // mode 6: the kernel's metadata addressing: k-step s = i & 3 reads column
      // e_tmem + (s & 2) with sparse selector id2 = s & 1
      const uint32_t et6 = kMode == 6 ? e_tmem + (b & 2) : et;
      const uint32_t id6 = kMode == 6 ? (idesc | (uint32_t)(b & 1)) : idesc;
      if constexpr (kPair)
        tc_mma_sp_f16_pair(d, adesc, bdesc, et6, id6, i > 1);
      else
        tc_mma_sp_f16(d, adesc, bdesc, et6, id6, i > 1);
    }
    if constexpr (kPair)
      tc_commit_pair(&bar);
    else
      tc_commit(&bar);
    mbar_wait(&bar, 0);
    const long long t1 = clock64();
    cycles[blockIdx.x] = t1 - t0;
    g_stop[blockIdx.x] = 1;
    if (kPair) g_stop[blockIdx.x + 1] = 1;
  } else if (kPair && tid == 0) {
    mbar_wait(&bar, 0);
  }
  tc_fence_before();
  if constexpr (kPair)
    cluster_sync_all();
  else
    __syncthreads();
  if (tid < 32) {
    if constexpr (kPair)
      tmem_dealloc_pair<512>(tb);
    else
      tmem_dealloc<512>(tb);
  }
}

template <int N, bool kPair, int kMode>
void run(long long* d) {
  auto k = rate_kernel<N, kPair, kMode>;
  const int smem = 1024 + 4 * 32 * (kPair ? N / 2 : N) * 2 + 4 * 4096 + 2048 + (kMode == 4 ? 32768 : 0);
  int zero[148] = {0};
  cudaMemcpyToSymbol(g_stop, zero, sizeof zero);
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(148);
  cfg.blockDim = dim3(kMode == 4 ? 384 : 128);
  cfg.dynamicSmemBytes = smem;
  cudaLaunchAttribute a[1];
  a[0].id = cudaLaunchAttributeClusterDimension;
  a[0].val.clusterDim.x = kPair ? 2 : 1;
  a[0].val.clusterDim.y = 1;
  a[0].val.clusterDim.z = 1;
  cfg.attrs = a;
  cfg.numAttrs = 1;
  float best = 1e30f;
  for (int r = 0; r < 3; ++r) {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaMemcpyToSymbol(g_stop, zero, sizeof zero);
    cudaEventRecord(e0);
    cudaLaunchKernelEx(&cfg, k, d);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    best = ms < best ? ms : best;
  }
  long long h[148];
  cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
  long long cyc = 0;
  int n = 0;
  for (int i = 0; i < 148; ++i)
    if (!kPair || i % 2 == 0) {
      cyc += h[i];
      ++n;
    }
  cyc /= n;
  const double flop_per_instr = 2.0 * (kPair ? 256 : 128) * N * 32;  // logical (dense-equivalent) K = 32
  const double total = flop_per_instr * kIters * (kPair ? 74 : 148);
  long long bgit = 0;
  if (kMode == 4) cudaMemcpy(&bgit, d + 148, sizeof bgit, cudaMemcpyDeviceToHost);
  printf("[bg iters CTA0 %lld = %.0f KB] mode %d %s M=%d N=%3d: %7.1f cycles / instr (per issuing CTA), %6.0f TFLOP/s logical over 148 SMs "
         "(event %.1f us) %s\n",
         bgit, bgit * 256 * 32 / 1024.0, kMode, kPair ? "pair  " : "single", kPair ? 256 : 128, N, (double)cyc / kIters, total / (best * 1e-3) / 1e12,
         best * 1e3, cudaGetErrorString(cudaGetLastError()));
}

int main() {
  long long* d;
  cudaMalloc(&d, 2 * 148 * sizeof(long long));
  run<64, false, 0>(d);
  run<128, false, 0>(d);
  run<256, false, 0>(d);
  run<128, true, 0>(d);
  run<256, true, 0>(d);
  run<128, false, 1>(d);
  run<256, false, 1>(d);
  run<128, true, 1>(d);
  run<256, true, 1>(d);
  run<128, false, 2>(d);
  run<128, true, 2>(d);
  run<256, true, 2>(d);
  run<128, true, 3>(d);
  run<128, false, 3>(d);

  run<128, false, 6>(d);
  run<128, true, 6>(d);
  run<256, true, 6>(d);
  return 0;
}
