// mc_bench.cu -- L2 -> SM ingest microbenchmark: does sharing the compressed-A
// stream between CTAs (TMA multicast inside a cluster, or plain unicast of the
// same addresses at the same time) raise the bytes per clock an SM receives,
// alone and mixed with the 16-byte cp.async B-row gather of k_spmm?
//
// Per CTA and stage: `abytes` of A-like data by cp.async.bulk (one 1-D bulk copy,
// or its 1/csz slice multicast to every CTA of the cluster) + `gbytes` of B-like
// rows gathered by 8 LDGSTS warps (256 B per row, random rows of a 4 MB matrix).
// Developer tool.  Build:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/mc_bench tools/mc_bench.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <vector>

#include "ptx_tools.cuh"

using namespace jig;

__device__ __forceinline__ uint32_t cluster_nctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(r));
  return r;
}

constexpr int kStages = 4, kMaxStage = 48 * 1024, KB = 192;

__device__ __forceinline__ void bulk_g2s_mc(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar,
                                            uint16_t mask) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1], %2, [%3], %4;" ::"r"(
          dst),
      "l"(src), "r"(bytes), "r"(bar), "h"(mask)
      : "memory");
}

__device__ __forceinline__ int hrow(int b, int kb, int row, int K) {
  uint32_t x = (uint32_t)(b * 7919 + kb * 104729 + row * 2654435761u);
  x ^= x >> 15; x *= 0x2c1b3c6du; x ^= x >> 12;
  return (int)(x % (uint32_t)K);
}

// mode: 0 = unicast distinct, 1 = unicast, same address in the cluster, 2 = multicast
__global__ void __launch_bounds__(320, 1) ingest(const uint8_t* Asrc, size_t asz, const uint16_t* B, int K,
                                                 int abytes, int gbytes, int mode, long long* out) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t full[kStages], empty[kStages];
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const uint32_t csz = cluster_nctarank(), rank = cluster_ctarank();
  const int cid = blockIdx.x / csz;
  const int grows = gbytes / 256;  // gathered rows per stage
  if (threadIdx.x == 0) {
    for (int s = 0; s < kStages; ++s) {
      mbar_init(&full[s], 1 + (grows ? 8 * 32 : 0));
      mbar_init(&empty[s], mode == 2 ? csz : 1);
    }
    fence_barrier_init();
  }
  cluster_sync_all();
  const int stage_bytes = abytes + gbytes;
  long long t0 = clock64();
  if (warp == 0) {  // consumer: frees the stage in every CTA that writes into it
    if (lane == 0) {
      int stage = 0;
      uint32_t ph = 0;
      for (int kb = 0; kb < KB; ++kb) {
        mbar_wait(&full[stage], ph);
        if (mode == 2) {
          for (uint32_t r = 0; r < csz; ++r) mbar_arrive_cluster(mapa_shared(smem_u32(&empty[stage]), r));
        } else {
          mbar_arrive(&empty[stage]);
        }
        if (++stage == kStages) { stage = 0; ph ^= 1; }
      }
      out[blockIdx.x] = clock64() - t0;
    }
  } else if (warp == 1) {  // A-like bulk producer
    if (lane == 0) {
      int stage = 0;
      uint32_t ph = 0;
      for (int kb = 0; kb < KB; ++kb) {
        mbar_wait(&empty[stage], ph ^ 1);
        uint8_t* dst = sm + stage * kMaxStage;
        const size_t chunk = (size_t)((mode == 0 ? blockIdx.x : cid) * KB + kb) * abytes % asz;
        if (abytes) {
          mbar_arrive_expect_tx(&full[stage], abytes);
          if (mode == 2) {
            const uint32_t slice = abytes / csz;
            bulk_g2s_mc(smem_u32(dst) + rank * slice, Asrc + chunk + rank * slice, slice, smem_u32(&full[stage]),
                        (uint16_t)((1u << csz) - 1));
          } else {
            bulk_g2s(dst, Asrc + chunk, abytes, &full[stage]);
          }
        } else {
          mbar_arrive(&full[stage]);
        }
        if (++stage == kStages) { stage = 0; ph ^= 1; }
      }
    }
  } else if (warp >= 2 && warp < 10 && grows) {  // B-like gather: 8 LDGSTS warps
    const int w = warp - 2;
    const int c = lane & 15;
    int stage = 0;
    uint32_t ph = 0;
    for (int kb = 0; kb < KB; ++kb) {
      mbar_wait(&empty[stage], ph ^ 1);
      uint8_t* st = sm + stage * kMaxStage + abytes;
      for (int j2 = w; j2 < grows / 2; j2 += 8) {
        const int row = 2 * j2 + (lane >> 4);
        const int g = hrow(blockIdx.x, kb, row, K);
        cp_async_16(st + (c >> 3) * (grows * 128) + row * 128 + (((c & 7) ^ (row & 7)) << 4), B + (size_t)g * 128 + 8 * c,
                    16);
      }
      cp_async_mbar_arrive_noinc(&full[stage]);
      if (++stage == kStages) { stage = 0; ph ^= 1; }
    }
  }
  (void)stage_bytes;
  __syncwarp();
  cluster_sync_all();
}

int main(int argc, char** argv) {
  const int grid = 148;
  const size_t asz = 64 << 20;
  const int K = 16384;
  uint8_t* dA;
  uint16_t* dB;
  long long* dout;
  cudaMalloc(&dA, asz);
  cudaMemset(dA, 1, asz);
  cudaMalloc(&dB, (size_t)K * 128 * 2);
  cudaMemset(dB, 0, (size_t)K * 128 * 2);
  cudaMalloc(&dout, grid * 8);
  const int smem = kStages * kMaxStage + 1024;
  cudaFuncSetAttribute(ingest, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaFuncSetAttribute(ingest, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  struct Case { const char* name; int csz, mode, abytes, gbytes; };
  std::vector<Case> cases = {
      {"bulk 32K unicast distinct       ", 1, 0, 32768, 0},
      {"bulk 32K unicast same, csz 2    ", 2, 1, 32768, 0},
      {"bulk 32K unicast same, csz 4    ", 4, 1, 32768, 0},
      {"bulk 32K multicast csz 2        ", 2, 2, 32768, 0},
      {"bulk 32K multicast csz 4        ", 4, 2, 32768, 0},
      {"gather 32K only                 ", 1, 0, 0, 32768},
      {"A 16K distinct + gather 32K     ", 1, 0, 16384, 32768},
      {"A 16K same csz2 + gather 32K    ", 2, 1, 16384, 32768},
      {"A 16K same csz4 + gather 32K    ", 4, 1, 16384, 32768},
      {"A 16K mc csz2 + gather 32K      ", 2, 2, 16384, 32768},
      {"A 16K mc csz4 + gather 32K      ", 4, 2, 16384, 32768},
      {"A 8K distinct + gather 32K      ", 1, 0, 8192, 32768},
      {"A 16K distinct + gather 16K     ", 1, 0, 16384, 16384},
      {"A 16K mc csz4 + gather 16K      ", 4, 2, 16384, 16384},
      {"bulk 32K multicast csz 8        ", 8, 2, 32768, 0},
      {"A 16K mc csz8 + gather 32K      ", 8, 2, 16384, 32768},
      {"A 16K same csz8 + gather 32K    ", 8, 1, 16384, 32768},
  };
  // cluster of 8: 144 CTAs (whole clusters only)
  for (const Case& c : cases) {
    const int g = grid / c.csz * c.csz;
    float best = 1e30f;
    long long maxcyc = 0;
    for (int rep = 0; rep < 4; ++rep) {
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(g);
      cfg.blockDim = dim3(320);
      cfg.dynamicSmemBytes = smem;
      cudaLaunchAttribute attr[1];
      attr[0].id = cudaLaunchAttributeClusterDimension;
      attr[0].val.clusterDim.x = c.csz;
      attr[0].val.clusterDim.y = 1;
      attr[0].val.clusterDim.z = 1;
      cfg.attrs = attr;
      cfg.numAttrs = 1;
      cudaEvent_t a, b;
      cudaEventCreate(&a);
      cudaEventCreate(&b);
      cudaEventRecord(a);
      cudaError_t e = cudaLaunchKernelEx(&cfg, ingest, (const uint8_t*)dA, asz, (const uint16_t*)dB, K, c.abytes,
                                         c.gbytes, c.mode, dout);
      cudaEventRecord(b);
      if (e == cudaSuccess) e = cudaDeviceSynchronize();
      if (e != cudaSuccess) {
        printf("%s error %s\n", c.name, cudaGetErrorString(e));
        return 1;
      }
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (rep > 0 && ms < best) {
        best = ms;
        std::vector<long long> h(g);
        cudaMemcpy(h.data(), dout, g * 8, cudaMemcpyDeviceToHost);
        maxcyc = 0;
        for (long long x : h) maxcyc = x > maxcyc ? x : maxcyc;
      }
    }
    const double per_cta = (double)KB * (c.abytes + c.gbytes);
    printf("%s %8.1f us  %7.1f GB/s into SMEM (all CTAs)  %5.1f B/clk/SM  (max CTA %lld cyc, %lld cyc/stage)\n", c.name,
           best * 1e3, per_cta * g / (best * 1e-3) / 1e9, per_cta / maxcyc, maxcyc, maxcyc / KB);
  }
  return 0;
}
