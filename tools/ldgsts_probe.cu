// ldgsts_probe.cu -- is the 16-byte cp.async (LDGSTS) B-row gather limited by one
// in-flight batch per warp (each warp's next stage waits for its previous stage's
// cp.async.mbarrier.arrive to fire)?  Compares the k_spmm organisation (all B
// warps split every stage's rows) with warp GROUPS that own alternate stages, so
// several stages are in flight from different warps.  Developer tool.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/lp tools/ldgsts_probe.cu
#include <cuda_runtime.h>

#include <cstdio>
#include <vector>

#include "ptx_tools.cuh"

using namespace jig;

constexpr int kRows = 128, KB = 96, kMaxStages = 6;

__device__ __forceinline__ int hrow(int b, int kb, int row, int K) {
  uint32_t x = (uint32_t)(b * 7919 + kb * 104729 + row * 2654435761u);
  x ^= x >> 15; x *= 0x2c1b3c6du; x ^= x >> 12;
  return (int)(x % (uint32_t)K);
}

// nw producer warps in ng groups; group g fills stages kb = g, g + ng, ...; the
// warps of a group split the stage's 128 rows.  rowbytes = B bytes per row (NT*2).
__global__ void __launch_bounds__(544, 1) probe(const uint16_t* B, int K, int ldb, int nw, int ng, int rowbytes,
                                                int stages, long long* out) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t full[kMaxStages], empty[kMaxStages];
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int wpg = ng > 0 ? nw / ng : nw;  // warps per group
  const int stage_bytes = kRows * rowbytes;
  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) {
      mbar_init(&full[s], 32 * wpg);
      mbar_init(&empty[s], 1);
    }
    fence_barrier_init();
  }
  __syncthreads();
  long long t0 = clock64();
  if (warp == 0) {
    if (lane == 0) {
      int stage = 0;
      uint32_t ph = 0;
      for (int kb = 0; kb < KB; ++kb) {
        mbar_wait(&full[stage], ph);
        mbar_arrive(&empty[stage]);
        if (++stage == stages) { stage = 0; ph ^= 1; }
      }
      out[blockIdx.x] = clock64() - t0;
    }
  } else if (warp - 1 < nw && ng < 0) {
    // one group, completion tracked with commit_group / wait_group: up to D = -ng
    // k-blocks in flight per warp, then a plain arrive for the oldest
    const int D = -ng, w = warp - 1;
    const int lpr = rowbytes / 16, rpi = 32 / lpr;
    const int c = lane % lpr;
    const int rows_per_warp = kRows / nw;
    for (int kb = 0; kb < KB + D - 1; ++kb) {
      if (kb < KB) {
        const int stage = kb % stages;
        const uint32_t ph = (uint32_t)((kb / stages) & 1);
        mbar_wait(&empty[stage], ph ^ 1);
        uint8_t* st = sm + stage * stage_bytes;
        for (int r0 = w * rows_per_warp; r0 < (w + 1) * rows_per_warp; r0 += rpi) {
          const int row = r0 + lane / lpr;
          const int gr = hrow(blockIdx.x, kb, row, K);
          cp_async_16(st + row * rowbytes + ((c ^ (row & 7)) & (lpr - 1)) * 16, B + (size_t)gr * ldb + 8 * c, 16);
        }
      }
      asm volatile("cp.async.commit_group;" ::: "memory");
      const int old = kb - (D - 1);
      if (old >= 0) {
        switch (D) {
          case 1: asm volatile("cp.async.wait_group 0;" ::: "memory"); break;
          case 2: asm volatile("cp.async.wait_group 1;" ::: "memory"); break;
          case 3: asm volatile("cp.async.wait_group 2;" ::: "memory"); break;
          default: asm volatile("cp.async.wait_group 3;" ::: "memory"); break;
        }
        fence_proxy_async();
        mbar_arrive(&full[old % stages]);
      }
    }
  } else if (warp - 1 < nw) {
    const int w = warp - 1, g = w / wpg, wi = w % wpg;
    const int lpr = rowbytes / 16, rpi = 32 / lpr;  // lanes per row, rows per instruction
    const int c = lane % lpr;
    const int rows_per_warp = kRows / wpg;
    for (int kb = g; kb < KB; kb += ng) {
      const int stage = kb % stages;
      const uint32_t ph = (uint32_t)((kb / stages) & 1);
      mbar_wait(&empty[stage], ph ^ 1);
      uint8_t* st = sm + stage * stage_bytes;
      for (int r0 = wi * rows_per_warp; r0 < (wi + 1) * rows_per_warp; r0 += rpi) {
        const int row = r0 + lane / lpr;
        const int gr = hrow(blockIdx.x, kb, row, K);
        cp_async_16(st + row * rowbytes + ((c ^ (row & 7)) & (lpr - 1)) * 16, B + (size_t)gr * ldb + 8 * c, 16);
      }
      cp_async_mbar_arrive_noinc(&full[stage]);
    }
  }
  __syncthreads();
}

int main() {
  const int grid = 148, K = 8192, ldb = 2048;
  uint16_t* dB;
  long long* dout;
  cudaMalloc(&dB, (size_t)K * ldb * 2);
  cudaMemset(dB, 0, (size_t)K * ldb * 2);
  cudaMalloc(&dout, grid * 8);
  const int smem = 200 * 1024;
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  struct Case { int nw, ng, rowbytes, stages; };
  std::vector<Case> cases = {
      // groups <= stages (a group's parity waits must stay within one phase)
      {8, -2, 64, 6}, {8, -4, 64, 6}, {8, -2, 256, 4}, {8, -4, 256, 4}, {16, -4, 256, 4},
      {8, 1, 64, 6},  {8, 2, 64, 6},  {8, 4, 64, 6},  {12, 6, 64, 6}, {16, 4, 64, 6},
      {8, 1, 128, 6}, {8, 2, 128, 6}, {8, 4, 128, 6}, {16, 4, 128, 6}, {12, 6, 128, 6},
      {8, 1, 256, 4}, {8, 2, 256, 4}, {8, 4, 256, 4}, {16, 2, 256, 4}, {16, 4, 256, 4},
  };
  for (const Case& c : cases) {
    printf("case warps %d groups %d row %d stages %d ...\n", c.nw, c.ng, c.rowbytes, c.stages);
    fflush(stdout);
    float best = 1e30f;
    long long mx = 0;
    for (int rep = 0; rep < 4; ++rep) {
      cudaEvent_t a, b;
      cudaEventCreate(&a);
      cudaEventCreate(&b);
      cudaEventRecord(a);
      probe<<<grid, 32 * (1 + c.nw), smem>>>(dB, K, ldb, c.nw, c.ng, c.rowbytes, c.stages, dout);
      cudaEventRecord(b);
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (rep > 0 && ms < best) {
        best = ms;
        std::vector<long long> h(grid);
        cudaMemcpy(h.data(), dout, grid * 8, cudaMemcpyDeviceToHost);
        mx = 0;
        for (long long x : h) mx = x > mx ? x : mx;
      }
    }
    const double bytes = (double)KB * kRows * c.rowbytes;
    printf("warps %2d groups %d row %3d B stages %d: %7.1f us  %5.1f B/clk/SM  %5.0f cyc/stage\n", c.nw, c.ng,
           c.rowbytes, c.stages, best * 1e3, bytes / mx, (double)mx / KB);
    fflush(stdout);
  }
  return 0;
}
