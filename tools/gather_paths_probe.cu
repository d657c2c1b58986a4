// gather_paths_probe.cu -- developer microbenchmark: which load path gathers
// random 256-byte B rows from an L2-resident matrix into shared memory fastest,
// per SM, with 148 CTAs of 16 warps (the k_spmm B-producer access pattern)?
//   0  cp.async 16 B (LDGSTS), commit/wait groups, D batches in flight per warp
//   1  ld.global.v4 into registers (U loads in flight per lane) + st.shared.v4
//   2  ld.global.nc.v4 (texture path) into registers + st.shared.v4
//   3  cp.async.bulk (non-tensor TMA) of one 256 B row per lane, mbarrier completion
// Prints B/clk/SM.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17
//   -o /tmp/gpp tools/gather_paths_probe.cu
#include <cuda_runtime.h>

#include <cstdio>
#include <vector>

#include "ptx_tools.cuh"

using namespace jig;

constexpr int kRowBytes = 256, kIters = 64;  // rows per warp per iteration = 32 (bulk) / 2 per instr (others)

__device__ __forceinline__ uint32_t hrow(uint32_t b, uint32_t it, uint32_t r, uint32_t K) {
  uint32_t x = b * 7919u + it * 104729u + r * 2654435761u;
  x ^= x >> 15; x *= 0x2c1b3c6du; x ^= x >> 12;
  return x % K;
}

template <int MODE, int D>
__global__ void __launch_bounds__(512, 1) probe(const uint8_t* __restrict__ B, uint32_t K, uint32_t pitch,
                                                int nwarps, long long* out) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t bars[16][4];
  __shared__ uint64_t cbar[4];  // MODE 5: one CTA-wide barrier per batch slot
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // per warp: one 32-row x 256 B = 8 KB region, rewritten by every batch (the
  // contents do not matter here, only the throughput)
  uint8_t* ws = sm + (size_t)warp * 32 * kRowBytes;
  if (MODE == 3 && lane == 0)
    for (int d = 0; d < D; ++d) mbar_init(&bars[warp][d], 1);
  if (MODE == 4 && lane == 0)
    for (int d = 0; d < D; ++d) mbar_init(&bars[warp][d], 32);
  if (MODE == 5 && threadIdx.x == 0)
    for (int d = 0; d < D; ++d) mbar_init(&cbar[d], 32 * nwarps);
  if (MODE == 6 && lane == 0)
    for (int d = 0; d < D; ++d) mbar_init(&bars[warp][d], 1);
  fence_barrier_init();
  __syncthreads();
  const long long t0 = clock64();
  if (warp >= nwarps) {
  } else if (MODE == 0 || MODE == 4 || MODE == 5 || MODE == 6) {
    // 16 lanes per row: 2 rows per instruction, 16 instructions per 32-row batch
    const int c = lane & 15;
    for (int it = 0; it < kIters; ++it) {
      uint8_t* dst = ws;
      for (int r = 0; r < 32; r += 2) {
        const int row = r + (lane >> 4);
        const uint32_t g = hrow(blockIdx.x * 16 + warp, it, row, K);
        const uint32_t d = smem_u32(dst + row * kRowBytes + c * 16);
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(B + (size_t)g * pitch + c * 16)
                     : "memory");
      }
      if (MODE == 4 || MODE == 5) {  // completion through an mbarrier (k_spmm's cp.async.mbarrier.arrive.noinc)
        const int s = it % D;
        uint64_t* bb = MODE == 4 ? bars[warp] : cbar;
        cp_async_mbar_arrive_noinc(&bb[s]);
        if (it >= D - 1) {
          const int so = (it - (D - 1)) % D;
          mbar_wait(&bb[so], (uint32_t)(((it - (D - 1)) / D) & 1));
        }
        continue;
      }
      if (MODE == 6) {  // commit groups; one plain arrive per warp once a group has landed
        asm volatile("cp.async.commit_group;" ::: "memory");
        if (it >= D - 1) {
          if (D == 4) asm volatile("cp.async.wait_group 3;" ::: "memory");
          else if (D == 2) asm volatile("cp.async.wait_group 1;" ::: "memory");
          else asm volatile("cp.async.wait_group 0;" ::: "memory");
          __syncwarp();
          const int so = (it - (D - 1)) % D;
          if (lane == 0) mbar_arrive(&bars[warp][so]);
          mbar_wait(&bars[warp][so], (uint32_t)(((it - (D - 1)) / D) & 1));
        }
        continue;
      }
      asm volatile("cp.async.commit_group;" ::: "memory");
      if (it >= D - 1) {
        if (D == 4) asm volatile("cp.async.wait_group 3;" ::: "memory");
        else if (D == 2) asm volatile("cp.async.wait_group 1;" ::: "memory");
        else asm volatile("cp.async.wait_group 0;" ::: "memory");
      }
    }
    if (MODE == 0 || MODE == 6) asm volatile("cp.async.wait_group 0;" ::: "memory");
    else
      for (int it = kIters - (D - 1); it < kIters; ++it)
        if (it >= 0) mbar_wait(MODE == 4 ? &bars[warp][it % D] : &cbar[it % D], (uint32_t)((it / D) & 1));
  } else if (MODE == 1 || MODE == 2) {
    // each lane loads D 16-byte pieces (rows r = 2i + lane/16) before storing them
    const int c = lane & 15;
    for (int it = 0; it < kIters; ++it) {
      uint8_t* dst = ws;
      for (int r0 = 0; r0 < 32; r0 += 2 * D) {
        uint4 v[D];
#pragma unroll
        for (int i = 0; i < D; ++i) {
          const int row = r0 + 2 * i + (lane >> 4);
          const uint32_t g = hrow(blockIdx.x * 16 + warp, it, row, K);
          const uint4* src = reinterpret_cast<const uint4*>(B + (size_t)g * pitch + c * 16);
          if (MODE == 1)
            asm volatile("ld.global.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v[i].x), "=r"(v[i].y), "=r"(v[i].z), "=r"(v[i].w)
                         : "l"(src));
          else
            v[i] = __ldg(src);
        }
#pragma unroll
        for (int i = 0; i < D; ++i) {
          const int row = r0 + 2 * i + (lane >> 4);
          st_shared_v4u(smem_u32(dst + row * kRowBytes + c * 16), v[i]);
        }
      }
    }
  } else {
    // one bulk copy per lane per batch (32 rows x 256 B), D batches in flight
    uint32_t ph[4] = {0, 0, 0, 0};
    for (int it = 0; it < kIters; ++it) {
      const int s = it % D;
      if (it >= D) {
        mbar_wait(&bars[warp][s], ph[s]);
        ph[s] ^= 1;
      }
      if (lane == 0) mbar_arrive_expect_tx(&bars[warp][s], 32 * kRowBytes);
      __syncwarp();
      const uint32_t g = hrow(blockIdx.x * 16 + warp, it, lane, K);
      bulk_g2s(ws + lane * kRowBytes, B + (size_t)g * pitch, kRowBytes, &bars[warp][s]);
    }
    for (int it = kIters; it < kIters + D; ++it) {
      const int s = it % D;
      mbar_wait(&bars[warp][s], ph[s]);
      ph[s] ^= 1;
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = clock64() - t0;
}

template <int MODE, int D>
void run(const char* name, const uint8_t* dB, uint32_t K, uint32_t pitch, int nwarps, long long* dout) {
  const int grid = 148;
  const int smem = 1024 + 16 * 32 * kRowBytes;
  cudaFuncSetAttribute(probe<MODE, D>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  long long best = -1;
  for (int rep = 0; rep < 5; ++rep) {
    probe<MODE, D><<<grid, 512, smem>>>(dB, K, pitch, nwarps, dout);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
      printf("%s: error %s\n", name, cudaGetErrorString(e));
      return;
    }
    std::vector<long long> h(grid);
    cudaMemcpy(h.data(), dout, grid * 8, cudaMemcpyDeviceToHost);
    long long mx = 0;
    for (long long x : h) mx = x > mx ? x : mx;
    if (rep > 0 && (best < 0 || mx < best)) best = mx;
  }
  const double bytes = (double)nwarps * kIters * 32 * kRowBytes;  // per CTA
  printf("%-44s pitch %5u warps %2d %6.1f B/clk/SM\n", name, pitch, nwarps, bytes / best);
  fflush(stdout);
}

int main() {
  uint8_t* dB;
  long long* dout;
  const size_t bytes = 64u << 20;
  cudaMalloc(&dB, bytes);
  cudaMemset(dB, 1, bytes);
  cudaMalloc(&dout, 148 * 8);
  const uint32_t pitch = 512, K = (uint32_t)((16u << 20) / pitch);
  for (int nw : {8, 16}) {
    run<4, 2>("noinc arrive, per-warp barrier, 2 in flight", dB, K, pitch, nw, dout);
    run<4, 4>("noinc arrive, per-warp barrier, 4 in flight", dB, K, pitch, nw, dout);
    run<5, 2>("noinc arrive, ONE CTA barrier, 2 in flight", dB, K, pitch, nw, dout);
    run<5, 4>("noinc arrive, ONE CTA barrier, 4 in flight", dB, K, pitch, nw, dout);
    run<6, 2>("wait_group + 1 arrive/warp, 2 in flight", dB, K, pitch, nw, dout);
    run<6, 4>("wait_group + 1 arrive/warp, 4 in flight", dB, K, pitch, nw, dout);
  }
  return 0;
}
