// tools/gather_bench.cu -- developer microbenchmark (not product): throughput of
// gathering random 256-byte B-row segments into a 4-stage shared-memory ring,
// all 148 SMs busy, B resident in L2.  Decides how k_spmm stages B.
//   mode 0: cp.async 16 B (LDGSTS), 4 warps      mode 1: same, 8 warps
//   mode 2: TMA tile::gather4 (box {64,1}, SW128), 1 issuing thread
//   mode 3: TMA gather4 issued by 4 warps (one elected lane each)
//   mode 4/5: LDGSTS with 12 / 16 warps          mode 6: LDG.128 + STS.128, 16 warps
//   mode 7/8: TMA gather4 from 8 / 16 issuing warps
//   mode 9: half the rows by 8 LDGSTS warps, half by 8 TMA gather4 warps
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o gb tools/gather_bench.cu
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "ptx_tools.cuh"

using namespace jig;

constexpr int kRows = 128, kStages = 4, kRowBytes = 256, kStageBytes = kRows * kRowBytes;
constexpr int KB = 64;  // k-blocks per CTA

// pseudo-random row index computed in registers (no memory dependency in the loop)
__device__ __forceinline__ int hrow(int b, int kb, int row, int K) {
  uint32_t x = (uint32_t)(b * 7919 + kb * 104729 + row * 2654435761u);
  x ^= x >> 15; x *= 0x2c1b3c6du; x ^= x >> 12;
  return (int)(x % (uint32_t)K);
}

__global__ void __launch_bounds__(544, 1) gather_kernel(const __grid_constant__ CUtensorMap tm, const uint16_t* B,
                                                        int ldb, int K, const int* idx, int mode, long long* out) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t full[kStages], empty[kStages];
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int nprod = mode == 1 ? 8 : mode == 4 ? 12 : (mode == 5 || mode == 6 || mode == 8 || mode == 9) ? 16
                    : (mode == 7 || mode == 10) ? 8 : 4;
  const bool ldgsts = mode <= 1 || mode == 4 || mode == 5;
  const int N = ldb;
  if (threadIdx.x == 0) {
    for (int s = 0; s < kStages; ++s) {
      mbar_init(&full[s], (ldgsts || mode == 6) ? nprod * 32
                          : mode == 9 ? 8 * 32 + 8
                          : (mode == 7 || mode == 8 || mode == 10) ? nprod : 1 + (mode == 3 ? 3 : 0));
      mbar_init(&empty[s], 1);
    }
    fence_barrier_init();
  }
  __syncthreads();
  const int* myidx = idx + (size_t)blockIdx.x * KB * kRows;
  long long t0 = clock64();
  if (warp == 0) {  // consumer
    if (lane == 0) {
      int stage = 0;
      uint32_t ph = 0;
      for (int kb = 0; kb < KB; ++kb) {
        mbar_wait(&full[stage], ph);
        mbar_arrive(&empty[stage]);
        if (++stage == kStages) { stage = 0; ph ^= 1; }
      }
      out[blockIdx.x] = clock64() - t0;
    }
  } else if (warp - 1 < nprod) {
    const int w = warp - 1;
    int stage = 0;
    uint32_t ph = 0;
    for (int kb = 0; kb < KB; ++kb) {
      const int* ri = myidx + kb * kRows;
      mbar_wait(&empty[stage], ph ^ 1);
      uint8_t* st = sm + stage * kStageBytes;
      if (ldgsts || mode == 6) {
        // 256 rows-halves: 16 lanes per row (256 B), 2 rows per instruction; rows dealt round-robin
        const int c = lane & 15;
        if (ldgsts) {
          for (int j2 = w; j2 < kRows / 2; j2 += nprod) {
            const int row = 2 * j2 + (lane >> 4);
            const int g = hrow(blockIdx.x, kb, row, K);
            cp_async_16(st + (c >> 3) * (kRows * 128) + row * 128 + (((c & 7) ^ (row & 7)) << 4),
                        B + (size_t)g * ldb + 8 * c, 16);
          }
          cp_async_mbar_arrive_noinc(&full[stage]);
        } else {
          uint4 v[4];
          int rows[4];
          int n = 0;
          for (int j2 = w; j2 < kRows / 2; j2 += nprod) {
            rows[n] = 2 * j2 + (lane >> 4);
            v[n] = *reinterpret_cast<const uint4*>(B + (size_t)hrow(blockIdx.x, kb, rows[n], K) * ldb + 8 * c);
            ++n;
          }
          for (int i = 0; i < n; ++i) {
            const int row = rows[i];
            *reinterpret_cast<uint4*>(st + (c >> 3) * (kRows * 128) + row * 128 + (((c & 7) ^ (row & 7)) << 4)) = v[i];
          }
          fence_proxy_async();
          mbar_arrive(&full[stage]);
        }
      } else if (mode == 7 || mode == 8 || (mode == 9 && w >= 8)) {
        // TMA gather4: each issuing warp takes a share of the 32 row-quads x 2 chunks
        const int nt = mode == 9 ? 8 : nprod, wt = mode == 9 ? w - 8 : w;
        const int q0 = mode == 9 ? 16 : 0;                      // mode 9: rows 64..127
        const int nq = mode == 9 ? 16 : 32;
        if (lane == 0) {
          uint32_t bytes = 0;
          for (int q = q0 + wt; q < q0 + nq; q += nt) bytes += 2 * 512;
          mbar_arrive_expect_tx(&full[stage], bytes);
          for (int q = q0 + wt; q < q0 + nq; q += nt)
            for (int ch = 0; ch < 2; ++ch)
              tma_gather4(st + ch * (kRows * 128) + q * 512, &tm, 64 * ch, hrow(blockIdx.x, kb, 4 * q, K),
                          hrow(blockIdx.x, kb, 4 * q + 1, K), hrow(blockIdx.x, kb, 4 * q + 2, K),
                          hrow(blockIdx.x, kb, 4 * q + 3, K), &full[stage]);
        }
      } else if (mode == 9) {
        // LDGSTS warps 0..7: rows 0..63
        const int c = lane & 15;
        for (int j2 = w; j2 < 32; j2 += 8) {
          const int row = 2 * j2 + (lane >> 4);
          const int g = hrow(blockIdx.x, kb, row, K);
          cp_async_16(st + (c >> 3) * (kRows * 128) + row * 128 + (((c & 7) ^ (row & 7)) << 4),
                      B + (size_t)g * ldb + 8 * c, 16);
        }
        cp_async_mbar_arrive_noinc(&full[stage]);
      } else if (mode == 2) {
        if (w == 0 && lane == 0) {
          mbar_arrive_expect_tx(&full[stage], kStageBytes);
          for (int q = 0; q < kRows / 4; ++q)
            for (int ch = 0; ch < 2; ++ch)
              tma_gather4(st + ch * (kRows * 128) + q * 512, &tm, 64 * ch, hrow(blockIdx.x, kb, 4 * q, K),
                          hrow(blockIdx.x, kb, 4 * q + 1, K), hrow(blockIdx.x, kb, 4 * q + 2, K),
                          hrow(blockIdx.x, kb, 4 * q + 3, K), &full[stage]);
        }
      } else if (mode == 10) {
        // TMA 2-D tile per row (box {64, 1}, SW128): 8 issuing warps, 32 rows x 2 chunks each
        if (lane == 0) {
          mbar_arrive_expect_tx(&full[stage], kStageBytes / nprod);
          for (int row = w; row < kRows; row += nprod)
            for (int ch = 0; ch < 2; ++ch)
              tma_load_2d(st + ch * (kRows * 128) + row * 128, &tm, 64 * ch, hrow(blockIdx.x, kb, row, K), &full[stage]);
        }
      } else if (mode == 11) {
        // contiguous 1-D bulk copies (the compressed-A path): 4 x 8 KB per stage, one issuer
        if (w == 0 && lane == 0) {
          mbar_arrive_expect_tx(&full[stage], kStageBytes);
          for (int i = 0; i < 4; ++i) {
            const int off = hrow(blockIdx.x, kb, i, K * N * 2 / 8192 - 1) * 8192;
            bulk_g2s(st + i * 8192, reinterpret_cast<const uint8_t*>(B) + off, 8192, &full[stage]);
          }
        }
      } else {
        if (lane == 0) {
          if (w == 0) mbar_arrive_expect_tx(&full[stage], kStageBytes);
          else mbar_arrive(&full[stage]);
          for (int q = w * 8; q < w * 8 + 8; ++q)
            for (int ch = 0; ch < 2; ++ch)
              tma_gather4(st + ch * (kRows * 128) + q * 512, &tm, 64 * ch, hrow(blockIdx.x, kb, 4 * q, K),
                          hrow(blockIdx.x, kb, 4 * q + 1, K), hrow(blockIdx.x, kb, 4 * q + 2, K),
                          hrow(blockIdx.x, kb, 4 * q + 3, K), &full[stage]);
        }
      }
      if (++stage == kStages) { stage = 0; ph ^= 1; }
    }
  }
  __syncthreads();
}

typedef CUresult (*EncodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main(int argc, char** argv) {
  const int K = 4096, N = 256, grid = argc > 1 ? atoi(argv[1]) : 148;
  std::vector<int> modes;
  if (argc > 2) {
    for (char* t = strtok(argv[2], ","); t; t = strtok(nullptr, ",")) modes.push_back(atoi(t));
  } else {
    for (int m = 0; m < 12; ++m) modes.push_back(m);
  }
  uint16_t* dB;
  int* didx;
  long long* dout;
  cudaMalloc(&dB, (size_t)K * N * 2);
  cudaMemset(dB, 0, (size_t)K * N * 2);
  std::vector<int> h((size_t)grid * KB * kRows);
  srand(3);
  for (auto& x : h) x = rand() % K;
  cudaMalloc(&didx, h.size() * 4);
  cudaMemcpy(didx, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  cudaMalloc(&dout, grid * 8);
  EncodeTiled enc;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q);
  CUtensorMap tm;
  cuuint64_t gdim[2] = {(cuuint64_t)N, (cuuint64_t)K};
  cuuint64_t gstr[1] = {(cuuint64_t)N * 2};
  cuuint32_t box[2] = {64, 1}, es[2] = {1, 1};
  enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, dB, gdim, gstr, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
      CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  const int smem = kStages * kStageBytes + 1024;
  cudaFuncSetAttribute(gather_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const char* names[] = {"LDGSTS 4 warps", "LDGSTS 8 warps", "TMA gather4, 1 issuer", "TMA gather4, 4 issuers",
                         "LDGSTS 12 warps", "LDGSTS 16 warps", "LDG+STS 16 warps", "TMA gather4, 8 issuers",
                         "TMA gather4, 16 issuers", "LDGSTS 8w + gather4 8w", "TMA tile row, 8 issuers",
                         "bulk 1-D 8 KB x 4"};
  for (int mode : modes) {
    for (int rep = 0; rep < 3; ++rep) {
      cudaEvent_t a, b;
      cudaEventCreate(&a);
      cudaEventCreate(&b);
      cudaEventRecord(a);
      gather_kernel<<<grid, 544, smem>>>(tm, dB, N, K, didx, mode, dout);
      cudaEventRecord(b);
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) { printf("mode %d error %s\n", mode, cudaGetErrorString(e)); return 1; }
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      std::vector<long long> cyc(grid);
      cudaMemcpy(cyc.data(), dout, grid * 8, cudaMemcpyDeviceToHost);
      long long mx = 0;
      for (auto c : cyc) mx = c > mx ? c : mx;
      const double bytes = (double)grid * KB * kStageBytes;
      if (rep == 2)
        printf("grid %3d %-24s %8.1f us  %7.1f GB/s total  %5.1f B/clk/SM (max CTA %lld cyc, %.0f cyc per k-block)\n",
               grid, names[mode], ms * 1e3, bytes / ms / 1e6, (double)KB * kStageBytes / mx, mx, (double)mx / KB);
    }
  }
  return 0;
}
