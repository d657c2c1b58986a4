// tools/probe_sp.cu -- developer probe (not product, not a test): pins the
// sm_100a layouts the SpMM kernel relies on, on real hardware.
//   1. tcgen05.mma.sp.kind::f16, M=128, N=64, K=32 logical, A no-swizzle K-major
//      (compressed, 16 halves/row), B MN-major SW128, metadata via tcgen05.cp
//      128x128b into TMEM -- several candidate metadata lane layouts.
//   2. B staged by TMA tile::gather4 (tensor-map box {64,1} and {64,4}) vs. a
//      manual swizzled fill, with a row permutation and an out-of-bounds row.
//   3. throughput of back-to-back sparse vs dense MMAs (M=128, N=256).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -o probe tools/probe_sp.cu
#include <cuda.h>
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

constexpr int N = 64;  // one SW128 MN chunk

// A_img: 4096 B (no-swizzle K-major image), E_img: 2048 B (128 x 16 B), B: K x ldb fp16
// bmode: 0 manual fill from global, 1 gather4 via tmap
__global__ void probe_kernel(const uint8_t* A_img, const uint8_t* E_img, const __half* B, int ldb,
                             const int* rows, const __grid_constant__ CUtensorMap tmap, int bmode,
                             int lbo_a, int sbo_a, int ecol_off, int id2, float* D) {
  __shared__ __align__(1024) uint8_t sB[32 * 128];
  __shared__ __align__(128) uint8_t sA[4096];
  __shared__ __align__(128) uint8_t sE[2048];
  __shared__ uint64_t bar_ld, bar_mma;
  __shared__ uint32_t tmem_base;
  const int tid = threadIdx.x, warp = tid / 32;

  for (int i = tid; i < 4096; i += blockDim.x) sA[i] = A_img[i];
  for (int i = tid; i < 2048; i += blockDim.x) sE[i] = E_img[i];
  if (bmode == 0) {
    // manual SW128 MN-major: row k at k*128, 16B chunk c stored at chunk c ^ (k % 8)
    for (int i = tid; i < 32 * 8; i += blockDim.x) {
      int k = i / 8, c = i % 8;
      int r = rows[k];
      uint4 v = make_uint4(0, 0, 0, 0);
      if (r >= 0) v = *reinterpret_cast<const uint4*>(B + (size_t)r * ldb + c * 8);
      *reinterpret_cast<uint4*>(sB + k * 128 + ((c ^ (k % 8)) * 16)) = v;
    }
  }
  if (tid == 0) {
    mbar_init(&bar_ld, 1);
    mbar_init(&bar_mma, 1);
    fence_barrier_init();
  }
  if (warp == 0) tmem_alloc<128>(&tmem_base);
  __syncthreads();
  tc_fence_after();
  if (bmode == 1 && tid == 0) {
    mbar_arrive_expect_tx(&bar_ld, 32 * 128);
    for (int g = 0; g < 8; ++g)
      tma_gather4(sB + g * 512, &tmap, 0, rows[4 * g], rows[4 * g + 1], rows[4 * g + 2],
                  rows[4 * g + 3], &bar_ld);
  }
  if (bmode == 1) mbar_wait(&bar_ld, 0);
  fence_proxy_async();  // generic-proxy smem writes -> async proxy (tensor core)
  __syncthreads();
  uint32_t tbase = tmem_base;
  if (tid == 0) {
    tc_fence_after();
    uint64_t edesc = smem_desc(smem_u32(sE), 16 /*unused*/, 128, 0);
    tc_cp_128x128b(tbase + 64, edesc);
    uint64_t adesc = smem_desc(smem_u32(sA), lbo_a, sbo_a, 0);
    uint64_t bdesc = smem_desc(smem_u32(sB), 4096 /*next 64-col chunk, unused*/, 1024, 2);
    uint32_t idesc = idesc_f16(128, N, 0, 1, 1, id2);
    tc_mma_sp_f16(tbase, adesc, bdesc, tbase + 64 + ecol_off, idesc, 0);
    tc_commit(&bar_mma);
  }
  mbar_wait(&bar_mma, 0);
  tc_fence_after();
  if (warp < 4) {
    for (int c0 = 0; c0 < N; c0 += 32) {
      uint32_t r[32];
      tc_ld_32x32b_x32(tbase + ((uint32_t)(warp * 32) << 16) + c0, r);
      tc_wait_ld();
      int row = warp * 32 + (tid % 32);
      for (int j = 0; j < 32; ++j) D[row * N + c0 + j] = __uint_as_float(r[j]);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc<128>(tbase);
}

// throughput: loop of MMAs on garbage smem data
//   alay: A smem layout 0 = no swizzle (LBO 128, SBO 256), 6 = SW32 K-major, 2 = SW128 K-major
__global__ void tput_kernel(int iters, int sparse, int N, int alay, long long* cycles) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint64_t bar;
  __shared__ uint32_t tmem_base;
  const int tid = threadIdx.x;
  if (tid == 0) { mbar_init(&bar, 1); fence_barrier_init(); }
  if (tid < 32) tmem_alloc<512>(&tmem_base);
  __syncthreads();
  tc_fence_after();
  uint32_t tb = tmem_base;
  if (tid == 0) {
    uint64_t adesc = alay == 0 ? smem_desc(smem_u32(sm), 128, 256, 0)
                   : alay == 6 ? smem_desc(smem_u32(sm), 16, 256, 6)
                               : smem_desc(smem_u32(sm), 16, 1024, 2);
    uint64_t bdesc = smem_desc(smem_u32(sm + 32768), 4096 * 2, 1024, 2);
    uint32_t idesc = idesc_f16(128, N, 0, 1, sparse, 0);
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      if (sparse) tc_mma_sp_f16(tb, adesc, bdesc, tb + 256, idesc, 1);
      else tc_mma_f16(tb, adesc, bdesc, idesc, 1);
    }
    tc_commit(&bar);
    mbar_wait(&bar, 0);
    cycles[blockIdx.x] = clock64() - t0;
  }
  __syncthreads();
  if (tid < 32) tmem_dealloc<512>(tb);
}

typedef CUresult (*EncodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                const cuuint64_t*, const cuuint32_t*, const cuuint32_t*,
                                CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion,
                                CUtensorMapFloatOOBfill);

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
  srand(1);
  const int M = 128, KL = 32, KROWS = 40;  // B has 40 rows; gather picks 32 (one OOB)
  // logical A with 2:4 pattern per group of 4, and compressed form
  std::vector<float> Al(M * KL, 0.f);
  std::vector<uint16_t> vals(M * 16);
  std::vector<uint32_t> meta32(M, 0);  // row's 8 nibbles (32 logical)
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
  // A image: [mgroup 16][kcore 2][row 8][8 halves]
  std::vector<uint8_t> Aimg(4096);
  for (int r = 0; r < M; ++r)
    for (int c = 0; c < 2; ++c)
      memcpy(&Aimg[(r / 8) * 256 + c * 128 + (r % 8) * 16], &vals[r * 16 + c * 8], 16);
  // B: KROWS x 64
  std::vector<uint16_t> Bh(KROWS * N);
  for (auto& x : Bh) x = f2h((float)((rand() % 9) - 4) * 0.5f);
  int rows[32];
  for (int k = 0; k < 32; ++k) rows[k] = (k * 7 + 3) % KROWS;
  rows[5] = KROWS + 3;  // out of bounds: TMA zero fill; manual path uses -1
  std::vector<float> Bl(32 * N, 0.f);
  for (int k = 0; k < 32; ++k)
    for (int n = 0; n < N; ++n) Bl[k * N + n] = rows[k] < KROWS ? h2f(Bh[rows[k] * N + n]) : 0.f;
  std::vector<float> Dref(M * N, 0.f);
  for (int r = 0; r < M; ++r)
    for (int n = 0; n < N; ++n) {
      double s = 0;
      for (int k = 0; k < KL; ++k) s += (double)Al[r * KL + k] * Bl[k * N + n];
      Dref[r * N + n] = (float)s;
    }

  // candidate E images
  auto make_E = [&](int variant, int vc) {
    std::vector<uint32_t> E(128 * 4, 0);
    for (int L = 0; L < 128; ++L) {
      uint32_t w = 0;
      if (variant == 0) {  // CUTLASS-derived interleave: lane = m0 + 8*k1 + 16*m2
        int r = 16 * (L / 16) + (L % 8), k1 = (L / 8) % 2;
        uint32_t lo = (meta32[r] >> (16 * k1)) & 0xFFFF, hi = (meta32[r + 8] >> (16 * k1)) & 0xFFFF;
        w = lo | (hi << 16);
      } else {  // naive: lane = row, word = row's 32 logical
        w = meta32[L];
      }
      for (int c = 0; c < 4; ++c) E[L * 4 + c] = (c == vc) ? w : 0x44444444u;  // others: (0,1) everywhere
    }
    return E;
  };

  uint8_t *dA, *dE;
  __half* dB;
  int* dRows;
  float* dD;
  CK(cudaMalloc(&dA, 4096));
  CK(cudaMalloc(&dE, 2048));
  CK(cudaMalloc(&dB, KROWS * N * 2));
  CK(cudaMalloc(&dRows, 32 * 4));
  CK(cudaMalloc(&dD, M * N * 4));
  CK(cudaMemcpy(dA, Aimg.data(), 4096, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dB, Bh.data(), KROWS * N * 2, cudaMemcpyHostToDevice));

  EncodeTiled enc = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q));
  CUtensorMap tm1, tm4;
  cuuint64_t gdim[2] = {(cuuint64_t)N, (cuuint64_t)KROWS};
  cuuint64_t gstr[1] = {(cuuint64_t)N * 2};
  cuuint32_t estr[2] = {1, 1};
  cuuint32_t box1[2] = {64, 1}, box4[2] = {64, 4};
  CUresult r1 = enc(&tm1, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, dB, gdim, gstr, box1, estr,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                    CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  CUresult r4 = enc(&tm4, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, dB, gdim, gstr, box4, estr,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                    CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("encode box{64,1}=%d box{64,4}=%d\n", (int)r1, (int)r4);

  struct V { const char* name; int evar, bmode, tmap4, lbo, sbo, ecol, id2, vc; };
  V vs[] = {
      {"E-interleave manualB lbo128/sbo256", 0, 0, 0, 128, 256, 0, 0, 0},
      {"E-interleave manualB ecol=0 id2=1 vc=1", 0, 0, 0, 128, 256, 0, 1, 1},
      {"E-interleave manualB ecol=2 id2=0 vc=2", 0, 0, 0, 128, 256, 2, 0, 2},
      {"E-interleave manualB ecol=2 id2=1 vc=3", 0, 0, 0, 128, 256, 2, 1, 3},
      {"E-interleave gather4 box{64,1}    ", 0, 1, 0, 128, 256, 0, 0, 0},
  };
  int hrows_manual[32];
  for (int k = 0; k < 32; ++k) hrows_manual[k] = rows[k] < KROWS ? rows[k] : -1;
  for (auto& v : vs) {
    if (v.bmode == 1 && ((v.tmap4 ? r4 : r1) != CUDA_SUCCESS)) {
      printf("%s : tensor map encode failed\n", v.name);
      continue;
    }
    auto E = make_E(v.evar, v.vc);
    CK(cudaMemcpy(dE, E.data(), 2048, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dRows, v.bmode ? rows : hrows_manual, 32 * 4, cudaMemcpyHostToDevice));
    CK(cudaMemset(dD, 0, M * N * 4));
    probe_kernel<<<1, 128>>>(dA, dE, dB, N, dRows, v.tmap4 ? tm4 : tm1, v.bmode, v.lbo, v.sbo,
                             v.ecol, v.id2, dD);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
      printf("%s : kernel error %s\n", v.name, cudaGetErrorString(e));
      return 1;
    }
    std::vector<float> D(M * N);
    CK(cudaMemcpy(D.data(), dD, M * N * 4, cudaMemcpyDeviceToHost));
    int bad = 0;
    double maxerr = 0;
    for (int i = 0; i < M * N; ++i) {
      double err = fabs(D[i] - Dref[i]);
      if (err > 1e-3) ++bad;
      maxerr = fmax(maxerr, err);
    }
    printf("%s : mismatches %d / %d  maxerr %g  D[0..3]=%g %g %g %g ref %g %g %g %g\n", v.name,
           bad, M * N, maxerr, D[0], D[1], D[2], D[3], Dref[0], Dref[1], Dref[2], Dref[3]);
  }

  // throughput
  long long* dcyc;
  CK(cudaMalloc(&dcyc, 148 * 8));
  struct TV { int sp, N, alay; const char* name; };
  TV tvs[] = {{0, 256, 0, "dense  N256 A noswz"}, {1, 256, 0, "sparse N256 A noswz"},
              {1, 128, 0, "sparse N128 A noswz"}, {1, 64, 0, "sparse N64  A noswz"},
              {1, 128, 6, "sparse N128 A SW32 "}, {1, 128, 2, "sparse N128 A SW128"},
              {0, 128, 0, "dense  N128 A noswz"}, {0, 128, 2, "dense  N128 A SW128"}};
  CK(cudaFuncSetAttribute(tput_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024));
  for (auto& tv : tvs) {
    int iters = 4096;
    tput_kernel<<<148, 128, 100 * 1024>>>(iters, tv.sp, tv.N, tv.alay, dcyc);
    CK(cudaDeviceSynchronize());
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a);
    tput_kernel<<<148, 128, 100 * 1024>>>(iters, tv.sp, tv.N, tv.alay, dcyc);
    cudaEventRecord(b);
    CK(cudaDeviceSynchronize());
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    long long cyc;
    CK(cudaMemcpy(&cyc, dcyc, 8, cudaMemcpyDeviceToHost));
    double flops = 2.0 * 128 * tv.N * (tv.sp ? 32 : 16) * (double)iters * 148;  // logical
    printf("%s: %.1f cycles/mma (SM0), %.1f TFLOP/s logical (event %.3f ms)\n", tv.name,
           (double)cyc / iters, flops / ms / 1e9, ms);
  }
  return 0;
}
