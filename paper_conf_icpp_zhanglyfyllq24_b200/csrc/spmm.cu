// spmm.cu -- S1: the SpMM mainloop C = A x B on sm_100a sparse tensor cores
// (DESIGN.md §5.2).  PAPER.md P:120-128 (CTA per C tile, B gathered by the
// reorder indices, C written straight from the accumulators)
// (deepened pipeline: gather indices are read >= one stage ahead of the MMA),
// re-designed for tcgen05:
//
//   persistent CTA per SM, 6 warps, warp-specialised:
//     warp 0  producer : per k-block (4 k-steps = 128 logical columns)
//                        cp.async.bulk of the compressed A image (16 KB) and the
//                        metadata block (2 KB), and 2 x 32 TMA tile::gather4 of
//                        the B rows named by the gather list (SW128, MN-major)
//     warp 1  MMA      : tcgen05.cp metadata -> TMEM, then per k-step one
//                        tcgen05.mma.sp.kind::f16  M=128 N=128 K=32 (logical)
//                        into a double-buffered fp32 TMEM accumulator
//     warps 2-5 epilogue: tcgen05.ld -> fp16 (RN) -> C rows < M
//   work unit = (panel p of 128 rows, 128-column slice of C); units are
//   scheduled round-robin, panels fastest, so co-resident CTAs share B in L2.
#include <cuda_fp16.h>

#include <cstdio>

#include "internal.h"
#include "ptx.cuh"

namespace jig {

namespace {

constexpr int kNTile = 128;                         // C columns per unit (UMMA N)
constexpr int kStages = 4;
constexpr int kRowsPerBlock = 32 * kStepsPerBlock;  // B rows per k-block (128)
constexpr int kChunkB = kRowsPerBlock * 128;        // one 64-column SW128 chunk: 16 KB
constexpr int kStageB = 2 * kChunkB;                // 32 KB
constexpr int kStageA = kStepsPerBlock * kKStepBytesA;  // 16 KB
constexpr int kStageE = kEBlockBytes;               // 2 KB
constexpr int kThreads = 192;
constexpr int kTmemCols = 512;
constexpr int kAccCols = kNTile;                    // fp32 accumulator: 1 column per C column
constexpr int kEColBase = 2 * kAccCols;             // metadata ring after the two accumulators
constexpr size_t kSmemBytes = 1024 + (size_t)kStages * (kStageB + kStageA + kStageE) + 256;

struct SpmmParams {
  const uint8_t* Aimg;
  const uint8_t* Eimg;
  const int32_t* G;
  const int32_t* ksn;
  const int32_t* ksoff;
  const int32_t* kboff;
  __half* C;
  int64_t M, N;
  int npanels, nunits;
};

__global__ void __launch_bounds__(kThreads, 1)
    k_spmm(const __grid_constant__ CUtensorMap tmB, const SpmmParams prm) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sB = smem;                                // kStages x 32 KB (1024-aligned)
  uint8_t* sA = sB + kStages * kStageB;              // kStages x 16 KB
  uint8_t* sE = sA + kStages * kStageA;              // kStages x 2 KB
  uint64_t* full = reinterpret_cast<uint64_t*>(sE + kStages * kStageE);
  uint64_t* empty = full + kStages;
  uint64_t* tfull = empty + kStages;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < kStages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(&tfull[a], 1);
      mbar_init(&tempty[a], 4);
    }
    fence_barrier_init();
  }
  if (warp == 0 && lane == 0) prefetch_tmap(&tmB);
  if (warp == 1) tmem_alloc<kTmemCols>(tmem_slot);
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------ producer
    int stage = 0;
    uint32_t phase = 0;
    for (int u = blockIdx.x; u < prm.nunits; u += gridDim.x) {
      const int p = u % prm.npanels;
      const int n0 = (u / prm.npanels) * kNTile;
      const int nks = prm.ksn[p];
      const int ks0 = prm.ksoff[p];
      const int kb0 = prm.kboff[p];
      for (int kb = 0; kb * kStepsPerBlock < nks; ++kb) {
        const int steps = min(kStepsPerBlock, nks - kb * kStepsPerBlock);
        const int gks = ks0 + kb * kStepsPerBlock;
        // gather rows for this k-block (issued before waiting: index load latency
        // overlaps the wait, the P:222 "col_idx one stage ahead" idea)
        int4 rows = make_int4(0, 0, 0, 0);
        if (lane < steps * 8) rows = *reinterpret_cast<const int4*>(prm.G + (int64_t)gks * 32 + 4 * lane);
        mbar_wait(&empty[stage], phase ^ 1);
        if (lane == 0) {
          mbar_arrive_expect_tx(&full[stage], (uint32_t)(steps * kKStepBytesA + kStageE + steps * 32 * 128 * 2));
          bulk_g2s(sA + stage * kStageA, prm.Aimg + (int64_t)gks * kKStepBytesA, steps * kKStepBytesA, &full[stage]);
          bulk_g2s(sE + stage * kStageE, prm.Eimg + (int64_t)(kb0 + kb) * kEBlockBytes, kStageE, &full[stage]);
        }
        __syncwarp();
        if (lane < steps * 8) {
          uint8_t* dst = sB + stage * kStageB + lane * 512;
#pragma unroll
          for (int ch = 0; ch < 2; ++ch)
            tma_gather4(dst + ch * kChunkB, &tmB, n0 + 64 * ch, rows.x, rows.y, rows.z, rows.w, &full[stage]);
        }
        if (++stage == kStages) { stage = 0; phase ^= 1; }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer
    if (lane == 0) {
      const uint32_t idesc0 = idesc_f16(128, kNTile, 0, 1, 1, 0);
      const uint32_t idesc1 = idesc_f16(128, kNTile, 0, 1, 1, 1);
      int stage = 0;
      uint32_t phase = 0;
      int it = 0;
      for (int u = blockIdx.x; u < prm.nunits; u += gridDim.x) {
        const int p = u % prm.npanels;
        const int nks = prm.ksn[p];
        if (nks == 0) continue;
        const int a = it & 1;
        const uint32_t use = (uint32_t)(it >> 1);
        mbar_wait(&tempty[a], (use & 1) ^ 1);
        tc_fence_after();
        const uint32_t d_tmem = tbase + a * kAccCols;
        for (int kb = 0; kb * kStepsPerBlock < nks; ++kb) {
          const int steps = min(kStepsPerBlock, nks - kb * kStepsPerBlock);
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          const uint32_t e_tmem = tbase + kEColBase + 4 * stage;
          tc_cp_128x128b(e_tmem, smem_desc(smem_u32(sE + stage * kStageE), 16, 128, 0));
          const uint32_t a_base = smem_u32(sA + stage * kStageA);
          const uint32_t b_base = smem_u32(sB + stage * kStageB);
          for (int s = 0; s < steps; ++s) {
            const uint64_t adesc = smem_desc(a_base + s * kKStepBytesA, 128, 256, 0);
            const uint64_t bdesc = smem_desc(b_base + s * 32 * 128, kChunkB, 1024, 2);
            tc_mma_sp_f16(d_tmem, adesc, bdesc, e_tmem + (s & 2), (s & 1) ? idesc1 : idesc0,
                          (kb | s) != 0);
          }
          tc_commit(&empty[stage]);
          if (++stage == kStages) { stage = 0; phase ^= 1; }
        }
        tc_commit(&tfull[a]);
        ++it;
      }
    }
    __syncwarp();
  } else {
    // ------------------------------------------------------------ epilogue
    const int q = warp & 3;  // TMEM lane quarter this warp may access
    int it = 0;
    for (int u = blockIdx.x; u < prm.nunits; u += gridDim.x) {
      const int p = u % prm.npanels;
      const int n0 = (u / prm.npanels) * kNTile;
      const int nks = prm.ksn[p];
      const int64_t row = (int64_t)p * 128 + q * 32 + lane;
      __half* crow = prm.C + row * prm.N + n0;
      if (nks == 0) {  // all-zero panel (R-Q21): C rows are zeros
        if (row < prm.M)
          for (int c = 0; c < kNTile && n0 + c < prm.N; c += 8)
            *reinterpret_cast<uint4*>(crow + c) = make_uint4(0, 0, 0, 0);
        continue;
      }
      const int a = it & 1;
      const uint32_t use = (uint32_t)(it >> 1);
      mbar_wait(&tfull[a], use & 1);
      tc_fence_after();
#pragma unroll 1
      for (int c0 = 0; c0 < kNTile; c0 += 32) {
        uint32_t r[32];
        tc_ld_32x32b_x32(tbase + ((uint32_t)(q * 32) << 16) + a * kAccCols + c0, r);
        tc_wait_ld();
        if (row < prm.M) {
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            if (n0 + c0 + 8 * j < prm.N) {
              uint4 pk;
              __half2 h0 = __floats2half2_rn(__uint_as_float(r[8 * j + 0]), __uint_as_float(r[8 * j + 1]));
              __half2 h1 = __floats2half2_rn(__uint_as_float(r[8 * j + 2]), __uint_as_float(r[8 * j + 3]));
              __half2 h2 = __floats2half2_rn(__uint_as_float(r[8 * j + 4]), __uint_as_float(r[8 * j + 5]));
              __half2 h3 = __floats2half2_rn(__uint_as_float(r[8 * j + 6]), __uint_as_float(r[8 * j + 7]));
              pk.x = *reinterpret_cast<uint32_t*>(&h0);
              pk.y = *reinterpret_cast<uint32_t*>(&h1);
              pk.z = *reinterpret_cast<uint32_t*>(&h2);
              pk.w = *reinterpret_cast<uint32_t*>(&h3);
              *reinterpret_cast<uint4*>(crow + c0 + 8 * j) = pk;
            }
          }
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&tempty[a]);
      ++it;
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<kTmemCols>(tbase);
}

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*,
                                  CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion,
                                  CUtensorMapFloatOOBfill);

EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFn>(p);
  }
  return fn;
}

int g_num_sms[64] = {0};
bool g_attr_set[64] = {false};

}  // namespace

int spmm_num_sms() {
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 64) return 148;
  if (!g_num_sms[dev]) cudaDeviceGetAttribute(&g_num_sms[dev], cudaDevAttrMultiProcessorCount, dev);
  return g_num_sms[dev];
}

jigsaw_status_t launch_spmm(const Format& f, const void* dB, int64_t N, void* dC, cudaStream_t s) {
  EncodeTiledFn enc = encode_fn();
  if (!enc) return set_status(JIGSAW_ERROR_CUDA, "cuTensorMapEncodeTiled unavailable");
  CUtensorMap tm;
  cuuint64_t gdim[2] = {(cuuint64_t)N, (cuuint64_t)f.K};
  cuuint64_t gstr[1] = {(cuuint64_t)N * 2};
  cuuint32_t box[2] = {64, 1};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, const_cast<void*>(dB), gdim, gstr, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_status(JIGSAW_ERROR_CUDA, "cuTensorMapEncodeTiled failed (" + std::to_string((int)r) + ")");
  SpmmParams prm;
  prm.Aimg = f.d_Aimg;
  prm.Eimg = f.d_Eimg;
  prm.G = f.d_G;
  prm.ksn = f.d_ksn;
  prm.ksoff = f.d_ksoff;
  prm.kboff = f.d_kboff;
  prm.C = reinterpret_cast<__half*>(dC);
  prm.M = f.M;
  prm.N = N;
  prm.npanels = (int)f.npanels;
  const int64_t ntn = (N + kNTile - 1) / kNTile;
  prm.nunits = (int)(f.npanels * ntn);
  int dev = f.device;
  if (dev >= 0 && dev < 64 && !g_attr_set[dev]) {
    cudaError_t e = cudaFuncSetAttribute(k_spmm, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemBytes);
    if (e != cudaSuccess) return cuda_status(e, "cudaFuncSetAttribute(k_spmm)");
    g_attr_set[dev] = true;
  }
  const int grid = (int)std::min<int64_t>(prm.nunits, spmm_num_sms());
  k_spmm<<<grid, kThreads, kSmemBytes, s>>>(tm, prm);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_status(e, "k_spmm launch");
  return JIGSAW_SUCCESS;
}

}  // namespace jig
