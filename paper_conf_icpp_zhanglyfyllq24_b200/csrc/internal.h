// internal.h -- shared declarations of libjigsaw.so (host side + kernel launchers).
// Not part of the ABI (include/jigsaw.h is).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <string>
#include <vector>

#include "../../include/jigsaw.h"

namespace jig {

constexpr int kTileCols = 16;     // logical columns per tile (the paper's MMA_TILE width)
constexpr int kPanelRows = 128;   // P = tcgen05 M of one CTA (R-Q5); the default panel height
constexpr int kPairPanelRows = 256;  // P = tcgen05 M of a CTA pair (cta_group::2, R-Q6)
constexpr int kKStepBytesA = 4096;  // 128 rows x 16 halves (compressed 32 logical) per k-step and half
constexpr int kStepsPerBlock = 4;   // k-steps per E block (tcgen05.cp 128x128b = 4 TMEM columns)
constexpr int kEBlockBytes = 2048;  // 128 lanes x 16 B
constexpr int kPad = -1;
constexpr int kPinCC = 1 << 30;     // flag in the device copy of a panel's pin.w: the panel has CUDA-core entries

// Device-resident prepared matrix (the reorder-aware format).
struct Format {
  int64_t M = 0, K = 0;
  int v = 0, P = kPanelRows, mode = 0, device = 0;
  int c_dtype = JIGSAW_C_F16;  // element type of C written by jigsaw_spmm (jigsaw_options_t.c_dtype)
  int row_order = JIGSAW_ROWS_GIVEN;
  int32_t* d_rowmap = nullptr;  // [M] (row-clustered panels only): C row of panel row r
  int64_t npanels = 0, ntiles = 0, nksteps = 0, nkblocks = 0, ndtiles = 0;
  // host copies of per-panel counts / offsets
  std::vector<int32_t> T, D, tile_off, ks_off, kb_off;
  // device per-panel arrays
  int4* d_pin = nullptr;       // [npanels] {k-steps = ceil(T_p/2), first k-step, first E block, dense k-steps},
                               // .w | kPinCC on the device when the panel has CUDA-core entries (f3)
  std::vector<int4> pin;       // host copy of d_pin, without the kPinCC flag
  int4 pin_dev(int64_t p) const {  // the device form of pin[p]
    int4 x = pin[p];
    if (!ccT.empty() && ccT[p] > 0) x.w |= kPinCC;
    return x;
  }
  // canonical arrays (device)
  int32_t* d_colidx = nullptr;  // [ntiles][16]
  uint8_t* d_perm = nullptr;    // [ntiles][16]
  uint8_t* d_kind = nullptr;    // [ntiles]
  uint8_t* d_nevict = nullptr;  // [ntiles]
  // device layout consumed by the SpMM kernel
  // A and E are stored as P/128 planes, one per 128-row half of every panel (the
  // CTA of a pair that owns those rows), each plane contiguous per k-block.
  uint8_t* d_Aimg = nullptr;  // [halves][nksteps][4096]: UMMA K-major no-swizzle core matrices
  uint8_t* d_Eimg = nullptr;  // [halves][nkblocks][128][4] u32: TMEM metadata lanes
  int32_t* d_G = nullptr;     // [nksteps][32]: B row per logical column (PAD -> K, TMA zero fill)
  // CUDA-core tiles (f3, R-Q28; jigsaw_options_t.cc_max_nnz): the entries of row
  // r of the (padded) panel rows -- global panel-row index pr = p * P + r -- are
  // d_ccent[d_ccoff[pr] .. d_ccoff[pr + 1]), each {column, fp16 bits}, ordered
  // by column; null when no tile moved
  int cc_max_nnz = 0;
  int64_t cc_tiles = 0, cc_entries = 0;
  std::vector<int32_t> ccT;     // [npanels] tiles moved per panel
  int32_t* d_ccoff = nullptr;   // [npanels * P + 1]
  int2* d_ccent = nullptr;      // [cc_entries]
  int halves() const { return P > kPanelRows ? P / kPanelRows : 1; }
  int64_t planeA() const { return nksteps * (int64_t)kKStepBytesA; }
  int64_t planeE() const { return nkblocks * (int64_t)kEBlockBytes; }
  // stats
  int64_t nnz = 0, kp_total = 0, evictions = 0, overflow_tiles = 0, max_tiles = 0;
  int64_t device_bytes = 0;
  double reorder_ms = 0;
  std::vector<void*> allocs;
};

// status plumbing (api.cu)
jigsaw_status_t set_status(jigsaw_status_t s, const std::string& msg = "");
jigsaw_status_t cuda_status(cudaError_t e, const char* what);
// stream-ordered allocation from the library's private pool of the current
// device (api.cu); under stream capture it becomes a graph allocation node
cudaError_t pool_alloc_async(void** p, size_t bytes, cudaStream_t s);

// Diagnostic launch override (jigsaw_set_launch_override), per host thread.
struct LaunchOverride {
  int tile_n = 0;       // 0 = library choice; 32 / 64 / 128 / 256
  int split_k = 0;      // 0 = library choice; 1 / 2 / 4 / 8 (single products, NT 64 or 32)
  int no_pieces = 0;    // 1: grouped launches never cut units into k-range pieces
  int host_chunks = 0;  // 0 = default; > 0: chunks of jigsaw_spmm_batched_host
  int k_pieces = 0;     // 1: split long units by k-range pieces (workspace) instead of N slices
};
LaunchOverride& launch_override();
jigsaw_launch_desc_t& last_launch();  // this thread's most recent jigsaw_spmm* call

// reorder.cu: builds *f from device A (M x K fp16) on `stream`; synchronous.
jigsaw_status_t build_format(const uint16_t* dA, int64_t M, int64_t K, int v, int P, int mode, int row_order,
                             int cc_max_nnz, cudaStream_t stream, Format* f);
void free_format(Format* f);

// spmm.cu
jigsaw_status_t launch_spmm(const Format& f, const void* dB, int64_t N, void* dC, cudaStream_t s);
jigsaw_status_t launch_spmm_grouped(const Format* const* fs, const void* const* Bs, const int64_t* Ns,
                                    void* const* Cs, int count, cudaStream_t s);
int spmm_num_sms();
int debug_trace_read(long long* host, int max_ctas);

}  // namespace jig
