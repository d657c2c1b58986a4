// spmm.cu -- S1: the SpMM mainloop C = A x B on sm_100a sparse tensor cores
// (DESIGN.md §5.2).  PAPER.md P:120-128 (CTA per C tile, B gathered through the
// reorder indices, C written straight from the accumulators)
// (deepened pipeline: gather indices fetched ahead of the B copies), re-designed
// for tcgen05:
//
//   512 threads (16 warps), warp-specialised, mbarrier ring of kStages k-blocks
//   (k-block = 4 k-steps = 128 logical columns = 8 tiles):
//     warp 0      A/E producer : cp.async.bulk of the compressed A image (4 KB per
//                               k-step) and of the TMEM metadata block (2 KB); a
//                               second cursor fills the gather-list ring ahead
//     warps 9, 13  (static schedules) metadata blocks / gather-list ring, split
//                               off warp 0, whose one thread paced the k-blocks
//     warps 6-15  B producers  : 8 warps (9 and 13 not: SM sub-partition 1 is
//     except 9,13               left to the MMA warp) gather the B rows of the
//                               k-block with 16-byte cp.async straight into the
//                               SW128 MN-major UMMA layout (PAD rows / columns
//                               >= N zero-filled)
//     warp 1      MMA issuer   : tcgen05.cp metadata -> TMEM, then per k-step one
//                               tcgen05.mma.sp.kind::f16 (M = 128, or M = 256 on a
//                               CTA pair) x N = NT x K = 32 (logical) into fp32
//                               TMEM accumulators; odd CTA of a pair: the relay
//     warps 2-5   epilogue     : tcgen05.ld -> fp16 (RN) -> C rows < M (and the
//                               first unit's initial loads at kernel start)
//   Launched with programmatic stream serialization: everything before
//   griddepcontrol.wait touches only handle-owned data.
//   Work unit = (panel, NT columns of C).  Persistent grouped launches (a
//   dynamic tile scheduler, or a static LPT schedule for CTA pairs) split long
//   units into k-range pieces reduced by the last piece to finish.  Split-K for
//   single small products: a cluster of S CTAs shares one unit, each CTA runs
//   1/S of the panel's k-blocks, and the fp32 partial tiles are reduce-scattered
//   through DSMEM by bulk copies (owner CTA r sums rows [r*128/S, (r+1)*128/S)
//   and writes them to C).
#include <cuda_fp16.h>

#include <algorithm>
#include <atomic>
#include <cstdio>
#include <mutex>
#include <utility>
#include <vector>
#include <string>
#include <type_traits>
#include <unordered_map>

#include "internal.h"
#include "ptx.cuh"

#ifndef JIG_BGROUPS
#define JIG_BGROUPS 1  // B-producer warp groups (see Cfg::kBGroups); > 1 measured slower in k_spmm
#endif
#ifndef JIG_RELAY
#define JIG_RELAY 1  // pair relay: bit 0 fence.proxy.async, bit 1 release.cluster arrive (else relaxed; release: C4 +16 %)
#endif
#ifndef JIG_EARLY_TRIGGER
#define JIG_EARLY_TRIGGER 1  // griddepcontrol.launch_dependents once a CTA has fetched its last unit
#endif
#ifndef JIG_DEV
#define JIG_DEV 0  // developer build (-DJIG_DEV=1): timing-only JIGSAW_DBG modes and schedule experiments
#endif
#ifndef JIG_AE_SPLIT
#define JIG_AE_SPLIT 1  // static schedules: metadata copies on warp 9, gather lists on warp 13 (else all on warp 0)
#endif

namespace jig {

namespace {

constexpr unsigned kFullMask = 0xFFFFFFFFu;
constexpr int kBProdWarp0 = 6;
#ifndef JIG_BWARPS
#define JIG_BWARPS 8
#endif
constexpr int kBProdWarps = JIG_BWARPS;  // B-producer (cp.async) warps
                                 // reach ~36 B/clk/SM vs ~28 with 4 (profiles/r01_gather_bench.txt)
// Warps 6-15 except 9 and 13 are the B producers: warp w runs on SM
// sub-partition w % 4, and sub-partition 1 is left to the MMA warp (1) and one
// epilogue warp (5), so the single-thread tcgen05 issue loop is not starved of
// issue slots by producer warps (warps 9 and 13 idle).
#ifndef JIG_SPARE_SMSP1
#define JIG_SPARE_SMSP1 1
#endif
constexpr int kThreads = JIG_SPARE_SMSP1 ? 32 * 16 : 32 * (kBProdWarp0 + kBProdWarps);
__device__ __forceinline__ int bprod_index(int warp) {  // -1: not a B producer
  if (warp < kBProdWarp0) return -1;
  if (!JIG_SPARE_SMSP1) return warp - kBProdWarp0;
  if ((warp & 3) == 1) return -1;
  const int i = warp - kBProdWarp0;  // 0..9 -> skip 3 (warp 9) and 7 (warp 13)
  return i - (i > 3) - (i > 7);
}
constexpr int kBarInit = 2, kBarTmem = 3;  // named barriers (1: epilogue warps, split pieces)
constexpr int kRowsPerBlock = 32 * kStepsPerBlock;  // B rows per k-block (128)
constexpr int kChunkB = kRowsPerBlock * 128;        // one 64-column SW128 chunk: 16 KB
constexpr int kStageA = kStepsPerBlock * kKStepBytesA;  // 16 KB
constexpr int kStageE = kEBlockBytes;               // 2 KB
constexpr int kStageG = kRowsPerBlock * 4;          // gather list of a k-block: 512 B

// NT = the MMA's N (C columns per work unit).  kPair: a cluster of two CTAs runs
// one 256-row panel with tcgen05 cta_group::2 (M = 256); each CTA stages NT/2 of
// the B columns and holds its 128 rows x NT accumulator.
template <int NT, bool kSplit, bool kPair = false>
struct Cfg {
  static constexpr int kNTL = kPair ? NT / 2 : NT;  // B columns staged by this CTA
  // B is staged as 64-column SW128 chunks; NT = 32 fills the first half of one
  // chunk (the MMA with N = 32 reads only those columns of the swizzled atom)
  static constexpr int kChunks = kNTL >= 64 ? kNTL / 64 : 1;
  static constexpr int kStageB = kChunks * kChunkB;
#ifndef JIG_STAGE_DELTA
#define JIG_STAGE_DELTA 0  // developer: stage-count sensitivity experiments
#endif
  static constexpr int kStages = (kPair ? (NT == 256 ? 4 : 6) : NT == 256 ? 2 : NT == 128 ? 4 : 5) + JIG_STAGE_DELTA;
  static constexpr int kAccCols = NT;
  // TMEM (512 columns): double-buffered fp32 accumulators, one for NT = 256
  // (two half-width accumulators issued as N = 128 MMAs measured slower in
  // round 1); then 4 metadata columns per stage
  static constexpr int kAccBufs = NT == 256 ? 1 : 2;
  static constexpr int kEColBase = kAccBufs * NT;
  static constexpr uint32_t kTmemCols = kAccBufs * NT + 4 * kStages <= 256 ? 256 : 512;
  static constexpr int kRecvStride = NT * 4 + 16;          // bytes per received row (padded)
  static constexpr int kRecvBytes = kSplit ? 128 * kRecvStride : 0;
  static constexpr int kStageC = 4 * 32 * 64;  // epilogue: per warp 32 rows x 32 fp16 columns
  // gather-list ring: twice as deep as the stage ring, filled kStages k-blocks
  // ahead of the A/E copies, so the B producers never wait on the gather list
  // B-producer warp groups: group g fills the k-blocks j (CTA-wide k-block
  // sequence number) with j % kBGroups == g, its 8 / kBGroups warps splitting the
  // 128 rows.  A warp's cp.async batches complete one after another, so k_spmm's
  // gather rate grows with the number of k-blocks in flight from DIFFERENT warps
  // (tools/ldgsts_probe.cu, profiles/r01s_ldgsts_probe.txt: 64-byte rows 9.6 ->
  // 22.6 B/clk/SM, 256-byte rows 18.7 -> 32.6).  kBGroups <= kStages keeps every
  // parity wait within one phase; kGS is a multiple of kBGroups so each gather
  // ring slot always belongs to the same group.
  static constexpr int kBGroups = JIG_BGROUPS < kStages ? JIG_BGROUPS : kStages;
  static constexpr int kWPG = kBProdWarps / kBGroups;  // warps per group
  static constexpr int kGS = (2 * kStages + kBGroups - 1) / kBGroups * kBGroups;
#ifndef JIG_GAHEAD_EXTRA
#define JIG_GAHEAD_EXTRA 0  // developer: gather-list lead beyond the stage count
#endif
  static constexpr int kGAhead = kStages + JIG_GAHEAD_EXTRA;
  static constexpr size_t kSmem =
      1024 + (size_t)kStages * (kStageB + kStageA + kStageE) + (size_t)kGS * kStageG + kRecvBytes + kStageC + 512;
  static_assert(kSmem <= 232448, "shared memory budget");
};

// One product of a (possibly grouped) launch.
struct Problem {
  const uint8_t* Aimg;
  const uint8_t* Eimg;
  const int32_t* G;
  const int4* pin;  // per panel {k-steps, first k-step, first E block, 0} (device)
  const __half* B;
  void* C;  // fp16 or fp32 (c32) row-major M x N
  const int32_t* rowmap;  // row-clustered panels: C row of panel row r (nullptr: identity)
  const int32_t* ccoff;   // CUDA-core entries (f3): offsets per padded panel row (nullptr: none)
  const int2* ccent;      //   {column, fp16 bits} per entry
  int64_t boff;  // offset of this problem's B in the concatenation of all B's (L2 prefetch)
  // 32-bit fields keep the 64-problem table of grouped launches in parameter space
  int32_t M, N, K;  // M < 2^31, N, K <= 2^30 (validated)
  int32_t nksA, nkbE;  // k-steps / E blocks between the A / E planes of the two 128-row halves (P = 256)
  int npanels;
  int unit0;  // first global work unit of this problem
  int pin0;   // offset of this problem's panels in ParamsT::pin (if use_pin)
  int c32;    // 1: C is fp32 (jigsaw_options_t.c_dtype), else fp16
};
// Kernel parameters: a problem table and the panel table, kept in parameter space
// (read with LDC, no dependent global load at kernel start).  Two sizes: a
// small block for single products (cheap to launch) and a large one for grouped
// launches.
template <int MAXP, int MAXPIN, int MAXU, int MAXC = 1>
struct ParamsT {
  static constexpr int kMaxProblems = MAXP;
  static constexpr int kMaxPin = MAXPIN;
  static constexpr int kMaxUnits = MAXU;
  static constexpr int kMaxCta = MAXC;
  Problem pr[MAXP];
  int4 pin[MAXPIN];
  // single products: the first unit of every CTA pre-decoded on the host, indexed
  // by blockIdx.x (one level of parameter loads instead of a dependent chain):
  // [c][0] = {panel, first C column, kb_lo, kb_hi}, [c][1] = {k-steps, dense
  // k-steps, first k-step, first E block} of the panel
  int4 ctab[MAXC][2];
  int use_ctab;
  // L2 prefetch of B at kernel start (when all B's of the launch fit in L2 with
  // room to spare): CTA c prefetches bytes [c*bpf_chunk, (c+1)*bpf_chunk) of the
  // concatenation of the problems' B matrices (bpf_bytes in total), in parallel
  // with the gather-list fetches the B row gathers depend on
  int64_t bpf_bytes, bpf_chunk;
  // grouped launches: schedule position -> work piece, packed as
  //   problem (6 bits) | local unit (11) | piece (3) | pieces - 1 (3) | partial slot (9)
  // a unit split into `pieces` k-ranges (split-K inside the persistent launch)
  // reduces its fp32 partials through `ws` (slots pslot .. pslot + pieces - 1)
  uint32_t ulist[MAXU];
  // Per-launch workspace (a region owned by the launching stream, or a graph-owned
  // allocation under stream capture; spmm.cu acquire_workspace): counters that
  // are zero at launch start and left zero, and the fp32 partial tiles of split units
  float* ws;       // partial tiles: [slot][rank][NT / 32][warp 4][8][lane 32][4] fp32
  int* wcnt;       // per split unit and CTA rank: pieces finished (reset by the last piece)
  int* sched_ctr;  // dynamic tile scheduler: [next ticket, CTAs done fetching] (reset by the last CTA)
  int nprob, nunits, S, use_pin, use_ulist;
  int dyn;    // 1: dynamic tile scheduler on sched_ctr; 0: static (round-robin / host schedule)
  int trace;  // 1: record a per-CTA timeline into g_trace (JIGSAW_TRACE=1)
  int prefetch;  // 1: prefetch each unit's gather lists / metadata into L2 at unit start
  int dbg;       // developer timing experiments (JIGSAW_DBG, results invalid): 1 skip tcgen05.cp, 2 skip MMAs,
                 // 8 no B reads (zero fill), 16 no A / metadata loads after the initial fill
};
using ParamsOne = ParamsT<1, 128, 1, 160>;   // single product (~7.3 KB of parameters)
using ParamsGroup = ParamsT<64, 1024, 2048>; // grouped launch (~31 KB)
constexpr int kMaxProblems = ParamsGroup::kMaxProblems;

// Opt-in per-CTA timeline (clock64 / %globaltimer), read by jigsaw_debug_trace.
constexpr int kTraceCTAs = 1024, kTraceSlots = 24;
__device__ long long g_trace[kTraceCTAs * kTraceSlots];
constexpr int kTraceKB = 32;
__device__ long long g_trace_kb[8 * 6 * kTraceKB];  // [cta<8][AE issue, B issue, full seen, commit, after cp, after mma][kb]
// Per-k-block timeline (developer builds only: -DJIG_TRACE_KB_ON=1); in the
// product build the hot loops carry no per-k-block trace code.
#ifndef JIG_TRACE_KB_ON
#define JIG_TRACE_KB_ON 0
#endif
#define JIG_TRACE_KB(role, n)                                                        \
  do {                                                                               \
    if (JIG_TRACE_KB_ON && prm.trace && blockIdx.x < 8 && (n) < kTraceKB)            \
      g_trace_kb[(blockIdx.x * 6 + (role)) * kTraceKB + (n)] = clock64();            \
  } while (0)
__device__ __forceinline__ long long gtimer() {
  long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ uint32_t smid() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}
#define JIG_TRACE(k)                                                                  \
  do {                                                                                \
    if (prm.trace && blockIdx.x < kTraceCTAs) g_trace[blockIdx.x * kTraceSlots + (k)] = clock64(); \
  } while (0)

// Work unit u -> (problem, panel, first C column, k-block range of this CTA).
// Fields are copied out of the parameter space by value (LDC); a pointer into the
// kernel parameters would turn every access into a slow generic load.
struct Work {
  const uint8_t* Aimg;
  const uint8_t* Eimg;
  const int32_t* G;
  const __half* B;
  void* C;
  int c32;
  const int32_t* rowmap;
  const int32_t* ccoff;
  const int2* ccent;
  int64_t M, N, K;
  int p, n0, nks, ndk, nkb_s, kb_lo, kb_hi;
  int piece, npieces, pslot;  // split-K piece of a grouped launch (npieces = 1: whole unit)
  bool ccp;                   // the panel has CUDA-core entries (f3; kPinCC)
  int ncols;                  // C columns of this unit (NT, or NT / nsplit for an N-split unit)
  bool valid;                 // false: padding entry of a static per-slot schedule
  int64_t ks0, kb0;  // first k-step / E block of the panel
  int64_t row0;      // first C row written by this CTA
  // k-block kb of the panel: the first nkb_s are 2:4 sparse (4 k-steps of 32
  // logical columns each, metadata block kb0 + kb); the rest (DENSE residual mode)
  // hold up to 4 dense K = 16 steps each, stored after the sparse k-steps.
  __device__ __forceinline__ bool dense(int kb) const { return kb >= nkb_s; }
  __device__ __forceinline__ int steps(int kb) const {
    return kb < nkb_s ? min(kStepsPerBlock, nks - kb * kStepsPerBlock)
                      : min(kStepsPerBlock, ndk - (kb - nkb_s) * kStepsPerBlock);
  }
  __device__ __forceinline__ int64_t gks(int kb) const { return ks0 + (int64_t)kb * kStepsPerBlock; }
};
constexpr uint32_t kNoWork = 0xFFFFFFFFu;  // schedule padding
// Schedule code with partial-slot field kNSplit: an N-split unit, piece `piece`
// of `pieces` column slices of width NT / pieces (full k-range, no workspace).
constexpr uint32_t kNSplit = 0x1FFu;
// `hint` = problem index of this thread's previous unit: units are visited in
// increasing order, so the scan is amortised O(1) instead of O(problems).
// kPair: `rank` selects this CTA's 128-row half of the 256-row panel (its A / E
// plane); otherwise it selects the CTA's k-block share of a split-K cluster of S.
template <int NT, bool kPair, class Prm>
__device__ __forceinline__ Work decode_unit(const Prm& prm, int u, uint32_t rank, int S, int& hint) {
  int i, lu, piece = 0, npieces = 1, pslot = 0;
  Work w;
  w.valid = true;
  if constexpr (Prm::kMaxCta > 1 && !kPair) {
    if (prm.use_ctab && (int)blockIdx.x == u * S + (int)rank) {  // the CTA's first unit, host-decoded
      const int4 a = prm.ctab[blockIdx.x][0], b = prm.ctab[blockIdx.x][1];
      w.Aimg = prm.pr[0].Aimg;
      w.Eimg = prm.pr[0].Eimg;
      w.G = prm.pr[0].G;
      w.B = prm.pr[0].B;
      w.C = prm.pr[0].C;
      w.c32 = prm.pr[0].c32;
      w.rowmap = prm.pr[0].rowmap;
      w.ccoff = prm.pr[0].ccoff;
      w.ccent = prm.pr[0].ccent;
      w.M = prm.pr[0].M;
      w.N = prm.pr[0].N;
      w.K = prm.pr[0].K;
      w.p = a.x;
      w.n0 = a.y;
      w.kb_lo = a.z;
      w.kb_hi = a.w;
      w.nks = b.x;
      w.ndk = b.y & ~kPinCC;
      w.ccp = (b.y & kPinCC) != 0;
      w.ks0 = b.z;
      w.kb0 = b.w;
      w.nkb_s = (w.nks + kStepsPerBlock - 1) / kStepsPerBlock;
      w.piece = 0;
      w.npieces = 1;
      w.pslot = 0;
      w.ncols = NT;
      w.row0 = (int64_t)w.p * kPanelRows;
      return w;
    }
  }
  if (Prm::kMaxUnits > 1 && prm.use_ulist) {  // host-ordered schedule (longest pieces first)
    const uint32_t code = prm.ulist[u];
    if (code == kNoWork) {
      w.valid = false;
      return w;
    }
    i = (int)(code >> 26);
    lu = (int)((code >> 15) & 0x7FFu);
    piece = (int)((code >> 12) & 7u);
    npieces = (int)((code >> 9) & 7u) + 1;
    pslot = (int)(code & 0x1FFu);
  } else {
    i = hint;
    if (prm.pr[i].unit0 > u) i = 0;
    while (i + 1 < prm.nprob && prm.pr[i + 1].unit0 <= u) ++i;
    hint = i;
    lu = u - prm.pr[i].unit0;
  }
  w.Aimg = prm.pr[i].Aimg;
  w.Eimg = prm.pr[i].Eimg;
  w.G = prm.pr[i].G;
  w.B = prm.pr[i].B;
  w.C = prm.pr[i].C;
  w.c32 = prm.pr[i].c32;
  w.rowmap = prm.pr[i].rowmap;
  w.ccoff = prm.pr[i].ccoff;
  w.ccent = prm.pr[i].ccent;
  w.M = prm.pr[i].M;
  w.N = prm.pr[i].N;
  w.K = prm.pr[i].K;
  const int np = prm.pr[i].npanels;
  w.p = lu % np;
  w.n0 = (lu / np) * NT;
  w.ncols = NT;
  if (pslot == (int)kNSplit) {  // column slice `piece` of the N tile, whole k-range
    w.ncols = NT / npieces;
    w.n0 += piece * w.ncols;
    piece = 0;
    npieces = 1;
    pslot = 0;
  }
  // panel table from parameter space (no dependent global load at kernel start)
  const int4 pi = prm.use_pin ? prm.pin[prm.pr[i].pin0 + w.p] : prm.pr[i].pin[w.p];
  w.nks = pi.x;
  w.ks0 = pi.y;
  w.kb0 = pi.z;
  w.ndk = pi.w & ~kPinCC;
  w.ccp = (pi.w & kPinCC) != 0;
  w.nkb_s = (w.nks + kStepsPerBlock - 1) / kStepsPerBlock;
  const int nkb = w.nkb_s + (w.ndk + kStepsPerBlock - 1) / kStepsPerBlock;
  w.piece = piece;
  w.npieces = npieces;
  w.pslot = pslot;
  if constexpr (kPair) {
    w.Aimg += rank * (int64_t)prm.pr[i].nksA * kKStepBytesA;
    w.Eimg += rank * (int64_t)prm.pr[i].nkbE * kEBlockBytes;
    w.row0 = (int64_t)w.p * kPairPanelRows + rank * kPanelRows;
    w.kb_lo = piece * nkb / npieces;
    w.kb_hi = (piece + 1) * nkb / npieces;
  } else if (npieces > 1) {
    w.row0 = (int64_t)w.p * kPanelRows;
    w.kb_lo = piece * nkb / npieces;
    w.kb_hi = (piece + 1) * nkb / npieces;
  } else {
    w.row0 = (int64_t)w.p * kPanelRows;
    w.kb_lo = (int)(rank * nkb / S);
    w.kb_hi = (int)((rank + 1) * nkb / S);
  }
  return w;
}

// Dynamic tile scheduler (persistent launches): CTA b starts with unit b, then
// takes gridDim.x + atomicAdd(ticket).  The counters live in the launch's
// workspace (zero when the launch starts: see acquire_workspace) and are reset
// to zero by the last CTA to stop fetching, so the next launch that uses the
// same workspace (the next one on the stream) finds them zero.  (%gridid cannot
// tag launches instead: CUDA-graph replays reuse the value fixed at
// instantiation, tools/gridid_probe.cu.)
constexpr int kSD = 4;  // unit-ring depth

// Unit-ring consumer: the A/E producer publishes each unit id (or -1 = done)
// into a kSD-deep ring in shared memory; every consumer warp reads the same
// sequence and releases the slot (one arrival per warp).
__device__ __forceinline__ int ring_take(const volatile int* ring, uint64_t* rfull, uint64_t* rempty, int& slot,
                                         uint32_t& ph, bool full_warp, int lane) {
  mbar_wait(&rfull[slot], ph);
  const int u = ring[slot];
  if (full_warp) __syncwarp();
  if (lane == 0) mbar_arrive(&rempty[slot]);
  if (++slot == kSD) { slot = 0; ph ^= 1; }
  return u;
}

__device__ __forceinline__ float4 ld_shared_f4(uint32_t saddr) {
  float4 v;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(saddr));
  return v;
}

__device__ __forceinline__ uint32_t pack_h2(float a, float b) {
  __half2 h = __floats2half2_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}

// CUDA-core tiles (f3, §4.7; DESIGN.md R-Q28): acc[j] += a * B[col][col0 + j]
// for the entries {col, a} of this lane's panel row, j < width (columns past N
// are skipped: N % 8 == 0, 16-byte B reads).  fp32 FMA into the tensor-core
// accumulator before C is written.
__device__ __forceinline__ float cc_f(float x) { return x; }
__device__ __forceinline__ float cc_f(uint32_t x) { return __uint_as_float(x); }
__device__ __forceinline__ void cc_set(float& d, float x) { d = x; }
__device__ __forceinline__ void cc_set(uint32_t& d, float x) { d = __float_as_uint(x); }
template <int W, class T>
__device__ __forceinline__ void cc_accum(T (&acc)[W], const int2* __restrict__ ent, int e0, int e1,
                                         const __half* __restrict__ B, int64_t N, int64_t col0, int width) {
  for (int e = e0; e < e1; ++e) {
    const int2 en = __ldg(ent + e);
    const float a = __half2float(__ushort_as_half((unsigned short)en.y));
    const __half* brow = B + (int64_t)en.x * N + col0;
#pragma unroll
    for (int j = 0; j < W / 8; ++j) {
      if (8 * j < width && col0 + 8 * j < N) {
        const uint4 b = __ldg(reinterpret_cast<const uint4*>(brow + 8 * j));
        const __half2* h = reinterpret_cast<const __half2*>(&b);
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const float2 f = __half22float2(h[k]);
          cc_set(acc[8 * j + 2 * k], fmaf(a, f.x, cc_f(acc[8 * j + 2 * k])));
          cc_set(acc[8 * j + 2 * k + 1], fmaf(a, f.y, cc_f(acc[8 * j + 2 * k + 1])));
        }
      }
    }
  }
}

// Entries two at a time: both entries, then both B row segments are loaded
// before the FMAs (two dependent chains in flight instead of one per entry).
template <class T>
__device__ __forceinline__ void cc_accum2(T (&acc)[32], const int2* __restrict__ ent, int e0, int e1,
                                          const __half* __restrict__ B, int64_t N, int64_t col0, int width) {
  for (int e = e0; e < e1; e += 2) {
    const int n = min(e1 - e, 2);
    int2 en[2];
#pragma unroll
    for (int i = 0; i < 2; ++i) en[i] = i < n ? __ldg(ent + e + i) : make_int2(0, 0);
    uint4 b[2][4];
#pragma unroll
    for (int i = 0; i < 2; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j)
        b[i][j] = (i < n && 8 * j < width && col0 + 8 * j < N)
                      ? __ldg(reinterpret_cast<const uint4*>(B + (int64_t)en[i].x * N + col0 + 8 * j))
                      : make_uint4(0, 0, 0, 0);
#pragma unroll
    for (int i = 0; i < 2; ++i) {
      const float a = __half2float(__ushort_as_half((unsigned short)en[i].y));  // 0 for the padding entry
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const __half2* h = reinterpret_cast<const __half2*>(&b[i][j]);
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const float2 f = __half22float2(h[k]);
          cc_set(acc[8 * j + 2 * k], fmaf(a, f.x, cc_f(acc[8 * j + 2 * k])));
          cc_set(acc[8 * j + 2 * k + 1], fmaf(a, f.y, cc_f(acc[8 * j + 2 * k + 1])));
        }
      }
    }
  }
}

// Adds the CUDA-core entries of the warp's 32 rows (lane = row; panel-row index
// pr) to the fp32 accumulator in TMEM (taddr: the warp's lane quarter, column 0
// of the unit's buffer): tcgen05.ld -> FMAs -> tcgen05.st per 32 columns.
__device__ __noinline__ void cc_tmem_add(uint32_t taddr, int ncols, const int32_t* __restrict__ ccoff,
                                         const int2* __restrict__ ent, const __half* __restrict__ B, int64_t N,
                                         int64_t n0, int64_t pr) {
  const int e0 = ccoff[pr], e1 = ccoff[pr + 1];
  if (!__any_sync(kFullMask, e1 > e0)) return;
  for (int c0 = 0; c0 < ncols; c0 += 32) {
    uint32_t v[32];
    tc_ld_32x32b_x32(taddr + (uint32_t)c0, v);
    tc_wait_ld();
    if (e1 > e0) cc_accum2(v, ent, e0, e1, B, N, n0 + c0, ncols - c0);
    tc_st_32x32b_x32(taddr + (uint32_t)c0, v);
    tc_wait_st();
  }
}

// A unit whose panel has no tensor-core tile (every tile moved to the CUDA
// cores): this lane's C row (crow, -1: a padding row) is the sum of its
// entries, written directly (fp16 RN or fp32), 32 columns at a time.
__device__ __noinline__ void cc_only_store(void* C, int c32, int64_t crow, int ncols, int64_t N, int64_t n0,
                                           const int32_t* __restrict__ ccoff, const int2* __restrict__ ent,
                                           const __half* __restrict__ B, int64_t pr) {
  const int e0 = ccoff[pr], e1 = ccoff[pr + 1];
  for (int c0 = 0; c0 < ncols; c0 += 32) {
    float v[32];
#pragma unroll
    for (int j = 0; j < 32; ++j) v[j] = 0.f;
    if (e1 > e0) cc_accum2(v, ent, e0, e1, B, N, n0 + c0, ncols - c0);
    if (crow < 0) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int64_t col = n0 + c0 + 8 * j;
      if (8 * j >= ncols - c0 || col >= N) continue;
      if (c32) {
        float4* dst = reinterpret_cast<float4*>(static_cast<float*>(C) + crow * N + col);
        dst[0] = make_float4(v[8 * j], v[8 * j + 1], v[8 * j + 2], v[8 * j + 3]);
        dst[1] = make_float4(v[8 * j + 4], v[8 * j + 5], v[8 * j + 6], v[8 * j + 7]);
      } else {
        uint4 pk;
        pk.x = pack_h2(v[8 * j], v[8 * j + 1]);
        pk.y = pack_h2(v[8 * j + 2], v[8 * j + 3]);
        pk.z = pack_h2(v[8 * j + 4], v[8 * j + 5]);
        pk.w = pack_h2(v[8 * j + 6], v[8 * j + 7]);
        *reinterpret_cast<uint4*>(static_cast<__half*>(C) + crow * N + col) = pk;
      }
    }
  }
}

// kCC: the launch has CUDA-core entries (f3).  A separate instantiation, so the
// launches without them run the epilogue without the entry code (inlined or as a
// call, it cost C4 1-1.5 %: profiles/r02ab_*).
template <int NT, bool kSplit, bool kPair, class Prm, bool kCC>
__global__ void __launch_bounds__(kThreads, 1) k_spmm(const Prm prm) {
  static_assert(!(kSplit && kPair), "split-K and CTA pairs are separate variants");
  using C_ = Cfg<NT, kSplit, kPair>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sB = smem;                                   // kStages x kStageB (1024-aligned)
  uint8_t* sA = sB + C_::kStages * C_::kStageB;         // kStages x 16 KB
  uint8_t* sE = sA + C_::kStages * kStageA;             // kStages x 2 KB
  int32_t* sG = reinterpret_cast<int32_t*>(sE + C_::kStages * kStageE);  // kGS x 128 gather rows
  uint8_t* sRecv = reinterpret_cast<uint8_t*>(sG) + C_::kGS * kStageG;     // split-K receive buffer
  uint8_t* sC = sRecv + C_::kRecvBytes;                                       // epilogue staging
  uint64_t* full = reinterpret_cast<uint64_t*>(sC + C_::kStageC);
  uint64_t* empty = full + C_::kStages;
  uint64_t* gfull = empty + C_::kStages;  // gather-list ring slot has landed
  uint64_t* gempty = gfull + C_::kGS;     // gather-list ring slot read by all B producers
  uint64_t* tfull = gempty + C_::kGS;
  uint64_t* tempty = tfull + 3;
  uint64_t* recv_full = tempty + 3;
  uint64_t* rfull = recv_full + 1;   // unit ring (dynamic scheduler)
  uint64_t* rempty = rfull + kSD;
  uint64_t* pfull = rempty + kSD;    // kPair, even CTA: the odd CTA's stage has landed
  volatile int* ring = reinterpret_cast<volatile int*>(pfull + C_::kStages);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(pfull + C_::kStages) + kSD;
  const uint32_t s_last = smem_u32(tmem_slot + 1);  // split piece: this CTA reduces (int flag)

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (JIG_EARLY_TRIGGER == 2 && threadIdx.x == 0) griddep_launch_dependents();  // at entry (A/B option)
  const int S = kSplit ? prm.S : 1;
  const int CS = kPair ? 2 : S;  // CTAs per cluster
  const uint32_t rank = (kSplit || kPair) ? cluster_ctarank() : 0;
  const int cluster_id = blockIdx.x / CS, nclusters = gridDim.x / CS;
  const bool dyn = !kSplit && !kPair && prm.dyn;  // CTA pairs always run a static plan
  if (threadIdx.x == 0 && prm.trace && blockIdx.x < kTraceCTAs) {
    g_trace[blockIdx.x * kTraceSlots + 15] = gtimer();
    g_trace[blockIdx.x * kTraceSlots + 14] = smid();
    JIG_TRACE(0);
  }

  // The CTA's first unit, decoded from parameter space by the warps that issue
  // its first loads (the epilogue warps, idle until the first accumulator is
  // ready) while warp 0 initialises the barriers; warp 0 decodes it afterwards
  // for its own bookkeeping.
  int nA0 = 0, nG0 = 0;
  Work w0;
  w0.valid = false;
  auto decode_first = [&]() {
    if (cluster_id < prm.nunits) {
      int h0 = 0;
      w0 = decode_unit<NT, kPair, Prm>(prm, cluster_id, rank, S, h0);
      if (w0.valid) {
        const int nkb = w0.kb_hi - w0.kb_lo;
        nA0 = min(nkb, C_::kStages);
        nG0 = min(nkb, C_::kGAhead + 1);
      }
    }
  };
  // Static schedules split warp 0's per-k-block issue work (each mbarrier /
  // bulk-copy operation costs ~100 cycles from one thread, and warp 0 paced the
  // k-blocks: its copies left ~1,000 cycles after the B producers saw the same
  // free stage, profiles/r02ac_kblock_timeline_c4.txt): warp 0 the compressed A,
  // warp 9 the metadata blocks, warp 13 the gather-list ring (9 and 13 were idle).
  const bool split_ae = JIG_AE_SPLIT && JIG_SPARE_SMSP1 && !dyn;
  if ((warp >= 2 && warp <= 5) || (split_ae && (warp == 9 || warp == 13))) decode_first();

  // Barrier initialisation spread over the lanes of warp 0 (~50 barriers; one
  // thread initialising them all costs ~0.5 us of kernel start).  The barriers
  // are contiguous in shared memory: full, empty, gfull, gempty, tfull, tempty,
  // recv_full, rfull, rempty, pfull.
  if (warp == 0) {
    constexpr int nb = 3 * C_::kStages + 2 * C_::kGS + 7 + 2 * kSD;
    for (int i = lane; i < nb; i += 32) {
      int k = i;
      uint32_t cnt;
      if (k < C_::kStages) cnt = (split_ae ? 2 : 1) + 32 * C_::kWPG;  // full: A (and E) expect_tx + the B group's cp.async
      else if ((k -= C_::kStages) < C_::kStages) cnt = 1;  // empty
      else if ((k -= C_::kStages) < C_::kGS) cnt = 1;      // gfull
      else if ((k -= C_::kGS) < C_::kGS) cnt = C_::kWPG;   // gempty
      else if ((k -= C_::kGS) < 3) cnt = 1;                // tfull
      else if ((k -= 3) < 3) cnt = kPair ? 8 : 4;          // tempty: epilogue warps (of both CTAs of a pair)
      else if ((k -= 3) < 1) cnt = 1;                      // recv_full
      else if ((k -= 1) < kSD) cnt = 1;                    // rfull
      else if ((k -= kSD) < kSD) cnt = kBProdWarps + 1 + 4;  // rempty: B-producer warps + MMA + epilogue warps
      else cnt = 1;                                        // pfull
      mbar_init(full + i, cnt);
    }
    fence_barrier_init();
    fence_proxy_async();
    if (lane == 0) JIG_TRACE(17);
    named_bar_arrive(kBarInit, kThreads);  // the barriers are valid
    decode_first();
  } else {
    if (warp == 1) {  // the TMEM allocation overlaps the barrier initialisation
      if constexpr (kPair)
        tmem_alloc_pair<C_::kTmemCols>(tmem_slot);
      else
        tmem_alloc<C_::kTmemCols>(tmem_slot);
    }
    named_bar_sync(kBarInit, kThreads);
  }
  // Cluster variants: peers' barriers must be initialised before any remote
  // arrive / st.async / pair MMA targets them.  Every thread arrives here; only
  // the warps that touch peer shared memory (MMA, relay, epilogue) wait before
  // their first remote operation, the others at exit.
  if constexpr (kSplit || kPair) cluster_arrive_relaxed();
  bool cl_waited = !(kSplit || kPair);
  // Initial fill, spread over warps so the first loads leave at once (each
  // mbarrier / bulk-copy operation costs ~100 cycles of issue from one thread,
  // and a per-lane bulk copy is serialised): warp 2 issues the gather lists of
  // the first unit's first k-blocks (ring slots 0 .. nG0-1; the B producers
  // depend on them), warps 3-5 the compressed A / metadata of stages
  // (warp - 3) + 3i.  All of it is handle-owned, immutable data, so it runs
  // before griddepcontrol.wait.
  if (warp == 2) {
    if (lane == 0) {
      JIG_TRACE(18);
      for (int l = 0; l < nG0; ++l) {
        const int kb = w0.kb_lo + l;
        const int steps = w0.steps(kb);
        mbar_arrive_expect_tx(&gfull[l], (uint32_t)(steps * 128));
        bulk_g2s(sG + l * kRowsPerBlock, w0.G + w0.gks(kb) * 32, steps * 128, &gfull[l]);
      }
    }
    __syncwarp();
  } else if (warp >= 3 && warp <= 5) {
    if (lane == 0) {
      for (int l = warp - 3; l < nA0; l += 3) {
        const int kb = w0.kb_lo + l;
        const int steps = w0.steps(kb);
        const bool dense = w0.dense(kb);
        mbar_arrive_expect_tx(&full[l], (uint32_t)(steps * kKStepBytesA + (dense ? 0 : kStageE)));
        bulk_g2s(sA + l * kStageA, w0.Aimg + w0.gks(kb) * kKStepBytesA, steps * kKStepBytesA, &full[l]);
        if (!dense) bulk_g2s(sE + l * kStageE, w0.Eimg + (w0.kb0 + kb) * kEBlockBytes, kStageE, &full[l]);
        if (split_ae) mbar_arrive(&full[l]);  // the metadata warp's arrival for this stage
      }
      if (warp == 3 && nA0 > 0) JIG_TRACE(2);
    }
    __syncwarp();
  } else if (warp == 0 && prm.bpf_bytes > 0) {
    const int64_t lo = (int64_t)blockIdx.x * prm.bpf_chunk, hi = min(prm.bpf_bytes, lo + prm.bpf_chunk);
    for (int i = 31 - lane; i < prm.nprob; i += 32) {  // lane 31 takes problem 0
      const int64_t b0 = prm.pr[i].boff, b1 = b0 + (int64_t)prm.pr[i].K * prm.pr[i].N * 2;
      const int64_t x0 = max(lo, b0), x1 = min(hi, b1);
      if (x0 < x1)
        bulk_prefetch_l2(reinterpret_cast<const uint8_t*>(prm.pr[i].B) + (x0 - b0), (uint32_t)(x1 - x0));
    }
    if (lane == 31) JIG_TRACE(22);
    __syncwarp();
  }
  // TMEM address: warp 1 (allocator, MMA issuer) and the epilogue warps 2-5
  uint32_t tbase = 0;
  if (warp >= 1 && warp <= 5) {
    tc_fence_before();
    named_bar_sync(kBarTmem, 5 * 32);
    tc_fence_after();
    tbase = *tmem_slot;
    if (threadIdx.x == 32) JIG_TRACE(1);
    if constexpr (kSplit || kPair) {
      cluster_wait();
      cl_waited = true;
    }
  }

  if (warp == 0) {
    // ------------------------------------------------------------ A / E producer
    if (lane == 0) {
      // the dynamic scheduler's ticket is shared with the previous launch on the stream
      if (dyn) griddep_wait();
      // state after the parallel initial fill: stages 0..nA0-1 and gather slots
      // 0..nG0-1 hold the first unit's first k-blocks
      int stage = nA0 % C_::kStages, hint = 0, nkb_issued = nA0, rslot = 0;
      uint32_t phase = nA0 == C_::kStages ? 1u : 0u, rph = 0;
      int* const ctr = prm.sched_ctr;
      // Unit sequence of this CTA (static stride or dynamic scheduler), fetched
      // into a small queue shared by two cursors over the same (unit, k-block)
      // sequence: the gather-list cursor runs kGAhead k-blocks ahead of the A/E
      // cursor, so gather lists land long before their B rows are needed
      // (the P:220-226 dependency, pipelined one level further).
      constexpr int kQ = 16;
      int uq[kQ];
      int qn = 0, mq = 0, next_un = cluster_id;
      // Queues the CTA's next unit (-1 = none left); the dynamic scheduler's
      // ticket for the one after is taken here, its value needed only then
      auto fetch = [&]() {
        const int un = next_un < prm.nunits ? next_un : -1;
        if (un >= 0) next_un = dyn ? (int)gridDim.x + atomicAdd(ctr, 1) : un + nclusters;
        uq[qn % kQ] = un;
        ++qn;
      };
      // gather-list cursor
      int gq = 0, ghint = 0, gkb = 0, gkbe = 0, gslot = nG0 % C_::kGS;
      uint32_t gph = nG0 == C_::kGS ? 1u : 0u;
      int64_t gj = nG0;
      bool gend = false;
      Work gwk = w0;
      if (nG0 > 0) {  // the gather cursor continues inside the first unit
        fetch();
        gq = 1;
        gkb = w0.kb_lo + nG0;
        gkbe = w0.kb_hi;
      }
      auto g_issue_upto = [&](int64_t limit) {
        while (gj < limit && !gend) {
          if (gkb >= gkbe) {  // next unit with work
            if (gq == qn) {
              if (qn - mq >= kQ) return;  // queue full: the A/E cursor catches up first
              fetch();
            }
            const int u = uq[gq % kQ];
            if (u < 0) {
              gend = true;
              return;
            }
            ++gq;
            gwk = decode_unit<NT, kPair, Prm>(prm, u, rank, S, ghint);
            if (!gwk.valid) continue;
            gkb = gwk.kb_lo;
            gkbe = gwk.kb_hi;
            continue;
          }
          const int steps = gwk.steps(gkb);
          mbar_wait(&gempty[gslot], gph ^ 1);
          mbar_arrive_expect_tx(&gfull[gslot], (uint32_t)(steps * 128));
          bulk_g2s(sG + gslot * kRowsPerBlock, gwk.G + gwk.gks(gkb) * 32, steps * 128, &gfull[gslot]);
          ++gkb;
          ++gj;
          if (++gslot == C_::kGS) { gslot = 0; gph ^= 1; }
        }
      };
      int64_t mi = nA0;  // k-blocks issued by the A/E cursor
      for (;;) {
        if (mq == qn) fetch();
        if (mq == 0) JIG_TRACE(16);
        const int u = uq[mq % kQ];
        ++mq;
        if (dyn) {  // publish the unit to the other warp roles
          mbar_wait(&rempty[rslot], rph ^ 1);
          ring[rslot] = u;
          mbar_arrive(&rfull[rslot]);
          if (++rslot == kSD) { rslot = 0; rph ^= 1; }
        }
        if (u < 0) break;
        const Work wk = decode_unit<NT, kPair, Prm>(prm, u, rank, S, hint);
        if (!wk.valid) continue;
        const int64_t kb0 = wk.kb0;
        if (prm.prefetch && wk.kb_hi > wk.kb_lo) {
          // the unit's metadata into L2 up front
          const int kbe = min(wk.kb_hi, wk.nkb_s);
          if (kbe > wk.kb_lo)
            bulk_prefetch_l2(wk.Eimg + (kb0 + wk.kb_lo) * kEBlockBytes, (uint32_t)(kbe - wk.kb_lo) * kEBlockBytes);
        }
        for (int kb = wk.kb_lo + (mq == 1 ? nA0 : 0); kb < wk.kb_hi; ++kb) {
          if (!split_ae) g_issue_upto(mi + 1 + C_::kGAhead);
          const int steps = wk.steps(kb);
          const bool dense = wk.dense(kb);
          const int64_t gks = wk.gks(kb);
          mbar_wait(&empty[stage], phase ^ 1);
          if (JIG_DEV && (prm.dbg & 16)) {  // timing only: no A / metadata loads
            mbar_arrive(&full[stage]);
          } else if (split_ae) {
            mbar_arrive_expect_tx(&full[stage], (uint32_t)(steps * kKStepBytesA));
            bulk_g2s(sA + stage * kStageA, wk.Aimg + gks * kKStepBytesA, steps * kKStepBytesA, &full[stage]);
          } else {
            mbar_arrive_expect_tx(&full[stage], (uint32_t)(steps * kKStepBytesA + (dense ? 0 : kStageE)));
            bulk_g2s(sA + stage * kStageA, wk.Aimg + gks * kKStepBytesA, steps * kKStepBytesA, &full[stage]);
            if (!dense) bulk_g2s(sE + stage * kStageE, wk.Eimg + (kb0 + kb) * kEBlockBytes, kStageE, &full[stage]);
          }
          if (u == cluster_id && kb == wk.kb_lo) JIG_TRACE(2);
          JIG_TRACE_KB(0, nkb_issued);
          ++nkb_issued;
          ++mi;
          if (++stage == C_::kStages) { stage = 0; phase ^= 1; }
        }
      }
      if (dyn) {  // the last CTA to stop fetching resets the ticket for the next launch
        __threadfence();
        if (atomicAdd(ctr + 1, 1) == (int)gridDim.x - 1) {
          atomicExch(ctr, 0);
          atomicExch(ctr + 1, 0);
        }
      }
      // This CTA takes no more units: once every CTA got here (all of them are
      // resident, so this cannot starve the grid), the next kernel of the stream
      // may launch and run its prologue on the SMs this grid frees; its B / C /
      // workspace / scheduler accesses still wait for this grid to complete.
      if (JIG_EARLY_TRIGGER == 1) griddep_launch_dependents();
    }
  } else if (split_ae && warp == 9) {
    // ------------------------------------------------------------ metadata producer (static schedules)
    // The same (unit, k-block) sequence and stage ring as warp 0: per k-block one
    // metadata bulk copy (its own expect_tx), or a plain arrival for a DENSE
    // k-block; the first unit's first nA0 stages were filled by the initial fill.
    if (lane == 0) {
      int stage = nA0 % C_::kStages, hint = 0;
      uint32_t phase = nA0 == C_::kStages ? 1u : 0u;
      for (int us = cluster_id; us < prm.nunits; us += nclusters) {
        const Work wk = decode_unit<NT, kPair, Prm>(prm, us, rank, S, hint);
        if (!wk.valid) continue;
        for (int kb = wk.kb_lo + (us == cluster_id ? nA0 : 0); kb < wk.kb_hi; ++kb) {
          mbar_wait(&empty[stage], phase ^ 1);
          if (wk.dense(kb) || (JIG_DEV && (prm.dbg & 16))) {
            mbar_arrive(&full[stage]);
          } else {
            mbar_arrive_expect_tx(&full[stage], (uint32_t)kStageE);
            bulk_g2s(sE + stage * kStageE, wk.Eimg + (wk.kb0 + kb) * kEBlockBytes, kStageE, &full[stage]);
          }
          if (++stage == C_::kStages) { stage = 0; phase ^= 1; }
        }
      }
    }
    __syncwarp();
  } else if (split_ae && warp == 13) {
    // ------------------------------------------------------------ gather-list producer (static schedules)
    // Fills the gather-list ring in (unit, k-block) order, paced only by the ring
    // (kGS = 2 x stages slots freed by the B producers): the lists land long
    // before their B rows are needed; the initial fill issued the
    // first unit's first nG0 lists.
    if (lane == 0) {
      int gslot = nG0 % C_::kGS, hint = 0;
      uint32_t gph = nG0 == C_::kGS ? 1u : 0u;
      for (int us = cluster_id; us < prm.nunits; us += nclusters) {
        const Work wk = decode_unit<NT, kPair, Prm>(prm, us, rank, S, hint);
        if (!wk.valid) continue;
        for (int kb = wk.kb_lo + (us == cluster_id ? nG0 : 0); kb < wk.kb_hi; ++kb) {
          const int steps = wk.steps(kb);
          mbar_wait(&gempty[gslot], gph ^ 1);
          mbar_arrive_expect_tx(&gfull[gslot], (uint32_t)(steps * 128));
          bulk_g2s(sG + gslot * kRowsPerBlock, wk.G + wk.gks(kb) * 32, steps * 128, &gfull[gslot]);
          if (++gslot == C_::kGS) { gslot = 0; gph ^= 1; }
        }
      }
    }
    __syncwarp();
  } else if (bprod_index(warp) >= 0) {
    // ------------------------------------------------------------ B producers
    // Group grp copies the B rows of the k-blocks j with j % kBGroups == grp; warp
    // wi of the group copies rows [wi*R, wi*R + R) of the k-block (R = 128 / kWPG,
    // 32 rows per k-step), their indices taken from the k-block's gather list in
    // shared memory (TMA-loaded by warp 0).
    const int bw = bprod_index(warp);
    const int grp = bw / C_::kWPG, wi = bw % C_::kWPG;
    griddep_wait();  // B may be the previous kernel's output
    constexpr int R = kRowsPerBlock / C_::kWPG;   // rows per warp and k-block
    constexpr int LPR = C_::kNTL / 8;      // lanes per B row (16-byte chunks per row)
    constexpr int RPI = 32 / LPR;          // rows per iteration
    const int c = lane % LPR;
    int hint = 0, traced = 0, rslot = 0;
    uint32_t rph = 0;
    int j = 0;  // CTA-wide k-block sequence number (the stage ring's order)
    for (int us = cluster_id;; us += nclusters) {
      const int u = dyn ? ring_take(ring, rfull, rempty, rslot, rph, true, lane) : (us < prm.nunits ? us : -1);
      if (u < 0) break;
      const Work wk = decode_unit<NT, kPair, Prm>(prm, u, rank, S, hint);
      if (bw == 0 && lane == 0 && traced == 0) JIG_TRACE(19);
      if (!wk.valid) continue;
      // Per-lane constants of the unit: the 16-byte column chunk this lane copies
      // (global byte address of row 0), the row pitch, and the row bound -- PAD
      // rows (index K) and chunks past column N are zero-filled.  The inner loop
      // is then SHFL (row index) + IMAD.WIDE (address) + ISETP (bound) + LDGSTS
      // per 16 bytes: the B producers are issue-bound (a few extra instructions
      // per copy measured -25 % on C4).
      // CTA r of a pair stages columns [r * ncols / 2, (r + 1) * ncols / 2) of the
      // unit; lanes whose 16-byte chunk lies beyond the unit's width (an N-split
      // unit narrower than NT) zero-fill it without reading (the MMA reads only
      // ncols columns) -- the same ignore-src path as columns past N, so the hot
      // loop carries no extra predicate
      const int wl = kPair ? wk.ncols / 2 : wk.ncols;   // columns staged by this CTA
      const int col = wk.n0 + (kPair ? (int)rank * wl : 0) + 8 * c;
      const char* const colbase = reinterpret_cast<const char*>(wk.B) + (int64_t)col * 2;
      const uint32_t ldb_bytes = (uint32_t)wk.N * 2u;
      const uint32_t kbound = col < wk.N && 8 * c < wl && !(JIG_DEV && (prm.dbg & 8)) ? (uint32_t)wk.K : 0u;
      const uint32_t hsw = (uint32_t)((c & 7) ^ (lane / LPR));  // SW128 chunk of this lane, row phase 0
      int kb = wk.kb_lo + (int)((grp - j % C_::kBGroups + C_::kBGroups) % C_::kBGroups);
      j += kb - wk.kb_lo;
      for (; kb < wk.kb_hi; kb += C_::kBGroups, j += C_::kBGroups) {
        const int stage = (int)(j % C_::kStages), gslot = (int)(j % C_::kGS);
        const uint32_t phase = (uint32_t)((j / C_::kStages) & 1), gph = (uint32_t)((j / C_::kGS) & 1);
        const int steps = wk.steps(kb);
        const bool dense = wk.dense(kb);   // a dense step uses 16 B rows
        mbar_wait(&gfull[gslot], gph);
        int32_t gl[(R + 31) / 32];
#pragma unroll
        for (int t = 0; t < (R + 31) / 32; ++t)
          gl[t] = ld_shared_s32(smem_u32(sG + gslot * kRowsPerBlock + ((wi * R) & ~31) + 32 * t + lane));
        if (bw == grp * C_::kWPG && lane == 0 && traced == 0) JIG_TRACE(20);
        __syncwarp();
        if (lane == 0) mbar_arrive(&gempty[gslot]);
        mbar_wait(&empty[stage], phase ^ 1);
        const uint32_t sb = smem_u32(sB + stage * C_::kStageB + (c >> 3) * kChunkB) + (uint32_t)(lane / LPR) * 128u;
#pragma unroll
        for (int t = 0; t < (R + 31) / 32; ++t) {
          const int ks = (wi * R) / 32 + t;          // k-step of these rows
          const int jlo = R < 32 ? (wi * R) & 31 : 0;  // rows [jlo, jlo + min(R, 32)) of the k-step
          if (ks >= steps || (dense && jlo >= 16)) continue;
#pragma unroll
          for (int it = 0; it < (R < 32 ? R : 32) / RPI; ++it) {
            if (dense && jlo + it * RPI >= 16) break;
            const int jr0 = jlo + it * RPI;             // row of lane group 0 (multiple of RPI)
            const uint32_t g = (uint32_t)__shfl_sync(kFullMask, gl[t], jr0 + lane / LPR);
            const char* src = colbase + (uint64_t)g * ldb_bytes;
            // row = 32 ks + jr0 + lane / LPR; its SW128 phase (row & 7) = (jr0 & 7) ^ (lane / LPR)
            const uint32_t dst = sb + (uint32_t)(32 * ks + jr0) * 128u + ((hsw ^ (uint32_t)(jr0 & 7)) << 4);
            cp_async_16_zfill(dst, src, g >= kbound);
          }
        }
        cp_async_mbar_arrive_noinc(&full[stage]);
        if (lane == 0 && bw == 0) {
          if (traced == 0) JIG_TRACE(3);
          JIG_TRACE_KB(1, traced);
        }
        if (kPair && rank != 0 && lane == 0 && bw == kBProdWarps - 1) JIG_TRACE_KB(3, traced);  // last B warp (odd CTA)
        ++traced;
      }
      j -= kb - wk.kb_hi;  // the k-blocks of this unit past the last one of this group
    }
  } else if (warp == 1 && kPair && rank != 0) {
    // ------------------------------------------------------------ pair relay (odd CTA)
    // The even CTA issues the pair's MMAs; it may read this CTA's stage only once
    // this CTA's A/E bulk copies and B cp.async have landed: relay full -> pfull.
    if (lane == 0) {
      int stage = 0, hint = 0, nrel = 0;
      uint32_t phase = 0;
      const uint32_t rpfull = mapa_shared(smem_u32(pfull), 0);
      for (int us = cluster_id; us < prm.nunits; us += nclusters) {
        const Work wk = decode_unit<NT, kPair, Prm>(prm, us, rank, S, hint);
        if (!wk.valid) continue;
        for (int kb = wk.kb_lo; kb < wk.kb_hi; ++kb) {
          mbar_wait(&full[stage], phase);
          JIG_TRACE_KB(2, nrel);  // odd CTA: own stage landed
          ++nrel;
          if (JIG_RELAY & 1) fence_proxy_async();
          if (JIG_RELAY & 2)
            mbar_arrive_cluster(rpfull + 8 * stage);
          else
            mbar_arrive_cluster_relaxed(rpfull + 8 * stage);
          if (++stage == C_::kStages) { stage = 0; phase ^= 1; }
        }
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer
    // The whole warp runs the loop; the tcgen05 ops are issued by a lane elected
    // inside their asm blocks, so the compiler sees warp-uniform code and moves
    // the operands to uniform registers without a per-instruction R2UR
    // waterfall (the single-lane loop spent more issue slots than the MMAs took).
    {
      const bool issuer = lane == 0;
      const uint32_t tbase_u = __shfl_sync(kFullMask, tbase, 0);
      constexpr int MM = kPair ? 256 : 128;
      int stage = 0, hint = 0, nkb_mma = 0, rslot = 0;
      uint32_t phase = 0, rph = 0;
      int it = 0;
      long long wait_cycles = 0;
      for (int us = cluster_id;; us += nclusters) {
        const int u = dyn ? __shfl_sync(kFullMask, ring_take(ring, rfull, rempty, rslot, rph, true, lane), 0) : (us < prm.nunits ? us : -1);
        if (u < 0) break;
        const Work wk = decode_unit<NT, kPair, Prm>(prm, u, rank, S, hint);
        if (it == 0 && lane == 0) JIG_TRACE(21);
        if (!wk.valid) continue;
        const int kb_lo = wk.kb_lo, kb_hi = wk.kb_hi;
        if (kb_lo == kb_hi) continue;
        // MMA N = the unit's width (NT, or a column slice of an N-split unit)
        const uint32_t idesc0 = idesc_f16(MM, wk.ncols, 0, 1, 1, 0);
        const uint32_t idesc1 = idesc0 | 1u;  // metadata selector id2 = 1
        const uint32_t idesc_dense = idesc_f16(MM, wk.ncols, 0, 1, 0, 0);
        const int a = it % C_::kAccBufs;  // accumulator buffer of this unit
        const uint32_t use = (uint32_t)(it / C_::kAccBufs);
        if (kPair)
          mbar_wait_cluster(&tempty[a], (use & 1) ^ 1);
        else
          mbar_wait(&tempty[a], (use & 1) ^ 1);
        tc_fence_after();
        const uint32_t d_tmem = tbase_u + a * C_::kAccCols;
        for (int kb = kb_lo; kb < kb_hi; ++kb) {
          const int steps = wk.steps(kb);
          const bool dense = wk.dense(kb);
          const long long tw0 = JIG_TRACE_KB_ON && prm.trace ? clock64() : 0;
          mbar_wait(&full[stage], phase);
          if (kPair) JIG_TRACE_KB(4, nkb_mma);  // pair: own stage landed (the relay's wait follows)
          // pfull: CTA-scope acquire.  The odd CTA released its stage at cluster scope
          // after observing its own copies complete; the data is read by the tensor
          // core (async proxy, ordered by tcgen05.fence), not by this thread, and a
          // cluster-scope acquire would add an L1 invalidate (CCTL.IVALL) per k-block.
          if (kPair) mbar_wait(&pfull[stage], phase);
          if (JIG_TRACE_KB_ON && prm.trace) wait_cycles += clock64() - tw0;
          // the stage's B rows were written by cp.async (generic proxy) and are
          // read by the tensor core (async proxy): proxy fence after observing them
          fence_proxy_async();
          tc_fence_after();
          if (it == 0 && kb == kb_lo) JIG_TRACE(4);
          JIG_TRACE_KB(2, nkb_mma);
          const uint32_t e_tmem = tbase_u + C_::kEColBase + 4 * stage;
          if (!dense && !(JIG_DEV && (prm.dbg & 1))) {
            const uint64_t edesc = smem_desc(smem_u32(sE + stage * kStageE), 16, 128, 0);
            tc_cp_128x128b_warp<kPair>(e_tmem, edesc);
          }
          if (!kPair) JIG_TRACE_KB(4, nkb_mma);
          const uint32_t a_base = smem_u32(sA + stage * kStageA);
          const uint32_t b_base = smem_u32(sB + stage * C_::kStageB);
          if (!dense && steps == kStepsPerBlock && !(JIG_DEV && (prm.dbg & 2))) {
            // full sparse k-block: one asm block for the 4 MMAs (descriptors stepped in PTX)
            tc_mma_sp_f16_x4_warp<kPair>(d_tmem, smem_desc(a_base, 128, 256, 0),
                                         smem_desc(b_base, kChunkB, 1024, 2), kKStepBytesA >> 4,
                                         (32 * 128) >> 4, e_tmem, idesc0, kb != kb_lo);
          } else
          for (int s = 0; s < (JIG_DEV && (prm.dbg & 2) ? 0 : steps); ++s) {
            const uint64_t adesc = smem_desc(a_base + s * kKStepBytesA, 128, 256, 0);
            const uint64_t bdesc = smem_desc(b_base + s * 32 * 128, kChunkB, 1024, 2);
            const uint32_t acc = (kb != kb_lo) || (s != 0);
            if constexpr (kPair) {
              if (issuer) {
                if (dense)
                  tc_mma_f16_pair(d_tmem, adesc, bdesc, idesc_dense, acc);
                else
                  tc_mma_sp_f16_pair(d_tmem, adesc, bdesc, e_tmem + (s & 2), (s & 1) ? idesc1 : idesc0, acc);
              }
            } else {
              if (issuer) {   // residual tile on the dense tensor path, K = 16
                if (dense)
                  tc_mma_f16(d_tmem, adesc, bdesc, idesc_dense, acc);
                else
                  tc_mma_sp_f16(d_tmem, adesc, bdesc, e_tmem + (s & 2), (s & 1) ? idesc1 : idesc0, acc);
              }
            }
          }
          JIG_TRACE_KB(5, nkb_mma);
          tc_commit_warp<kPair>(&empty[stage]);   // frees the stage (in both CTAs of a pair)
          JIG_TRACE_KB(3, nkb_mma);
          ++nkb_mma;
          if (++stage == C_::kStages) { stage = 0; phase ^= 1; }
        }
        tc_commit_warp<kPair>(&tfull[a]);
        JIG_TRACE(5);
        ++it;
      }
      if (!kSplit && prm.trace && blockIdx.x < kTraceCTAs) {  // slots 7/8 are split-K-only otherwise
        g_trace[blockIdx.x * kTraceSlots + 7] = wait_cycles;  // MMA issuer: cycles waiting for data
        g_trace[blockIdx.x * kTraceSlots + 8] = nkb_mma;      // k-blocks issued
      }
    }
    __syncwarp();
  } else if (warp >= 2 && warp <= 5) {
    // ------------------------------------------------------------ epilogue (warps 2-5)
    const int q = warp & 3;  // TMEM lane quarter this warp may access
    griddep_wait();          // C and the split workspace may still be in use by the previous kernel
    int it = 0, hint = 0, rslot = 0;
    uint32_t rph = 0;
    for (int us = cluster_id;; us += nclusters) {
      const int u = dyn ? ring_take(ring, rfull, rempty, rslot, rph, true, lane) : (us < prm.nunits ? us : -1);
      if (u < 0) break;
      const Work wk = decode_unit<NT, kPair, Prm>(prm, u, rank, S, hint);
      if (!wk.valid) continue;
      const int p = wk.p, n0 = wk.n0;
      const int64_t M = wk.M, N = wk.N;
      void* const Cm = wk.C;
      const bool c32 = wk.c32 != 0;
      const bool has_acc = wk.kb_hi > wk.kb_lo;
      const int r = q * 32 + lane;                       // row of the panel (= TMEM lane)
      const int a = it % C_::kAccBufs;
      const int ncols = wk.ncols;                        // C columns of this unit
      if (kCC && !kSplit && wk.ccp) {
        // CUDA-core entries of this lane's row (f3): their B row segments are
        // prefetched into L2 while the accumulator is still being built
        const int64_t pr = wk.row0 + q * 32 + lane;
        const int e0 = wk.ccoff[pr], e1 = wk.ccoff[pr + 1];
        for (int e = e0; e < e1 && e < e0 + 8; ++e)
          bulk_prefetch_l2(wk.B + (int64_t)__ldg(wk.ccent + e).x * N + n0, (uint32_t)wk.ncols * 2u);
      }
      if (has_acc) {
        mbar_wait(&tfull[a], (uint32_t)(it / C_::kAccBufs) & 1);
        tc_fence_after();
      }
      // CUDA-core entries (f3, kCC launches only): added into the TMEM
      // accumulator once per unit (piece 0 of a k-range split), or -- a panel
      // with no tensor-core tile -- written to C directly
      bool cc_done = false;
      if (kCC && !kSplit && wk.ccp) {
        const int64_t pr = wk.row0 + q * 32 + lane;  // padded panel-row index
        if (has_acc) {
          if (wk.piece == 0)
            cc_tmem_add(tbase + ((uint32_t)(q * 32) << 16) + (uint32_t)(a * C_::kAccCols), wk.ncols, wk.ccoff,
                        wk.ccent, wk.B, N, n0, pr);
        } else if (wk.npieces == 1) {
          cc_only_store(wk.C, wk.c32, pr < M ? (wk.rowmap ? (int64_t)wk.rowmap[pr] : pr) : -1, wk.ncols, N, n0,
                        wk.ccoff, wk.ccent, wk.B, pr);
          cc_done = true;
        }
      }
      // 32-column chunk k of the unit: its TMEM column and its C column offset
      auto tcol = [&](int k) -> uint32_t { return (uint32_t)(a * C_::kAccCols + 32 * k); };
      auto ucol = [&](int k) -> int { return 32 * k; };
      auto release = [&](int buf) {  // this warp is done reading accumulator buffer `buf`
        tc_fence_before();
        __syncwarp();
        if (lane == 0) {
          if (kPair && rank != 0)
            mbar_arrive_cluster(mapa_shared(smem_u32(&tempty[buf]), 0));  // the pair's issuer
          else
            mbar_arrive(&tempty[buf]);
        }
      };
      if (warp == 2 && lane == 0 && it == 0) JIG_TRACE(6);
      if constexpr (!kSplit) {
        const uint32_t stg = smem_u32(sC + q * (32 * 64));
        bool write_c = !cc_done;
        // C rows of the 4 rows this lane stores (rr = 8i + lane / 4 of the warp's
        // 32): row-clustered panels scatter panel row r to C row rowmap[r]; once
        // per unit, outside the store loop (M < 2^31 by validation)
        int64_t srow[4];
        {
          const int64_t prow = wk.row0 + q * 32 + lane;
          int crow = (int)prow;
          if (wk.rowmap && prow < M) crow = wk.rowmap[prow];
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const int64_t lrow = wk.row0 + q * 32 + 8 * i + (lane >> 2);
            const int mrow = __shfl_sync(kFullMask, crow, 8 * i + (lane >> 2));
            srow[i] = lrow < M ? (wk.rowmap ? (int64_t)mrow : lrow) : -1;
          }
        }
        const int npc = wk.npieces;
        if (npc > 1) {
          // split-K piece: publish the fp32 partial tile, count the pieces done;
          // the last piece of the unit adds the others' partials to its own and
          // writes C (the last-arriver reduction never waits on another CTA)
          constexpr size_t kTile = (size_t)128 * NT;  // floats per partial tile
          float* part = prm.ws + ((size_t)(wk.pslot + wk.piece) * CS + rank) * kTile;
#pragma unroll 1
          for (int c0 = 0; c0 < ncols; c0 += 32) {
            uint32_t v[32];
            if (has_acc) {
              tc_ld_32x32b_x32(tbase + ((uint32_t)(q * 32) << 16) + tcol(c0 / 32), v);
              tc_wait_ld();
            } else {
#pragma unroll
              for (int j = 0; j < 32; ++j) v[j] = 0;
            }
            // [chunk][warp][j][lane] float4s: each store instruction is 512 contiguous bytes
            float4* dst = reinterpret_cast<float4*>(part + ((size_t)(c0 / 32) * 128 + q * 32) * 32) + lane;
#pragma unroll
            for (int j = 0; j < 8; ++j)
              __stcg(dst + 32 * j, make_float4(__uint_as_float(v[4 * j]), __uint_as_float(v[4 * j + 1]),
                                         __uint_as_float(v[4 * j + 2]), __uint_as_float(v[4 * j + 3])));
          }
          __threadfence();
          asm volatile("bar.sync 1, 128;" ::: "memory");
          if (threadIdx.x == 64) {
            int* cnt = prm.wcnt + wk.pslot * CS + rank;
            const int done = atomicAdd(cnt, 1);
            st_shared_s32(s_last, done == npc - 1);
            if (done == npc - 1) atomicExch(cnt, 0);  // zero again for the next launch
          }
          asm volatile("bar.sync 1, 128;" ::: "memory");
          write_c = ld_shared_s32(s_last) != 0;
          if (write_c) __threadfence();
        }
#pragma unroll 1
        for (int c0 = 0; write_c && c0 < ncols; c0 += 32) {
          uint32_t v[32];
          if (has_acc) {
            tc_ld_32x32b_x32(tbase + ((uint32_t)(q * 32) << 16) + tcol(c0 / 32), v);
            tc_wait_ld();
          } else {
#pragma unroll
            for (int j = 0; j < 32; ++j) v[j] = 0;     // all-zero panel (R-Q21)
          }
          if (npc > 1) {
            constexpr size_t kTile = (size_t)128 * NT;
            for (int pc = 0; pc < npc; ++pc) {
              if (pc == wk.piece) continue;
              const float4* src = reinterpret_cast<const float4*>(
                  prm.ws + ((size_t)(wk.pslot + pc) * CS + rank) * kTile + ((size_t)(c0 / 32) * 128 + q * 32) * 32) + lane;
#pragma unroll
              for (int j = 0; j < 8; ++j) {
                const float4 x = __ldcg(src + 32 * j);
                v[4 * j] = __float_as_uint(__uint_as_float(v[4 * j]) + x.x);
                v[4 * j + 1] = __float_as_uint(__uint_as_float(v[4 * j + 1]) + x.y);
                v[4 * j + 2] = __float_as_uint(__uint_as_float(v[4 * j + 2]) + x.z);
                v[4 * j + 3] = __float_as_uint(__uint_as_float(v[4 * j + 3]) + x.w);
              }
            }
          }
          // Transposed through shared memory so that each store instruction
          // writes 8 rows x 64 contiguous bytes (4 lanes per row) instead of 32
          // rows x 16 bytes; 16-byte chunks swizzled by (row >> 1) & 3.
          // fp16 C (RN): the 32 columns are one 64-byte row segment; fp32 C
          // (c_dtype = 1): two 16-column halves of 64 bytes each.
          if (!c32) {
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              uint4 pk;
              pk.x = pack_h2(__uint_as_float(v[8 * j + 0]), __uint_as_float(v[8 * j + 1]));
              pk.y = pack_h2(__uint_as_float(v[8 * j + 2]), __uint_as_float(v[8 * j + 3]));
              pk.z = pack_h2(__uint_as_float(v[8 * j + 4]), __uint_as_float(v[8 * j + 5]));
              pk.w = pack_h2(__uint_as_float(v[8 * j + 6]), __uint_as_float(v[8 * j + 7]));
              st_shared_v4u(stg + lane * 64 + ((j ^ ((lane >> 1) & 3)) << 4), pk);
            }
            __syncwarp();
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              const int rr = 8 * i + (lane >> 2), c = lane & 3;
              const uint4 pk = ld_shared_v4u(stg + rr * 64 + ((c ^ ((rr >> 1) & 3)) << 4));
              const int col = n0 + ucol(c0 / 32) + 8 * c;
              if (srow[i] >= 0 && col < N) *reinterpret_cast<uint4*>(static_cast<__half*>(Cm) + srow[i] * N + col) = pk;
            }
            __syncwarp();
          } else {
#pragma unroll
            for (int h = 0; h < 2; ++h) {
#pragma unroll
              for (int j = 0; j < 4; ++j)
                st_shared_v4u(stg + lane * 64 + ((j ^ ((lane >> 1) & 3)) << 4),
                              make_uint4(v[16 * h + 4 * j], v[16 * h + 4 * j + 1], v[16 * h + 4 * j + 2],
                                         v[16 * h + 4 * j + 3]));
              __syncwarp();
#pragma unroll
              for (int i = 0; i < 4; ++i) {
                const int rr = 8 * i + (lane >> 2), c = lane & 3;
                const uint4 pk = ld_shared_v4u(stg + rr * 64 + ((c ^ ((rr >> 1) & 3)) << 4));
                const int col = n0 + ucol(c0 / 32) + 16 * h + 4 * c;
                if (srow[i] >= 0 && col < N) *reinterpret_cast<uint4*>(static_cast<float*>(Cm) + srow[i] * N + col) = pk;
              }
              __syncwarp();
            }
          }
        }
      } else {
        // reduce-scatter of the fp32 partial tile through DSMEM: each warp stages
        // its 32 rows (padded stride, the receive layout) in the B stage ring --
        // free once the accumulator is ready, a split CTA runs exactly one unit --
        // and sends them with ONE bulk copy to the owner's receive slot (16-byte
        // st.async per lane moved ~15 B/clk)
        const int rpo = 128 / S;                           // rows owned per CTA
        constexpr int kMaxRun = 32;                        // rows of a warp sent by one copy
        // the S - 1 peers' slices of this CTA's rows arrive by bulk copy
        if (warp == 2 && lane == 0) mbar_arrive_expect_tx(recv_full, (uint32_t)((128 - rpo) * C_::kRecvStride));
        const uint32_t stg = smem_u32(sB + q * 32 * C_::kRecvStride);
#pragma unroll 1
        for (int c0 = 0; c0 < NT; c0 += 32) {
          uint32_t v[32];
          if (has_acc) {
            tc_ld_32x32b_x32(tbase + ((uint32_t)(q * 32) << 16) + a * C_::kAccCols + c0, v);
            tc_wait_ld();
          } else {
#pragma unroll
            for (int j = 0; j < 32; ++j) v[j] = 0;
          }
#pragma unroll
          for (int j = 0; j < 8; ++j)
            st_shared_v4u(stg + lane * C_::kRecvStride + (c0 + 4 * j) * 4,
                          make_uint4(v[4 * j], v[4 * j + 1], v[4 * j + 2], v[4 * j + 3]));
        }
        fence_proxy_async();  // the staged rows are read by the bulk copy (async proxy)
        __syncwarp();
        // one copy per owner of the warp's rows (S = 8: 16-row owners, two runs);
        // rows this CTA owns itself are moved inside its shared memory by the warp
        const int run = rpo < kMaxRun ? rpo : kMaxRun;
#pragma unroll 1
        for (int ri = 0; ri < 32 / run; ++ri) {
          const int r0 = q * 32 + ri * run;
          const uint32_t owner = (uint32_t)(r0 / rpo);
          const uint32_t src = stg + ri * run * C_::kRecvStride;
          const uint32_t dst = smem_u32(sRecv + (rank * rpo + r0 % rpo) * C_::kRecvStride);
          if (owner == rank) {
            for (int o = lane * 16; o < run * C_::kRecvStride; o += 32 * 16) st_shared_v4u(dst + o, ld_shared_v4u(src + o));
          } else if (lane == 0) {
            bulk_s2cluster(mapa_shared(dst, owner), src, run * C_::kRecvStride, mapa_shared(smem_u32(recv_full), owner));
          }
        }
        // owner: wait for all S partial slices of its rows, sum, convert, store
        if (warp == 2 && lane == 0) JIG_TRACE(7);
        mbar_wait(recv_full, 0);
        asm volatile("bar.sync 1, 128;" ::: "memory");  // the local slice, copied by all four warps
        if (warp == 2 && lane == 0) JIG_TRACE(8);
        const int t = threadIdx.x - 64;                    // 0..127
        constexpr int C8 = NT / 8;                         // 8-column groups per row
        for (int item = t; item < rpo * C8; item += 128) {
          const int i = item / C8, c8 = item % C8;
          float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
          for (int s = 0; s < S; ++s) {
            const uint32_t src = smem_u32(sRecv + (s * rpo + i) * C_::kRecvStride + c8 * 32);
            const float4 x = ld_shared_f4(src), y = ld_shared_f4(src + 16);
            acc[0] += x.x; acc[1] += x.y; acc[2] += x.z; acc[3] += x.w;
            acc[4] += y.x; acc[5] += y.y; acc[6] += y.z; acc[7] += y.w;
          }
          const int64_t lrow = (int64_t)p * 128 + rank * rpo + i;
          const int64_t colg = n0 + c8 * 8;
          if (kCC && wk.ccp) {  // CUDA-core entries of this row (f3)
            const int e0 = wk.ccoff[lrow], e1 = wk.ccoff[lrow + 1];
            if (e1 > e0) cc_accum(acc, wk.ccent, e0, e1, wk.B, N, colg, 8);
          }
          if (lrow < M && colg < N) {
            const int64_t row = wk.rowmap ? (int64_t)wk.rowmap[lrow] : lrow;
            if (c32) {
              float4* dst = reinterpret_cast<float4*>(static_cast<float*>(Cm) + row * N + colg);
              dst[0] = make_float4(acc[0], acc[1], acc[2], acc[3]);
              dst[1] = make_float4(acc[4], acc[5], acc[6], acc[7]);
            } else {
              uint4 pk;
              pk.x = pack_h2(acc[0], acc[1]);
              pk.y = pack_h2(acc[2], acc[3]);
              pk.z = pack_h2(acc[4], acc[5]);
              pk.w = pack_h2(acc[6], acc[7]);
              *reinterpret_cast<uint4*>(static_cast<__half*>(Cm) + row * N + colg) = pk;
            }
          }
        }
      }
      if (warp == 2 && lane == 0) JIG_TRACE(9);
      if (has_acc) {
        release(a);
        ++it;
      }
    }
    if (warp == 2 && lane == 0 && prm.trace && blockIdx.x < kTraceCTAs)
      g_trace[blockIdx.x * kTraceSlots + 12] = it;  // units with an accumulator run by this CTA
  }
  if (threadIdx.x == 0) JIG_TRACE(10);
  tc_fence_before();
  if constexpr (kSplit || kPair) {
    // no CTA leaves while peers may still target its shared memory (DSMEM
    // sends, pair commits); the C stores need no cluster-scope release here
    __syncwarp();
    if (!cl_waited) cluster_wait();  // complete the prologue's barrier phase first
    cluster_sync_relaxed();
  } else {
    __syncthreads();
  }
  if (threadIdx.x == 0) JIG_TRACE(23);
  if (warp == 1) {
    if constexpr (kPair)
      tmem_dealloc_pair<C_::kTmemCols>(tbase);
    else
      tmem_dealloc<C_::kTmemCols>(tbase);
  }
  if (threadIdx.x == 0 && prm.trace && blockIdx.x < kTraceCTAs) {
    JIG_TRACE(11);
    g_trace[blockIdx.x * kTraceSlots + 13] = gtimer();
  }
}

int g_num_sms[64] = {0};

// Environment read ONCE per process (library load): JIGSAW_PDL=0 launches
// without the programmatic-dependency attribute, JIGSAW_TRACE=1 records the
// per-CTA timeline of jigsaw_debug_trace.  Developer builds (-DJIG_DEV=1) also
// read the schedule / timing experiments below; product builds compile them
// out (the constants are the product defaults).
struct Knobs {
  bool pdl = true, trace = false;
  int dbg = 0;               // JIGSAW_DBG (timing only, results invalid)
  bool no_prefetch = false;  // JIGSAW_NO_PREFETCH: no per-unit metadata prefetch into L2
  bool dyn_sched = false;    // JIGSAW_DYN_SCHEDULE: dynamic tile scheduler for grouped launches
                             // (measured 4-12 % slower than the static LPT plan, profiles/r02x)
  int unit_cost = -1;        // JIGSAW_UNIT_COST: per-unit cost in k-block equivalents
  bool sched_loc = false;    // JIGSAW_SCHED=loc: locality order, no cost sort, no pieces
  bool debug_sched = false;  // JIGSAW_DEBUG_SCHED: print the pair schedule balance
  int64_t group_bpf = 0;     // JIGSAW_GROUP_BPF (MB): L2 prefetch of all B's of a grouped launch
  bool bpf = false;          // JIGSAW_BPF: L2 prefetch of B for single products
  bool no_ctab = false;      // JIGSAW_NO_CTAB: no host-decoded first units
  int split_pct = 125;       // JIGSAW_SPLIT_PCT: split a unit into pieces above this % of the per-slot load
};
const Knobs& knobs() {
  static const Knobs k = [] {
    Knobs r;
    auto env = [](const char* n) -> const char* { return getenv(n); };
    r.pdl = !(env("JIGSAW_PDL") && atoi(env("JIGSAW_PDL")) == 0);
    r.trace = env("JIGSAW_TRACE") && env("JIGSAW_TRACE")[0] == '1';
#if JIG_DEV
    r.dbg = env("JIGSAW_DBG") ? atoi(env("JIGSAW_DBG")) : 0;
    r.no_prefetch = env("JIGSAW_NO_PREFETCH") != nullptr;
    r.dyn_sched = env("JIGSAW_DYN_SCHEDULE") != nullptr;
    r.unit_cost = env("JIGSAW_UNIT_COST") ? atoi(env("JIGSAW_UNIT_COST")) : -1;
    r.sched_loc = env("JIGSAW_SCHED") && std::string(env("JIGSAW_SCHED")) == "loc";
    r.debug_sched = env("JIGSAW_DEBUG_SCHED") != nullptr;
    r.group_bpf = env("JIGSAW_GROUP_BPF") ? atoll(env("JIGSAW_GROUP_BPF")) : 0;
    r.bpf = env("JIGSAW_BPF") != nullptr;
    r.no_ctab = env("JIGSAW_NO_CTAB") != nullptr;
    r.split_pct = env("JIGSAW_SPLIT_PCT") ? atoi(env("JIGSAW_SPLIT_PCT")) : 125;
#endif
    return r;
  }();
  return k;
}
std::atomic<bool> g_attr_set[64][32] = {};  // [device][variant (+16: kCC)]

template <int NT, bool kSplit, bool kPair, bool kCC, class Prm>
jigsaw_status_t launch_variant(const Prm& prm, int grid, int S, int dev, int vid, cudaStream_t s) {
  using C_ = Cfg<NT, kSplit, kPair>;
  auto kern = k_spmm<NT, kSplit, kPair, Prm, kCC>;
  vid += kCC ? 16 : 0;
  if (dev >= 0 && dev < 64 && !g_attr_set[dev][vid].load(std::memory_order_acquire)) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C_::kSmem);
    if (e != cudaSuccess) return cuda_status(e, "cudaFuncSetAttribute(k_spmm)");
    if (kSplit) {
      e = cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
      if (e != cudaSuccess) return cuda_status(e, "cudaFuncSetAttribute(cluster)");
    }
    g_attr_set[dev][vid].store(true, std::memory_order_release);
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = C_::kSmem;
  cfg.stream = s;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = kPair ? 2 : kSplit ? S : 1;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  // Programmatic dependent launch: the CTAs may start while the previous kernel
  // of the stream drains.  The prologue (barrier init, TMEM allocation, the
  // first k-blocks' compressed A / metadata / gather lists -- handle-owned,
  // immutable) runs before griddepcontrol.wait; every access to B, C and the
  // launch workspace (counters, partial tiles) comes after it.
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = knobs().pdl ? 2 : 1;
  cudaError_t e = cudaLaunchKernelEx(&cfg, kern, prm);
  if (e != cudaSuccess) return cuda_status(e, "k_spmm launch");
  return JIGSAW_SUCCESS;
}

}  // namespace

LaunchOverride& launch_override() {
  thread_local LaunchOverride o;
  return o;
}
jigsaw_launch_desc_t& last_launch() {
  thread_local jigsaw_launch_desc_t d = {};
  return d;
}

int spmm_num_sms() {
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 64) return 148;
  if (!g_num_sms[dev]) cudaDeviceGetAttribute(&g_num_sms[dev], cudaDevAttrMultiProcessorCount, dev);
  return g_num_sms[dev];
}

// Tile / split selection: enough units for every SM -> NT = 128
// (or 256), persistent; otherwise NT = 32 / 64 and split-K over a cluster of
// S = 1/2/4 CTAs by the cost model below.  256-row panels (CTA pairs): NT = 256
// when there is a unit for every pair, else NT = 128; grid = 2 x pairs.
void choose_config(const Format& f, int64_t N, int sms, int* NT, int* S, int* grid) {
  const int force = launch_override().tile_n;
  if (f.P == kPairPanelRows) {
    const int64_t u256 = f.npanels * ((N + 255) / 256);
    *NT = ((u256 >= sms / 2 && force != 128) || force == 256) ? 256 : 128;
    *S = 1;
    const int64_t units = f.npanels * ((N + *NT - 1) / *NT);
    *grid = 2 * (int)std::min<int64_t>(units, sms / 2);
    return;
  }
  const int64_t u256 = f.npanels * ((N + 255) / 256), u128 = f.npanels * ((N + 127) / 128);
  int64_t kbs = 0;
  for (int64_t p = 0; p < f.npanels; ++p) kbs += (f.pin[p].x + 3) / 4 + (f.pin[p].w + 3) / 4;
  const bool long_units = kbs >= 24 * f.npanels;  // NT = 256 runs a 2-stage ring: needs long units
  if ((u256 >= sms && long_units && force == 0) || force == 256) {   // large: A read once per 256 columns
    *NT = 256;
    *S = 1;
    *grid = (int)std::min<int64_t>(u256, sms);
    return;
  }
  if (u128 >= sms || force == 128) {
    *NT = 128;
    *S = 1;
    *grid = (int)std::min<int64_t>(u128, sms);
    return;
  }
  // Small products (fewer 128-column units than SMs): latency-bound.  Pick the
  // tile width NT (32 or 64 columns) and the split-K factor S (1, 2, 4 CTAs of a
  // cluster per unit, one wave) that minimise a per-CTA cost model in SM cycles
  // (profiles/r01s_*: compressed A/E arrive by bulk TMA at ~70 B/clk/SM, the B
  // row gather by 16-byte cp.async at ~35 B/clk/SM, the two overlap; the split
  // reduction moves (S-1)/S of the fp32 partial tile through DSMEM at ~15 B/clk
  // plus ~1500 cycles of cluster-wide skew and synchronisation).
  int64_t kb_max = 0;
  for (int64_t p = 0; p < f.npanels; ++p)
    kb_max = std::max<int64_t>(kb_max, (f.pin[p].x + 3) / 4 + (f.pin[p].w + 3) / 4);
  double best = 1e30;
  *NT = 64;
  *S = 1;
  *grid = (int)std::min<int64_t>(f.npanels * ((N + 63) / 64), sms);
  for (int nt : {32, 64}) {
    if (force && force != nt) continue;
    const int64_t units = f.npanels * ((N + nt - 1) / nt);
    for (int s = 1; s <= 4; s *= 2) {
      if (units * s > sms && !(s == 1 && units > sms && nt == 64)) continue;  // one wave (S = 1 may loop)
      if (s > 1 && kb_max < 2 * s) continue;
      const double waves = (double)((units * s + sms - 1) / sms);
      const double nkb = (double)((kb_max + s - 1) / s) * waves;
      const double t_ae = nkb * (kStepsPerBlock * kKStepBytesA + kEBlockBytes) / 70.0;
      const double t_b = nkb * 128.0 * nt * 2 / 35.0;
      const double t_red = s > 1 ? (double)(s - 1) / s * 128.0 * nt * 4 / 15.0 + 1500.0 : 0.0;
      const double cost = std::max(t_ae, t_b) + t_red + 128.0 * nt * 2 / 32.0;
      if (cost < best - 1.0) {
        best = cost;
        *NT = nt;
        *S = s;
        *grid = s > 1 ? (int)(units * s) : (int)std::min<int64_t>(units, sms);
      }
    }
  }
}

template <class Prm>
static void fill_problem(Prm& prm, int i, const Format& f, const void* dB, int64_t N, void* dC) {
  Problem& P = prm.pr[i];
  P.pin0 = i == 0 ? 0 : prm.pr[i - 1].pin0 + prm.pr[i - 1].npanels;
  if (P.pin0 + f.npanels <= Prm::kMaxPin)
    for (int64_t p = 0; p < f.npanels; ++p) prm.pin[P.pin0 + p] = f.pin_dev(p);
  else
    prm.use_pin = 0;
  P.Aimg = f.d_Aimg;
  P.Eimg = f.d_Eimg;
  P.nksA = (int32_t)f.nksteps;
  P.nkbE = (int32_t)f.nkblocks;
  P.G = f.d_G;
  P.pin = f.d_pin;
  P.B = reinterpret_cast<const __half*>(dB);
  P.C = dC;
  P.c32 = f.c_dtype == JIGSAW_C_F32 ? 1 : 0;
  P.rowmap = f.d_rowmap;
  P.ccoff = f.d_ccoff;
  P.ccent = f.d_ccent;
  P.M = (int32_t)f.M;
  P.N = (int32_t)N;
  P.K = (int32_t)f.K;
  P.npanels = (int)f.npanels;
  P.boff = i == 0 ? 0 : prm.pr[i - 1].boff + prm.pr[i - 1].K * prm.pr[i - 1].N * 2;
}

int g_trace_ctas = 0;

// ---------------------------------------------------------------- launch workspace
// A launch that uses the dynamic tile scheduler or k-range pieces needs a small
// device workspace: [ticket (256 B) | piece counters (512 slots x 2 ranks x 4 B) |
// fp32 partial tiles].  The counters must be zero when a launch starts; each
// launch leaves them zero (reset by the last CTA / last piece).  A workspace is
// owned by exactly one launch at a time:
//   * eager launches: one region per stream (keyed by cudaStreamGetId, which is
//     unique for the life of the process), used only by launches on that
//     stream; consecutive launches of a stream share it because every workspace
//     access of a launch comes after griddepcontrol.wait (the previous kernel of
//     the stream has completed and left the counters zero).  A region is taken
//     from the library's stream-ordered pool on that stream and its counters
//     zeroed on that stream; it grows by a new allocation and a stream-ordered
//     free of the old region on the same stream -- no host or device
//     synchronisation, no free of memory another stream may still use.
//   * launches captured into a CUDA graph: a graph-owned allocation
//     (cudaMallocFromPoolAsync during capture = an allocation node), a memset
//     node zeroing its counters, and a free node right after the kernel node:
//     every replay zeroes its own workspace, and graph replays never share one
//     with any other launch (a graph exec never runs concurrently with itself).
constexpr size_t kWsTicket = 256, kWsHead = kWsTicket + 512 * 2 * 4;
// Regions of streams that are no longer used are reclaimed once more than
// kMaxRegions streams of a device have one: a region whose last launch has
// completed (its event) and that no host thread is launching on is freed.
constexpr size_t kMaxRegions = 64;
struct StreamRegion {
  char* base = nullptr;
  size_t size = 0;
  cudaEvent_t done = nullptr;  // recorded after every launch that used the region
  int inflight = 0;            // host threads between acquire and the event record
};
std::mutex g_ws_mu;
std::unordered_map<unsigned long long, StreamRegion> g_ws[64];

struct Workspace {
  char* base = nullptr;
  bool graph_owned = false;
  int dev = -1;
  unsigned long long stream_id = 0;
};

// Eager launches: after the kernel that used the stream's region is enqueued.
static void release_workspace(const Workspace& w, cudaStream_t s) {
  if (w.graph_owned || !w.base || w.dev < 0) return;
  std::lock_guard<std::mutex> lock(g_ws_mu);
  auto it = g_ws[w.dev].find(w.stream_id);
  if (it == g_ws[w.dev].end()) return;
  if (it->second.done) cudaEventRecord(it->second.done, s);
  --it->second.inflight;
}

static jigsaw_status_t acquire_workspace(int dev, size_t bytes, cudaStream_t s, Workspace* w) {
  if (dev < 0 || dev >= 64) return set_status(JIGSAW_ERROR_INTERNAL, "device ordinal out of range");
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  cudaError_t e = cudaStreamIsCapturing(s, &cs);
  if (e != cudaSuccess) return cuda_status(e, "cudaStreamIsCapturing");
  void* p = nullptr;
  if (cs != cudaStreamCaptureStatusNone) {
    e = pool_alloc_async(&p, bytes, s);
    if (e != cudaSuccess) return cuda_status(e, "workspace allocation node (stream capture)");
    e = cudaMemsetAsync(p, 0, kWsHead, s);
    if (e != cudaSuccess) return cuda_status(e, "workspace memset node (stream capture)");
    w->base = static_cast<char*>(p);
    w->graph_owned = true;
    return JIGSAW_SUCCESS;
  }
  unsigned long long id = 0;
  e = cudaStreamGetId(s, &id);
  if (e != cudaSuccess) return cuda_status(e, "cudaStreamGetId");
  std::lock_guard<std::mutex> lock(g_ws_mu);
  auto& map = g_ws[dev];
  if (map.size() >= kMaxRegions && map.find(id) == map.end()) {
    for (auto it = map.begin(); it != map.end();) {
      StreamRegion& o = it->second;
      if (o.inflight == 0 && (!o.done || cudaEventQuery(o.done) == cudaSuccess)) {
        if (o.base) cudaFreeAsync(o.base, s);  // idle: its last launch has completed
        if (o.done) cudaEventDestroy(o.done);
        it = map.erase(it);
      } else {
        ++it;
      }
    }
    cudaGetLastError();  // cudaEventQuery's cudaErrorNotReady is not an error here
  }
  StreamRegion& r = map[id];
  if (!r.done && cudaEventCreateWithFlags(&r.done, cudaEventDisableTiming) != cudaSuccess) {
    cudaGetLastError();
    r.done = nullptr;
  }
  if (r.size < bytes) {
    const size_t sz = std::max<size_t>({bytes, (size_t)4 << 20, 2 * r.size});
    e = pool_alloc_async(&p, sz, s);
    if (e != cudaSuccess) return cuda_status(e, "workspace allocation");
    e = cudaMemsetAsync(p, 0, kWsHead, s);
    if (e != cudaSuccess) return cuda_status(e, "workspace counters");
    if (r.base) cudaFreeAsync(r.base, s);  // after every earlier launch of this stream
    r.base = static_cast<char*>(p);
    r.size = sz;
  }
  w->base = r.base;
  w->graph_owned = false;
  w->dev = dev;
  w->stream_id = id;
  ++r.inflight;
  return JIGSAW_SUCCESS;
}

template <class Prm>
static void set_workspace(Prm& prm, const Workspace& w) {
  prm.sched_ctr = reinterpret_cast<int*>(w.base);
  prm.wcnt = w.base ? reinterpret_cast<int*>(w.base + kWsTicket) : nullptr;
  prm.ws = w.base ? reinterpret_cast<float*>(w.base + kWsHead) : nullptr;
}

// Launches k_spmm for the parameter block.  `pslots` split-piece slots of
// `tile_bytes` each need workspace; the dynamic scheduler is used when a
// single-CTA launch has more units than CTAs.
// The kernel instantiation for a launch shape (tile width, split-K, CTA pairs).
template <bool kCC, class Prm>
static jigsaw_status_t launch_shape(const Prm& prm, int NT, int S, int grid, int dev, bool pair, int vb,
                                    cudaStream_t s) {
  if (pair)
    return NT == 256 ? launch_variant<256, false, true, kCC>(prm, grid, 2, dev, vb + 5, s)
                     : launch_variant<128, false, true, kCC>(prm, grid, 2, dev, vb + 4, s);
  if (NT == 256) return launch_variant<256, false, false, kCC>(prm, grid, 1, dev, vb + 3, s);
  if (NT == 128) return launch_variant<128, false, false, kCC>(prm, grid, 1, dev, vb + 0, s);
  if (NT == 32 && S == 1) return launch_variant<32, false, false, kCC>(prm, grid, 1, dev, vb + 6, s);
  if (S == 1) return launch_variant<64, false, false, kCC>(prm, grid, 1, dev, vb + 1, s);
  if constexpr (std::is_same<Prm, ParamsOne>::value)
    return NT == 32 ? launch_variant<32, true, false, kCC>(prm, grid, S, dev, vb + 7, s)
                    : launch_variant<64, true, false, kCC>(prm, grid, S, dev, vb + 2, s);
  return set_status(JIGSAW_ERROR_INTERNAL, "split-K is only built for single products");
}

template <class Prm>
static jigsaw_status_t launch_params(Prm& prm, int NT, int S, int grid, int dev, bool pair, cudaStream_t s,
                                     int npieces_total = -1, int pslots = 0, size_t tile_bytes = 0) {
  prm.S = S;
  prm.prefetch = knobs().no_prefetch ? 0 : 1;

  prm.dbg = JIG_DEV ? knobs().dbg : 0;
  prm.trace = knobs().trace ? 1 : 0;
  if (prm.trace) g_trace_ctas = std::min(grid, kTraceCTAs);
  int u = 0;
  for (int i = 0; i < prm.nprob; ++i) {
    prm.pr[i].unit0 = u;
    u += (int)(prm.pr[i].npanels * ((prm.pr[i].N + NT - 1) / NT));
  }
  prm.nunits = npieces_total >= 0 ? npieces_total : u;
  // (a CTA per unit needs no scheduler: its one unit is known at kernel start)
  // Grouped launches run the host's static greedy-LPT plan (prm.use_ulist): the
  // dynamic tile scheduler measured 4-12 % slower on C2 / C3 / C5a (units taken
  // ahead of time unbalance the tail; profiles/r02w, r02x) and is a developer
  // option there; a CTA-pair variant (the even CTA forwarding tickets through a
  // mailbox) measured 8-20 % slower on C2 / C4 and was removed (profiles/r02e).
  // Single products whose units outnumber the CTAs (no host plan) use it.
  prm.dyn = (S == 1 && !pair && grid < prm.nunits && (!prm.use_ulist || knobs().dyn_sched)) ? 1 : 0;
  Workspace w;
  if (prm.dyn || pslots > 0) {
    jigsaw_status_t st = acquire_workspace(dev, kWsHead + (size_t)pslots * tile_bytes, s, &w);
    if (st != JIGSAW_SUCCESS) return st;
  }
  set_workspace(prm, w);
  jigsaw_launch_desc_t& d = last_launch();
  d.tile_n = NT;
  d.split_k = S;
  d.grid = grid;
  d.cta_pair = pair ? 1 : 0;
  d.problems = prm.nprob;
  d.work_items = prm.nunits;
  d.split_slots = pslots;
  d.dynamic_schedule = prm.dyn;
  d.graph_owned_workspace = w.graph_owned ? 1 : 0;
  d.launches += 1;
  constexpr int vb = std::is_same<Prm, ParamsOne>::value ? 0 : 8;
  bool cc = false;  // some product of the launch has CUDA-core entries (f3)
  for (int i = 0; i < prm.nprob; ++i) cc = cc || prm.pr[i].ccent != nullptr;
  jigsaw_status_t st = cc ? launch_shape<true>(prm, NT, S, grid, dev, pair, vb, s)
                          : launch_shape<false>(prm, NT, S, grid, dev, pair, vb, s);
  if (w.graph_owned) {
    cudaError_t e = cudaFreeAsync(w.base, s);  // free node right after the kernel node
    if (st == JIGSAW_SUCCESS && e != cudaSuccess) st = cuda_status(e, "workspace free node");
  } else {
    release_workspace(w, s);
  }
  return st;
}

static jigsaw_status_t launch_group(const Format* const* fs, const void* const* Bs, const int64_t* Ns,
                                    void* const* Cs, int count, cudaStream_t s);

jigsaw_status_t launch_spmm(const Format& f, const void* dB, int64_t N, void* dC, cudaStream_t s) {
  last_launch() = jigsaw_launch_desc_t{};
  thread_local ParamsOne prm;  // host-side scratch for the parameter block
  prm.nprob = 1;
  prm.use_pin = 1;
  prm.use_ulist = 0;
  fill_problem(prm, 0, f, dB, N, dC);
  int NT = 128, S = 1, grid = 1;
  choose_config(f, N, spmm_num_sms(), &NT, &S, &grid);
  const bool pair = f.P == kPairPanelRows;
  const int force_split = launch_override().split_k;
  if (pair || (S == 1 && NT >= 128 && !force_split)) {
    // large products: the grouped persistent path (cost-ordered schedule, long
    // units split into pieces; CTA pairs are only scheduled there)
    const Format* fp = &f;
    return launch_group(&fp, &dB, &N, &dC, 1, s);
  }
  prm.use_ctab = 0;
  prm.bpf_bytes = 0;
  prm.bpf_chunk = 0;
  if (force_split == 1 || force_split == 2 || force_split == 4 || force_split == 8) {
    // diagnostic override: split-K S over a cluster (NT = 64, or 32 with tile_n = 32)
    NT = launch_override().tile_n == 32 ? 32 : 64;
    S = force_split;
    const int64_t un = f.npanels * ((N + NT - 1) / NT);
    grid = S > 1 ? (int)(un * S) : (int)std::min<int64_t>(un, spmm_num_sms());
  }
  // host-decoded first unit of every CTA (see ParamsT::ctab)
  if (grid <= ParamsOne::kMaxCta && !knobs().no_ctab) {
    const int64_t nkb_units = f.npanels * ((N + NT - 1) / NT);
    for (int c = 0; c < grid; ++c) {
      const int u = S > 1 ? c / S : c, r = S > 1 ? c % S : 0;
      if (u >= nkb_units) {
        prm.ctab[c][0] = make_int4(0, 0, 0, 0);
        prm.ctab[c][1] = make_int4(0, 0, 0, 0);
        continue;
      }
      const int p = (int)(u % f.npanels), n0 = (int)(u / f.npanels) * NT;
      const int4 pi = f.pin[p];  // {k-steps, first k-step, first E block, dense k-steps}
      const int nkb = (pi.x + 3) / 4 + (pi.w + 3) / 4;
      prm.ctab[c][0] = make_int4(p, n0, r * nkb / S, (r + 1) * nkb / S);
      prm.ctab[c][1] = make_int4(pi.x, f.pin_dev(p).w, pi.y, pi.z);
    }
    prm.use_ctab = 1;
  }
  // small B: prefetch it into L2 at kernel start, spread over the CTAs
  // (developer option: measured 0.1-0.2 us slower)
  const int64_t bbytes = f.K * N * 2;
  if (bbytes <= ((int64_t)16 << 20) && knobs().bpf) {
    prm.bpf_bytes = bbytes;
    prm.bpf_chunk = ((bbytes + grid - 1) / grid + 255) & ~int64_t(255);
  }
  return launch_params(prm, NT, S, grid, f.device, pair, s);
}

// Grouped launch: many independent products in ONE persistent kernel (units of
// all problems are dealt round-robin to the CTAs), up to kMaxProblems per launch.
// Products with 128-row and 256-row panels go to separate launches (one CTA vs
// one CTA pair per unit).
static jigsaw_status_t launch_group(const Format* const* fs, const void* const* Bs, const int64_t* Ns,
                                    void* const* Cs, int count, cudaStream_t s) {
  thread_local ParamsGroup prm;
  const int sms = spmm_num_sms();
  const bool pair = count > 0 && fs[0]->P == kPairPanelRows;
  const Knobs& kn = knobs();
  for (int i0 = 0; i0 < count; i0 += kMaxProblems) {
    const int n = std::min(kMaxProblems, count - i0);
    prm.nprob = n;
    prm.use_pin = 1;
    prm.use_ctab = 0;
    prm.bpf_bytes = 0;
    prm.bpf_chunk = 0;
    int64_t u128 = 0, u64 = 0;
    for (int i = 0; i < n; ++i) {
      fill_problem(prm, i, *fs[i0 + i], Bs[i0 + i], Ns[i0 + i], Cs[i0 + i]);
      u128 += fs[i0 + i]->npanels * ((Ns[i0 + i] + 127) / 128);
      u64 += fs[i0 + i]->npanels * ((Ns[i0 + i] + 63) / 64);
    }
    int64_t u256 = 0, kbs = 0, npan = 0;
    for (int i = 0; i < n; ++i) {
      const Format& f = *fs[i0 + i];
      u256 += f.npanels * ((Ns[i0 + i] + 255) / 256);
      for (int64_t p = 0; p < f.npanels; ++p) kbs += (f.pin[p].x + 3) / 4 + (f.pin[p].w + 3) / 4;
      npan += f.npanels;
    }
    const int force = launch_override().tile_n;
    int NT;
    if (pair) {
      NT = ((u256 >= sms / 2 && force != 128) || force == 256) ? 256 : 128;
    } else {
      NT = u128 >= 2 * sms ? 128 : 64;
      if ((u256 >= sms && kbs >= 24 * npan && force == 0) || force == 256) NT = 256;
      if (force == 128 || force == 64 || force == 32) NT = force;
    }
    const int64_t units = NT == 256 ? u256 : NT == 128 ? u128 : u64;
    const int slots_max = pair ? sms / 2 : sms;                  // CTAs or CTA pairs
    int slots = (int)std::min<int64_t>(units, slots_max);
    // Schedule: units sorted by cost (k-blocks of their panel + a fixed per-unit
    // cost), longest first, dealt by greedy LPT to the least loaded CTA (or CTA
    // pair); every slot runs its own queue, known at launch.  A unit much longer
    // than the per-slot average is cut into column slices (or, on request,
    // k-range pieces reduced through the workspace) so one long panel does not
    // set the makespan.
    prm.use_ulist = 0;
    int npieces_total = -1, pslots = 0, nsplit_items = 0;
    const size_t tile = (size_t)128 * NT * sizeof(float) * (pair ? 2 : 1);
    if (units <= ParamsGroup::kMaxUnits) {
      struct U { int cost; int nkb; uint32_t code; int n0; int64_t N; };
      thread_local std::vector<U> us;
      us.clear();
      int64_t total = 0;
      // fixed per-unit cost in k-block equivalents (accumulator drain, pipeline
      // refill): 2 for single CTAs (C2 static plan: 1 -> 32.4, 2 -> 31.8 us,
      // profiles/r02w); pairs with NT = 256 have a single accumulator buffer, so a
      // unit's epilogue is not overlapped with the next unit's mainloop: 4
      // (C2 at P = 256: 41.1 -> 35.3 us; the larger cost also stops the split
      // pieces whose workspace reduction cost more than the balance they bought,
      // profiles/r01w_unit_cost.txt).
      const int unit_cost = kn.unit_cost >= 0 ? kn.unit_cost : (pair && NT == 256 ? 4 : 2);
      for (int i = 0; i < n; ++i) {
        const Format& f = *fs[i0 + i];
        const int ntn = (int)((Ns[i0 + i] + NT - 1) / NT);
        for (int p = 0; p < f.npanels; ++p)
          for (int t = 0; t < ntn; ++t) {  // N tiles of a panel adjacent: they share its A stream
            const int nkb = (f.pin[p].x + 3) / 4 + (f.pin[p].w + 3) / 4;
            us.push_back({nkb + unit_cost, nkb, ((uint32_t)i << 26) | ((uint32_t)(t * f.npanels + p) << 15), t * NT,
                          Ns[i0 + i]});
            total += nkb + unit_cost;
          }
      }
      const bool loc = kn.sched_loc;  // developer experiment: locality order, no cost sort, no pieces
      const int64_t target = std::max<int64_t>(4, (total + slots_max - 1) / slots_max);
      const bool allow_split = !launch_override().no_pieces && !loc;
      thread_local std::vector<std::pair<int, uint32_t>> order;
      order.clear();
      if (!loc) std::stable_sort(us.begin(), us.end(), [](const U& a, const U& b) { return a.cost > b.cost; });
      // Bytes a CTA ingests per k-block: compressed A + metadata, and the B rows
      // of its NT_L columns (the cost of a column slice scales only the B part).
      const double kb_a = kStepsPerBlock * kKStepBytesA + kEBlockBytes;
      const double kb_b = 128.0 * 2 * (pair ? NT / 2 : NT);
      const int ns_max = pair ? NT / 64 : NT / 32;  // narrowest slice: 32 B columns per CTA
      for (const U& x : us) {
        int np = 1;
        const bool too_long = allow_split && (int64_t)x.cost * 100 > target * kn.split_pct;
        if (too_long && ns_max >= 2 && !launch_override().k_pieces &&
            (int64_t)order.size() + ns_max <= ParamsGroup::kMaxUnits) {
          // N-split: column slices of the N tile over the whole k-range (each
          // re-reads the unit's compressed A, none needs a partial-tile
          // workspace or a reduction); the fewest slices that bring the unit
          // to the per-slot load
          int ns = 2;
          auto slice_cost = [&](int n) {
            return (int)(x.nkb * (kb_a + kb_b / n) / (kb_a + kb_b)) + unit_cost;
          };
          while (ns < ns_max && slice_cost(ns) > target) ns *= 2;
          const int w = NT / ns;
          for (int h = 0; h < ns; ++h)
            if (x.n0 + h * w < x.N) {
              order.push_back({-slice_cost(ns), x.code | ((uint32_t)h << 12) | ((uint32_t)(ns - 1) << 9) | kNSplit});
              ++nsplit_items;
            }
          continue;
        }
        if (too_long && x.nkb >= 8) {
          np = (int)std::min<int64_t>({8, (x.cost + target - 1) / target, x.nkb / 4});
          if (pslots + np > 511 || (int64_t)order.size() + np > ParamsGroup::kMaxUnits) np = 1;
        }
        if (np > 1) {
          for (int pc = 0; pc < np; ++pc)
            order.push_back({-(x.cost / np), x.code | ((uint32_t)pc << 12) | ((uint32_t)(np - 1) << 9) |
                                                 (uint32_t)pslots});
          pslots += np;
        } else {
          order.push_back({-x.cost, x.code});
        }
      }
      if (!loc)
        std::stable_sort(order.begin(), order.end(),
                         [](const std::pair<int, uint32_t>& a, const std::pair<int, uint32_t>& b) { return a.first < b.first; });
      const int nslots = (int)std::min<int64_t>(slots_max, (int64_t)order.size());
      npieces_total = (int)order.size();
      if (kn.dyn_sched && !pair) {
        // developer option: cost order, handed out by the dynamic scheduler
        for (size_t k = 0; k < order.size(); ++k) prm.ulist[k] = order[k].second;
      } else {
        // static schedule: greedy LPT (each piece, longest first, to the least
        // loaded CTA or CTA pair); slot c runs positions c, c + nslots, ... of
        // the list, padded with kNoWork where its queue is shorter than the longest
        thread_local std::vector<std::vector<uint32_t>> q;
        q.assign(nslots, {});
        std::vector<std::pair<int64_t, int>> heap;  // (load, slot), min-heap
        for (int c = 0; c < nslots; ++c) heap.push_back({0, c});
        auto cmp = [](const std::pair<int64_t, int>& a, const std::pair<int64_t, int>& b) { return a > b; };
        std::make_heap(heap.begin(), heap.end(), cmp);
        size_t maxlen = 0;
        size_t k_rr = 0;
        for (const auto& o : order) {
          if (loc) {  // round-robin: consecutive (same-panel) units run concurrently
            const int c = (int)(k_rr++ % nslots);
            q[c].push_back(o.second);
            maxlen = std::max(maxlen, q[c].size());
            continue;
          }
          std::pop_heap(heap.begin(), heap.end(), cmp);
          auto& h = heap.back();
          q[h.second].push_back(o.second);
          h.first += -o.first;
          maxlen = std::max(maxlen, q[h.second].size());
          std::push_heap(heap.begin(), heap.end(), cmp);
        }
        // Units of panels with CUDA-core entries (f3) go first in their slot's
        // queue: their epilogue (the entries' B loads) then overlaps the next
        // units' mainloops instead of extending the slot's tail.  The set of
        // units per slot -- the LPT balance -- is unchanged.
        for (auto& qc : q)
          std::stable_partition(qc.begin(), qc.end(), [&](uint32_t code) {
            const Format& f = *fs[i0 + (int)(code >> 26)];
            return !f.ccT.empty() && f.ccT[((code >> 15) & 0x7FFu) % f.npanels] > 0;
          });
        if (JIG_DEV && kn.debug_sched) {
          int64_t lo = INT64_MAX, hi = 0;
          for (const auto& h : heap) lo = std::min(lo, h.first), hi = std::max(hi, h.first);
          fprintf(stderr, "[jigsaw] pair schedule: %zu pieces (%d split slots) on %d pairs, load min %lld max %lld "
                  "(target %lld), longest queue %zu\n", order.size(), pslots, nslots, (long long)lo, (long long)hi,
                  (long long)target, maxlen);
        }
        if (maxlen * nslots <= (size_t)ParamsGroup::kMaxUnits) {
          for (size_t r = 0; r < maxlen; ++r)
            for (int c = 0; c < nslots; ++c) prm.ulist[r * nslots + c] = r < q[c].size() ? q[c][r] : kNoWork;
          npieces_total = (int)(maxlen * nslots);
        } else {  // snake order (no padding)
          for (size_t k = 0; k < order.size(); ++k) {
            const int r = (int)(k / nslots), c = (int)(k % nslots);
            const int mr = (int)std::min<int64_t>(nslots, (int64_t)order.size() - (int64_t)r * nslots);
            prm.ulist[r * nslots + ((r & 1) ? mr - 1 - c : c)] = order[k].second;
          }
        }
      }
      prm.use_ulist = 1;
      slots = nslots;
    }
    const int grid = pair ? 2 * slots : slots;
    // all B's of the launch small enough to sit in L2 next to the A stream:
    // prefetch them at kernel start (developer option; measured slower for C2,
    // 44.7 vs 41.0 us)
    if (kn.group_bpf > 0) {
      int64_t bsum = 0;
      for (int i = 0; i < n; ++i) bsum += fs[i0 + i]->K * Ns[i0 + i] * 2;
      if (bsum <= (kn.group_bpf << 20)) {
        prm.bpf_bytes = bsum;
        prm.bpf_chunk = ((bsum + grid - 1) / grid + 255) & ~int64_t(255);
      }
    }
    jigsaw_status_t st = launch_params(prm, NT, 1, grid, fs[i0]->device, pair, s, npieces_total, pslots, tile);
    last_launch().nsplit_items = nsplit_items;
    if (st != JIGSAW_SUCCESS) return st;
  }
  return JIGSAW_SUCCESS;
}

jigsaw_status_t launch_spmm_grouped(const Format* const* fs, const void* const* Bs, const int64_t* Ns,
                                    void* const* Cs, int count, cudaStream_t s) {
  last_launch() = jigsaw_launch_desc_t{};
  bool mixed = false;
  for (int i = 1; i < count; ++i) mixed |= fs[i]->P != fs[0]->P;
  if (!mixed) return launch_group(fs, Bs, Ns, Cs, count, s);
  for (int P : {kPanelRows, kPairPanelRows}) {
    std::vector<const Format*> f2;
    std::vector<const void*> b2;
    std::vector<int64_t> n2;
    std::vector<void*> c2;
    for (int i = 0; i < count; ++i)
      if (fs[i]->P == P) {
        f2.push_back(fs[i]);
        b2.push_back(Bs[i]);
        n2.push_back(Ns[i]);
        c2.push_back(Cs[i]);
      }
    if (f2.empty()) continue;
    jigsaw_status_t st = launch_group(f2.data(), b2.data(), n2.data(), c2.data(), (int)f2.size(), s);
    if (st != JIGSAW_SUCCESS) return st;
  }
  return JIGSAW_SUCCESS;
}

// Copies the timeline of the last traced launch (JIGSAW_TRACE=1): per CTA 16
// int64 slots (clock64 at the trace points 0-11, 13 = %globaltimer at exit,
// 14 = SM id, 15 = %globaltimer at entry).  Returns the CTA count.
int debug_trace_read(long long* host, int max_ctas) {
  if (max_ctas < 0) {  // per-k-block timeline of CTAs 0..7: 8*6*32 int64
    if (cudaMemcpyFromSymbol(host, g_trace_kb, sizeof(long long) * 8 * 6 * kTraceKB) != cudaSuccess) return -1;
    return 8;
  }
  const int n = std::min(max_ctas, g_trace_ctas);
  if (n <= 0) return 0;
  if (cudaMemcpyFromSymbol(host, g_trace, sizeof(long long) * kTraceSlots * n) != cudaSuccess) return -1;
  return n;
}

}  // namespace jig
