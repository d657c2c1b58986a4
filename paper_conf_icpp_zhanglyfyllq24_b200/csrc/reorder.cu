// reorder.cu -- GPU builder of the reorder-aware format (R1..R5).
//
//   R1 k_colmask     per panel and column: the P-bit row mask of nonzeros
//                    (BLOCK_TILE granularity)
//   R2 k_compact     S_p = ascending list of the panel's nonzero columns
//                    (col_idx_array; R-Q4)
//   R3 k_main_tiles  one warp per full 16-column tile of S_p: Alg. 1
//                    + reorder retry -- tiles are independent
//   R4 k_overflow    one CTA per panel (waves of warps): the remainder of S_p and the evicted
//                    columns, re-tiled in FIFO order (R-Q12)
//   R5 k_emit        2:4 compression straight into the device
//                    layout the SpMM kernel consumes (A image, TMEM metadata
//                    lanes, B gather rows) + the canonical col_idx / perm
//
// The tile search returns the lexicographically first cover (R-Q8) and evicts
// the real column in the fewest compatible groups, ties to the smallest slot
// (R-Q11) -- the definition the oracle (oracle/oracle.c) implements
// independently; tests/test_gpu_parity.py compares the two bit for bit.
#include <climits>
#include <atomic>
#include <cstdio>
#include <cstring>
#include <mutex>

#include "internal.h"

namespace jig {

namespace {

constexpr int kNumSubsets = 1820;  // C(16, 4)
constexpr int kNumG0 = 455;        // 4-subsets containing slot 0 = C(15, 3)
constexpr unsigned kFull = 0xFFFFFFFFu;

__device__ uint16_t g_subs[kNumSubsets];  // all 4-subsets of 16 slots, lexicographic

std::atomic<bool> g_tables_ready[64] = {};
std::mutex g_tables_mu;

jigsaw_status_t init_tables(int dev) {
  if (dev >= 0 && dev < 64 && g_tables_ready[dev].load(std::memory_order_acquire)) return JIGSAW_SUCCESS;
  std::lock_guard<std::mutex> lock(g_tables_mu);
  if (dev >= 0 && dev < 64 && g_tables_ready[dev].load(std::memory_order_acquire)) return JIGSAW_SUCCESS;
  uint16_t subs[kNumSubsets];
  int n = 0;
  for (int a = 0; a < 16; ++a)
    for (int b = a + 1; b < 16; ++b)
      for (int c = b + 1; c < 16; ++c)
        for (int d = c + 1; d < 16; ++d)
          subs[n++] = (uint16_t)((1u << a) | (1u << b) | (1u << c) | (1u << d));
  cudaError_t e = cudaMemcpyToSymbol(g_subs, subs, sizeof subs);
  if (e != cudaSuccess) return cuda_status(e, "cudaMemcpyToSymbol(subsets)");
  if (dev >= 0 && dev < 64) g_tables_ready[dev].store(true, std::memory_order_release);
  return JIGSAW_SUCCESS;
}

// Row mask of one column inside a panel of up to 256 rows (row r = bit r%32 of word r/32).
struct RowMask {
  uint4 lo, hi;
};
__device__ __forceinline__ RowMask zero_mask() { return RowMask{make_uint4(0, 0, 0, 0), make_uint4(0, 0, 0, 0)}; }
// bits set where >= 3 of the 4 masks are set (the Alg. 1 compatibility test)
__device__ __forceinline__ uint32_t three_of_four(uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
  return (a & b & (c | d)) | (c & d & (a | b));
}
__device__ __forceinline__ uint32_t any_three_of_four(const RowMask& a, const RowMask& b, const RowMask& c,
                                                      const RowMask& d) {
  return three_of_four(a.lo.x, b.lo.x, c.lo.x, d.lo.x) | three_of_four(a.lo.y, b.lo.y, c.lo.y, d.lo.y) |
         three_of_four(a.lo.z, b.lo.z, c.lo.z, d.lo.z) | three_of_four(a.lo.w, b.lo.w, c.lo.w, d.lo.w) |
         three_of_four(a.hi.x, b.hi.x, c.hi.x, d.hi.x) | three_of_four(a.hi.y, b.hi.y, c.hi.y, d.hi.y) |
         three_of_four(a.hi.z, b.hi.z, c.hi.z, d.hi.z) | three_of_four(a.hi.w, b.hi.w, c.hi.w, d.hi.w);
}
__device__ __forceinline__ uint32_t all_three(const RowMask& a, const RowMask& b, const RowMask& c) {
  return (a.lo.x & b.lo.x & c.lo.x) | (a.lo.y & b.lo.y & c.lo.y) | (a.lo.z & b.lo.z & c.lo.z) |
         (a.lo.w & b.lo.w & c.lo.w) | (a.hi.x & b.hi.x & c.hi.x) | (a.hi.y & b.hi.y & c.hi.y) |
         (a.hi.z & b.hi.z & c.hi.z) | (a.hi.w & b.hi.w & c.hi.w);
}

// ------------------------------------------------------------------ R1
__global__ void k_colmask(const uint16_t* __restrict__ A, int64_t M, int64_t K, int P,
                          RowMask* __restrict__ masks, unsigned long long* __restrict__ nnz) {
  const int p = blockIdx.y;
  const int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  uint32_t w[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  int cnt = 0;
  if (c < K) {
    const int64_t row0 = (int64_t)p * P;
    const int nr = (int)min((int64_t)P, M - row0);
#pragma unroll 8
    for (int r = 0; r < nr; ++r) {
      const uint16_t x = A[(row0 + r) * K + c];
      if (x & 0x7FFFu) {  // R-Q3: +-0 are zeros
        w[r >> 5] |= 1u << (r & 31);
        ++cnt;
      }
    }
    masks[(int64_t)p * K + c] = RowMask{make_uint4(w[0], w[1], w[2], w[3]), make_uint4(w[4], w[5], w[6], w[7])};
  }
  for (int o = 16; o; o >>= 1) cnt += __shfl_xor_sync(kFull, cnt, o);
  if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(nnz, (unsigned long long)cnt);
}

// ------------------------------------------------------------------ R2
__global__ void k_compact(const RowMask* __restrict__ masks, int64_t K, int32_t* __restrict__ S,
                          int32_t* __restrict__ Kp) {
  __shared__ int wsum[32];
  __shared__ int total;
  const int p = blockIdx.x, tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int nw = blockDim.x >> 5;
  int base = 0;
  for (int64_t c0 = 0; c0 < K; c0 += blockDim.x) {
    const int64_t c = c0 + tid;
    bool flag = false;
    if (c < K) {
      const RowMask m = masks[(int64_t)p * K + c];
      flag = (m.lo.x | m.lo.y | m.lo.z | m.lo.w | m.hi.x | m.hi.y | m.hi.z | m.hi.w) != 0;
    }
    const unsigned b = __ballot_sync(kFull, flag);
    const int lpre = __popc(b & ((1u << lane) - 1u));
    if (lane == 0) wsum[warp] = __popc(b);
    __syncthreads();
    if (warp == 0) {
      int x = lane < nw ? wsum[lane] : 0;
      int incl = x;
      for (int o = 1; o < 32; o <<= 1) {
        int y = __shfl_up_sync(kFull, incl, o);
        if (lane >= o) incl += y;
      }
      if (lane < nw) wsum[lane] = incl - x;  // exclusive
      if (lane == 31) total = incl;
    }
    __syncthreads();
    if (flag) S[(int64_t)p * K + base + wsum[warp] + lpre] = (int32_t)c;
    base += total;
    __syncthreads();
  }
  if (tid == 0) Kp[p] = base;
}

// ------------------------------------------------------------------ tile search
constexpr int kMaxBig = 256;
struct TileSmem {
  uint32_t bitmap[2048];  // compat[S] for every 4-subset S, indexed by the 16-bit slot mask
  uint32_t half[2048];    // cover_dp: 8-slot unions g0 | g1 of two disjoint compatible groups
  uint16_t big[kMaxBig];  // compatible 3- and 4-subsets of the real slots (existence test)
  int nbig;
  RowMask m[16];          // row masks per slot (PAD: 0)
  int32_t cols[16];       // column per slot (kPad = -1)
  int32_t ev[16];         // evicted columns, in eviction order
  uint8_t perm[16];
  int nev;
  int stop;               // cover_exists: some lane found a cover (the others stop)
};

__device__ __forceinline__ bool compat(const TileSmem& s, uint32_t sub) {
  return (s.bitmap[sub >> 5] >> (sub & 31)) & 1u;
}

// Lexicographically first completion of the cover given g0 (R-Q8): g1 holds the
// smallest uncovered slot, candidates tried in lexicographic order; then g2; g3
// is the rest.
// Pruning (exact, never changes the result): no compatible group holds more than
// `hmax` real columns, so the real columns still uncovered must fit hmax per
// remaining group.
__device__ bool complete_cover(const TileSmem& s, uint32_t used, uint32_t& o1, uint32_t& o2,
                               uint32_t& o3, uint32_t realset, int hmax) {
  const int lo1 = __ffs(~used & 0xFFFFu) - 1;
  const uint32_t av1 = ~used & 0xFFFFu & ~(1u << lo1);
  for (uint32_t x = av1; x; x &= x - 1) {
    const int b = __ffs(x) - 1;
    for (uint32_t y = x & (x - 1); y; y &= y - 1) {
      const int c = __ffs(y) - 1;
      for (uint32_t z = y & (y - 1); z; z &= z - 1) {
        const int d = __ffs(z) - 1;
        const uint32_t s1 = (1u << lo1) | (1u << b) | (1u << c) | (1u << d);
        if (!compat(s, s1)) continue;
        const uint32_t u2 = used | s1;
        if (__popc(realset & ~u2) > 2 * hmax) continue;
        const int lo2 = __ffs(~u2 & 0xFFFFu) - 1;
        const uint32_t av2 = ~u2 & 0xFFFFu & ~(1u << lo2);
        for (uint32_t x2 = av2; x2; x2 &= x2 - 1) {
          const int b2 = __ffs(x2) - 1;
          for (uint32_t y2 = x2 & (x2 - 1); y2; y2 &= y2 - 1) {
            const int c2 = __ffs(y2) - 1;
            for (uint32_t z2 = y2 & (y2 - 1); z2; z2 &= z2 - 1) {
              const int d2 = __ffs(z2) - 1;
              const uint32_t s2 = (1u << lo2) | (1u << b2) | (1u << c2) | (1u << d2);
              if (!compat(s, s2)) continue;
              const uint32_t s3 = ~(u2 | s2) & 0xFFFFu;
              if (compat(s, s3)) {
                o1 = s1; o2 = s2; o3 = s3;
                return true;
              }
            }
          }
        }
      }
    }
  }
  return false;
}

// Exact existence test for a cover of all 16 slots by 4 disjoint compatible
// groups, by levels (the oracle's DFS memoises dead used-sets instead; both only
// decide existence): level 2 marks every union g0 | g1 of a compatible group g0
// holding slot 0 and a compatible g1 holding the smallest slot outside g0 (at
// most C(16,8) distinct 8-slot sets, deduplicated in a bitmap); a cover exists
// iff the 8 remaining slots of some marked set split into two compatible groups
// (the one holding their smallest slot, and the rest).  Work is bounded
// (<= 455 x 165 level-2 checks, <= 12870 x 35 level-3 checks per warp), unlike
// the depth-first search of complete_cover when no cover exists.
__device__ bool cover_dp(TileSmem& s, uint32_t realset, int hmax, int lane) {
  for (int i = lane; i < 2048; i += 32) s.half[i] = 0;
  __syncwarp();
  for (int k = lane; k < kNumG0; k += 32) {
    const uint32_t g0 = g_subs[k];
    // (exact pruning, as in complete_cover: no compatible group holds more than
    // hmax real columns, so the real columns left must fit hmax per group)
    if (!compat(s, g0) || __popc(realset & ~g0) > 3 * hmax) continue;
    const int l1 = __ffs(~g0 & 0xFFFFu) - 1;
    const uint32_t av = ~g0 & 0xFFFFu & ~(1u << l1);
    for (uint32_t x = av; x; x &= x - 1) {
      const uint32_t bb = x & (0u - x);
      for (uint32_t y = x & (x - 1); y; y &= y - 1) {
        const uint32_t cb = y & (0u - y);
        for (uint32_t z = y & (y - 1); z; z &= z - 1) {
          const uint32_t g1 = (1u << l1) | bb | cb | (z & (0u - z));
          if (compat(s, g1) && __popc(realset & ~(g0 | g1)) <= 2 * hmax) {
            const uint32_t u = g0 | g1;
            atomicOr(&s.half[u >> 5], 1u << (u & 31));
          }
        }
      }
    }
  }
  __syncwarp();
  bool found = false;
  for (int w = lane; w < 2048 && !__any_sync(kFull, found); w += 32) {
    for (uint32_t bits = s.half[w]; bits && !found; bits &= bits - 1) {
      const uint32_t u = (uint32_t)w * 32u + (uint32_t)(__ffs(bits) - 1);
      const uint32_t rest = ~u & 0xFFFFu;
      const int l2 = __ffs(rest) - 1;
      const uint32_t av = rest & ~(1u << l2);
      for (uint32_t x = av; x && !found; x &= x - 1) {
        const uint32_t bb = x & (0u - x);
        for (uint32_t y = x & (x - 1); y && !found; y &= y - 1) {
          const uint32_t cb = y & (0u - y);
          for (uint32_t z = y & (y - 1); z && !found; z &= z - 1) {
            const uint32_t g2 = (1u << l2) | bb | cb | (z & (0u - z));
            if (compat(s, g2) && compat(s, rest & ~g2)) found = true;
          }
        }
      }
    }
  }
  return __any_sync(kFull, found) != 0;
}

// Exact existence test for a cover (used to skip exhaustive searches that must
// fail; it never changes WHICH cover is chosen).  PAD slots are interchangeable
// zero columns and any group with <= 2 real columns is compatible, so a cover
// exists iff some k <= 4 disjoint compatible "big" groups (3 or 4 real columns)
// hold enough real columns that the rest fits 2 per remaining group:
// sum(|b_i| - 2) >= nreal - 8.  When the candidate list or the search budget
// overflows, the level-wise exact test cover_dp decides.
__device__ bool cover_exists(TileSmem& s, uint32_t realset, int hmax, int lane) {
  if (lane == 0) {
    s.nbig = 0;
    s.stop = 0;
  }
  __syncwarp();
  for (int k = lane; k < kNumSubsets; k += 32) {          // 4 real columns
    const uint32_t sub = g_subs[k];
    if ((sub & ~realset) == 0 && compat(s, sub)) {
      const int i = atomicAdd(&s.nbig, 1);
      if (i < kMaxBig) s.big[i] = (uint16_t)sub;
    }
  }
  if (lane < 16 && ((realset >> lane) & 1u)) {              // 3 real columns, min slot = lane
    const RowMask ma = s.m[lane];
    for (uint32_t x = realset & ~((2u << lane) - 1u); x; x &= x - 1) {
      const int b = __ffs(x) - 1;
      const RowMask mb = s.m[b];
      for (uint32_t y = x & (x - 1); y; y &= y - 1) {
        const int c = __ffs(y) - 1;
        const RowMask mc = s.m[c];
        const uint32_t all3 = all_three(ma, mb, mc);
        if (!all3) {
          const int i = atomicAdd(&s.nbig, 1);
          if (i < kMaxBig) s.big[i] = (uint16_t)((1u << lane) | (1u << b) | (1u << c));
        }
      }
    }
  }
  __syncwarp();
  // depth-first over up to 4 disjoint blocks, the first block dealt to the lanes
  // (lane l starts from blocks l, l + 32, ...): a search that must fail -- the
  // common case once a tile has more than 8 hard columns -- is exhausted 32
  // lanes at a time instead of by one thread
  int found = 0;
  bool maybe = false;
  const int n = s.nbig, need = __popc(realset) - 8;
  if (n > kMaxBig) {
    maybe = true;
  } else {
    int budget = 1 << 13;  // per lane; exceeding it answers "maybe" (exactness kept)
    volatile int* stop = &s.stop;
    for (int i0 = lane; i0 < n && !found && !maybe && !*stop; i0 += 32) {
      const uint32_t b0 = s.big[i0];
      int idx[3];
      uint32_t used[4];
      int exc[4];
      used[0] = b0;
      exc[0] = __popc(b0) - 2;
      if (exc[0] >= need) { found = 1; break; }
      int d = 0;
      idx[0] = i0 + 1;
      while (d >= 0) {
        if (--budget < 0) { maybe = true; break; }
        if ((budget & 63) == 0 && *stop) break;  // another lane already answered
        if (idx[d] >= n) {                    // level exhausted: backtrack
          --d;
          if (d >= 0) ++idx[d];
          continue;
        }
        const uint32_t b = s.big[idx[d]];
        if (b & used[d]) { ++idx[d]; continue; }
        used[d + 1] = used[d] | b;
        exc[d + 1] = exc[d] + __popc(b) - 2;
        if (exc[d + 1] >= need) { found = 1; break; }
        if (d + 1 < 3) { idx[d + 1] = idx[d] + 1; ++d; } else { ++idx[d]; }
      }
      if (found || maybe) *stop = 1;  // answered (or inconclusive: the exact test decides)
    }
  }
  if (__any_sync(kFull, found)) return true;
  // inconclusive (candidate list or search budget exceeded): the exact test below
  if (__any_sync(kFull, maybe)) return cover_dp(s, realset, hmax, lane);
  return false;
}

// Alg. 1 + reorder retry on one tile, executed by one full warp.  On entry
// s.cols / s.m hold the 16 popped columns; on exit s.cols has evicted slots set
// to PAD, s.perm the new column order g0||g1||g2||g3, s.ev[0..s.nev) the evictions.
__device__ void tile_search(TileSmem& s, int lane) {
  if (lane == 0) s.nev = 0;
  __syncwarp();
  uint32_t realset = __ballot_sync(kFull, lane < 16 && s.cols[lane] != kPad) & 0xFFFFu;
  for (;;) {
    // Alg. 1 lines 1-8: compatibility of all 1820 4-column groups; a group is
    // compatible iff no row has >= 3 nonzeros among its 4 columns.
    for (int i = lane; i < 2048; i += 32) s.bitmap[i] = 0;
    __syncwarp();
    int fr = 0, hmax = 0;
    // freq counters, per lane: slot j counts in byte (j & 3) of word j >> 2 (<= 57
    // subsets per lane, no byte overflow); reduced over the warp once, below
    uint32_t pc0 = 0, pc1 = 0, pc2 = 0, pc3 = 0;
    for (int k0 = 0; k0 < kNumSubsets; k0 += 32) {
      const int k = k0 + lane;
      bool ok = false;
      uint32_t sub = 0;
      if (k < kNumSubsets) {
        sub = g_subs[k];
        uint32_t r = sub;
        const int a = __ffs(r) - 1; r &= r - 1;
        const int b = __ffs(r) - 1; r &= r - 1;
        const int c = __ffs(r) - 1; r &= r - 1;
        const int d = __ffs(r) - 1;
        const uint32_t bad = any_three_of_four(s.m[a], s.m[b], s.m[c], s.m[d]);
        ok = bad == 0;
        if (ok) {
          atomicOr(&s.bitmap[sub >> 5], 1u << (sub & 31));
          hmax = max(hmax, __popc(sub & realset));
          // nibble -> one count per byte: (n * 0x00204081) & 0x01010101
          pc0 += ((sub & 0xFu) * 0x00204081u) & 0x01010101u;
          pc1 += (((sub >> 4) & 0xFu) * 0x00204081u) & 0x01010101u;
          pc2 += (((sub >> 8) & 0xFu) * 0x00204081u) & 0x01010101u;
          pc3 += (((sub >> 12) & 0xFu) * 0x00204081u) & 0x01010101u;
        }
      }
    }
    {
      // freq[j] = number of compatible groups containing slot j: the byte
      // counters widened to 16-bit halves (<= 455 each) and summed over the warp
      const uint32_t pw[4] = {pc0, pc1, pc2, pc3};
      uint32_t tot[8];
#pragma unroll
      for (int w = 0; w < 4; ++w) {
        tot[2 * w] = __reduce_add_sync(kFull, pw[w] & 0x00FF00FFu);             // bytes 0, 2
        tot[2 * w + 1] = __reduce_add_sync(kFull, (pw[w] >> 8) & 0x00FF00FFu);  // bytes 1, 3
      }
      if (lane < 16) {
        const int w = lane >> 2, b = lane & 3;
        uint32_t t = 0;
#pragma unroll
        for (int i = 0; i < 8; ++i)
          if (i == 2 * w + (b & 1)) t = tot[i];
        fr = (int)((t >> (16 * (b >> 1))) & 0xFFFFu);
      }
    }
    for (int o = 16; o; o >>= 1) hmax = max(hmax, __shfl_xor_sync(kFull, hmax, o));
    __syncwarp();
    // Necessary conditions for a cover (they only skip searches that must fail):
    // every slot lies in some compatible group; 4 groups can hold all real columns.
    bool coverable = __all_sync(kFull, lane >= 16 || fr > 0) && hmax * 4 >= __popc(realset);
    const int nreal = __popc(realset);
    // (hmax >= 3 and a necessary condition already failed: no cover, and some
    // compatible group holds 3+ real columns, so the shortcut below cannot apply --
    // the existence test is skipped, the result is the same)
    if (nreal > 8 && (hmax < 3 || coverable)) {
      const bool ex = cover_exists(s, realset, hmax, lane);
      if (s.nbig == 0) {
        // No compatible group holds 3+ real columns, and none will after more
        // evictions: every real column is in the same number of compatible groups
        // (C(pad,3) + (real-1)*C(pad,2)), so the retry evicts the smallest real
        // slots one by one until 8 remain -- done here in one step (identical result).
        if (lane == 0) {
          int need = nreal - 8;
          for (int j = 0; j < 16 && need > 0; ++j) {
            if (!((realset >> j) & 1u)) continue;
            s.ev[s.nev++] = s.cols[j];
            s.cols[j] = kPad;
            s.m[j] = zero_mask();
            --need;
          }
        }
        __syncwarp();
        realset = __ballot_sync(kFull, lane < 16 && s.cols[lane] != kPad) & 0xFFFFu;
        continue;
      }
      coverable = coverable && ex;
    }
    // Alg. 1 lines 9-17: lanes try the candidates for g0 (groups containing slot 0)
    // in lexicographic order, 32 at a time; the lowest successful one wins.
    if (coverable) {
      for (int k0 = 0; k0 < kNumG0; k0 += 32) {
        const int k = k0 + lane;
        uint32_t g0 = 0, a1 = 0, a2 = 0, a3 = 0;
        bool ok = false;
        if (k < kNumG0) {
          g0 = g_subs[k];
          ok = compat(s, g0) && __popc(realset & ~g0) <= 3 * hmax &&
               complete_cover(s, g0, a1, a2, a3, realset, hmax);
        }
        const unsigned b = __ballot_sync(kFull, ok);
        if (b) {
          const int w = __ffs(b) - 1;
          g0 = __shfl_sync(kFull, g0, w);
          a1 = __shfl_sync(kFull, a1, w);
          a2 = __shfl_sync(kFull, a2, w);
          a3 = __shfl_sync(kFull, a3, w);
          if (lane == 0) {
            int o = 0;
            const uint32_t gs[4] = {g0, a1, a2, a3};
            for (int g = 0; g < 4; ++g)
              for (uint32_t x = gs[g]; x; x &= x - 1) s.perm[o++] = (uint8_t)(__ffs(x) - 1);
          }
          __syncwarp();
          return;
        }
      }
    }
    // Reorder retry: evict the least frequent real column (ties: smallest slot).
    const int key = (lane < 16 && ((realset >> lane) & 1u)) ? (fr << 5) | lane : INT_MAX;
    int best = key;
    for (int o = 16; o; o >>= 1) best = min(best, __shfl_xor_sync(kFull, best, o));
    const int e = best & 31;
    if (lane == 0) {
      s.ev[s.nev++] = s.cols[e];
      s.cols[e] = kPad;
      s.m[e] = zero_mask();
    }
    realset &= ~(1u << e);
    __syncwarp();
  }
}

struct Scratch {
  int32_t* tcols;  // [npan][cap][16]
  uint8_t* tperm;  // [npan][cap][16]
  int32_t* tev;    // [npan][cap][16]
  uint8_t* tnev;   // [npan][cap]
  int32_t* tmap;   // [npan][cap] (CUDA-core split only, else null): tile t of the final list is
                   // tile tmap[t] of the canonical reorder
  int cap;
};

__device__ void store_tile(const TileSmem& s, const Scratch& sc, int p, int t, int lane) {
  const int64_t o = ((int64_t)p * sc.cap + t) * 16;
  if (lane < 16) {
    sc.tcols[o + lane] = s.cols[lane];
    sc.tperm[o + lane] = s.perm[lane];
    sc.tev[o + lane] = lane < s.nev ? s.ev[lane] : kPad;
  }
  if (lane == 0) sc.tnev[(int64_t)p * sc.cap + t] = (uint8_t)s.nev;
}

// ------------------------------------------------------------------ R3
constexpr int kR3Warps = 2;  // 2 x sizeof(TileSmem) (~17.6 KB) of static shared memory
__global__ void __launch_bounds__(32 * kR3Warps) k_main_tiles(const RowMask* __restrict__ masks,
                                                              const int32_t* __restrict__ S,
                                                              const int32_t* __restrict__ Kp,
                                                              int64_t K, Scratch sc) {
  __shared__ TileSmem sm[kR3Warps];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int p = blockIdx.y;
  const int t = blockIdx.x * kR3Warps + warp;
  if (t >= Kp[p] / 16) return;  // only full tiles of S_p (warp-uniform)
  TileSmem& s = sm[warp];
  if (lane < 16) {
    const int32_t c = S[(int64_t)p * K + 16 * t + lane];
    s.cols[lane] = c;
    s.m[lane] = masks[(int64_t)p * K + c];
  }
  __syncwarp();
  tile_search(s, lane);
  store_tile(s, sc, p, t, lane);
}

// ------------------------------------------------------------------ R4
// SPTC mode (paper): evicted columns are re-queued and re-tiled (overflow tiles).
// DENSE mode: only the partial last tile of S_p is built here, and the
// evicted columns of all tiles, in tile and eviction order, form the residual
// list R_p (left at the front of the panel's queue buffer, count in nres[p]).
//
// One CTA of kR4Warps warps per panel, in waves.  CR1 pops the FIFO one tile at a
// time, each tile appending its evictions at the back; so every tile whose 16
// columns are already in the queue when a wave starts sees exactly the columns
// the sequential algorithm would give it (appends only go behind it).  A wave
// searches all such tiles in parallel (one warp per tile), then appends their
// evictions in tile order.  When fewer than 16 columns are queued, every earlier
// tile is done and the one (partial) tile is popped exactly as in CR1.  The
// result is bit-identical to the sequential queue (tests compare with the oracle).
constexpr int kR4Warps = 8;
__global__ void __launch_bounds__(32 * kR4Warps) k_overflow(const RowMask* __restrict__ masks,
                                                            const int32_t* __restrict__ S,
                                                            const int32_t* __restrict__ Kp, int64_t K,
                                                            Scratch sc, int32_t* __restrict__ queue,
                                                            int64_t qcap, int32_t* __restrict__ T,
                                                            int* __restrict__ err, int mode,
                                                            int32_t* __restrict__ nres) {
  extern __shared__ __align__(16) uint8_t r4_smem[];
  TileSmem* sm = reinterpret_cast<TileSmem*>(r4_smem);
  __shared__ int64_t s_head, s_tail;
  __shared__ int s_t, s_nw, s_stop;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int p = blockIdx.x;
  const int kp = Kp[p], nfull = kp / 16, rem = kp - 16 * nfull;
  int32_t* q = queue + (int64_t)p * qcap;
  if (mode == 1) {
    if (warp != 0) return;
    TileSmem& s = sm[0];
    int t = nfull;
    if (rem > 0) {
      if (lane < 16) {
        const int32_t c = lane < rem ? S[(int64_t)p * K + 16 * nfull + lane] : kPad;
        s.cols[lane] = c;
        s.m[lane] = c == kPad ? zero_mask() : masks[(int64_t)p * K + c];
      }
      __syncwarp();
      tile_search(s, lane);
      store_tile(s, sc, p, t, lane);
      ++t;
      __syncwarp();
    }
    int64_t n = 0;
    for (int tt = 0; tt < t; ++tt) {
      const int e = sc.tnev[(int64_t)p * sc.cap + tt];
      if (lane < e) q[n + lane] = sc.tev[((int64_t)p * sc.cap + tt) * 16 + lane];
      n += e;
    }
    if (lane == 0) {
      T[p] = t;
      nres[p] = (int32_t)n;
    }
    return;
  }
  // FIFO contents after the full tiles: the rest of S_p, then the columns the full
  // tiles evicted, in tile order and eviction order (exactly CR1's sequential queue).
  if (warp == 0) {
    for (int i = lane; i < rem; i += 32) q[i] = S[(int64_t)p * K + 16 * nfull + i];
    int64_t tail = rem;
    for (int t = 0; t < nfull; ++t) {
      const int n = sc.tnev[(int64_t)p * sc.cap + t];
      if (lane < n) q[tail + lane] = sc.tev[((int64_t)p * sc.cap + t) * 16 + lane];
      tail += n;
    }
    if (lane == 0) {
      s_head = 0;
      s_tail = tail;
      s_t = nfull;
      s_stop = 0;
    }
  }
  __syncthreads();
  for (;;) {
    if (threadIdx.x == 0) {
      const int64_t avail = s_tail - s_head;
      int nw = avail >= 16 ? (int)(avail / 16) : (avail > 0 ? 1 : 0);
      if (nw > 0 && (s_t + nw > sc.cap || s_tail + 16 * (int64_t)nw > qcap)) {
        atomicExch(err, 1);
        nw = 0;
      }
      s_nw = nw;
    }
    __syncthreads();
    const int nw = s_nw;
    if (nw == 0) break;
    const int64_t head = s_head, tail0 = s_tail;
    const int t0 = s_t;
    for (int k = warp; k < nw; k += kR4Warps) {
      TileSmem& s = sm[warp];
      if (lane < 16) {
        const int64_t pos = head + 16 * (int64_t)k + lane;
        const int32_t c = pos < tail0 ? q[pos] : kPad;
        s.cols[lane] = c;
        s.m[lane] = c == kPad ? zero_mask() : masks[(int64_t)p * K + c];
      }
      __syncwarp();
      tile_search(s, lane);
      store_tile(s, sc, p, t0 + k, lane);
      __syncwarp();
    }
    __syncthreads();
    if (warp == 0) {  // the wave's evictions, in tile order
      int64_t tail = tail0;
      for (int k = 0; k < nw; ++k) {
        const int n = sc.tnev[(int64_t)p * sc.cap + t0 + k];
        if (lane < n) q[tail + lane] = sc.tev[((int64_t)p * sc.cap + t0 + k) * 16 + lane];
        tail += n;
      }
      if (lane == 0) {
        s_head = min(head + 16 * (int64_t)nw, tail0);
        s_tail = tail;
        s_t = t0 + nw;
      }
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    T[p] = s_t;
    nres[p] = 0;
  }
}

// ------------------------------------------------------------------ R5
// One CTA (P threads = rows) per (panel, k-step): compresses the two tiles of
// the k-step (R-Q15, R-Q16) and writes, per 128-row half of the
// panel (P = 256 -> two halves, one per CTA of the pair), into that half's plane
//   A image : 4096 B = [row group 16][tile 2][row 8][8 halves]  (UMMA K-major,
//             no swizzle: LBO = 128 B between the two tiles, SBO = 256 B)
//   E lanes : TMEM metadata layout of tcgen05.mma.sp kind::f16 -- lane
//             L = m0 + 8*h + 16*m2 holds rows r = 16*m2 + m0 and r + 8 of tile half h
//   G rows  : B row per logical column, PAD -> K (TMA zero fill); one list per k-step
__global__ void __launch_bounds__(256) k_emit(const uint16_t* __restrict__ A, int64_t M, int64_t K, int P,
                                              Scratch sc, const int32_t* __restrict__ T,
                                              const int32_t* __restrict__ tile_off,
                                              const int32_t* __restrict__ ksoff,
                                              const int32_t* __restrict__ kboff,
                                              uint8_t* __restrict__ Aimg, int64_t planeA,
                                              uint32_t* __restrict__ Eimg, int64_t planeE,
                                              int32_t* __restrict__ G, int32_t* __restrict__ colidx,
                                              uint8_t* __restrict__ perm, uint8_t* __restrict__ kind,
                                              uint8_t* __restrict__ nevict, const int32_t* __restrict__ Kp) {
  __shared__ int32_t gat[2][16];
  __shared__ uint16_t smeta[2][256];
  const int p = blockIdx.y, ks = blockIdx.x, tid = threadIdx.x;
  const int Tp = T[p];
  const int nks = (Tp + 1) / 2;
  if (ks >= nks) return;
  const int64_t gks = ksoff[p] + ks;
  if (tid < 32) {
    const int h = tid >> 4, j = tid & 15, t = 2 * ks + h;
    int32_t g = kPad;
    if (t < Tp) {
      const int to = sc.tmap ? sc.tmap[(int64_t)p * sc.cap + t] : t;  // canonical tile index
      const int64_t o = ((int64_t)p * sc.cap + to) * 16;
      g = sc.tcols[o + sc.tperm[o + j]];
      const int64_t ft = (int64_t)tile_off[p] + t;
      colidx[ft * 16 + j] = sc.tcols[o + j];
      perm[ft * 16 + j] = sc.tperm[o + j];
      if (j == 0) {
        kind[ft] = to < (Kp[p] + 15) / 16 ? 0 : 1;
        nevict[ft] = sc.tnev[(int64_t)p * sc.cap + to];
      }
    }
    gat[h][j] = g;
    G[gks * 32 + tid] = g == kPad ? (int32_t)K : g;
  }
  __syncthreads();
  const int r = tid, half = r >> 7, rr = r & 127;
  const int64_t row = (int64_t)p * P + r;
  uint8_t* Ah = Aimg + half * planeA + gks * kKStepBytesA;
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    if (r >= P) break;  // P = 16: 32 threads (the gather list), 16 rows
    uint16_t v[8];
    uint16_t meta = 0;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      uint16_t bits[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int32_t c = gat[h][4 * q + i];
        bits[i] = (c == kPad || row >= M) ? (uint16_t)0 : A[row * K + c];
      }
      int keep[2], nk = 0;
#pragma unroll
      for (int i = 0; i < 4; ++i)
        if (nk < 2 && (bits[i] & 0x7FFFu)) keep[nk++] = i;
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        if (nk >= 2) break;
        if (bits[i] & 0x7FFFu) continue;
        if (nk == 1 && keep[0] == i) continue;
        keep[nk++] = i;
      }
      if (keep[0] > keep[1]) { const int x = keep[0]; keep[0] = keep[1]; keep[1] = x; }
#pragma unroll
      for (int k = 0; k < 2; ++k) {
        const uint16_t b = bits[keep[k]];
        v[2 * q + k] = (b & 0x7FFFu) ? b : (uint16_t)0;
      }
      meta |= (uint16_t)((keep[0] + 4 * keep[1]) << (4 * q));
    }
    uint4 pk;
    pk.x = v[0] | ((uint32_t)v[1] << 16);
    pk.y = v[2] | ((uint32_t)v[3] << 16);
    pk.z = v[4] | ((uint32_t)v[5] << 16);
    pk.w = v[6] | ((uint32_t)v[7] << 16);
    *reinterpret_cast<uint4*>(Ah + (rr >> 3) * 256 + h * 128 + (rr & 7) * 16) = pk;
    smeta[h][r] = meta;
  }
  __syncthreads();
  if (tid < P) {
    const int L = tid & 127, m0 = L & 7, h = (L >> 3) & 1, m2 = L >> 4;
    const int r0 = half * 128 + 16 * m2 + m0;
    const uint32_t w = (uint32_t)smeta[h][r0] | ((uint32_t)smeta[h][r0 + 8] << 16);
    Eimg[half * planeE + ((int64_t)(kboff[p] + ks / kStepsPerBlock) * 128 + L) * 4 + (ks % kStepsPerBlock)] = w;
  }
}

// R5 (DENSE mode): one CTA per (panel, dense step): dense step j holds residual
// columns R_p[16j .. 16j+16) as an uncompressed K = 16 A image in the same UMMA
// K-major no-swizzle layout ([row group 16][8-column half 2][row 8][8 halves]);
// its gather list is the 16 columns (PAD -> K) followed by 16 PAD rows.
__global__ void __launch_bounds__(256) k_emit_dense(const uint16_t* __restrict__ A, int64_t M, int64_t K, int P,
                                                    const int32_t* __restrict__ queue, int64_t qcap,
                                                    const int32_t* __restrict__ nres,
                                                    const int4* __restrict__ pin,
                                                    uint8_t* __restrict__ Aimg, int64_t planeA,
                                                    int32_t* __restrict__ G) {
  __shared__ int32_t cols[16];
  const int p = blockIdx.y, j = blockIdx.x, tid = threadIdx.x;
  const int4 pi = pin[p];
  if (j >= (pi.w & ~kPinCC)) return;
  const int64_t gks = (int64_t)pi.y + ((pi.x + kStepsPerBlock - 1) / kStepsPerBlock) * kStepsPerBlock + j;
  const int n = nres[p];
  if (tid < 32) {
    const int i = 16 * j + (tid & 15);
    const int32_t c = (tid < 16 && i < n) ? queue[(int64_t)p * qcap + i] : kPad;
    if (tid < 16) cols[tid] = c;
    G[gks * 32 + tid] = c == kPad ? (int32_t)K : c;
  }
  __syncthreads();
  const int r = tid, rr = r & 127;
  const int64_t row = (int64_t)p * P + r;
  uint8_t* Ah = Aimg + (r >> 7) * planeA + gks * kKStepBytesA;
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    if (r >= P) break;
    uint16_t v[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int32_t c = cols[8 * h + i];
      const uint16_t b = (c == kPad || row >= M) ? (uint16_t)0 : A[row * K + c];
      v[i] = (b & 0x7FFFu) ? b : (uint16_t)0;   // canonical +0 (R-Q3)
    }
    uint4 pk;
    pk.x = v[0] | ((uint32_t)v[1] << 16);
    pk.y = v[2] | ((uint32_t)v[3] << 16);
    pk.z = v[4] | ((uint32_t)v[5] << 16);
    pk.w = v[6] | ((uint32_t)v[7] << 16);
    *reinterpret_cast<uint4*>(Ah + (rr >> 3) * 256 + h * 128 + (rr & 7) * 16) = pk;
  }
}

// ------------------------------------------------------------------ CC (f3)
// CUDA-core tiles (DESIGN.md R-Q28).  CC1: one CTA
// per panel; thread i of a chunk takes tile t = base + i of the canonical list,
// counts its nonzeros (popcounts of its real columns' row masks) and keeps it
// iff the count exceeds Z.  Kept tiles are numbered in list order (tmap: final
// tile -> canonical tile); the real columns of the others are marked in the
// panel's column bitmap ccbm (bit c of word c / 32).  T[p] becomes the kept count.
__global__ void __launch_bounds__(256) k_cc_split(const RowMask* __restrict__ masks, int64_t K, Scratch sc,
                                                  int32_t* __restrict__ T, int32_t* __restrict__ ccT,
                                                  uint32_t* __restrict__ ccbm, int64_t KW, int Z) {
  __shared__ int wsum[8];
  const int p = blockIdx.x, tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int Tp = T[p];
  int kept = 0;
  for (int base = 0; base < Tp; base += 256) {
    const int t = base + tid;
    bool keep = false;
    if (t < Tp) {
      const int64_t o = ((int64_t)p * sc.cap + t) * 16;
      int nnz = 0;
      for (int j = 0; j < 16; ++j) {
        const int32_t c = sc.tcols[o + j];
        if (c == kPad) continue;
        const RowMask m = masks[(int64_t)p * K + c];
        nnz += __popc(m.lo.x) + __popc(m.lo.y) + __popc(m.lo.z) + __popc(m.lo.w) + __popc(m.hi.x) +
               __popc(m.hi.y) + __popc(m.hi.z) + __popc(m.hi.w);
      }
      keep = nnz > Z;
      if (!keep)
        for (int j = 0; j < 16; ++j) {
          const int32_t c = sc.tcols[o + j];
          if (c != kPad) atomicOr(ccbm + (int64_t)p * KW + (c >> 5), 1u << (c & 31));
        }
    }
    const unsigned b = __ballot_sync(kFull, keep);
    if (lane == 0) wsum[warp] = __popc(b);
    __syncthreads();
    int pre = kept;
    for (int w = 0; w < warp; ++w) pre += wsum[w];
    int tot = 0;
    for (int w = 0; w < 8; ++w) tot += wsum[w];
    if (keep) sc.tmap[(int64_t)p * sc.cap + pre + __popc(b & ((1u << lane) - 1u))] = t;
    kept += tot;
    __syncthreads();
  }
  if (tid == 0) {
    T[p] = kept;
    ccT[p] = Tp - kept;
  }
}

// CC2: one thread per panel row: the nonzeros of A in the panel's CUDA-core
// columns (bitmap order = ascending column).  fill == 0: count them into
// cnt[p * P + r]; fill == 1: write them as {column, fp16 bits} from off[p * P + r].
__global__ void k_cc_entries(const uint16_t* __restrict__ A, int64_t M, int64_t K, int P,
                             const uint32_t* __restrict__ ccbm, int64_t KW, int fill,
                             int32_t* __restrict__ cnt, const int32_t* __restrict__ off, int2* __restrict__ ent) {
  const int p = blockIdx.x, r = threadIdx.x;
  if (r >= P) return;
  const int64_t row = (int64_t)p * P + r;
  int n = 0;
  int64_t o = fill ? off[row] : 0;
  if (row < M) {
    const uint32_t* bm = ccbm + (int64_t)p * KW;
    for (int64_t w = 0; w < KW; ++w) {
      uint32_t b = bm[w];
      while (b) {
        const int c = (int)(w * 32) + __ffs(b) - 1;
        b &= b - 1;
        const uint16_t x = A[row * K + c];
        if (x & 0x7FFFu) {
          if (fill) ent[o++] = make_int2(c, x);
          ++n;
        }
      }
    }
  }
  if (!fill) cnt[row] = n;
}

template <class T>
jigsaw_status_t dalloc(T** p, size_t bytes, std::vector<void*>& list) {
  *p = nullptr;
  if (bytes == 0) bytes = 16;
  cudaError_t e = cudaMalloc((void**)p, bytes);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return set_status(JIGSAW_ERROR_OUT_OF_MEMORY, std::string("cudaMalloc failed: ") + cudaGetErrorString(e));
  }
  list.push_back(*p);
  return JIGSAW_SUCCESS;
}

// Scratch of one build: stream-ordered (the library's pool), released with
// cudaFreeAsync on the build's stream -- no implicit device synchronisation, so
// builds on different streams (jigsaw_reorder_batched) overlap.
template <class T>
jigsaw_status_t salloc(T** p, size_t bytes, std::vector<void*>& list, cudaStream_t s) {
  *p = nullptr;
  if (bytes == 0) bytes = 16;
  cudaError_t e = pool_alloc_async((void**)p, bytes, s);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return set_status(JIGSAW_ERROR_OUT_OF_MEMORY, std::string("scratch allocation failed: ") + cudaGetErrorString(e));
  }
  list.push_back(*p);
  return JIGSAW_SUCCESS;
}

}  // namespace

void free_format(Format* f) {
  for (void* p : f->allocs) cudaFree(p);
  f->allocs.clear();
}

#define JIG_TRY(x)                          \
  do {                                      \
    jigsaw_status_t _s = (x);               \
    if (_s != JIGSAW_SUCCESS) goto fail;    \
  } while (0)
#define JIG_CU(x, what)                                   \
  do {                                                    \
    cudaError_t _e = (x);                                 \
    if (_e != cudaSuccess) { cuda_status(_e, what); goto fail; } \
  } while (0)

// ------------------------------------------------------------------ row-clustered panels (f2)
// RC1: nonzero count of every row of A (one CTA per row).
__global__ void __launch_bounds__(256) k_rownnz(const uint16_t* __restrict__ A, int64_t K, int32_t* __restrict__ cnt) {
  const int64_t r = blockIdx.x;
  int c = 0;
  for (int64_t k = threadIdx.x; k < K; k += blockDim.x) c += (A[r * K + k] & 0x7FFF) != 0;
  for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xFFFFFFFFu, c, o);
  __shared__ int part[8];
  if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = c;
  __syncthreads();
  if (threadIdx.x == 0) {
    int t = 0;
    for (int w = 0; w < 8; ++w) t += part[w];
    cnt[r] = t;
  }
}
// RC2: A'[i][:] = A[rowmap[i]][:] (one CTA per row).
__global__ void __launch_bounds__(256) k_permute_rows(const uint16_t* __restrict__ A, int64_t K,
                                                      const int32_t* __restrict__ rowmap, uint16_t* __restrict__ Ap) {
  const int64_t i = blockIdx.x, r = rowmap[i];
  for (int64_t k = threadIdx.x; k < K; k += blockDim.x) Ap[i * K + k] = A[r * K + k];
}

static jigsaw_status_t build_format_rows(const uint16_t* dA, int64_t M, int64_t K, int v, int P, int mode,
                                         int Z, cudaStream_t stream, Format* f);

// Row-clustered panels (DESIGN.md R-Q27): the rows are ordered by
// nonzero count, descending, ties by ascending row index (a stable counting sort
// on the host), the format is built for A[rowmap] exactly as for any matrix, and
// the SpMM epilogue writes panel row r to C row rowmap[r].  Panels of sparse
// rows then have fewer nonzero columns (K_p), hence fewer tiles and fewer B rows
// to gather.  The row order of vector-sparse rows (v identical rows) is kept.
jigsaw_status_t build_format(const uint16_t* dA, int64_t M, int64_t K, int v, int P, int mode, int row_order,
                             int cc_max_nnz, cudaStream_t stream, Format* f) {
  if (row_order != JIGSAW_ROWS_CLUSTERED) return build_format_rows(dA, M, K, v, P, mode, cc_max_nnz, stream, f);
  int32_t *cnt = nullptr, *rmap = nullptr;
  uint16_t* Ap = nullptr;
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  std::vector<int32_t> hc(M), hmap(M);
  jigsaw_status_t st = JIGSAW_SUCCESS;
  float ms = 0;
  auto cleanup = [&]() {
    if (cnt) cudaFreeAsync(cnt, stream);
    if (Ap) cudaFreeAsync(Ap, stream);
    if (e0) cudaEventDestroy(e0);
    if (e1) cudaEventDestroy(e1);
  };
  if (pool_alloc_async((void**)&cnt, sizeof(int32_t) * M, stream) != cudaSuccess ||
      pool_alloc_async((void**)&Ap, sizeof(uint16_t) * M * K, stream) != cudaSuccess ||
      cudaMalloc(&rmap, sizeof(int32_t) * M) != cudaSuccess) {
    cudaGetLastError();
    if (rmap) cudaFree(rmap);
    cleanup();
    return set_status(JIGSAW_ERROR_OUT_OF_MEMORY, "reorder: row clustering buffers");
  }
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0, stream);
  k_rownnz<<<(unsigned)M, 256, 0, stream>>>(dA, K, cnt);
  cudaError_t e = cudaMemcpyAsync(hc.data(), cnt, sizeof(int32_t) * M, cudaMemcpyDeviceToHost, stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(stream);
  if (e != cudaSuccess) {
    cudaFree(rmap);
    cleanup();
    return cuda_status(e, "reorder: row nonzero counts");
  }
  {  // stable counting sort by descending count
    std::vector<int64_t> start(K + 2, 0);
    for (int64_t r = 0; r < M; ++r) ++start[K - hc[r] + 1];
    for (int64_t c = 1; c <= K + 1; ++c) start[c] += start[c - 1];
    for (int64_t r = 0; r < M; ++r) hmap[start[K - hc[r]]++] = (int32_t)r;
  }
  e = cudaMemcpyAsync(rmap, hmap.data(), sizeof(int32_t) * M, cudaMemcpyHostToDevice, stream);
  if (e == cudaSuccess) {
    k_permute_rows<<<(unsigned)M, 256, 0, stream>>>(dA, K, rmap, Ap);
    e = cudaGetLastError();
  }
  if (e == cudaSuccess) e = cudaEventRecord(e1, stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(stream);
  if (e != cudaSuccess) {
    cudaFree(rmap);
    cleanup();
    return cuda_status(e, "reorder: row clustering");
  }
  cudaEventElapsedTime(&ms, e0, e1);
  st = build_format_rows(Ap, M, K, v, P, mode, cc_max_nnz, stream, f);
  cleanup();
  if (st != JIGSAW_SUCCESS) {
    cudaFree(rmap);
    return st;
  }
  f->row_order = JIGSAW_ROWS_CLUSTERED;
  f->d_rowmap = rmap;
  f->allocs.push_back(rmap);
  f->reorder_ms += ms;
  f->device_bytes += sizeof(int32_t) * M;
  return JIGSAW_SUCCESS;
}

static jigsaw_status_t build_format_rows(const uint16_t* dA, int64_t M, int64_t K, int v, int P, int mode,
                                         int Z, cudaStream_t stream, Format* f) {
  std::vector<void*> scratch;
  int dev = 0;
  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  jigsaw_status_t st = JIGSAW_SUCCESS;
  const int npan = (int)((M + P - 1) / P);
  const int cap = (int)(K / 8 + 2);
  const int64_t qcap = 2 * K + 64;
  RowMask* masks = nullptr;
  int32_t *S = nullptr, *Kp = nullptr, *T = nullptr, *queue = nullptr, *tile_off = nullptr;
  int32_t *d_ksoff = nullptr, *d_kboff = nullptr, *nres = nullptr;
  int* err = nullptr;
  unsigned long long* nnz = nullptr;
  Scratch sc{};
  std::vector<int32_t> hKp(npan), hT(npan), hR(npan);
  int maxdk = 0;
  unsigned long long hnnz = 0;
  int herr = 0;
  int maxks = 0;
  // CUDA-core split (f3): column bitmap per panel, per-row entry counts / offsets
  const int64_t KW = (K + 31) / 32;
  uint32_t* ccbm = nullptr;
  int32_t *ccT = nullptr, *cccnt = nullptr, *ccoff = nullptr;
  std::vector<int32_t> hccT(Z > 0 ? npan : 0), hcnt(Z > 0 ? (size_t)npan * P : 0);

  cudaGetDevice(&dev);
  f->M = M; f->K = K; f->v = v; f->P = P; f->mode = mode; f->device = dev;
  f->cc_max_nnz = Z;
  f->npanels = npan;
  if ((st = init_tables(dev)) != JIGSAW_SUCCESS) return st;

  JIG_TRY(salloc(&masks, sizeof(RowMask) * npan * K, scratch, stream));
  JIG_TRY(salloc(&S, sizeof(int32_t) * npan * K, scratch, stream));
  JIG_TRY(salloc(&Kp, sizeof(int32_t) * npan, scratch, stream));
  JIG_TRY(salloc(&T, sizeof(int32_t) * npan, scratch, stream));
  JIG_TRY(salloc(&nres, sizeof(int32_t) * npan, scratch, stream));
  JIG_TRY(salloc(&err, sizeof(int), scratch, stream));
  JIG_TRY(salloc(&nnz, sizeof(unsigned long long), scratch, stream));
  JIG_TRY(salloc(&queue, sizeof(int32_t) * npan * qcap, scratch, stream));
  JIG_TRY(salloc(&sc.tcols, sizeof(int32_t) * npan * cap * 16, scratch, stream));
  JIG_TRY(salloc(&sc.tperm, (size_t)npan * cap * 16, scratch, stream));
  JIG_TRY(salloc(&sc.tev, sizeof(int32_t) * npan * cap * 16, scratch, stream));
  JIG_TRY(salloc(&sc.tnev, (size_t)npan * cap, scratch, stream));
  sc.cap = cap;
  sc.tmap = nullptr;
  if (Z > 0) {
    JIG_TRY(salloc(&sc.tmap, sizeof(int32_t) * npan * cap, scratch, stream));
    JIG_TRY(salloc(&ccbm, sizeof(uint32_t) * npan * KW, scratch, stream));
    JIG_TRY(salloc(&ccT, sizeof(int32_t) * npan, scratch, stream));
    JIG_TRY(salloc(&cccnt, sizeof(int32_t) * npan * P, scratch, stream));
  }

  JIG_CU(cudaEventCreate(&ev0), "cudaEventCreate");
  JIG_CU(cudaEventCreate(&ev1), "cudaEventCreate");
  JIG_CU(cudaEventRecord(ev0, stream), "cudaEventRecord");
  JIG_CU(cudaMemsetAsync(err, 0, sizeof(int), stream), "memset");
  JIG_CU(cudaMemsetAsync(nnz, 0, sizeof(unsigned long long), stream), "memset");
  k_colmask<<<dim3((unsigned)((K + 127) / 128), npan), 128, 0, stream>>>(dA, M, K, P, masks, nnz);
  k_compact<<<npan, 1024, 0, stream>>>(masks, K, S, Kp);
  k_main_tiles<<<dim3((unsigned)((K / 16 + kR3Warps - 1) / kR3Warps), npan), 32 * kR3Warps, 0, stream>>>(
      masks, S, Kp, K, sc);
  {
    static std::atomic<bool> attr_set[64] = {};
    if (dev >= 0 && dev < 64 && !attr_set[dev]) {
      JIG_CU(cudaFuncSetAttribute(k_overflow, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  (int)(kR4Warps * sizeof(TileSmem))), "cudaFuncSetAttribute(k_overflow)");
      attr_set[dev] = true;
    }
  }
  k_overflow<<<npan, 32 * kR4Warps, kR4Warps * sizeof(TileSmem), stream>>>(masks, S, Kp, K, sc, queue, qcap, T, err,
                                                                          mode, nres);
  if (Z > 0) {  // f3: CUDA-core tiles leave the list (CC1), their entries are counted (CC2)
    JIG_CU(cudaMemsetAsync(ccbm, 0, sizeof(uint32_t) * npan * KW, stream), "memset");
    k_cc_split<<<npan, 256, 0, stream>>>(masks, K, sc, T, ccT, ccbm, KW, Z);
    k_cc_entries<<<npan, P < 32 ? 32 : P, 0, stream>>>(dA, M, K, P, ccbm, KW, 0, cccnt, nullptr, nullptr);
    JIG_CU(cudaMemcpyAsync(hccT.data(), ccT, sizeof(int32_t) * npan, cudaMemcpyDeviceToHost, stream), "copy ccT");
    JIG_CU(cudaMemcpyAsync(hcnt.data(), cccnt, sizeof(int32_t) * npan * P, cudaMemcpyDeviceToHost, stream), "copy cc counts");
  }
  JIG_CU(cudaGetLastError(), "reorder kernels launch");
  JIG_CU(cudaMemcpyAsync(hKp.data(), Kp, sizeof(int32_t) * npan, cudaMemcpyDeviceToHost, stream), "copy Kp");
  JIG_CU(cudaMemcpyAsync(hT.data(), T, sizeof(int32_t) * npan, cudaMemcpyDeviceToHost, stream), "copy T");
  JIG_CU(cudaMemcpyAsync(hR.data(), nres, sizeof(int32_t) * npan, cudaMemcpyDeviceToHost, stream), "copy nres");
  JIG_CU(cudaMemcpyAsync(&hnnz, nnz, sizeof hnnz, cudaMemcpyDeviceToHost, stream), "copy nnz");
  JIG_CU(cudaMemcpyAsync(&herr, err, sizeof herr, cudaMemcpyDeviceToHost, stream), "copy err");
  JIG_CU(cudaStreamSynchronize(stream), "reorder R1-R4");
  if (herr) {
    st = set_status(JIGSAW_ERROR_INTERNAL, "reorder: tile or queue capacity exceeded");
    goto fail;
  }
  // offsets (host): tiles, k-steps (ceil(T_p/2)), E blocks (ceil(ksteps/4))
  f->T = hT;
  f->D.assign(npan, 0);
  f->tile_off.assign(npan + 1, 0);
  f->ks_off.assign(npan + 1, 0);
  f->kb_off.assign(npan + 1, 0);
  f->kp_total = 0;
  f->max_tiles = 0;
  f->overflow_tiles = 0;
  for (int p = 0; p < npan; ++p) {
    const int nks = (hT[p] + 1) / 2;
    const int ndk = (hR[p] + 15) / 16;   // dense residual tiles (DENSE mode)
    f->D[p] = ndk;
    maxdk = std::max(maxdk, ndk);
    // k-step slots: sparse k-steps, then (DENSE mode) the dense steps starting on
    // a fresh E block boundary so every k-block is all-sparse or all-dense
    const int span = ndk ? (nks + kStepsPerBlock - 1) / kStepsPerBlock * kStepsPerBlock + ndk : nks;
    f->tile_off[p + 1] = f->tile_off[p] + hT[p];
    f->ks_off[p + 1] = f->ks_off[p] + span;
    f->kb_off[p + 1] = f->kb_off[p] + (nks + kStepsPerBlock - 1) / kStepsPerBlock;
    f->kp_total += hKp[p];
    f->max_tiles = std::max<int64_t>(f->max_tiles, hT[p]);
    maxks = std::max(maxks, nks);
  }
  f->ccT = hccT;
  f->cc_tiles = 0;
  for (int32_t x : hccT) f->cc_tiles += x;
  f->cc_entries = 0;
  if (f->cc_tiles > 0) {  // per-row entry offsets (host prefix sum), then the entries (CC2, fill)
    std::vector<int32_t> hoff((size_t)npan * P + 1);
    int64_t acc = 0;
    for (size_t i = 0; i < hcnt.size(); ++i) {
      hoff[i] = (int32_t)acc;
      acc += hcnt[i];
    }
    if (acc >= ((int64_t)1 << 31)) {
      st = set_status(JIGSAW_ERROR_UNSUPPORTED, "reorder: more than 2^31 CUDA-core entries");
      goto fail;
    }
    hoff.back() = (int32_t)acc;
    f->cc_entries = acc;
    JIG_TRY(dalloc(&f->d_ccoff, sizeof(int32_t) * hoff.size(), f->allocs));
    JIG_TRY(dalloc(&f->d_ccent, sizeof(int2) * acc, f->allocs));
    JIG_CU(cudaMemcpyAsync(f->d_ccoff, hoff.data(), sizeof(int32_t) * hoff.size(), cudaMemcpyHostToDevice, stream),
           "upload cc offsets");
    k_cc_entries<<<npan, P < 32 ? 32 : P, 0, stream>>>(dA, M, K, P, ccbm, KW, 1, nullptr, f->d_ccoff, f->d_ccent);
    JIG_CU(cudaGetLastError(), "k_cc_entries launch");
    // the host copy of the offsets must outlive the async upload
    JIG_CU(cudaStreamSynchronize(stream), "cc offsets");
  }
  f->ntiles = f->tile_off[npan];
  f->ndtiles = 0;
  for (int p = 0; p < npan; ++p) f->ndtiles += f->D[p];
  f->nksteps = f->ks_off[npan];
  f->nkblocks = f->kb_off[npan];
  f->nnz = (int64_t)hnnz;
  f->evictions = f->ntiles * 16 - f->kp_total - 0;  // placeholder, replaced below
  {
    f->pin.resize(npan);
    for (int p = 0; p < npan; ++p) f->pin[p] = make_int4((hT[p] + 1) / 2, f->ks_off[p], f->kb_off[p], f->D[p]);
    JIG_TRY(dalloc(&f->d_pin, sizeof(int4) * npan, f->allocs));
    JIG_TRY(salloc(&d_ksoff, sizeof(int32_t) * (npan + 1), scratch, stream));
    JIG_TRY(salloc(&d_kboff, sizeof(int32_t) * (npan + 1), scratch, stream));
    JIG_TRY(salloc(&tile_off, sizeof(int32_t) * (npan + 1), scratch, stream));
    JIG_TRY(dalloc(&f->d_colidx, sizeof(int32_t) * 16 * f->ntiles, f->allocs));
    JIG_TRY(dalloc(&f->d_perm, (size_t)16 * f->ntiles, f->allocs));
    JIG_TRY(dalloc(&f->d_kind, (size_t)f->ntiles, f->allocs));
    JIG_TRY(dalloc(&f->d_nevict, (size_t)f->ntiles, f->allocs));
    JIG_TRY(dalloc(&f->d_Aimg, (size_t)kKStepBytesA * f->nksteps * f->halves(), f->allocs));
    JIG_TRY(dalloc(&f->d_Eimg, (size_t)kEBlockBytes * f->nkblocks * f->halves(), f->allocs));
    JIG_TRY(dalloc(&f->d_G, sizeof(int32_t) * 32 * f->nksteps, f->allocs));
    std::vector<int4> pin_dev(npan);  // the device form (kPinCC flags); synchronised below before it goes
    for (int p = 0; p < npan; ++p) pin_dev[p] = f->pin_dev(p);
    JIG_CU(cudaMemcpyAsync(f->d_pin, pin_dev.data(), sizeof(int4) * npan, cudaMemcpyHostToDevice, stream), "upload");
    JIG_CU(cudaMemcpyAsync(d_ksoff, f->ks_off.data(), sizeof(int32_t) * (npan + 1), cudaMemcpyHostToDevice, stream), "upload");
    JIG_CU(cudaMemcpyAsync(d_kboff, f->kb_off.data(), sizeof(int32_t) * (npan + 1), cudaMemcpyHostToDevice, stream), "upload");
    JIG_CU(cudaMemcpyAsync(tile_off, f->tile_off.data(), sizeof(int32_t) * (npan + 1), cudaMemcpyHostToDevice, stream), "upload");
    JIG_CU(cudaMemsetAsync(f->d_Eimg, 0, (size_t)kEBlockBytes * f->nkblocks * f->halves(), stream), "memset E");
    if (maxks > 0)
      k_emit<<<dim3(maxks, npan), P < 32 ? 32 : P, 0, stream>>>(dA, M, K, P, sc, T, tile_off, d_ksoff, d_kboff, f->d_Aimg,
                                                f->planeA(), reinterpret_cast<uint32_t*>(f->d_Eimg),
                                                f->planeE() / 4, f->d_G, f->d_colidx, f->d_perm, f->d_kind,
                                                f->d_nevict, Kp);
    if (maxdk > 0)
      k_emit_dense<<<dim3(maxdk, npan), P < 32 ? 32 : P, 0, stream>>>(dA, M, K, P, queue, qcap, nres, f->d_pin, f->d_Aimg,
                                                      f->planeA(), f->d_G);
    JIG_CU(cudaGetLastError(), "k_emit launch");
    JIG_CU(cudaEventRecord(ev1, stream), "cudaEventRecord");
    // total evictions = sum of per-tile counts
    std::vector<uint8_t> hnev(f->ntiles), hkind(f->ntiles);
    if (f->ntiles) {
      JIG_CU(cudaMemcpyAsync(hnev.data(), f->d_nevict, f->ntiles, cudaMemcpyDeviceToHost, stream), "copy nevict");
      JIG_CU(cudaMemcpyAsync(hkind.data(), f->d_kind, f->ntiles, cudaMemcpyDeviceToHost, stream), "copy kind");
    }
    JIG_CU(cudaStreamSynchronize(stream), "reorder R5");
    f->evictions = 0;
    for (uint8_t x : hnev) f->evictions += x;
    f->overflow_tiles = 0;  // overflow tiles of the final list (kind 1)
    for (uint8_t x : hkind) f->overflow_tiles += x;
  }
  {
    float ms = 0;
    cudaEventElapsedTime(&ms, ev0, ev1);
    f->reorder_ms = ms;
  }
  f->device_bytes = 0;
  f->device_bytes += (int64_t)f->nksteps * (kKStepBytesA * f->halves() + 128) +
                     (int64_t)f->nkblocks * kEBlockBytes * f->halves() +
                     (int64_t)f->ntiles * (16 * 4 + 16 + 2) + (int64_t)npan * 12;
  if (f->cc_tiles > 0) f->device_bytes += ((int64_t)npan * P + 1) * 4 + f->cc_entries * 8;
  for (void* p : scratch) cudaFreeAsync(p, stream);
  cudaEventDestroy(ev0);
  cudaEventDestroy(ev1);
  return JIGSAW_SUCCESS;
fail:
  for (void* p : scratch) cudaFreeAsync(p, stream);
  if (ev0) cudaEventDestroy(ev0);
  if (ev1) cudaEventDestroy(ev1);
  free_format(f);
  {
    jigsaw_status_t s = jigsaw_last_status();
    return s == JIGSAW_SUCCESS ? set_status(JIGSAW_ERROR_INTERNAL, "reorder failed") : s;
  }
}

}  // namespace jig
