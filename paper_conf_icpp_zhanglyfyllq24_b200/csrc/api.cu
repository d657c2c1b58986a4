// api.cu -- the C ABI of libjigsaw.so (include/jigsaw.h): validation, handle
// lifetime, status reporting, export of the canonical format, launches.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstring>
#include <atomic>
#include <mutex>
#include <new>
#include <string>
#include <thread>
#include <vector>

#include "internal.h"

struct jigsaw_handle_s {
  jig::Format f;
};

namespace jig {

namespace {
thread_local jigsaw_status_t t_status = JIGSAW_SUCCESS;
thread_local std::string t_msg;
}  // namespace

jigsaw_status_t set_status(jigsaw_status_t s, const std::string& msg) {
  t_status = s;
  t_msg = msg;
  return s;
}

jigsaw_status_t cuda_status(cudaError_t e, const char* what) {
  cudaGetLastError();  // clear sticky-free errors
  return set_status(JIGSAW_ERROR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

namespace {

jigsaw_status_t check_device(int* dev_out) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return set_status(JIGSAW_ERROR_UNSUPPORTED, std::string("no CUDA device: ") + cudaGetErrorString(e));
  }
  int major = 0, minor = 0;
  cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
  cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev);
  if (major != 10 || minor != 0)
    return set_status(JIGSAW_ERROR_UNSUPPORTED, "libjigsaw is built for sm_100a (B200); device " +
                                                    std::to_string(dev) + " is sm_" + std::to_string(major) +
                                                    std::to_string(minor));
  *dev_out = dev;
  return JIGSAW_SUCCESS;
}

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

// Stream-ordered device memory of the library (host-buffer staging, launch
// workspaces): a private pool per device.  Memory up to the pool's release
// threshold stays reserved across synchronisations; anything above it goes back
// to the OS at the next synchronisation.  The threshold starts at 256 MB and
// rises to the largest host-buffer call's staging + 256 MB (high watermark,
// capped at 1/4 of the device's memory): with a fixed 256 MB a C4 batch
// (381 MB of staging) re-mapped ~125 MB every call, 7.8 vs 5.9 ms per call
// (profiles/r02au_e2e_calls.jsonl).
cudaMemPool_t g_pool[64] = {};
uint64_t g_pool_keep[64] = {};  // current release threshold, guarded by g_lazy_mu
std::mutex g_lazy_mu;           // guards the lazy creation of the pools and their thresholds
#ifndef JIG_POOL_KEEP_MB
#define JIG_POOL_KEEP_MB 256
#endif
constexpr uint64_t kPoolKeepBytes = (uint64_t)JIG_POOL_KEEP_MB << 20;

// Pool of device `dev`, created on first use; call with g_lazy_mu held.
static cudaError_t pool_locked(int dev, cudaMemPool_t* out) {
  if (!g_pool[dev]) {
    cudaMemPoolProps props = {};
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    cudaError_t e = cudaMemPoolCreate(&g_pool[dev], &props);
    if (e != cudaSuccess) return e;
    uint64_t thr = kPoolKeepBytes;
    cudaMemPoolSetAttribute(g_pool[dev], cudaMemPoolAttrReleaseThreshold, &thr);
    g_pool_keep[dev] = thr;
  }
  *out = g_pool[dev];
  return cudaSuccess;
}

cudaError_t staging_alloc(void** p, size_t bytes, cudaStream_t st) {
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 64) return cudaMallocAsync(p, bytes, st);
  cudaMemPool_t pool;
  {
    std::lock_guard<std::mutex> lock(g_lazy_mu);
    cudaError_t e = pool_locked(dev, &pool);
    if (e != cudaSuccess) return e;
  }
  return cudaMallocFromPoolAsync(p, bytes, pool, st);
}

// A host-buffer call about to stage `bytes`: raise the current device's release
// threshold so the staging stays reserved for the next call (see above).
static void staging_reserve(size_t bytes) {
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 64) return;
  static uint64_t total[64] = {};
  std::lock_guard<std::mutex> lock(g_lazy_mu);
  cudaMemPool_t pool;
  if (pool_locked(dev, &pool) != cudaSuccess) {
    cudaGetLastError();
    return;
  }
  if (!total[dev]) {
    size_t fr = 0, tot = 0;
    if (cudaMemGetInfo(&fr, &tot) != cudaSuccess) {
      cudaGetLastError();
      return;
    }
    total[dev] = tot;
  }
  const uint64_t want = std::min<uint64_t>((uint64_t)bytes + kPoolKeepBytes, total[dev] / 4);
  if (want > g_pool_keep[dev]) {
    uint64_t thr = want;
    if (cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr) == cudaSuccess)
      g_pool_keep[dev] = thr;
    else
      cudaGetLastError();
  }
}

// Helper streams of the host-buffer batch pipeline: a free list per device; a
// call takes a triple for its own use and returns it when done, so concurrent
// calls never share (or wait on) each other's helper streams.
struct HostPipe {
  cudaStream_t h2d = nullptr, comp = nullptr, d2h = nullptr;
};
std::vector<HostPipe> g_pipes_free[64];
bool take_pipe(int dev, HostPipe* out) {
  {
    std::lock_guard<std::mutex> lock(g_lazy_mu);
    if (!g_pipes_free[dev].empty()) {
      *out = g_pipes_free[dev].back();
      g_pipes_free[dev].pop_back();
      return true;
    }
  }
  HostPipe P;
  if (cudaStreamCreateWithFlags(&P.h2d, cudaStreamNonBlocking) != cudaSuccess ||
      cudaStreamCreateWithFlags(&P.comp, cudaStreamNonBlocking) != cudaSuccess ||
      cudaStreamCreateWithFlags(&P.d2h, cudaStreamNonBlocking) != cudaSuccess) {
    cudaGetLastError();
    if (P.h2d) cudaStreamDestroy(P.h2d);
    if (P.comp) cudaStreamDestroy(P.comp);
    return false;
  }
  *out = P;
  return true;
}
void give_pipe(int dev, const HostPipe& P) {
  std::lock_guard<std::mutex> lock(g_lazy_mu);
  g_pipes_free[dev].push_back(P);
}

size_t c_elem_bytes(const Format& f) { return f.c_dtype == JIGSAW_C_F32 ? 4 : 2; }

// panel_rows = 0 (auto): CTA pairs (256-row panels) for tall matrices, where the
// halved B traffic per output pays (4096 x 4096 N = 2048, +30 %);
// 128-row panels otherwise (more, shorter units for the small DLMC shapes).
constexpr int64_t kAutoPairMinRows = 4096;
int resolve_panel_rows(const jigsaw_options_t* opt, int64_t M) {
  if (!opt) return kPanelRows;
  if (opt->panel_rows == 0) return M >= kAutoPairMinRows ? kPairPanelRows : kPanelRows;
  return opt->panel_rows;
}

jigsaw_status_t validate_reorder(const void* A, int64_t M, int64_t K, int v, const jigsaw_options_t* opt) {
  if (!A) return set_status(JIGSAW_ERROR_INVALID_VALUE, "A is NULL");
  if (M <= 0 || K <= 0) return set_status(JIGSAW_ERROR_INVALID_VALUE, "M and K must be positive");
  if (K > (int64_t)1 << 30 || M > (int64_t)1 << 31)
    return set_status(JIGSAW_ERROR_INVALID_VALUE, "M or K too large");
  if (!(v == 1 || v == 2 || v == 4 || v == 8)) return set_status(JIGSAW_ERROR_INVALID_VALUE, "v must be 1, 2, 4 or 8");
  if (M % v) return set_status(JIGSAW_ERROR_INVALID_VALUE, "M must be a multiple of v");
  if (opt) {
    const int pr = opt->panel_rows;
    if (!(pr == 0 || pr == JIGSAW_PANEL_AUTOTUNE || pr == 16 || pr == 32 || pr == 64 || pr == kPanelRows ||
          pr == kPairPanelRows))
      return set_status(JIGSAW_ERROR_INVALID_VALUE, "panel_rows must be 0 (auto), -1 (autotune), 16, 32, 64, 128 or 256");
    if (opt->autotune_n < 0 || opt->autotune_n % 8 || (opt->autotune_n && pr != JIGSAW_PANEL_AUTOTUNE))
      return set_status(JIGSAW_ERROR_INVALID_VALUE, "autotune_n must be 0, or a multiple of 8 with panel_rows = -1");
    if (opt->residual_mode != JIGSAW_RESIDUAL_SPTC && opt->residual_mode != JIGSAW_RESIDUAL_DENSE)
      return set_status(JIGSAW_ERROR_INVALID_VALUE, "unknown residual_mode");
    if (opt->c_dtype != JIGSAW_C_F16 && opt->c_dtype != JIGSAW_C_F32)
      return set_status(JIGSAW_ERROR_INVALID_VALUE, "unknown c_dtype");
    if (opt->row_order != JIGSAW_ROWS_GIVEN && opt->row_order != JIGSAW_ROWS_CLUSTERED)
      return set_status(JIGSAW_ERROR_INVALID_VALUE, "unknown row_order");
    if (opt->cc_max_nnz < 0 || opt->cc_max_nnz >= (1 << 24))
      return set_status(JIGSAW_ERROR_INVALID_VALUE, "cc_max_nnz must be in [0, 2^24)");
    for (int i = 0; i < 2; ++i)
      if (opt->reserved[i]) return set_status(JIGSAW_ERROR_INVALID_VALUE, "reserved options must be zero");
  }
  return JIGSAW_SUCCESS;
}

jigsaw_status_t validate_spmm(jigsaw_handle_t h, const void* B, int64_t N, const void* C, bool device_ptrs) {
  if (!h) return set_status(JIGSAW_ERROR_INVALID_VALUE, "handle is NULL");
  if (!B || !C) return set_status(JIGSAW_ERROR_INVALID_VALUE, "B or C is NULL");
  if (N <= 0 || N % 8) return set_status(JIGSAW_ERROR_INVALID_VALUE, "N must be a positive multiple of 8");
  if (N > (int64_t)1 << 30) return set_status(JIGSAW_ERROR_INVALID_VALUE, "N too large");
  if (device_ptrs && (!aligned16(B) || !aligned16(C)))
    return set_status(JIGSAW_ERROR_INVALID_VALUE, "B and C must be 16-byte aligned");
  int dev = -1;
  cudaGetDevice(&dev);
  if (dev != h->f.device) return set_status(JIGSAW_ERROR_WRONG_DEVICE, "current device differs from the handle's");
  if (h->f.P < kPanelRows)
    return set_status(JIGSAW_ERROR_UNSUPPORTED,
                      "formats with panel_rows < 128 are for analysis (export / statistics); the SpMM needs "
                      "128 or 256 (tcgen05 M)");
  return JIGSAW_SUCCESS;
}

// Per-shape panel-height autotune: both formats are built,
// one jigsaw_spmm of each is timed on the device (zero B of autotune_n columns,
// best of 3 after a warm-up, CUDA events on the reorder's stream), the faster
// is kept.  Ties (within 2 %) go to 128-row panels (split-K for small products).
jigsaw_status_t autotune_panels(const uint16_t* dA, int64_t M, int64_t K, int v, int mode, int row_order, int n,
                                int cc, cudaStream_t st, Format* out) {
  Format f[2];
  const int P[2] = {kPanelRows, kPairPanelRows};
  for (int i = 0; i < 2; ++i) {
    jigsaw_status_t s = build_format(dA, M, K, v, P[i], mode, row_order, cc, st, &f[i]);
    if (s != JIGSAW_SUCCESS) {
      if (i) free_format(&f[0]);
      return s;
    }
  }
  const int64_t N = n > 0 ? n : 256;
  void *dB = nullptr, *dC = nullptr;
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  float best[2] = {1e30f, 1e30f};
  cudaError_t e = cudaMalloc(&dB, (size_t)K * N * 2);
  if (e == cudaSuccess) e = cudaMalloc(&dC, (size_t)M * N * 4);
  if (e == cudaSuccess) e = cudaMemsetAsync(dB, 0, (size_t)K * N * 2, st);
  if (e == cudaSuccess) e = cudaEventCreate(&e0);
  if (e == cudaSuccess) e = cudaEventCreate(&e1);
  jigsaw_status_t s = e == cudaSuccess ? JIGSAW_SUCCESS : cuda_status(e, "autotune buffers");
  for (int i = 0; i < 2 && s == JIGSAW_SUCCESS; ++i)
    for (int rep = 0; rep < 4 && s == JIGSAW_SUCCESS; ++rep) {
      cudaEventRecord(e0, st);
      s = launch_spmm(f[i], dB, N, dC, st);
      cudaEventRecord(e1, st);
      if (s == JIGSAW_SUCCESS && (e = cudaEventSynchronize(e1)) != cudaSuccess) s = cuda_status(e, "autotune timing");
      float ms = 0;
      if (s == JIGSAW_SUCCESS && rep > 0 && cudaEventElapsedTime(&ms, e0, e1) == cudaSuccess)
        best[i] = std::min(best[i], ms);
    }
  if (e0) cudaEventDestroy(e0);
  if (e1) cudaEventDestroy(e1);
  if (dB) cudaFree(dB);
  if (dC) cudaFree(dC);
  if (s != JIGSAW_SUCCESS) {
    free_format(&f[0]);
    free_format(&f[1]);
    return s;
  }
  const int keep = best[1] < 0.98f * best[0] ? 1 : 0;
  free_format(&f[1 - keep]);
  *out = std::move(f[keep]);
  out->reorder_ms = f[0].reorder_ms + f[1].reorder_ms + 4 * (best[0] + best[1]);
  return JIGSAW_SUCCESS;
}

}  // namespace

cudaError_t pool_alloc_async(void** p, size_t bytes, cudaStream_t s) { return staging_alloc(p, bytes, s); }

}  // namespace jig

using namespace jig;

extern "C" {

jigsaw_status_t jigsaw_last_status(void) { return t_status; }
const char* jigsaw_last_error_string(void) { return t_msg.c_str(); }
const char* jigsaw_version(void) { return "jigsaw-b200 0.1 (sm_100a, tcgen05.mma.sp)"; }

jigsaw_status_t jigsaw_reorder_ex(const void* A, int64_t M, int64_t K, int v, const jigsaw_options_t* opt,
                                  jigsaw_stream_t stream, jigsaw_handle_t* out) {
  if (!out) return set_status(JIGSAW_ERROR_INVALID_VALUE, "out is NULL");
  *out = nullptr;
  jigsaw_status_t s = validate_reorder(A, M, K, v, opt);
  if (s != JIGSAW_SUCCESS) return s;
  if (!aligned16(A)) return set_status(JIGSAW_ERROR_INVALID_VALUE, "A must be 16-byte aligned");
  int dev = 0;
  if ((s = check_device(&dev)) != JIGSAW_SUCCESS) return s;
  jigsaw_handle_s* h = new (std::nothrow) jigsaw_handle_s();
  if (!h) return set_status(JIGSAW_ERROR_OUT_OF_MEMORY, "host allocation failed");
  set_status(JIGSAW_SUCCESS);
  const int mode = opt ? opt->residual_mode : (int)JIGSAW_RESIDUAL_SPTC;
  const int rows = opt ? opt->row_order : (int)JIGSAW_ROWS_GIVEN;
  const int cc = opt ? opt->cc_max_nnz : 0;
  if (opt && opt->panel_rows == JIGSAW_PANEL_AUTOTUNE)
    s = autotune_panels(static_cast<const uint16_t*>(A), M, K, v, mode, rows, opt->autotune_n, cc,
                        reinterpret_cast<cudaStream_t>(stream), &h->f);
  else
    s = build_format(static_cast<const uint16_t*>(A), M, K, v, resolve_panel_rows(opt, M), mode, rows, cc,
                     reinterpret_cast<cudaStream_t>(stream), &h->f);
  if (s != JIGSAW_SUCCESS) {
    delete h;
    return s;
  }
  h->f.c_dtype = opt ? opt->c_dtype : (int)JIGSAW_C_F16;
  *out = h;
  return set_status(JIGSAW_SUCCESS);
}

jigsaw_status_t jigsaw_reorder_batched(const void* const* As, const int64_t* Ms, const int64_t* Ks, const int* vs,
                                       int count, const jigsaw_options_t* opt, jigsaw_stream_t stream,
                                       jigsaw_handle_t* out) {
  if (count < 0 || (count > 0 && (!As || !Ms || !Ks || !vs || !out)))
    return set_status(JIGSAW_ERROR_INVALID_VALUE, "bad batch arguments");
  for (int i = 0; i < count; ++i) out[i] = nullptr;
  for (int i = 0; i < count; ++i) {
    jigsaw_status_t s = validate_reorder(As[i], Ms[i], Ks[i], vs[i], opt);
    if (s != JIGSAW_SUCCESS) return s;
    if (!aligned16(As[i])) return set_status(JIGSAW_ERROR_INVALID_VALUE, "A must be 16-byte aligned");
  }
  if (count == 0) return set_status(JIGSAW_SUCCESS);
  int dev = 0;
  jigsaw_status_t s = check_device(&dev);
  if (s != JIGSAW_SUCCESS) return s;
  // ordered after prior work on the caller's stream
  cudaEvent_t ev = nullptr;
  if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventRecord(ev, reinterpret_cast<cudaStream_t>(stream)) != cudaSuccess) {
    cudaError_t e = cudaGetLastError();
    if (ev) cudaEventDestroy(ev);
    return cuda_status(e, "jigsaw_reorder_batched: event");
  }
  int nthreads = std::min(count, 8);
#if defined(JIG_DEV) && JIG_DEV
  if (getenv("JIGSAW_REORDER_THREADS")) nthreads = std::max(1, std::min(count, atoi(getenv("JIGSAW_REORDER_THREADS"))));
#endif
  std::atomic<int> next{0};
  std::vector<jigsaw_status_t> st(count, JIGSAW_SUCCESS);
  std::vector<std::string> msg(count);
  auto worker = [&]() {
    cudaSetDevice(dev);
    cudaStream_t ws = nullptr;
    if (cudaStreamCreateWithFlags(&ws, cudaStreamNonBlocking) != cudaSuccess) {
      cudaGetLastError();
      ws = nullptr;
    } else {
      cudaStreamWaitEvent(ws, ev, 0);
    }
    for (int i; (i = next.fetch_add(1)) < count;) {
      if (!ws) {
        st[i] = JIGSAW_ERROR_CUDA;
        msg[i] = "cudaStreamCreate failed";
        continue;
      }
      st[i] = jigsaw_reorder_ex(As[i], Ms[i], Ks[i], vs[i], opt, reinterpret_cast<jigsaw_stream_t>(ws), &out[i]);
      if (st[i] != JIGSAW_SUCCESS) msg[i] = jigsaw_last_error_string();
    }
    if (ws) cudaStreamDestroy(ws);
  };
  std::vector<std::thread> pool;
  for (int t = 0; t + 1 < nthreads; ++t) pool.emplace_back(worker);
  worker();
  for (auto& t : pool) t.join();
  cudaEventDestroy(ev);
  for (int i = 0; i < count; ++i)
    if (st[i] != JIGSAW_SUCCESS) {
      for (int j = 0; j < count; ++j) {
        jigsaw_free(out[j]);
        out[j] = nullptr;
      }
      return set_status(st[i], "matrix " + std::to_string(i) + ": " + msg[i]);
    }
  return set_status(JIGSAW_SUCCESS);
}

jigsaw_handle_t jigsaw_reorder(const void* A, int64_t M, int64_t K, int v) {
  jigsaw_handle_t h = nullptr;
  jigsaw_reorder_ex(A, M, K, v, nullptr, nullptr, &h);
  return h;
}

jigsaw_status_t jigsaw_reorder_host(const void* A_host, int64_t M, int64_t K, int v, const jigsaw_options_t* opt,
                                    jigsaw_stream_t stream, jigsaw_handle_t* out) {
  if (!out) return set_status(JIGSAW_ERROR_INVALID_VALUE, "out is NULL");
  *out = nullptr;
  jigsaw_status_t s = validate_reorder(A_host, M, K, v, opt);
  if (s != JIGSAW_SUCCESS) return s;
  int dev = 0;
  if ((s = check_device(&dev)) != JIGSAW_SUCCESS) return s;
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  void* dA = nullptr;
  const size_t bytes = (size_t)M * K * 2;
  staging_reserve(bytes);
  cudaError_t e = staging_alloc(&dA, bytes, st);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return set_status(JIGSAW_ERROR_OUT_OF_MEMORY, "cudaMallocAsync(A) failed");
  }
  e = cudaMemcpyAsync(dA, A_host, bytes, cudaMemcpyHostToDevice, st);
  if (e != cudaSuccess) {
    cudaFreeAsync(dA, st);
    return cuda_status(e, "copy A to device");
  }
  s = jigsaw_reorder_ex(dA, M, K, v, opt, stream, out);
  cudaFreeAsync(dA, st);
  cudaStreamSynchronize(st);
  return s;
}

jigsaw_status_t jigsaw_spmm(jigsaw_handle_t h, const void* B, int64_t N, void* C, jigsaw_stream_t stream) {
  jigsaw_status_t s = validate_spmm(h, B, N, C, true);
  if (s != JIGSAW_SUCCESS) return s;
  s = launch_spmm(h->f, B, N, C, reinterpret_cast<cudaStream_t>(stream));
  if (s != JIGSAW_SUCCESS) return s;
  return set_status(JIGSAW_SUCCESS);
}

jigsaw_status_t jigsaw_spmm_host(jigsaw_handle_t h, const void* B_host, int64_t N, void* C_host,
                                 jigsaw_stream_t stream) {
  jigsaw_status_t s = validate_spmm(h, B_host, N, C_host, false);
  if (s != JIGSAW_SUCCESS) return s;
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  const size_t bbytes = (size_t)h->f.K * N * 2, cbytes = (size_t)h->f.M * N * c_elem_bytes(h->f);
  void *dB = nullptr, *dC = nullptr;
  staging_reserve(bbytes + cbytes + 512);
  cudaError_t e = staging_alloc(&dB, bbytes, st);
  if (e == cudaSuccess) e = staging_alloc(&dC, cbytes, st);
  if (e != cudaSuccess) {
    cudaGetLastError();
    if (dB) cudaFreeAsync(dB, st);
    return set_status(JIGSAW_ERROR_OUT_OF_MEMORY, "cudaMallocAsync(B/C) failed");
  }
  e = cudaMemcpyAsync(dB, B_host, bbytes, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess) {
    s = launch_spmm(h->f, dB, N, dC, st);
    if (s == JIGSAW_SUCCESS) e = cudaMemcpyAsync(C_host, dC, cbytes, cudaMemcpyDeviceToHost, st);
  }
  cudaFreeAsync(dB, st);
  cudaFreeAsync(dC, st);
  cudaError_t e2 = cudaStreamSynchronize(st);
  if (s != JIGSAW_SUCCESS) return s;
  if (e != cudaSuccess) return cuda_status(e, "jigsaw_spmm_host copies");
  if (e2 != cudaSuccess) return cuda_status(e2, "jigsaw_spmm_host");
  return set_status(JIGSAW_SUCCESS);
}

jigsaw_status_t jigsaw_spmm_batched(const jigsaw_handle_t* hs, const void* const* Bs, const int64_t* Ns,
                                    void* const* Cs, int count, jigsaw_stream_t stream) {
  if (count < 0 || (count > 0 && (!hs || !Bs || !Ns || !Cs)))
    return set_status(JIGSAW_ERROR_INVALID_VALUE, "bad batch arguments");
  for (int i = 0; i < count; ++i) {
    jigsaw_status_t s = validate_spmm(hs[i], Bs[i], Ns[i], Cs[i], true);
    if (s != JIGSAW_SUCCESS) return s;
  }
  if (count == 0) return set_status(JIGSAW_SUCCESS);
  std::vector<const Format*> fs(count);
  for (int i = 0; i < count; ++i) fs[i] = &hs[i]->f;
  jigsaw_status_t s = launch_spmm_grouped(fs.data(), Bs, Ns, Cs, count, reinterpret_cast<cudaStream_t>(stream));
  if (s != JIGSAW_SUCCESS) return s;
  return set_status(JIGSAW_SUCCESS);
}

// Start of the CUDA allocation (pinned host or device) that holds p, or 0 for
// memory CUDA does not know (pageable host memory).  Driver entry point looked
// up once through the runtime (no link-time dependency on libcuda).
static uintptr_t alloc_start(const void* p) {
  using Fn = int (*)(void*, int, unsigned long long);
  static Fn fn = []() -> Fn {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuPointerGetAttribute", &f, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess) {
      cudaGetLastError();
      return nullptr;
    }
    return reinterpret_cast<Fn>(f);
  }();
  if (!fn) return 0;
  unsigned long long start = 0;
  constexpr int kRangeStartAddr = 11;  // CU_POINTER_ATTRIBUTE_RANGE_START_ADDR
  return fn(&start, kRangeStartAddr, (unsigned long long)reinterpret_cast<uintptr_t>(p)) == 0 ? (uintptr_t)start : 0;
}

// True when host buffer b starts right where a (of `bytes`) ends, inside the
// same CUDA allocation: the two copies can be one (two adjacent buffers of
// separate pinned registrations cannot -- such a copy is rejected).
static bool host_contiguous(const void* a, size_t bytes, const void* b) {
  if (reinterpret_cast<const char*>(a) + bytes != reinterpret_cast<const char*>(b)) return false;
  const uintptr_t s = alloc_start(a);
  return s != 0 && s == alloc_start(b);
}

// Independent copies on one stream, one cudaMemcpyAsync per run of copies whose
// host AND device sides are both contiguous (runs[] marks where a new copy
// starts).  (The one-submission batch-copy call is not used: it faulted the GPU
// on this pool's boxes.)
static cudaError_t copy_batch(std::vector<void*>& dst, std::vector<void*>& src, std::vector<size_t>& sz,
                              const std::vector<char>& joins, cudaMemcpyKind kind, cudaStream_t st) {
  cudaError_t e = cudaSuccess;
  for (size_t i = 0; i < dst.size() && e == cudaSuccess;) {
    size_t j = i + 1, bytes = sz[i];
    while (j < dst.size() && joins[j]) bytes += sz[j++];
    e = cudaMemcpyAsync(dst[i], src[i], bytes, kind, st);
    i = j;
  }
  return e;
}

static jigsaw_status_t spmm_batched_host_on(const HostPipe& P, const jigsaw_handle_t* hs, const void* const* Bs_host,
                                            const int64_t* Ns, void* const* Cs_host, int count,
                                            jigsaw_stream_t stream);

jigsaw_status_t jigsaw_spmm_batched_host(const jigsaw_handle_t* hs, const void* const* Bs_host, const int64_t* Ns,
                                         void* const* Cs_host, int count, jigsaw_stream_t stream) {
  if (count < 0 || (count > 0 && (!hs || !Bs_host || !Ns || !Cs_host)))
    return set_status(JIGSAW_ERROR_INVALID_VALUE, "bad batch arguments");
  for (int i = 0; i < count; ++i) {
    jigsaw_status_t s = validate_spmm(hs[i], Bs_host[i], Ns[i], Cs_host[i], false);
    if (s != JIGSAW_SUCCESS) return s;
    if (i > 0 && hs[i]->f.device != hs[0]->f.device)
      return set_status(JIGSAW_ERROR_INVALID_VALUE, "handles of a batch must live on one device");
  }
  if (count == 0) return set_status(JIGSAW_SUCCESS);
  const int dev = hs[0]->f.device;
  if (dev < 0 || dev >= 64) return set_status(JIGSAW_ERROR_INTERNAL, "device ordinal out of range");
  HostPipe P;
  if (!take_pipe(dev, &P)) return set_status(JIGSAW_ERROR_CUDA, "cudaStreamCreate failed");
  jigsaw_status_t rs = spmm_batched_host_on(P, hs, Bs_host, Ns, Cs_host, count, stream);
  give_pipe(dev, P);
  return rs;
}

static jigsaw_status_t spmm_batched_host_on(const HostPipe& P, const jigsaw_handle_t* hs, const void* const* Bs_host,
                                            const int64_t* Ns, void* const* Cs_host, int count,
                                            jigsaw_stream_t stream) {
  cudaStream_t user = reinterpret_cast<cudaStream_t>(stream);
  // staging for the whole batch (one pool allocation each for B and C)
  // Staging offsets: products whose host buffers are contiguous in one pinned
  // allocation (a caller that packs its batch) get contiguous staging too (16-byte
  // aligned: K*N*2 and M*N*esize are multiples of 16), so their copies merge
  // into one per chunk and direction; otherwise 256-byte aligned slots.
  size_t bb = 0, cb = 0;
  std::vector<size_t> boff(count), coff(count);
  std::vector<char> bjoin(count, 0), cjoin(count, 0);
  for (int i = 0; i < count; ++i) {
    const size_t bsz = (size_t)hs[i]->f.K * Ns[i] * 2, csz = (size_t)hs[i]->f.M * Ns[i] * c_elem_bytes(hs[i]->f);
    if (i > 0) {
      const size_t pb = (size_t)hs[i - 1]->f.K * Ns[i - 1] * 2, pc = (size_t)hs[i - 1]->f.M * Ns[i - 1] * c_elem_bytes(hs[i - 1]->f);
      bjoin[i] = host_contiguous(Bs_host[i - 1], pb, Bs_host[i]);
      cjoin[i] = host_contiguous(Cs_host[i - 1], pc, Cs_host[i]);
    }
    if (!bjoin[i]) bb = (bb + 255) & ~size_t(255);
    if (!cjoin[i]) cb = (cb + 255) & ~size_t(255);
    boff[i] = bb;
    coff[i] = cb;
    bb += bsz;
    cb += csz;
  }
  cudaEvent_t ev0;
  if (cudaEventCreateWithFlags(&ev0, cudaEventDisableTiming) != cudaSuccess) return cuda_status(cudaGetLastError(), "event");
  cudaEventRecord(ev0, user);  // ordered after prior work on the caller's stream
  cudaStreamWaitEvent(P.h2d, ev0, 0);
  char *dB = nullptr, *dC = nullptr;
  staging_reserve(bb + cb + 512);
  cudaError_t e = staging_alloc(reinterpret_cast<void**>(&dB), bb, P.h2d);
  if (e == cudaSuccess) e = staging_alloc(reinterpret_cast<void**>(&dC), cb, P.h2d);
  if (e != cudaSuccess) {
    cudaGetLastError();
    if (dB) cudaFreeAsync(dB, P.h2d);
    cudaStreamSynchronize(P.h2d);
    cudaEventDestroy(ev0);
    return set_status(JIGSAW_ERROR_OUT_OF_MEMORY, "staging allocation failed");
  }
  // chunks of ~1/16 of the batch's bytes (at least one product; diagnostic
  // override jigsaw_set_launch_override host_chunks): copy-in of chunk k+1 and copy-out of chunk
  // k-1 overlap the grouped launch of chunk k (16 measured best with one copy
  // per product and direction, profiles/r01zt_e2e_chunks.txt)
  // chunk count: ~6 MB chunks, 2..16 (per-copy costs ~6 us on this link: C2's
  // 47 MB run best in 8 chunks, C4's 382 MB in 16; profiles/r02_e2e_floor*.jsonl)
  const int nchunks = launch_override().host_chunks > 0
                          ? launch_override().host_chunks
                          : (int)std::min<size_t>(16, std::max<size_t>(2, ((bb + cb) + (3u << 20)) / (6u << 20)));
  const size_t target = std::max<size_t>((bb + cb) / nchunks, 1);
  std::vector<const Format*> fs;
  std::vector<const void*> pb;
  std::vector<int64_t> pn;
  std::vector<void*> pc;
  jigsaw_status_t st = JIGSAW_SUCCESS;
  std::vector<cudaEvent_t> evs;
  // Chunks are runs of consecutive products (so packed host buffers still merge
  // into one copy per chunk and direction), taken alternately from the front and
  // the back of the batch: a batch ordered from B-heavy to C-heavy products (the
  // C2 batch: 512 x 2048 products, then 2048 x 512) otherwise keeps one copy
  // direction idle for half of the call -- with the ends interleaved both
  // directions of the link stay busy (C2: 0.92 -> see DESIGN.md §8).
  std::vector<std::pair<int, int>> runs;
  for (int i0 = 0; i0 < count;) {
    int i1 = i0;
    size_t acc = 0;
    while (i1 < count && (i1 == i0 || acc < target)) {
      acc += (size_t)hs[i1]->f.K * Ns[i1] * 2 + (size_t)hs[i1]->f.M * Ns[i1] * c_elem_bytes(hs[i1]->f);
      ++i1;
    }
    runs.push_back({i0, i1});
    i0 = i1;
  }
  std::vector<std::pair<int, int>> order;
  for (size_t lo = 0, hi = runs.size(); lo < hi;) {
    order.push_back(runs[lo++]);
    if (lo < hi) order.push_back(runs[--hi]);
  }
  for (size_t r = 0; r < order.size() && st == JIGSAW_SUCCESS; ++r) {
    const int i0 = order[r].first, i1 = order[r].second;
    std::vector<void*> cd, cs;
    std::vector<size_t> cz;
    std::vector<char> jn;
    for (int i = i0; i < i1; ++i) {
      cd.push_back(dB + boff[i]);
      cs.push_back(const_cast<void*>(Bs_host[i]));
      cz.push_back((size_t)hs[i]->f.K * Ns[i] * 2);
      jn.push_back(i > i0 && bjoin[i]);
    }
    if (e == cudaSuccess) e = copy_batch(cd, cs, cz, jn, cudaMemcpyHostToDevice, P.h2d);
    cudaEvent_t in, done;
    cudaEventCreateWithFlags(&in, cudaEventDisableTiming);
    cudaEventCreateWithFlags(&done, cudaEventDisableTiming);
    evs.push_back(in);
    evs.push_back(done);
    cudaEventRecord(in, P.h2d);
    cudaStreamWaitEvent(P.comp, in, 0);
    fs.clear(); pb.clear(); pn.clear(); pc.clear();
    for (int i = i0; i < i1; ++i) {
      fs.push_back(&hs[i]->f);
      pb.push_back(dB + boff[i]);
      pn.push_back(Ns[i]);
      pc.push_back(dC + coff[i]);
    }
    if (e == cudaSuccess) st = launch_spmm_grouped(fs.data(), pb.data(), pn.data(), pc.data(), i1 - i0, P.comp);
    cudaEventRecord(done, P.comp);
    cudaStreamWaitEvent(P.d2h, done, 0);
    cd.clear(); cs.clear(); cz.clear(); jn.clear();
    for (int i = i0; i < i1; ++i) {
      cd.push_back(Cs_host[i]);
      cs.push_back(dC + coff[i]);
      cz.push_back((size_t)hs[i]->f.M * Ns[i] * c_elem_bytes(hs[i]->f));
      jn.push_back(i > i0 && cjoin[i]);
    }
    if (e == cudaSuccess && st == JIGSAW_SUCCESS) e = copy_batch(cd, cs, cz, jn, cudaMemcpyDeviceToHost, P.d2h);
  }
  // staging goes back to the pool after the last copy-out
  cudaEvent_t fin;
  cudaEventCreateWithFlags(&fin, cudaEventDisableTiming);
  cudaEventRecord(fin, P.d2h);
  cudaStreamWaitEvent(P.h2d, fin, 0);
  cudaFreeAsync(dB, P.h2d);
  cudaFreeAsync(dC, P.h2d);
  cudaEventRecord(fin, P.h2d);
  cudaStreamWaitEvent(user, fin, 0);
  cudaError_t e2 = cudaStreamSynchronize(P.h2d);
  cudaError_t e3 = cudaStreamSynchronize(P.comp);
  cudaError_t e4 = cudaStreamSynchronize(P.d2h);
  for (cudaEvent_t x : evs) cudaEventDestroy(x);
  cudaEventDestroy(ev0);
  cudaEventDestroy(fin);
  if (st != JIGSAW_SUCCESS) return st;
  if (e != cudaSuccess) return cuda_status(e, "jigsaw_spmm_batched_host copies");
  if (e2 != cudaSuccess || e3 != cudaSuccess || e4 != cudaSuccess)
    return cuda_status(e2 != cudaSuccess ? e2 : e3 != cudaSuccess ? e3 : e4, "jigsaw_spmm_batched_host");
  return set_status(JIGSAW_SUCCESS);
}

int jigsaw_spmm_launches_per_call(jigsaw_handle_t h, int64_t N) {
  (void)h;
  (void)N;
  return 1;  // jigsaw_spmm: one k_spmm launch; jigsaw_spmm_batched: one per 64 products
}

jigsaw_status_t jigsaw_last_launch(jigsaw_launch_desc_t* out) {
  if (!out) return set_status(JIGSAW_ERROR_INVALID_VALUE, "NULL argument");
  *out = last_launch();
  return set_status(JIGSAW_SUCCESS);
}

jigsaw_status_t jigsaw_set_launch_override(const jigsaw_launch_override_t* o) {
  LaunchOverride v;
  if (o) {
    for (int i = 0; i < 3; ++i)
      if (o->reserved[i]) return set_status(JIGSAW_ERROR_INVALID_VALUE, "reserved fields must be zero");
    if (!(o->tile_n == 0 || o->tile_n == 32 || o->tile_n == 64 || o->tile_n == 128 || o->tile_n == 256))
      return set_status(JIGSAW_ERROR_INVALID_VALUE, "tile_n must be 0, 32, 64, 128 or 256");
    if (!(o->split_k == 0 || o->split_k == 1 || o->split_k == 2 || o->split_k == 4 || o->split_k == 8))
      return set_status(JIGSAW_ERROR_INVALID_VALUE, "split_k must be 0, 1, 2, 4 or 8");
    if (o->host_chunks < 0) return set_status(JIGSAW_ERROR_INVALID_VALUE, "host_chunks must be >= 0");
    v.tile_n = o->tile_n;
    v.split_k = o->split_k;
    v.no_pieces = o->no_pieces ? 1 : 0;
    v.host_chunks = o->host_chunks;
    v.k_pieces = o->k_pieces ? 1 : 0;
  }
  launch_override() = v;
  return set_status(JIGSAW_SUCCESS);
}

int jigsaw_debug_trace(int64_t* out, int max_ctas) {
  if (!out || max_ctas == 0) return 0;
  return debug_trace_read(reinterpret_cast<long long*>(out), max_ctas);
}

void jigsaw_free(jigsaw_handle_t h) {
  if (!h) return;
  int cur = 0;
  cudaGetDevice(&cur);
  if (cur != h->f.device) cudaSetDevice(h->f.device);
  cudaDeviceSynchronize();
  free_format(&h->f);
  if (cur != h->f.device) cudaSetDevice(cur);
  delete h;
  set_status(JIGSAW_SUCCESS);
}

jigsaw_status_t jigsaw_get_info(jigsaw_handle_t h, jigsaw_info_t* out) {
  if (!h || !out) return set_status(JIGSAW_ERROR_INVALID_VALUE, "NULL argument");
  const Format& f = h->f;
  memset(out, 0, sizeof *out);
  out->M = f.M;
  out->K = f.K;
  out->v = f.v;
  out->panel_rows = f.P;
  out->residual_mode = f.mode;
  out->device = f.device;
  out->c_dtype = f.c_dtype;
  out->row_order = f.row_order;
  out->npanels = f.npanels;
  out->ntiles = f.ntiles;
  out->ndtiles = f.ndtiles;
  out->overflow_tiles = f.overflow_tiles;
  out->evictions = f.evictions;
  out->nnz = f.nnz;
  out->kp_total = f.kp_total;
  out->max_tiles = f.max_tiles;
  out->nksteps = f.nksteps;
  out->format_bytes = (int64_t)(16 * f.P + 2 * f.P + 64) * f.ntiles + (int64_t)(32 * f.P + 64) * f.ndtiles;
  out->device_bytes = f.device_bytes;
  out->reorder_ms = f.reorder_ms;
  out->cc_max_nnz = f.cc_max_nnz;
  out->cc_tiles = f.cc_tiles;
  out->cc_entries = f.cc_entries;
  return set_status(JIGSAW_SUCCESS);
}

jigsaw_status_t jigsaw_export_format(jigsaw_handle_t h, jigsaw_format_host_t* out) {
  if (!h || !out) return set_status(JIGSAW_ERROR_INVALID_VALUE, "NULL argument");
  const Format& f = h->f;
  int cur = -1;
  cudaGetDevice(&cur);
  if (cur != f.device) return set_status(JIGSAW_ERROR_WRONG_DEVICE, "current device differs from the handle's");
  const int64_t nt = f.ntiles, P = f.P;
  if (out->T)
    for (int64_t p = 0; p < f.npanels; ++p) out->T[p] = f.T[p];
  if (out->D)
    for (int64_t p = 0; p < f.npanels; ++p) out->D[p] = f.D.empty() ? 0 : f.D[p];
  cudaError_t e = cudaSuccess;
  if (out->rowmap) {
    if (f.d_rowmap)
      e = cudaMemcpy(out->rowmap, f.d_rowmap, sizeof(int32_t) * f.M, cudaMemcpyDeviceToHost);
    else
      for (int64_t r = 0; r < f.M; ++r) out->rowmap[r] = (int32_t)r;
  }
  if (nt && out->col_idx && e == cudaSuccess) e = cudaMemcpy(out->col_idx, f.d_colidx, nt * 16 * 4, cudaMemcpyDeviceToHost);
  if (nt && out->perm && e == cudaSuccess) e = cudaMemcpy(out->perm, f.d_perm, nt * 16, cudaMemcpyDeviceToHost);
  if (nt && out->kind && e == cudaSuccess) e = cudaMemcpy(out->kind, f.d_kind, nt, cudaMemcpyDeviceToHost);
  if (nt && out->nevict && e == cudaSuccess) e = cudaMemcpy(out->nevict, f.d_nevict, nt, cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return cuda_status(e, "export copy");
  if (out->cc_T)
    for (int64_t p = 0; p < f.npanels; ++p) out->cc_T[p] = f.ccT.empty() ? 0 : f.ccT[p];
  if (out->cc_eoff || out->cc_row || out->cc_col || out->cc_val) {
    // CUDA-core entries (f3): per-row offsets over the padded panel rows -> per panel
    std::vector<int32_t> off;
    std::vector<int2> ent((size_t)f.cc_entries);
    if (f.d_ccoff) {
      off.resize((size_t)f.npanels * P + 1);
      e = cudaMemcpy(off.data(), f.d_ccoff, off.size() * 4, cudaMemcpyDeviceToHost);
      if (e == cudaSuccess && !ent.empty()) e = cudaMemcpy(ent.data(), f.d_ccent, ent.size() * 8, cudaMemcpyDeviceToHost);
      if (e != cudaSuccess) return cuda_status(e, "export copy (CUDA-core entries)");
    }
    for (int64_t p = 0; p <= f.npanels; ++p)
      if (out->cc_eoff) out->cc_eoff[p] = off.empty() ? 0 : off[p * P];
    for (int64_t i = 0; !off.empty() && i < f.npanels * P; ++i)
      for (int32_t k = off[i]; k < off[i + 1]; ++k) {
        if (out->cc_row) out->cc_row[k] = (int32_t)(i % P);
        if (out->cc_col) out->cc_col[k] = ent[k].x;
        if (out->cc_val) out->cc_val[k] = (uint16_t)ent[k].y;
      }
  }
  if ((nt && (out->gather || out->vals || out->meta)) || (f.ndtiles && (out->rcol || out->dvals))) {
    // read back the device layout and invert it
    std::vector<uint8_t> A((size_t)f.planeA() * f.halves());
    std::vector<uint32_t> E((size_t)f.planeE() / 4 * f.halves());
    std::vector<int32_t> G((size_t)f.nksteps * 32);
    e = cudaMemcpy(A.data(), f.d_Aimg, A.size(), cudaMemcpyDeviceToHost);
    if (e == cudaSuccess) e = cudaMemcpy(E.data(), f.d_Eimg, E.size() * 4, cudaMemcpyDeviceToHost);
    if (e == cudaSuccess) e = cudaMemcpy(G.data(), f.d_G, G.size() * 4, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) return cuda_status(e, "export copy (device layout)");
    int64_t dt = 0;
    for (int64_t p = 0; p < f.npanels; ++p) {
      // DENSE mode residual tiles: columns from the gather list, values from the A image
      const int64_t dks0 = f.ks_off[p] + (f.T[p] / 2 + (f.T[p] & 1) + kStepsPerBlock - 1) / kStepsPerBlock * kStepsPerBlock;
      for (int j = 0; j < f.D[p]; ++j, ++dt) {
        const int64_t gks = dks0 + j;
        for (int c = 0; c < 16; ++c) {
          const int32_t g = G[gks * 32 + c];
          if (out->rcol) out->rcol[dt * 16 + c] = g >= f.K ? kPad : g;
        }
        if (out->dvals)
          for (int r = 0; r < P; ++r)
            for (int h2 = 0; h2 < 2; ++h2)
              memcpy(out->dvals + (dt * P + r) * 16 + 8 * h2,
                     &A[(r >> 7) * f.planeA() + gks * kKStepBytesA + ((r & 127) >> 3) * 256 + h2 * 128 +
                        (r & 7) * 16],
                     16);
      }
      for (int t = 0; t < f.T[p]; ++t) {
        const int64_t ft = f.tile_off[p] + t;
        const int64_t gks = f.ks_off[p] + t / 2;
        const int h2 = t & 1;
        const int64_t kb = f.kb_off[p] + (t / 2) / kStepsPerBlock;
        const int col = (t / 2) % kStepsPerBlock;
        if (out->gather)
          for (int j = 0; j < 16; ++j) {
            const int32_t g = G[gks * 32 + h2 * 16 + j];
            out->gather[ft * 16 + j] = g >= f.K ? kPad : g;
          }
        for (int r = 0; r < P; ++r) {
          const int half = r >> 7, rr = r & 127;
          if (out->vals)
            memcpy(out->vals + (ft * P + r) * 8,
                   &A[half * f.planeA() + gks * kKStepBytesA + (rr >> 3) * 256 + h2 * 128 + (rr & 7) * 16], 16);
          if (out->meta) {
            const int m2 = rr >> 4, m0 = rr & 7, hi = (rr >> 3) & 1;
            const int L = m0 + 8 * h2 + 16 * m2;
            const uint32_t w = E[half * (f.planeE() / 4) + (kb * 128 + L) * 4 + col];
            out->meta[ft * P + r] = (uint16_t)(hi ? (w >> 16) : (w & 0xFFFF));
          }
        }
      }
    }
  }
  return set_status(JIGSAW_SUCCESS);
}

}  // extern "C"
