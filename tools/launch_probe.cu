// tools/launch_probe.cu -- developer probe (not product): the fixed cost of one
// kernel launch on B200 as a function of its launch configuration, measured the
// way bench.py measures a single product (L2 flush, then event / kernel / event),
// both eagerly and as a one-node CUDA graph.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -std=c++17 -o launch_probe tools/launch_probe.cu
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <vector>

#include "../paper_conf_icpp_zhanglyfyllq24_b200/csrc/ptx.cuh"

using namespace jig;

struct Big {
  int x[512];  // 2 KB of kernel parameters
};

__global__ void k_empty(int* out) {
  if (threadIdx.x == 1023 && out) out[0] = 1;
}
__global__ void k_smem(int* out) {
  extern __shared__ uint8_t sm[];
  if (threadIdx.x == 0) sm[0] = 1;
  __syncthreads();
  if (threadIdx.x == 5000 && out) out[0] = sm[0];
}
__global__ void k_big(Big b, int* out) {
  if (threadIdx.x == 5000 && out) out[0] = b.x[threadIdx.x & 511];
}
__global__ void k_tmem(int* out) {
  __shared__ uint32_t slot;
  __shared__ uint64_t bar;
  extern __shared__ uint8_t sm[];
  if (threadIdx.x == 0) {
    mbar_init(&bar, 1);
    fence_barrier_init();
  }
  if (threadIdx.x < 32) tmem_alloc<512>(&slot);
  __syncthreads();
  tc_fence_after();
  const uint32_t t = slot;
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x < 32) tmem_dealloc<512>(t);
  if (threadIdx.x == 5000 && out) out[0] = sm[0];
}
// every CTA writes 64 KB of output (a C tile) and exits
__global__ void k_store(int4* out) {
  const int4 v = make_int4(threadIdx.x, 1, 2, 3);
  int4* p = out + (size_t)blockIdx.x * 4096;
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) p[i] = v;
}

#define CK(x)                                                                    \
  do {                                                                           \
    cudaError_t e = (x);                                                         \
    if (e != cudaSuccess) {                                                      \
      printf("CUDA error %s at line %d\n", cudaGetErrorString(e), __LINE__);    \
      return 1;                                                                  \
    }                                                                            \
  } while (0)

template <class F>
float measure(const char* name, F launch, void* flush, size_t fbytes, cudaStream_t s, bool graph) {
  cudaGraphExec_t ge = nullptr;
  if (graph) {
    cudaGraph_t g;
    cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal);
    launch();
    cudaStreamEndCapture(s, &g);
    cudaGraphInstantiate(&ge, g, 0);
    cudaGraphDestroy(g);
  }
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  std::vector<float> ts;
  for (int r = 0; r < 25; ++r) {
    cudaMemsetAsync(flush, r, fbytes, s);
    cudaEventRecord(e0, s);
    if (graph)
      cudaGraphLaunch(ge, s);
    else
      launch();
    cudaEventRecord(e1, s);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (r >= 5) ts.push_back(ms * 1e3f);
  }
  std::sort(ts.begin(), ts.end());
  const cudaError_t err = cudaGetLastError();
  printf("%-58s %s  median %6.2f us  min %6.2f us  %s\n", name, graph ? "graph" : "eager", ts[ts.size() / 2], ts[0],
         err == cudaSuccess ? "" : cudaGetErrorString(err));
  if (ge) cudaGraphExecDestroy(ge);
  return ts[ts.size() / 2];
}

int main() {
  const size_t fbytes = 256u << 20;
  void* flush;
  int* out;
  int4* cbuf;
  CK(cudaMalloc(&flush, fbytes));
  CK(cudaMalloc(&out, 64));
  CK(cudaMalloc(&cbuf, 148u * 65536));
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  const int smem = 200 * 1024;
  CK(cudaFuncSetAttribute(k_smem, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  CK(cudaFuncSetAttribute(k_tmem, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  Big big{};
  for (int graph = 0; graph < 2; ++graph) {
    measure("nothing (event, event)", [&] {}, flush, fbytes, s, graph);
    measure("empty kernel 64 CTAs x 128", [&] { k_empty<<<64, 128, 0, s>>>(nullptr); }, flush, fbytes, s, graph);
    measure("empty kernel 64 CTAs x 448", [&] { k_empty<<<64, 448, 0, s>>>(nullptr); }, flush, fbytes, s, graph);
    measure("2 KB params, 64 x 448", [&] { k_big<<<64, 448, 0, s>>>(big, nullptr); }, flush, fbytes, s, graph);
    measure("200 KB dyn smem, 64 x 448", [&] { k_smem<<<64, 448, smem, s>>>(nullptr); }, flush, fbytes, s, graph);
    measure("200 KB dyn smem, 148 x 448", [&] { k_smem<<<148, 448, smem, s>>>(nullptr); }, flush, fbytes, s, graph);
    measure("200 KB smem + TMEM alloc/dealloc 512, 64 x 448",
            [&] { k_tmem<<<64, 448, smem, s>>>(nullptr); }, flush, fbytes, s, graph);
    for (int cs : {2, 4}) {
      char name[96];
      snprintf(name, sizeof name, "200 KB smem, cluster %d, 64 x 448", cs);
      measure(name, [&] {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(64);
        cfg.blockDim = dim3(448);
        cfg.dynamicSmemBytes = smem;
        cfg.stream = s;
        cudaLaunchAttribute a[1];
        a[0].id = cudaLaunchAttributeClusterDimension;
        a[0].val.clusterDim.x = cs;
        a[0].val.clusterDim.y = 1;
        a[0].val.clusterDim.z = 1;
        cfg.attrs = a;
        cfg.numAttrs = 1;
        cudaLaunchKernelEx(&cfg, k_smem, (int*)nullptr);
      }, flush, fbytes, s, graph);
    }
    measure("64 CTAs store 64 KB each (C write), x 256", [&] { k_store<<<64, 256, 0, s>>>(cbuf); }, flush, fbytes, s,
            graph);
  }
  return 0;
}
