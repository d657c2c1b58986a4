// launch_latency_probe.cu -- developer microbenchmark: the bench's step timing
// (CUDA graph [event, kernel, event], replayed after a 256 MB L2-flush memset)
// around a trivial 148-CTA kernel, varying one launch property at a time:
// parameter-block size, threads per CTA, dynamic shared memory, cluster and
// programmatic-dependent-launch attributes.  Prints the median event time.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/llp tools/launch_latency_probe.cu
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdio>
#include <vector>

template <int BYTES>
struct P {
  int v[BYTES / 4];
};
template <int BYTES>
__global__ void k(const __grid_constant__ P<BYTES> p, int* out) {
  extern __shared__ int sm[];
  if (threadIdx.x == 0) out[blockIdx.x] = p.v[blockIdx.x % (BYTES / 4)] + (int)(size_t)sm;
}

template <int BYTES>
float run(int* d, void* flush, size_t fbytes, int threads, int smem, bool cluster, bool pdl, cudaStream_t s) {
  P<BYTES> p{};
  for (int i = 0; i < BYTES / 4; ++i) p.v[i] = i;
  cudaFuncSetAttribute(k<BYTES>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaEvent_t a, b;
  cudaEventCreateWithFlags(&a, cudaEventDefault);
  cudaEventCreateWithFlags(&b, cudaEventDefault);
  cudaGraph_t g;
  cudaGraphExec_t ge;
  cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal);
  cudaEventRecordWithFlags(a, s, cudaEventRecordExternal);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(148);
  cfg.blockDim = dim3(threads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[2];
  int na = 0;
  if (cluster) {
    at[na].id = cudaLaunchAttributeClusterDimension;
    at[na].val.clusterDim.x = 2;
    at[na].val.clusterDim.y = 1;
    at[na].val.clusterDim.z = 1;
    ++na;
  }
  if (pdl) {
    at[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[na].val.programmaticStreamSerializationAllowed = 1;
    ++na;
  }
  cfg.attrs = at;
  cfg.numAttrs = na;
  cudaLaunchKernelEx(&cfg, k<BYTES>, p, d);
  cudaEventRecordWithFlags(b, s, cudaEventRecordExternal);
  cudaStreamEndCapture(s, &g);
  if (cudaGraphInstantiate(&ge, g, 0) != cudaSuccess) return -1;
  std::vector<float> t;
  for (int r = 0; r < 30; ++r) {
    cudaMemsetAsync(flush, r & 0xFF, fbytes, s);
    cudaGraphLaunch(ge, s);
    cudaStreamSynchronize(s);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    t.push_back(ms * 1e3f);
  }
  std::sort(t.begin(), t.end());
  cudaGraphExecDestroy(ge);
  cudaGraphDestroy(g);
  return t[t.size() / 2];
}

int main() {
  int* d;
  void* flush;
  const size_t fb = 256u << 20;
  cudaMalloc(&d, 4096);
  cudaMalloc(&flush, fb);
  cudaStream_t s;
  cudaStreamCreate(&s);
  printf("base (256 B params, 128 thr, 0 smem)   %.2f us\n", run<256>(d, flush, fb, 128, 0, false, false, s));
  printf("31 KB params                           %.2f us\n", run<31744>(d, flush, fb, 128, 0, false, false, s));
  printf("7 KB params                            %.2f us\n", run<7424>(d, flush, fb, 128, 0, false, false, s));
  printf("512 threads                            %.2f us\n", run<256>(d, flush, fb, 512, 0, false, false, s));
  printf("227 KB dynamic smem                    %.2f us\n", run<256>(d, flush, fb, 128, 232448, false, false, s));
  printf("cluster 2                              %.2f us\n", run<256>(d, flush, fb, 128, 0, true, false, s));
  printf("PDL attribute                          %.2f us\n", run<256>(d, flush, fb, 128, 0, false, true, s));
  printf("all (31 KB, 512 thr, 227 KB, PDL)      %.2f us\n", run<31744>(d, flush, fb, 512, 232448, false, true, s));
  printf("all + cluster 2                        %.2f us\n", run<31744>(d, flush, fb, 512, 232448, true, true, s));
  return 0;
}
