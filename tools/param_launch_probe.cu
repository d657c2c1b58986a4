// param_launch_probe.cu -- developer microbenchmark: device time per launch of a
// trivial 148-CTA kernel as a function of its kernel-parameter block size (CUDA
// graph of 50 launches), i.e. what a 31 KB grouped-launch parameter block costs.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/plp tools/param_launch_probe.cu
#include <cuda_runtime.h>
#include <cstdio>

template <int BYTES>
struct P {
  int v[BYTES / 4];
};
template <int BYTES>
__global__ void k(const __grid_constant__ P<BYTES> p, int* out) {
  if (threadIdx.x == 0) out[blockIdx.x] = p.v[blockIdx.x % (BYTES / 4)];
}

template <int BYTES>
void run(int* d, cudaStream_t s) {
  P<BYTES> p{};
  for (int i = 0; i < BYTES / 4; ++i) p.v[i] = i;
  cudaGraph_t g;
  cudaGraphExec_t ge;
  cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal);
  for (int i = 0; i < 50; ++i) k<BYTES><<<148, 512, 0, s>>>(p, d);
  cudaStreamEndCapture(s, &g);
  cudaGraphInstantiate(&ge, g, 0);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float best = 1e9;
  for (int r = 0; r < 10; ++r) {
    cudaEventRecord(a, s);
    cudaGraphLaunch(ge, s);
    cudaEventRecord(b, s);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    best = ms < best ? ms : best;
  }
  printf("param block %6d B: %.2f us per launch\n", BYTES, best * 1e3 / 50);
}

int main() {
  int* d;
  cudaMalloc(&d, 4096);
  cudaStream_t s;
  cudaStreamCreate(&s);
  run<256>(d, s);
  run<2048>(d, s);
  run<8192>(d, s);
  run<16384>(d, s);
  run<31744>(d, s);
  return 0;
}
