// tools/gridid_probe.cu -- developer probe: is %gridid unique per launch (eager
// launches, CUDA-graph replays, concurrent streams)?  Prints the values seen.
#include <cuda_runtime.h>
#include <cstdio>
__global__ void k(unsigned long long* out, int slot) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    unsigned long long g;
    asm volatile("mov.u64 %0, %%gridid;" : "=l"(g));
    out[slot] = g;
  }
}
int main() {
  unsigned long long* d;
  cudaMalloc(&d, 64 * 8);
  cudaStream_t s0, s1;
  cudaStreamCreate(&s0);
  cudaStreamCreate(&s1);
  for (int i = 0; i < 6; ++i) k<<<4, 32, 0, s0>>>(d, i);
  cudaGraph_t g;
  cudaGraphExec_t ge;
  cudaStreamBeginCapture(s0, cudaStreamCaptureModeGlobal);
  k<<<4, 32, 0, s0>>>(d, 6);
  k<<<4, 32, 0, s0>>>(d, 7);
  cudaStreamEndCapture(s0, &g);
  cudaGraphInstantiate(&ge, g, 0);
  unsigned long long h[64];
  for (int r = 0; r < 4; ++r) {
    cudaGraphLaunch(ge, r % 2 ? s1 : s0);
    cudaDeviceSynchronize();
    cudaMemcpy(h, d, 64 * 8, cudaMemcpyDeviceToHost);
    printf("replay %d: graph kernels gridid %llu %llu\n", r, h[6], h[7]);
  }
  for (int i = 8; i < 12; ++i) k<<<4, 32, 0, i % 2 ? s1 : s0>>>(d, i);
  cudaDeviceSynchronize();
  cudaMemcpy(h, d, 64 * 8, cudaMemcpyDeviceToHost);
  for (int i = 0; i < 12; ++i) printf("slot %d gridid %llu\n", i, h[i]);
  return 0;
}
