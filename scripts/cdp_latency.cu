// Device-side launch latency on B200: a 1-thread parent stamps %globaltimer
// and launches a child grid (fire-and-forget or tail launch); the child's
// first CTA stamps its start.  Also a host launch for reference.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -rdc=true -o cdp_latency scripts/cdp_latency.cu -lcudadevrt
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint64_t gt() { uint64_t t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }
__global__ void child(unsigned long long *t) {
  if (threadIdx.x == 0) atomicMin(&t[1], (unsigned long long)gt());
}
__global__ void parent(unsigned long long *t, int mode, unsigned grid) {
  t[0] = gt();
  if (mode == 0) child<<<grid, 256, 0, cudaStreamFireAndForget>>>(t);
  else child<<<grid, 256, 0, cudaStreamTailLaunch>>>(t);
}
int main() {
  unsigned long long *d, h[2];
  cudaMalloc(&d, 16);
  for (int mode = 0; mode < 2; ++mode)
    for (unsigned grid : {1u, 148u, 888u}) {
      double s = 0; int n = 0;
      for (int r = 0; r < 12; ++r) {
        unsigned long long init[2] = {0, ~0ull};
        cudaMemcpy(d, init, 16, cudaMemcpyHostToDevice);
        parent<<<1, 1>>>(d, mode, grid);
        cudaDeviceSynchronize();
        cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
        if (r >= 2) { s += (double)(h[1] - h[0]); ++n; }
      }
      printf("%s grid %4u: child start - parent stamp = %.2f us (%s)\n", mode ? "tail  " : "f&f   ", grid, s / n / 1e3,
             cudaGetErrorString(cudaGetLastError()));
    }
  return 0;
}
