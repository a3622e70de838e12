// Minimal mbarrier patterns of sgemm_tma_kernel (thread 0 initialises, fence,
// __syncthreads, waiters in other warps) to tell the synccheck "Missing init"
// report on that kernel apart from a real bug.  Arrivals:
//   mode 0: mbarrier.arrive by 128 threads
//   mode 1: tcgen05.commit (the MMA issuer's stage release)
//   mode 2: cp.async.bulk global->shared with complete_tx (TMA-style)
//   nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/mbar scripts/mbar_synccheck.cu
//   compute-sanitizer --tool synccheck /tmp/mbar <mode>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void wait_parity(uint64_t *b, uint32_t ph) {
  asm volatile("{\n\t.reg .pred p;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n\t}"
               ::"r"(su32(b)), "r"(ph) : "memory");
}
__global__ void k(int mode, const float *src, int *out) {
  __shared__ __align__(8) uint64_t bar;
  __shared__ __align__(128) float buf[256];
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&bar)), "r"(mode == 0 ? 128 : 1));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (mode == 0) {
    if (threadIdx.x >= 64)
      asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.shared::cta.b64 st, [%0];\n\t}" ::"r"(su32(&bar)) : "memory");
  } else if (mode == 1) {
    if (threadIdx.x == 32)
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar))
                   : "memory");
  } else if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar)), "r"(1024) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(su32(buf)), "l"(src), "r"(1024), "r"(su32(&bar)) : "memory");
  }
  if (threadIdx.x == 32 || threadIdx.x == 64) {
    wait_parity(&bar, 0);
    if (threadIdx.x == 64) out[blockIdx.x] = mode == 2 ? (int)buf[5] : 1;
  }
}
int main(int argc, char **argv) {
  const int mode = argc > 1 ? atoi(argv[1]) : 0;
  int *d;
  float *src;
  cudaMalloc(&d, 8 * sizeof(int));
  cudaMalloc(&src, 1024);
  float h0[256];
  for (int i = 0; i < 256; ++i) h0[i] = (float)i;
  cudaMemcpy(src, h0, 1024, cudaMemcpyHostToDevice);
  k<<<2, 192>>>(mode, src, d);
  cudaError_t e = cudaDeviceSynchronize();
  int h[2] = {0, 0};
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  printf("mbar pattern mode %d: %s out %d %d\n", mode, cudaGetErrorString(e), h[0], h[1]);
  return 0;
}
