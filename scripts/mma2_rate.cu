// Issue rate of tcgen05.mma.cta_group::2.kind::tf32 (M = 256 over a CTA pair)
// with A from TMEM (ts) or shared memory (ss), N = 64 / 128 / 256.  One pair
// per TPC; the leader issues NI MMAs, commits (multicast), waits; cycles/MMA.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mma2_rate scripts/mma2_rate.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc_k_sw128(uint32_t a) {
  uint64_t d = 0;
  d |= (uint64_t)((a >> 4) & 0x3fff); d |= (uint64_t)1 << 16; d |= (uint64_t)(1024 >> 4) << 32;
  d |= (uint64_t)1 << 46; d |= (uint64_t)2 << 61; return d;
}
__device__ __forceinline__ uint64_t desc_mn_sw128_32b(uint32_t a) {
  uint64_t d = 0;
  d |= (uint64_t)((a >> 4) & 0x3fff); d |= (uint64_t)(4096 >> 4) << 16; d |= (uint64_t)(512 >> 4) << 32;
  d |= (uint64_t)1 << 46; d |= (uint64_t)1 << 61; return d;
}
template <int N, int TS>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128, 1) k(unsigned long long *out, int NI) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ __align__(8) uint64_t bar;
  __shared__ uint32_t tb;
  uint32_t rank; asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
  const uint32_t base = (su32(sm) + 1023u) & ~1023u;
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(su32(&tb)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = tb;
  if (rank == 0 && threadIdx.x == 0) {
    const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | (1u << 16) | ((uint32_t)(N >> 3) << 17) |
                           ((uint32_t)(256 >> 4) << 24);
    const uint64_t da = desc_k_sw128(base), db = desc_mn_sw128_32b(base + 16384);
    const uint32_t ta = tmem + 256, z = 0;
    unsigned long long t0 = clock64();
    for (int i = 0; i < NI; ++i) {
      const uint32_t acc = i > 0;
      if (TS)
        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                     "tcgen05.mma.cta_group::2.kind::tf32 [%0], [%1], %2, %3, {%5,%5,%5,%5,%5,%5,%5,%5}, p;\n\t}" ::"r"(tmem),
                     "r"(ta), "l"(db), "r"(idesc), "r"(acc), "r"(z) : "memory");
      else
        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                     "tcgen05.mma.cta_group::2.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem), "l"(da), "l"(db),
                     "r"(idesc), "r"(acc) : "memory");
    }
    asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(su32(&bar)), "h"((uint16_t)3) : "memory");
    asm volatile("{\n\t.reg .pred p;\n\tW:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n\t@!p bra W;\n\t}" ::"r"(su32(&bar)) : "memory");
    out[blockIdx.x / 2] = clock64() - t0;
  }
  if (rank == 1 && threadIdx.x == 0)
    asm volatile("{\n\t.reg .pred p;\n\tW:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n\t@!p bra W;\n\t}" ::"r"(su32(&bar)) : "memory");
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" ::"r"(tmem));
}
template <int N, int TS>
void run(const char *name, unsigned long long *d, int nsm) {
  auto f = k<N, TS>;
  cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
  const int NI = 4096, pairs = nsm / 2;
  f<<<2 * pairs, 128, 64 * 1024>>>(d, NI);
  f<<<2 * pairs, 128, 64 * 1024>>>(d, NI);
  cudaError_t e = cudaDeviceSynchronize();
  unsigned long long h[256];
  cudaMemcpy(h, d, pairs * 8, cudaMemcpyDeviceToHost);
  double s = 0; for (int i = 0; i < pairs; ++i) s += h[i];
  const double cyc = s / pairs / NI, flop = 2.0 * 256 * N * 8;
  printf("%-22s %s cycles/MMA %7.1f  flop/clk/SM %7.0f -> %6.0f TF/s @1.965GHz x %d SM\n", name, cudaGetErrorString(e),
         cyc, flop / cyc / 2, flop / cyc * 1.965e9 * pairs / 1e12, nsm);
}
int main() {
  int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  unsigned long long *d; cudaMalloc(&d, 256 * 8);
  run<64, 0>("2cta tf32 ss N64", d, nsm);
  run<128, 0>("2cta tf32 ss N128", d, nsm);
  run<256, 0>("2cta tf32 ss N256", d, nsm);
  run<64, 1>("2cta tf32 ts N64", d, nsm);
  run<128, 1>("2cta tf32 ts N128", d, nsm);
  run<256, 1>("2cta tf32 ts N256", d, nsm);
  return 0;
}
