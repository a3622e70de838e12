// Microbenchmark: issue rate of tcgen05.mma kind::tf32 / kind::f16 (M = 128)
// per SM for N = 64 / 128 / 256, A from shared memory (ss) or TMEM (ts).
// One CTA per SM; thread 0 issues NI MMAs into one accumulator, commits,
// waits; cycles / MMA.  Operand contents are irrelevant (timing only).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mma_rate scripts/mma_rate.cu
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
template <int KIND, int N, int TS, int BMN>
__global__ void __launch_bounds__(128, 1) k(unsigned long long *out, int NI) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ __align__(8) uint64_t bar;
  __shared__ uint32_t tb;
  const uint32_t base = (su32(sm) + 1023u) & ~1023u;
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(su32(&tb)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = tb;
  if (threadIdx.x == 0) {
    // kind::tf32: A/B fmt 2; kind::f16 (bf16): A/B fmt 1; D f32
    const uint32_t fmt = KIND == 0 ? 2u : 1u;
    const uint32_t idesc = (1u << 4) | (fmt << 7) | (fmt << 10) | ((uint32_t)BMN << 16) | ((uint32_t)(N >> 3) << 17) |
                           ((uint32_t)(128 >> 4) << 24);
    const uint64_t da = desc_k_sw128(base);
    const uint64_t db = BMN ? desc_mn_sw128_32b(base + 16384) : desc_k_sw128(base + 16384);
    const uint32_t ta = tmem + 256;
    unsigned long long t0 = clock64();
    for (int i = 0; i < NI; ++i) {
      const uint32_t acc = i > 0;
      if (TS) {
        const uint32_t z = 0;
        if (KIND == 0)
          asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                       "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, {%5,%5,%5,%5}, p;\n\t}" ::"r"(tmem),
                       "r"(ta), "l"(db), "r"(idesc), "r"(acc), "r"(z) : "memory");
        else
          asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                       "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, {%5,%5,%5,%5}, p;\n\t}" ::"r"(tmem),
                       "r"(ta), "l"(db), "r"(idesc), "r"(acc), "r"(z) : "memory");
      } else {
        if (KIND == 0)
          asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                       "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem), "l"(da), "l"(db),
                       "r"(idesc), "r"(acc) : "memory");
        else
          asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                       "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem), "l"(da), "l"(db),
                       "r"(idesc), "r"(acc) : "memory");
      }
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar)) : "memory");
    asm volatile("{\n\t.reg .pred p;\n\tW:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n\t@!p bra W;\n\t}" ::"r"(su32(&bar)) : "memory");
    unsigned long long t1 = clock64();
    out[blockIdx.x] = t1 - t0;
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
}
template <int KIND, int N, int TS, int BMN>
void run(const char *name, unsigned long long *d, int nsm) {
  auto f = k<KIND, N, TS, BMN>;
  cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
  const int NI = 4096;
  f<<<nsm, 128, 64 * 1024>>>(d, NI);
  f<<<nsm, 128, 64 * 1024>>>(d, NI);
  cudaError_t e = cudaDeviceSynchronize();
  unsigned long long h[256];
  cudaMemcpy(h, d, nsm * 8, cudaMemcpyDeviceToHost);
  double s = 0; for (int i = 0; i < nsm; ++i) s += h[i];
  const double cyc = s / nsm / NI;
  const double flop = 2.0 * 128 * N * (KIND == 0 ? 8 : 16);
  printf("%-28s %s cycles/MMA %7.1f  flop/clk/SM %7.0f  -> %6.0f TF/s @1.965GHz x %d SM\n", name, cudaGetErrorString(e), cyc,
         flop / cyc, flop / cyc * 1.965e9 * nsm / 1e12, nsm);
}
int main() {
  int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  unsigned long long *d; cudaMalloc(&d, 256 * 8);
  run<0, 64, 0, 0>("tf32 ss N64 Bk", d, nsm);
  run<0, 128, 0, 0>("tf32 ss N128 Bk", d, nsm);
  run<0, 256, 0, 0>("tf32 ss N256 Bk", d, nsm);
  run<0, 64, 0, 1>("tf32 ss N64 Bmn", d, nsm);
  run<0, 128, 0, 1>("tf32 ss N128 Bmn", d, nsm);
  run<0, 64, 1, 1>("tf32 ts N64 Bmn", d, nsm);
  run<0, 128, 1, 1>("tf32 ts N128 Bmn", d, nsm);
  run<0, 256, 1, 1>("tf32 ts N256 Bmn", d, nsm);
  run<1, 64, 0, 0>("bf16 ss N64", d, nsm);
  run<1, 128, 0, 0>("bf16 ss N128", d, nsm);
  run<1, 256, 0, 0>("bf16 ss N256", d, nsm);
  return 0;
}
