// Does kind::tf32 tcgen05.mma truncate, round, or keep the low 13 mantissa bits
// of fp32 operands?  A = B-independent constant a, B = 1: D = 8 a_hw (K = 8).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tf32_trunc scripts/tf32_trunc.cu
#include <cstdio>
#include <cstdint>
#include <cstring>
#include <cuda_runtime.h>
__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc_k_sw128(uint32_t a) {
  uint64_t d = 0;
  d |= (uint64_t)((a >> 4) & 0x3fff); d |= (uint64_t)1 << 16; d |= (uint64_t)(1024 >> 4) << 32;
  d |= (uint64_t)1 << 46; d |= (uint64_t)2 << 61; return d;
}
__global__ void k(float aval, float bval, float *out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ __align__(8) uint64_t bar;
  __shared__ uint32_t tb;
  const uint32_t base = (su32(sm) + 1023u) & ~1023u;
  float *sa = (float *)(sm + (base - su32(sm)));
  for (int i = threadIdx.x; i < 128 * 32; i += blockDim.x) sa[i] = aval;          // A 128 x 32 (K-major sw128)
  for (int i = threadIdx.x; i < 128 * 32; i += blockDim.x) sa[4096 + i] = bval;   // B 128 x 32 (K-major)
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" ::"r"(su32(&tb)));
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
    const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(128 >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    const uint64_t da = desc_k_sw128(base), db = desc_k_sw128(base + 16384);
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem), "l"(da), "l"(db),
                 "r"(idesc), "r"(0u) : "memory");
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar)) : "memory");
  }
  asm volatile("{\n\t.reg .pred p;\n\tW:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n\t@!p bra W;\n\t}" ::"r"(su32(&bar)) : "memory");
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  uint32_t r;
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x1.b32 {%0}, [%1];" : "=r"(r) : "r"(tmem + ((threadIdx.x & 96u) << 16)));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
  if (threadIdx.x == 0) out[0] = __uint_as_float(r);
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" ::"r"(tmem));
}
int main() {
  float *d; cudaMalloc(&d, 4);
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 40 * 1024);
  const double cases[] = {1.0 + 1.0 / 2048 + 1.0 / 1048576, 1.0 + 1.0 / 4096 + 1.0 / 1048576, -(1.0 + 1.0 / 2048 + 1.0 / 1048576),
                          1.0 + 3.0 / 4096};
  for (double a : cases) {
    float af = (float)a, h;
    k<<<1, 128, 40 * 1024>>>(af, 1.0f, d);
    cudaError_t e = cudaDeviceSynchronize();
    cudaMemcpy(&h, d, 4, cudaMemcpyDeviceToHost);
    uint32_t bits; memcpy(&bits, &af, 4);
    float tr, rn; uint32_t t = bits & 0xffffe000u; memcpy(&tr, &t, 4);
    uint32_t rb = (bits + 0x1000u) & 0xffffe000u; memcpy(&rn, &rb, 4);
    printf("%s a=%.9g  D/8=%.9g  trunc=%.9g rn=%.9g full=%.9g\n", cudaGetErrorString(e), af, h / 8, tr, rn, af);
  }
  return 0;
}
