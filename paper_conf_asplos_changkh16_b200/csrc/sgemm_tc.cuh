// tcgen05 (5th-gen tensor core) 3xTF32 SGEMM tilings 128x64 and 128x128.
//
// The one dense contraction on the path (north_star: "Tensor cores
// (tcgen05/TMEM, 3xTF32) appear only in the SGEMM variants").  fp32 inputs are
// split in shared memory into hi = rna_tf32(a) and lo = rna_tf32(a - hi);
// C += A_hi B_hi + A_hi B_lo + A_lo B_hi is accumulated in fp32 in TMEM by
// tcgen05.mma.cta_group::1.kind::tf32 (M = 128, N = BN, K = 8 per instruction)
// issued by one thread; the epilogue reads TMEM with tcgen05.ld and applies
// alpha / beta.  The per-element result is a fixed sequence of tensor-core
// accumulations over k-blocks, independent of the CTA position (c-6).
//
// Shared-memory operand layout: K-major, 128-byte swizzle (SW128) — row r of a
// 32-element (128 B) k-slab at (r/8)*1024 + (r%8)*128, 16-byte chunk c stored
// at chunk position c ^ (r%8); descriptor SBO = 1024 B, LBO = 16 B (unused),
// version 1, layout type 2.  A is naturally K-major; B (row-major K x N) is
// transposed to K-major by the split pass.
#pragma once

#include <stdint.h>

#include "dysel_device.cuh"
#include "sgemm_simt.cuh"

namespace dysel {

constexpr int kTcBM = 128;
constexpr int kTcBK = 32;            // fp32 elements per 128-byte swizzle row
constexpr int kTcThreads = 128;

template <int BN>
struct TcCfg {
  static constexpr int A_BYTES = kTcBM * 128;        // one operand copy (hi or lo)
  static constexpr int B_BYTES = BN * 128;
  static constexpr int STAGE = 2 * A_BYTES + 2 * B_BYTES;
  static constexpr int STAGES = 2;
  static constexpr int SMEM = STAGES * STAGE + 1024;  // + alignment slack
  static constexpr uint32_t TMEM_COLS = BN < 32 ? 32 : BN;
  // instruction descriptor, kind::tf32: D f32, A/B tf32, both K-major
  static constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(BN >> 3) << 17) |
                                    ((uint32_t)(kTcBM >> 4) << 24);
};

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint64_t umma_desc_sw128(uint32_t saddr) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3fff);          // start address
  d |= (uint64_t)1 << 16;                          // LBO (ignored for swizzled K-major)
  d |= (uint64_t)(1024 >> 4) << 32;                // SBO: 8-row group stride
  d |= (uint64_t)1 << 46;                          // version (sm_100)
  d |= (uint64_t)2 << 61;                          // SWIZZLE_128B
  return d;
}

__device__ __forceinline__ uint32_t swz(int r, int chunk) {   // byte offset of (row, 16B chunk)
  return (uint32_t)((r >> 3) * 1024 + (r & 7) * 128 + ((chunk ^ (r & 7)) << 4));
}

__device__ __forceinline__ uint32_t to_tf32(float a) {
  uint32_t r;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(a));
  return r;
}

__device__ __forceinline__ void split(float a, uint32_t &hi, uint32_t &lo) {
  hi = to_tf32(a);
  lo = to_tf32(a - __uint_as_float(hi));
}

__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count));
}

__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(b)),
      "r"(parity)
      : "memory");
}

__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

__device__ __forceinline__ void tc_mma_tf32(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t idesc,
                                            uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(da), "l"(db), "r"(idesc), "r"(accumulate)
      : "memory");
}

__device__ __forceinline__ void tc_commit(uint64_t *b) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(b))
               : "memory");
}

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, float (&v)[16]) {
  uint32_t r[16];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
}

template <int BN>
__global__ void __launch_bounds__(kTcThreads, 1) sgemm_tc_kernel(SgemmArgs g, float *__restrict__ C, dysel_slice s) {
  using Cfg = TcCfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  __shared__ __align__(8) uint64_t mbar[Cfg::STAGES];
  __shared__ uint32_t tmem_base_sh;
  __shared__ dysel_prof_smem psm;
  if (!dysel_gate_open(s)) return;
  const uint32_t wa[3] = {BN / 32, kTcBM / 32, 1};
  dysel_prof_begin(s, psm);
  uint64_t u[3];
  const bool ok = dysel_cta_origin(s, wa, blockIdx.x, u);
  if (!ok) {
    dysel_prof_end(s, psm, 0u);
    return;
  }
  const int m0 = (int)u[1] * 32, n0 = (int)u[0] * 32;
  uint8_t *smem = (uint8_t *)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  const uint32_t sbase = smem_u32(smem);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;

  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base_sh)),
                 "r"(Cfg::TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    for (int i = 0; i < Cfg::STAGES; ++i) mbar_init(&mbar[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_base_sh;

  const int nk = (g.K + kTcBK - 1) / kTcBK;
  const bool a_vec = ((((uintptr_t)g.A) | ((uintptr_t)g.lda * 4)) & 15) == 0;
  // register staging of one k-block: A 128 rows x 8 chunks -> 8 float4 per
  // thread; B 32 k x BN n -> (BN*8/128) (n, k-chunk) pairs per thread
  constexpr int B_PAIRS = BN * 8 / kTcThreads;
  float4 ra[8];
  float4 rb[B_PAIRS];
  auto load = [&](int kb) {
    const int k0 = kb * kTcBK;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int r = (tid >> 3) + 16 * i, c = tid & 7;
      const int gm = m0 + r, gk = k0 + c * 4;
      float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
      if (gm < g.M) {
        const float *p = g.A + (int64_t)gm * g.lda + gk;
        if (a_vec && gk + 3 < g.K) {
          v = __ldg((const float4 *)p);
        } else {
          if (gk + 0 < g.K) v.x = __ldg(p + 0);
          if (gk + 1 < g.K) v.y = __ldg(p + 1);
          if (gk + 2 < g.K) v.z = __ldg(p + 2);
          if (gk + 3 < g.K) v.w = __ldg(p + 3);
        }
      }
      ra[i] = v;
    }
#pragma unroll
    for (int i = 0; i < B_PAIRS; ++i) {
      const int e = tid + kTcThreads * i;        // n fastest across lanes: coalesced per k
      const int n = e % BN, c = e / BN;          // c = 16-byte k-chunk (4 k values)
      const int gn = n0 + n, gk = k0 + c * 4;
      float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
      if (gn < g.N) {
        const float *p = g.B + (int64_t)gk * g.ldb + gn;
        if (gk + 0 < g.K) v.x = __ldg(p);
        if (gk + 1 < g.K) v.y = __ldg(p + g.ldb);
        if (gk + 2 < g.K) v.z = __ldg(p + 2 * (int64_t)g.ldb);
        if (gk + 3 < g.K) v.w = __ldg(p + 3 * (int64_t)g.ldb);
      }
      rb[i] = v;
    }
  };
  auto store = [&](int st) {
    uint8_t *stage = smem + st * Cfg::STAGE;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int r = (tid >> 3) + 16 * i, c = tid & 7;
      uint4 h, l;
      split(ra[i].x, h.x, l.x);
      split(ra[i].y, h.y, l.y);
      split(ra[i].z, h.z, l.z);
      split(ra[i].w, h.w, l.w);
      const uint32_t off = swz(r, c);
      *(uint4 *)(stage + off) = h;
      *(uint4 *)(stage + Cfg::A_BYTES + off) = l;
    }
#pragma unroll
    for (int i = 0; i < B_PAIRS; ++i) {
      const int e = tid + kTcThreads * i;
      const int n = e % BN, c = e / BN;
      uint4 h, l;
      split(rb[i].x, h.x, l.x);
      split(rb[i].y, h.y, l.y);
      split(rb[i].z, h.z, l.z);
      split(rb[i].w, h.w, l.w);
      const uint32_t off = swz(n, c);
      *(uint4 *)(stage + 2 * Cfg::A_BYTES + off) = h;
      *(uint4 *)(stage + 2 * Cfg::A_BYTES + Cfg::B_BYTES + off) = l;
    }
  };

  if (nk > 0) load(0);
  for (int kb = 0; kb < nk; ++kb) {
    const int st = kb & 1;
    if (kb >= 2) mbar_wait(&mbar[st], (uint32_t)(((kb - 2) >> 1) & 1));
    store(st);
    if (kb + 1 < nk) load(kb + 1);   // next slab in flight while this one is multiplied
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    if (tid == 0) {
      tc_fence_after();
      const uint32_t sa = sbase + st * Cfg::STAGE;
      const uint32_t a_hi = sa, a_lo = sa + Cfg::A_BYTES, b_hi = sa + 2 * Cfg::A_BYTES,
                     b_lo = sa + 2 * Cfg::A_BYTES + Cfg::B_BYTES;
#pragma unroll
      for (int kk = 0; kk < kTcBK / 8; ++kk) {
        const uint32_t ko = kk * 32;   // 8 tf32 = 32 bytes along the swizzled row
        tc_mma_tf32(tmem, umma_desc_sw128(a_lo + ko), umma_desc_sw128(b_hi + ko), Cfg::IDESC, (kb | kk) != 0);
        tc_mma_tf32(tmem, umma_desc_sw128(a_hi + ko), umma_desc_sw128(b_lo + ko), Cfg::IDESC, 1u);
        tc_mma_tf32(tmem, umma_desc_sw128(a_hi + ko), umma_desc_sw128(b_hi + ko), Cfg::IDESC, 1u);
      }
      tc_commit(&mbar[st]);
    }
  }
  if (nk > 0) mbar_wait(&mbar[(nk - 1) & 1], (uint32_t)(((nk - 1) >> 1) & 1));
  tc_fence_after();
  // epilogue: warp w owns TMEM lanes (= C rows) 32w..32w+31
  const int row = warp * 32 + lane;
  const int gm = m0 + row;
#pragma unroll 1
  for (int c0 = 0; c0 < BN; c0 += 16) {
    float v[16];
    if (nk > 0) {
      tmem_ld16(tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)c0, v);
    } else {
#pragma unroll
      for (int i = 0; i < 16; ++i) v[i] = 0.0f;
    }
    if (gm < g.M) {
#pragma unroll
      for (int i = 0; i < 16; ++i) {
        const int gn = n0 + c0 + i;
        if (gn < g.N) {
          float r = g.alpha * v[i];
          if (g.beta != 0.0f) r = __fmaf_rn(g.beta, g.C_in[(int64_t)gm * g.ldc + gn], r);
          C[(int64_t)gm * g.ldc + gn] = r;
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(Cfg::TMEM_COLS));
  }
  dysel_prof_end(s, psm, wa[0] * wa[1]);   // units (32x32 tiles) this CTA covered
}

inline dysel_status tc_sgemm_init() {
  if (cudaFuncSetAttribute(sgemm_tc_kernel<64>, cudaFuncAttributeMaxDynamicSharedMemorySize, TcCfg<64>::SMEM) !=
          cudaSuccess ||
      cudaFuncSetAttribute(sgemm_tc_kernel<128>, cudaFuncAttributeMaxDynamicSharedMemorySize, TcCfg<128>::SMEM) !=
          cudaSuccess)
    return DYSEL_ERR_CUDA;
  return DYSEL_OK;
}

template <int BN>
inline dysel_status launch_tc_sgemm(const SgemmArgs &g, float *C, const dysel_slice &s, unsigned ctas,
                                    cudaStream_t st) {
  sgemm_tc_kernel<BN><<<ctas, kTcThreads, TcCfg<BN>::SMEM, st>>>(g, C, s);
  return cudaGetLastError() == cudaSuccess ? DYSEL_OK : DYSEL_ERR_CUDA;
}

}  // namespace dysel
