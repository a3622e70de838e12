// tcgen05 3xTF32 SGEMM, TMA-fed warp-specialised pipeline (128 x BN tiles),
// A operand staged in TMEM.
//
//   warp 0 (one lane)   TMA producer: per 32-wide k-slab, A box {32 k, 128 m}
//                       (fp32, 128-byte swizzle) and BN/32 B boxes {32 n, 32 k}
//                       (fp32, 128-byte swizzle with 32-byte atoms = the UMMA
//                       MN-major tf32 canonical layout, so B is never
//                       transposed) into a STAGES-deep ring (complete_tx).
//   warps 2..5          converters: the thread owning TMEM lane (row) r reads
//                       its row's 32 A values, splits hi = a with the low 13
//                       mantissa bits cleared (exact tf32) and lo = a - hi
//                       (exact), and writes both straight into TMEM
//                       (tcgen05.st 32x32b.x32): A never goes back to shared
//                       memory and the MMAs read it from TMEM.  B chunks are
//                       split in place (hi) + a lo buffer.  Afterwards the same
//                       warps run the epilogue (tcgen05.ld -> alpha/beta ->
//                       128-bit stores).
//   warp 1 (one lane)   MMA issuer: per slab, 4 x (A_lo B_hi + A_hi B_lo +
//                       A_hi B_hi) tcgen05.mma.cta_group::1.kind::tf32 with A
//                       from TMEM, B from shared memory (M 128, N BN, K 8).
// TMEM: columns [0, BN) accumulator, [128 + 64 s, +32) A_hi / [+32, +64) A_lo
// of stage s.  Ragged edges: TMA zero-fills out-of-bounds box elements.
// Requires 16-byte aligned A/B and lda, ldb multiples of 4 (TMA strides);
// otherwise the register-staged kernel (sgemm_tc.cuh) runs.
#pragma once

#include <cuda.h>

#include "sgemm_tc.cuh"

namespace dysel {

constexpr int kTmaThreads = 192;   // producer warp, MMA warp, 4 converter / epilogue warps

template <int BN>
struct TmaCfg {
  static constexpr int A_BYTES = 128 * 128;   // A staging: 128 rows x 32 fp32 (TMA lands here)
  static constexpr int B_BYTES = BN * 128;    // BN/32 boxes of 32 x 32 fp32
  static constexpr int STAGE = A_BYTES + 2 * B_BYTES;
  static constexpr int STAGES = BN == 64 ? 6 : 4;
  static constexpr int SMEM = STAGES * STAGE + 1024;
  static constexpr uint32_t TMEM_COLS = 512;
  static constexpr uint32_t A_COL0 = 128;     // TMEM column of stage 0's A_hi
  static constexpr uint32_t TX = A_BYTES + B_BYTES;
  static constexpr int B_CHUNKS = B_BYTES / 16;
  static_assert(A_COL0 + 64 * STAGES <= TMEM_COLS, "TMEM columns");
  // kind::tf32: D f32, A/B tf32, A from TMEM (K-major), B MN-major, N = BN, M = 128
  static constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | (1u << 16) | ((uint32_t)(BN >> 3) << 17) |
                                    ((uint32_t)(128 >> 4) << 24);
};

// MN-major tf32 operands must use the 128B swizzle with 32-byte atoms
// (UMMA layout type 1, SWIZZLE_128B_BASE32B; TMA CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B):
// 128-byte K-rows (32 fp32 along N) whose 32-byte granules are permuted with a
// 4-row period.  LBO = distance between 32-wide N atoms (one 4 KB TMA box),
// SBO = distance between 4-row K groups (512 B).
__device__ __forceinline__ uint64_t umma_desc_mn_sw128_32b(uint32_t saddr) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3fff);
  d |= (uint64_t)(4096 >> 4) << 16;
  d |= (uint64_t)(512 >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)1 << 61;
  return d;
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t *b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap *tm, int c0, int c1, uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          dst),
      "l"((uint64_t)tm), "r"(c0), "r"(c1), "r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ uint4 lds128(uint32_t a) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts128(uint32_t a, const uint4 &v) {
  asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}

__device__ __forceinline__ void split_trunc(uint32_t a_bits, uint32_t &hi, uint32_t &lo) {
  hi = a_bits & 0xffffe000u;   // exact tf32 (low 13 mantissa bits cleared)
  lo = __float_as_uint(__uint_as_float(a_bits) - __uint_as_float(hi));
}
__device__ __forceinline__ void split_trunc4(uint4 &v, uint4 &lo) {
  split_trunc(v.x, v.x, lo.x);
  split_trunc(v.y, v.y, lo.y);
  split_trunc(v.z, v.z, lo.z);
  split_trunc(v.w, v.w, lo.w);
}

__device__ __forceinline__ void tmem_st32(uint32_t taddr, const uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
      "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]),
      "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]), "r"(r[16]), "r"(r[17]), "r"(r[18]),
      "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]), "r"(r[24]), "r"(r[25]), "r"(r[26]), "r"(r[27]),
      "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31])
      : "memory");
}

// D[tmem] (+)= A[tmem] * B[smem], no disabled output lanes
__device__ __forceinline__ void tc_mma_tf32_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t db, uint32_t idesc,
                                               uint32_t accumulate) {
  const uint32_t z = 0;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, {%5, %5, %5, %5}, p;\n\t}" ::"r"(tmem_d),
      "r"(tmem_a), "l"(db), "r"(idesc), "r"(accumulate), "r"(z)
      : "memory");
}

template <int BN>
__global__ void __launch_bounds__(kTmaThreads, 1)
    sgemm_tma_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB, SgemmArgs g,
                     float *__restrict__ C, dysel_slice s) {
  using Cfg = TmaCfg<BN>;
  constexpr int S = Cfg::STAGES;
  extern __shared__ uint8_t smem_raw[];
  __shared__ __align__(8) uint64_t full[S], conv[S], empty_[S], tfull;
  __shared__ uint32_t tmem_base_sh;
  __shared__ dysel_prof_smem psm;
  if (!dysel_gate_open(s)) return;
  const uint32_t wa[3] = {BN / 32, 4, 1};
  dysel_prof_begin(s, psm);
  uint64_t u[3];
  const bool ok = dysel_cta_origin(s, wa, blockIdx.x, u);
  if (!ok) {
    dysel_prof_end(s, psm, 0u);
    return;
  }
  const int m0 = (int)u[1] * 32, n0 = (int)u[0] * 32;
  const uint32_t sbase = (smem_u32(smem_raw) + 1023u) & ~1023u;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base_sh)),
                 "r"(Cfg::TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&conv[i], 128);
      mbar_init(&empty_[i], 1);
    }
    mbar_init(&tfull, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmA) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmB) : "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_base_sh;
  const int nk = (g.K + 31) / 32;

  if (warp == 0) {
    if (lane == 0) {   // ---------------------------------- TMA producer
      for (int kb = 0; kb < nk; ++kb) {
        // dominance report (A-32): a losing tiling is decided without waiting
        // for its profiled tiles (they still complete: no abort inside the pipeline)
        if ((kb & 15) == 15) dysel_prof_poll_thread(s, psm, (uint32_t)(kb + 1), (uint32_t)nk);
        const int st = kb % S;
        if (kb >= S) mbar_wait(&empty_[st], (uint32_t)(((kb / S) - 1) & 1));
        mbar_expect_tx(&full[st], Cfg::TX);
        const uint32_t a = sbase + st * Cfg::STAGE;
        tma_load_2d(a, &tmA, kb * 32, m0, &full[st]);
#pragma unroll
        for (int q = 0; q < BN / 32; ++q)
          tma_load_2d(a + Cfg::A_BYTES + q * 4096, &tmB, n0 + 32 * q, kb * 32, &full[st]);
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    if (lane == 0) {   // ---------------------------------- MMA issuer
      for (int kb = 0; kb < nk; ++kb) {
        const int st = kb % S;
        mbar_wait(&conv[st], (uint32_t)((kb / S) & 1));
        tc_fence_after();
        const uint32_t b = sbase + st * Cfg::STAGE + Cfg::A_BYTES, b_lo = b + Cfg::B_BYTES;
        const uint32_t ta = tmem + Cfg::A_COL0 + 64u * st;   // A_hi; A_lo at +32 columns
#pragma unroll
        for (int kk = 0; kk < 4; ++kk) {
          const uint64_t dbh = umma_desc_mn_sw128_32b(b + kk * 1024), dbl = umma_desc_mn_sw128_32b(b_lo + kk * 1024);
          tc_mma_tf32_ts(tmem, ta + 32 + 8 * kk, dbh, Cfg::IDESC, (kb | kk) != 0);   // small terms first
          tc_mma_tf32_ts(tmem, ta + 8 * kk, dbl, Cfg::IDESC, 1u);
          tc_mma_tf32_ts(tmem, ta + 8 * kk, dbh, Cfg::IDESC, 1u);
        }
        tc_commit(&empty_[st]);
      }
      if (nk > 0) tc_commit(&tfull);
    }
    __syncwarp();
  } else {
    const int q = warp & 3;                    // TMEM lane quadrant of this warp
    const int row = q * 32 + lane;             // A row / TMEM lane owned by this thread
    const int ct = tid - 64;                   // 0..127 for the B chunks
    const uint32_t tlane = (uint32_t)(q * 32) << 16;
    for (int kb = 0; kb < nk; ++kb) {   // ---------------------- converters
      const int st = kb % S;
      mbar_wait(&full[st], (uint32_t)((kb / S) & 1));
      const uint32_t stage = sbase + st * Cfg::STAGE;
      // A: this thread's row, 8 swizzled 16-byte chunks (chunk c at c ^ (row & 7))
      uint4 av[8];
#pragma unroll
      for (int c = 0; c < 8; ++c) av[c] = lds128(stage + row * 128 + ((c ^ (row & 7)) << 4));
      constexpr int B_PER = Cfg::B_CHUNKS / 128;
      uint4 bv[B_PER];
#pragma unroll
      for (int j = 0; j < B_PER; ++j) bv[j] = lds128(stage + Cfg::A_BYTES + 16 * (ct + 128 * j));
      uint32_t hi[32], lo[32];
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        split_trunc(av[c].x, hi[4 * c + 0], lo[4 * c + 0]);
        split_trunc(av[c].y, hi[4 * c + 1], lo[4 * c + 1]);
        split_trunc(av[c].z, hi[4 * c + 2], lo[4 * c + 2]);
        split_trunc(av[c].w, hi[4 * c + 3], lo[4 * c + 3]);
      }
      const uint32_t ta = tmem + tlane + Cfg::A_COL0 + 64u * st;
      tmem_st32(ta, hi);
      tmem_st32(ta + 32, lo);
#pragma unroll
      for (int j = 0; j < B_PER; ++j) {
        uint4 l;
        split_trunc4(bv[j], l);
        const uint32_t p = stage + Cfg::A_BYTES + 16 * (ct + 128 * j);
        sts128(p, bv[j]);
        sts128(p + Cfg::B_BYTES, l);
      }
      asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      tc_fence_before();
      mbar_arrive(&conv[st]);
    }
    // -------------------------------------------------------- epilogue
    if (nk > 0) {
      mbar_wait(&tfull, 0);
      tc_fence_after();
    }
    const int gm = m0 + row;
#pragma unroll 1
    for (int c0 = 0; c0 < BN; c0 += 16) {
      float v[16];
      if (nk > 0) {
        tmem_ld16(tmem + tlane + (uint32_t)c0, v);
      } else {
#pragma unroll
        for (int i = 0; i < 16; ++i) v[i] = 0.0f;
      }
      if (gm < g.M) {
        float *crow = C + (int64_t)gm * g.ldc + n0 + c0;
        const float *cin = g.C_in + (int64_t)gm * g.ldc + n0 + c0;
        if (n0 + c0 + 16 <= g.N && ((((uintptr_t)crow) | ((uintptr_t)cin)) & 15) == 0) {
#pragma unroll
          for (int i = 0; i < 16; i += 4) {   // 128-bit stores
            float4 r = make_float4(g.alpha * v[i], g.alpha * v[i + 1], g.alpha * v[i + 2], g.alpha * v[i + 3]);
            if (g.beta != 0.0f) {
              const float4 c = *(const float4 *)(cin + i);
              r.x = __fmaf_rn(g.beta, c.x, r.x);
              r.y = __fmaf_rn(g.beta, c.y, r.y);
              r.z = __fmaf_rn(g.beta, c.z, r.z);
              r.w = __fmaf_rn(g.beta, c.w, r.w);
            }
            *(float4 *)(crow + i) = r;
          }
        } else {
#pragma unroll
          for (int i = 0; i < 16; ++i) {
            if (n0 + c0 + i < g.N) {
              float r = g.alpha * v[i];
              if (g.beta != 0.0f) r = __fmaf_rn(g.beta, cin[i], r);
              crow[i] = r;
            }
          }
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(Cfg::TMEM_COLS));
  }
  dysel_prof_end(s, psm, wa[0] * wa[1]);   // units (32x32 tiles) this CTA covered
}

}  // namespace dysel
