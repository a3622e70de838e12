// SIMT-FFMA SGEMM tilings (Parboil sgemm's "register-tiled with scratchpad"
// GPU version, §4.3; WA factor 16x between versions).
// C[m0:m0+BM, n0:n0+BN] = alpha * A B + beta * C_in, fp32, row-major.
// Each C element is one thread's sequential fma chain over k (ascending), so
// a tile's result does not depend on which CTA computed it (c-6).
#pragma once

#include <stdint.h>

#include "dysel_device.cuh"

namespace dysel {

struct SgemmArgs {
  int M, N, K;
  float alpha, beta;
  const float *A;
  int lda;
  const float *B;
  int ldb;
  const float *C_in;   // beta term source (may alias C_out)
  int ldc;
};

// BM x BN tile, TM x TN per thread, BK deep, 256 threads; register-staged
// double buffering of the next K-slab.
// poll(done, total): called by all threads every 4 K-slabs (progress for the
// projected dominance test, A-51); true => abandon the tile
// (a dominated sandbox copy, reading A-32: its output would be discarded).
template <int BM, int BN, int BK, int TM, int TN, class Poll>
__device__ __forceinline__ void simt_tile(const SgemmArgs &g, float *__restrict__ C, int m0, int n0,
                                          const Poll &poll) {
  static_assert((BM / TM) * (BN / TN) == 256, "256 threads");
  constexpr int A_PER = BM * BK / 256, B_PER = BK * BN / 256;
  __shared__ __align__(16) float As[2][BK][BM + 4];
  __shared__ __align__(16) float Bs[2][BK][BN + 4];
  const int tid = threadIdx.x;
  const int tx = tid % (BN / TN), ty = tid / (BN / TN);
  float acc[TM][TN];
#pragma unroll
  for (int i = 0; i < TM; ++i)
#pragma unroll
    for (int j = 0; j < TN; ++j) acc[i][j] = 0.0f;
  float ra[A_PER], rb[B_PER];
  auto load = [&](int k0) {
#pragma unroll
    for (int q = 0; q < A_PER; ++q) {
      const int e = tid + q * 256;           // A tile element (m, k), k fastest
      const int m = e / BK, k = e % BK;
      const int gm = m0 + m, gk = k0 + k;
      ra[q] = (gm < g.M && gk < g.K) ? __ldg(g.A + (int64_t)gm * g.lda + gk) : 0.0f;
    }
#pragma unroll
    for (int q = 0; q < B_PER; ++q) {
      const int e = tid + q * 256;           // B tile element (k, n), n fastest
      const int k = e / BN, n = e % BN;
      const int gk = k0 + k, gn = n0 + n;
      rb[q] = (gk < g.K && gn < g.N) ? __ldg(g.B + (int64_t)gk * g.ldb + gn) : 0.0f;
    }
  };
  auto store = [&](int buf) {
#pragma unroll
    for (int q = 0; q < A_PER; ++q) {
      const int e = tid + q * 256;
      As[buf][e % BK][e / BK] = ra[q];
    }
#pragma unroll
    for (int q = 0; q < B_PER; ++q) {
      const int e = tid + q * 256;
      Bs[buf][e / BN][e % BN] = rb[q];
    }
  };
  const int nk = (g.K + BK - 1) / BK;
  if (nk > 0) {
    load(0);
    store(0);
  }
  __syncthreads();
  for (int kt = 0; kt < nk; ++kt) {
    const int buf = kt & 1;
    if (kt + 1 < nk) load((kt + 1) * BK);
#pragma unroll
    for (int k = 0; k < BK; ++k) {
      float a[TM], b[TN];
#pragma unroll
      for (int i = 0; i < TM; ++i) a[i] = As[buf][k][ty * TM + i];
#pragma unroll
      for (int j = 0; j < TN; ++j) b[j] = Bs[buf][k][tx * TN + j];
#pragma unroll
      for (int i = 0; i < TM; ++i)
#pragma unroll
        for (int j = 0; j < TN; ++j) acc[i][j] = __fmaf_rn(a[i], b[j], acc[i][j]);
    }
    if (kt + 1 < nk) store(buf ^ 1);
    __syncthreads();
    if ((kt & 3) == 3 && poll(kt + 1, nk)) return;
  }
#pragma unroll
  for (int i = 0; i < TM; ++i) {
    const int gm = m0 + ty * TM + i;
    if (gm >= g.M) continue;
#pragma unroll
    for (int j = 0; j < TN; ++j) {
      const int gn = n0 + tx * TN + j;
      if (gn >= g.N) continue;
      float r = g.alpha * acc[i][j];
      if (g.beta != 0.0f) r = __fmaf_rn(g.beta, g.C_in[(int64_t)gm * g.ldc + gn], r);
      C[(int64_t)gm * g.ldc + gn] = r;
    }
  }
}

template <int BM, int BN, int BK, int TM, int TN>
__global__ void __launch_bounds__(256) sgemm_simt_kernel(SgemmArgs g, float *__restrict__ C, dysel_slice s) {
  __shared__ dysel_prof_smem psm;
  if (!dysel_gate_open(s)) return;
  const uint32_t wa[3] = {BN / 32, BM / 32, 1};
  if (s.timer == nullptr && s.gate != nullptr) {
    // gated remainder: a persistent grid of one wave walks the slice's tiles,
    // so a variant that lost the selection costs one wave of exiting CTAs,
    // not one per tile (they compete for slots with the winner's grid)
    const uint64_t n = dysel_slice_ctas(s, wa);
    for (uint64_t cta = blockIdx.x; cta < n; cta += gridDim.x) {
      uint64_t u[3];
      if (dysel_cta_origin(s, wa, cta, u))
        simt_tile<BM, BN, BK, TM, TN>(g, C, (int)u[1] * 32, (int)u[0] * 32, [](int, int) { return false; });
      __syncthreads();   // the tile's shared buffers are reused
    }
    return;
  }
  dysel_prof_begin(s, psm);
  uint64_t u[3];
  const bool ok = dysel_cta_origin(s, wa, blockIdx.x, u);
  if (ok)
    simt_tile<BM, BN, BK, TM, TN>(g, C, (int)u[1] * 32, (int)u[0] * 32,
                                  [&](int done, int total) {
                                    return dysel_prof_poll(s, psm, (uint32_t)done, (uint32_t)total) &&
                                           s.role == DYSEL_ROLE_SANDBOX;
                                  });
  dysel_prof_end(s, psm, ok ? wa[0] * wa[1] : 0u);   // units (32x32 tiles) this CTA covered
}

}  // namespace dysel
