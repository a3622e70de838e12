// DySel SGEMM: the built-in variant pool registered through the generic
// launcher (dysel_launch), so SGEMM exercises the same slice planner, device
// timing and gated device-side remainder as user-registered kernels.
// Unit = one 32x32 tile of C; wa = (tile_N/32, tile_M/32) (SURVEY §8 notation).
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstring>
#include <string>

#include "internal.h"
#include "sgemm_simt.cuh"
#include "sgemm_tc.cuh"
#include "sgemm_tma.cuh"

namespace dysel {

static const char *kSgemmSig = "dysel.sgemm";

static PFN_cuTensorMapEncodeTiled_v12000 tensor_map_encoder() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (PFN_cuTensorMapEncodeTiled_v12000)p;
    cudaGetLastError();
  }
  return fn;
}

// 2-D fp32 tensor map, 128-byte swizzle, zero fill out of bounds.  Encoded
// maps are cached per thread (a few us of driver work per encode; a DySel
// SGEMM launches up to K profiling copies, the eager wave and K gated
// remainders, each with the same two maps).
struct MapKey {
  const float *base;
  uint64_t inner, outer, ld;
  uint32_t box_inner, box_outer;
  int swz;
  bool operator==(const MapKey &o) const {
    return base == o.base && inner == o.inner && outer == o.outer && ld == o.ld && box_inner == o.box_inner &&
           box_outer == o.box_outer && swz == o.swz;
  }
};
static bool make_map(CUtensorMap *m, const float *base, uint64_t inner, uint64_t outer, uint64_t ld_elems,
                     uint32_t box_inner, uint32_t box_outer, CUtensorMapSwizzle swz) {
  constexpr int kSlots = 8;
  thread_local MapKey keys[kSlots] = {};
  thread_local CUtensorMap maps[kSlots];
  thread_local int next = 0;
  const MapKey k{base, inner, outer, ld_elems, box_inner, box_outer, (int)swz};
  for (int i = 0; i < kSlots; ++i)
    if (keys[i].base && keys[i] == k) {
      *m = maps[i];
      return true;
    }
  auto enc = tensor_map_encoder();
  if (!enc) return false;
  const cuuint64_t dims[2] = {inner, outer};
  const cuuint64_t strides[1] = {ld_elems * sizeof(float)};
  const cuuint32_t box[2] = {box_inner, box_outer};
  const cuuint32_t estr[2] = {1, 1};
  if (enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void *)base, dims, strides, box, estr,
          CU_TENSOR_MAP_INTERLEAVE_NONE, swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
          CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
    return false;
  keys[next] = k;
  maps[next] = *m;
  next = (next + 1) % kSlots;
  return true;
}

// tcgen05 path: TMA pipeline when the operands allow TMA (16-byte aligned
// bases, lda / ldb multiples of 4), else the register-staged kernel.
template <int BN>
static dysel_status launch_tc(const SgemmArgs &g, float *C, const dysel_slice &s, unsigned ctas, cudaStream_t st) {
  const bool tma_ok = g.K > 0 && ((((uintptr_t)g.A) | ((uintptr_t)g.B)) & 15) == 0 && (g.lda % 4) == 0 &&
                      (g.ldb % 4) == 0;
  if (tma_ok) {
    CUtensorMap ta, tb;
    // A: K-major SW128 (16-byte granules); B: MN-major tf32 needs 32-byte atoms
    if (make_map(&ta, g.A, (uint64_t)g.K, (uint64_t)g.M, (uint64_t)g.lda, 32, 128, CU_TENSOR_MAP_SWIZZLE_128B) &&
        make_map(&tb, g.B, (uint64_t)g.N, (uint64_t)g.K, (uint64_t)g.ldb, 32, 32, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B)) {
      sgemm_tma_kernel<BN><<<ctas, kTmaThreads, TmaCfg<BN>::SMEM, st>>>(ta, tb, g, C, s);
      return cudaGetLastError() == cudaSuccess ? DYSEL_OK : DYSEL_ERR_CUDA;
    }
  }
  return launch_tc_sgemm<BN>(g, C, s, ctas, st);
}

static uint64_t g_simt_wave[2] = {0, 0};   // resident CTAs (occupancy x #SM) of the two SIMT kernels
static uint64_t g_tc128_wave = 0;          // ... of the 128x128 tcgen05 kernel

template <int VID>
static dysel_status sgemm_variant_fn(const dysel_slice *s, void *const *args, void *stream, void *) {
  const SgemmArgs &g = *(const SgemmArgs *)args[1];
  float *C = (float *)args[0];
  cudaStream_t st = (cudaStream_t)stream;
  uint32_t wa[3];
  if constexpr (VID == DYSEL_SGEMM_S64) {
    wa[0] = 2; wa[1] = 2; wa[2] = 1;
  } else if constexpr (VID == DYSEL_SGEMM_S128) {
    wa[0] = 4; wa[1] = 4; wa[2] = 1;
  } else if constexpr (VID == DYSEL_SGEMM_T128x64) {
    wa[0] = 2; wa[1] = 4; wa[2] = 1;
  } else {
    wa[0] = 4; wa[1] = 4; wa[2] = 1;
  }
  const uint64_t ctas = dysel_slice_ctas(*s, wa);
  if (ctas == 0) return DYSEL_OK;
  // gated remainder of a SIMT variant: one persistent wave (sgemm_simt_kernel)
  const uint64_t grid = (s->gate && s->timer == nullptr && !s->gate_full_grid && g_simt_wave[VID & 1] > 0)
                            ? std::min<uint64_t>(ctas, g_simt_wave[VID & 1]) : ctas;
  if constexpr (VID == DYSEL_SGEMM_S64) {
    sgemm_simt_kernel<64, 64, 16, 4, 4><<<(unsigned)grid, 256, 0, st>>>(g, C, *s);
  } else if constexpr (VID == DYSEL_SGEMM_S128) {
    sgemm_simt_kernel<128, 128, 8, 8, 8><<<(unsigned)grid, 256, 0, st>>>(g, C, *s);
  } else if constexpr (VID == DYSEL_SGEMM_T128x64) {
    DYSEL_TRY(launch_tc<64>(g, C, *s, (unsigned)ctas, st));
  } else {
    DYSEL_TRY(launch_tc<128>(g, C, *s, (unsigned)ctas, st));
  }
  return cudaGetLastError() == cudaSuccess ? DYSEL_OK : DYSEL_ERR_CUDA;
}

dysel_status sgemm_register(dysel_ctx *ctx) {
  static const int sb[1] = {0};
  DYSEL_TRY(tc_sgemm_init());
  if (cudaFuncSetAttribute(sgemm_tma_kernel<64>, cudaFuncAttributeMaxDynamicSharedMemorySize, TmaCfg<64>::SMEM) !=
          cudaSuccess ||
      cudaFuncSetAttribute(sgemm_tma_kernel<128>, cudaFuncAttributeMaxDynamicSharedMemorySize, TmaCfg<128>::SMEM) !=
          cudaSuccess)
    return DYSEL_ERR_CUDA;
  // CTAs resident at once (reading A-3b: a grid within one wave is not profiled)
  int o[4] = {0, 0, 0, 0};
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o[0], sgemm_simt_kernel<64, 64, 16, 4, 4>, 256, 0);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o[1], sgemm_simt_kernel<128, 128, 8, 8, 8>, 256, 0);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o[2], sgemm_tma_kernel<64>, kTmaThreads, TmaCfg<64>::SMEM);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o[3], sgemm_tma_kernel<128>, kTmaThreads, TmaCfg<128>::SMEM);
  cudaGetLastError();
  const uint64_t n = (uint64_t)ctx->n_sm;
  g_simt_wave[0] = (uint64_t)o[0] * n;
  g_simt_wave[1] = (uint64_t)o[1] * n;
  g_tc128_wave = (uint64_t)o[3] * n;
  dysel_variant v[DYSEL_SGEMM_NVARIANTS] = {
      {"simt64x64", sgemm_variant_fn<0>, {2, 2, 1}, sb, 1, 0, nullptr, (uint64_t)o[0] * n},
      {"simt128x128", sgemm_variant_fn<1>, {4, 4, 1}, sb, 1, 0, nullptr, (uint64_t)o[1] * n},
      {"tc3xtf32_128x64", sgemm_variant_fn<2>, {2, 4, 1}, sb, 1, 0, nullptr, (uint64_t)o[2] * n},
      {"tc3xtf32_128x128", sgemm_variant_fn<3>, {4, 4, 1}, sb, 1, 0, nullptr, (uint64_t)o[3] * n},
  };
  // initial ("default") version on B200: the tensor-core tiling (A-5)
  DYSEL_TRY(dysel_register_variants(ctx, kSgemmSig, v, DYSEL_SGEMM_NVARIANTS, DYSEL_SGEMM_T128x64));
  mark_builtin(ctx, kSgemmSig);
  return DYSEL_OK;
}

static dysel_status check_args(dysel_ctx *ctx, int M, int N, int K, const float *A, int lda, const float *B, int ldb,
                               float *C, int ldc) {
  if (M < 0 || N < 0 || K < 0 || (M > 0 && N > 0 && (!C || ldc < N)) || (M > 0 && K > 0 && (!A || lda < K)) ||
      (N > 0 && K > 0 && (!B || ldb < N))) {
    set_error(ctx, "dysel_sgemm: invalid arguments");
    return DYSEL_ERR_INVALID;
  }
  return DYSEL_OK;
}

}  // namespace dysel

using namespace dysel;

extern "C" {

dysel_status dysel_sgemm(dysel_ctx *ctx, int M, int N, int K, float alpha, const float *d_A, int lda, const float *d_B,
                         int ldb, float beta, float *d_C, int ldc, float f, uint32_t mode, void *stream,
                         dysel_report *rep) {
  if (!ctx) return DYSEL_ERR_INVALID;
  DYSEL_TRY(check_args(ctx, M, N, K, d_A, lda, d_B, ldb, d_C, ldc));
  if (rep) rep->n_slices = 0;
  if ((int64_t)M * N == 0) return DYSEL_OK;
  SgemmArgs g{M, N, K, alpha, beta, d_A, lda, d_B, ldb, d_C, ldc};
  const uint64_t U[3] = {(uint64_t)(N + 31) / 32, (uint64_t)(M + 31) / 32, 1};
  void *args[2] = {d_C, &g};
  const size_t sbytes[1] = {(size_t)M * ldc * sizeof(float)};
  const std::string key = std::string(kSgemmSig) + "#" + std::to_string(M) + "x" + std::to_string(N) + "x" +
                          std::to_string(K);
  // reading A-39: the initial version is the 128x128 tcgen05 tiling when its
  // grid spans at least two waves (large GEMMs: fewest passes over A and B),
  // else the 128x64 tiling (more CTAs: fills the SMs of a small GEMM)
  const uint64_t t128 = (uint64_t)((M + 127) / 128) * (uint64_t)((N + 127) / 128);
  const int def = (g_tc128_wave > 0 && t128 >= 2 * g_tc128_wave) ? DYSEL_SGEMM_T128x128 : DYSEL_SGEMM_T128x64;
  return launch_keyed(ctx, kSgemmSig, key.c_str(), U, f, mode, args, 2, sbytes, stream, rep, def);
}

dysel_status dysel_sgemm_variant(dysel_ctx *ctx, int variant_id, int M, int N, int K, float alpha, const float *d_A,
                                 int lda, const float *d_B, int ldb, float beta, float *d_C, int ldc, void *stream) {
  if (!ctx || variant_id < 0 || variant_id >= DYSEL_SGEMM_NVARIANTS) {
    set_error(ctx, "dysel_sgemm_variant: invalid variant");
    return DYSEL_ERR_INVALID;
  }
  DYSEL_TRY(check_args(ctx, M, N, K, d_A, lda, d_B, ldb, d_C, ldc));
  if ((int64_t)M * N == 0) return DYSEL_OK;
  SgemmArgs g{M, N, K, alpha, beta, d_A, lda, d_B, ldb, d_C, ldc};
  const uint64_t U[3] = {(uint64_t)(N + 31) / 32, (uint64_t)(M + 31) / 32, 1};
  void *args[2] = {d_C, &g};
  // one full-grid batch copy of the variant: a slice over every granule
  dysel_slice s;
  memset(&s, 0, sizeof(s));
  const uint32_t gg[3] = {4, 4, 1};
  for (int d = 0; d < 3; ++d) {
    s.g[d] = gg[d];
    s.U[d] = U[d];
    s.G[d] = (uint32_t)((U[d] + gg[d] - 1) / gg[d]);
  }
  s.granule_count = (uint64_t)s.G[0] * s.G[1] * s.G[2];
  s.granule_stride = 1;
  s.role = DYSEL_ROLE_BATCH;
  s.variant = variant_id;
  static dysel_variant_fn fns[DYSEL_SGEMM_NVARIANTS] = {sgemm_variant_fn<0>, sgemm_variant_fn<1>, sgemm_variant_fn<2>,
                                                        sgemm_variant_fn<3>};
  DYSEL_TRY(fns[variant_id](&s, args, stream, nullptr));
  return check_launch(ctx, "sgemm full-grid variant");
}

}  // extern "C"
