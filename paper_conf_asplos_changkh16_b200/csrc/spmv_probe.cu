// Measurement only (not part of DySel): the gather-probe kernels behind
// dysel_spmv_gather_probe (include/dysel.h; DESIGN.md §6 "floor").  They move
// the memory traffic every CSR SpMV of a plan's matrix must move -- col / val
// streamed once, x gathered at col (or read sequentially, or gathered by the
// TMA unit) -- with no row structure, so their time is the practical floor the
// SpMV variant kernels are judged against.  The result is not y = A x.
#include <cudaTypedefs.h>

#include <algorithm>

#include "spmv_plan.h"

namespace dysel {

// ------------------------------------------------------------ gather probe
// Measurement only (dysel_spmv_gather_probe): the memory traffic
// every CSR SpMV of this matrix must generate and nothing else -- col / val
// streamed with 128-bit evict_first loads, x[col] gathered (evict_last), one
// fma per nonzero, row_ptr read and y written once -- with no row structure
// (no segmented sums, no per-row work imbalance).  Its time is the practical
// floor of the variant kernels on this box; the result is not y = Ax.
// FLAV 0: x gathered at col (the matrix's access pattern); FLAV 1: x read at
// the nonzero's own index modulo a power of two <= n_cols (same bytes,
// sequential: the stream floor).
template <int FLAV>
__global__ void __launch_bounds__(kUnitRows) spmv_gather_probe_kernel(SpmvDev A, float *out, int64_t nnz, int64_t xmask) {
  const uint64_t ps = policy_evict_first(), px = policy_evict_last();
  const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
  const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t n4 = nnz >> 2;
  float acc = 0.0f;
  auto xat = [&](int c, int64_t k) -> float {
    if (FLAV == 0) return ld_x(A.x + c, px);
    return ld_x(A.x + ((k ^ (int64_t)(c & 1)) & xmask), px);   // keeps the col stream live
  };
  for (int64_t q = t; q < n4; q += 2 * nthr) {
    const int64_t q1 = q + nthr;
    const bool h1 = q1 < n4;
    const int4 c0 = ld_stream4(A.col + 4 * q, ps);
    const float4 v0 = ld_stream4(A.val + 4 * q, ps);
    const int4 c1 = h1 ? ld_stream4(A.col + 4 * q1, ps) : make_int4(0, 0, 0, 0);
    const float4 v1 = h1 ? ld_stream4(A.val + 4 * q1, ps) : make_float4(0.f, 0.f, 0.f, 0.f);
    const float x0 = xat(c0.x, 4 * q), x1 = xat(c0.y, 4 * q + 1), x2 = xat(c0.z, 4 * q + 2), x3 = xat(c0.w, 4 * q + 3);
    const float z0 = xat(c1.x, 4 * q1), z1 = xat(c1.y, 4 * q1 + 1), z2 = xat(c1.z, 4 * q1 + 2),
                z3 = xat(c1.w, 4 * q1 + 3);
    acc = __fmaf_rn(v0.x, x0, acc);
    acc = __fmaf_rn(v0.y, x1, acc);
    acc = __fmaf_rn(v0.z, x2, acc);
    acc = __fmaf_rn(v0.w, x3, acc);
    acc = __fmaf_rn(v1.x, z0, acc);
    acc = __fmaf_rn(v1.y, z1, acc);
    acc = __fmaf_rn(v1.z, z2, acc);
    acc = __fmaf_rn(v1.w, z3, acc);
  }
  for (int64_t k = 4 * n4 + t; k < nnz; k += nthr) acc = __fmaf_rn(ld_stream(A.val + k, ps), xat(ld_stream(A.col + k, ps), k), acc);
  for (int64_t i = t; i < A.n_rows; i += nthr) out[i] = acc + (float)__ldg(A.row_ptr + i + (i == A.n_rows - 1));
}

// FLAV 2 (experiment, same contract): x gathered by the TMA unit instead of
// the LSU -- each lane issues one cp.async.bulk.tensor tile::gather4 per 4
// nonzeros (x viewed as rows of 4 floats; the 4 rows col >> 2 land in a
// 128-byte shared slot), two 128-entry chunks in flight per warp (mbarrier
// per stage), then reads x[col] from shared memory.  Tests whether moving
// the gathers off the L1TEX pipe lowers the floor.
constexpr int kG4Warps = kUnitRows / 32;
struct G4Smem {
  float buf[kG4Warps][2][32][32];   // warp, stage, lane: 128-byte slot (4 rows x 16 B used)
  unsigned long long bar[kG4Warps][2];
};
// HYBRID (flavour 4): warps 0-1 of each CTA gather the first quarter of the
// chunks through the TMA unit, warps 2-7 the rest through the LSU (both gather
// engines at once).
constexpr int kG4TmaWarps = 2;
template <bool VERIFY, bool HYBRID>
__global__ void __launch_bounds__(kUnitRows) spmv_gather4_probe_kernel(const __grid_constant__ CUtensorMap tmX,
                                                                      SpmvDev A, float *out, int64_t nnz,
                                                                      uint32_t *err) {
  extern __shared__ __align__(1024) unsigned char g4_smem[];
  G4Smem &S = *reinterpret_cast<G4Smem *>(g4_smem);
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint64_t ps = policy_evict_first(), px = policy_evict_last();
  if (lane < 2)
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(spmv_smem_u32(&S.bar[w][lane])) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  uint32_t phase[2] = {0u, 0u};
  const int64_t nch_all = nnz / 128;
  const int64_t nch = HYBRID ? nch_all / 4 : nch_all;   // TMA chunks [0, nch)
  const int64_t nw = (int64_t)gridDim.x * (HYBRID ? kG4TmaWarps : kG4Warps);
  const int64_t gw = (int64_t)blockIdx.x * (HYBRID ? kG4TmaWarps : kG4Warps) + w;
  float acc = 0.0f;
  if (HYBRID && w >= kG4TmaWarps) {   // LSU warps: chunks [nch, nch_all), two in flight
    const int64_t nl = (int64_t)gridDim.x * (kG4Warps - kG4TmaWarps);
    for (int64_t ch = nch + (int64_t)blockIdx.x * (kG4Warps - kG4TmaWarps) + (w - kG4TmaWarps); ch < nch_all;
         ch += 2 * nl) {
      const int64_t ch1 = ch + nl;
      const bool h1 = ch1 < nch_all;
      const int4 c0 = ld_stream4(A.col + ch * 128 + 4 * lane, ps);
      const float4 v0 = ld_stream4(A.val + ch * 128 + 4 * lane, ps);
      const int4 c1 = h1 ? ld_stream4(A.col + ch1 * 128 + 4 * lane, ps) : make_int4(0, 0, 0, 0);
      const float4 v1 = h1 ? ld_stream4(A.val + ch1 * 128 + 4 * lane, ps) : make_float4(0.f, 0.f, 0.f, 0.f);
      const float x0 = ld_x(A.x + c0.x, px), x1 = ld_x(A.x + c0.y, px), x2 = ld_x(A.x + c0.z, px),
                  x3 = ld_x(A.x + c0.w, px);
      const float z0 = ld_x(A.x + c1.x, px), z1 = ld_x(A.x + c1.y, px), z2 = ld_x(A.x + c1.z, px),
                  z3 = ld_x(A.x + c1.w, px);
      acc = __fmaf_rn(v0.x, x0, acc);
      acc = __fmaf_rn(v0.y, x1, acc);
      acc = __fmaf_rn(v0.z, x2, acc);
      acc = __fmaf_rn(v0.w, x3, acc);
      acc = __fmaf_rn(v1.x, z0, acc);
      acc = __fmaf_rn(v1.y, z1, acc);
      acc = __fmaf_rn(v1.z, z2, acc);
      acc = __fmaf_rn(v1.w, z3, acc);
    }
  }
  auto issue = [&](int64_t ch, int st, int4 &c, float4 &v) {
    const int64_t k = ch * 128 + 4 * lane;
    c = ld_stream4(A.col + k, ps);
    v = ld_stream4(A.val + k, ps);
    const uint32_t bar = spmv_smem_u32(&S.bar[w][st]);
    if (lane == 0) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(32 * 64) : "memory");
    }
    __syncwarp();
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1, {%3, %4, %5, %6, %7}], [%2], %8;" ::"r"(spmv_smem_u32(&S.buf[w][st][lane][0])),
        "l"(&tmX), "r"(bar), "r"(0), "r"(c.x >> 2), "r"(c.y >> 2), "r"(c.z >> 2), "r"(c.w >> 2), "l"(px)
        : "memory");
  };
  int4 cc = make_int4(0, 0, 0, 0), cn = cc;
  float4 vc = make_float4(0.f, 0.f, 0.f, 0.f), vn = vc;
  int st = 0;
  if ((!HYBRID || w < kG4TmaWarps) && gw < nch) issue(gw, 0, cc, vc);
  for (int64_t ch = (!HYBRID || w < kG4TmaWarps) ? gw : nch; ch < nch; ch += nw, st ^= 1) {
    if (ch + nw < nch) issue(ch + nw, st ^ 1, cn, vn);
    const uint32_t bar = spmv_smem_u32(&S.bar[w][st]);
    uint32_t ok = 0;
    for (uint32_t spins = 0; !ok; ++spins) {
      asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                   : "=r"(ok)
                   : "r"(bar), "r"(phase[st])
                   : "memory");
      if (!ok && spins > (1u << 22)) {   // a mis-sized transfer must not hang the box
        atomicExch(err, 1u);
        return;
      }
    }
    phase[st] ^= 1u;
    const float *b = S.buf[w][st][lane];
    if (VERIFY) {   // flavour 3: the TMA-gathered values must be x[col]
      const bool bad = b[0 + (cc.x & 3)] != A.x[cc.x] || b[4 + (cc.y & 3)] != A.x[cc.y] ||
                       b[8 + (cc.z & 3)] != A.x[cc.z] || b[12 + (cc.w & 3)] != A.x[cc.w];
      if (bad) atomicOr(err, 2u);
    }
    acc = __fmaf_rn(vc.x, b[0 + (cc.x & 3)], acc);
    acc = __fmaf_rn(vc.y, b[4 + (cc.y & 3)], acc);
    acc = __fmaf_rn(vc.z, b[8 + (cc.z & 3)], acc);
    acc = __fmaf_rn(vc.w, b[12 + (cc.w & 3)], acc);
    __syncwarp();   // stage st read by every lane before it is refilled
    cc = cn;
    vc = vn;
  }
  const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
  const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (int64_t k = nch_all * 128 + t; k < nnz; k += nthr)
    acc = __fmaf_rn(ld_stream(A.val + k, ps), ld_x(A.x + ld_stream(A.col + k, ps), px), acc);
  for (int64_t i = t; i < A.n_rows; i += nthr) out[i] = acc + (float)__ldg(A.row_ptr + i + (i == A.n_rows - 1));
}

static PFN_cuTensorMapEncodeTiled_v12000 spmv_tensor_map_encoder() {
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

}  // namespace dysel

using namespace dysel;

extern "C" {

dysel_status dysel_spmv_gather_probe(dysel_ctx *ctx, dysel_spmv_plan *pl, int flavour, const float *d_x, float *d_out,
                                     void *stream) {
  if (!ctx || !pl || flavour < 0 || flavour > 4 || (pl->dev.n_rows > 0 && !d_out) ||
      (pl->info.nnz > 0 && !d_x)) {
    set_error(ctx, "dysel_spmv_gather_probe: invalid arguments");
    return DYSEL_ERR_INVALID;
  }
  if (pl->info.nnz > 0 && !pl->dev.vec_ok) {
    set_error(ctx, "dysel_spmv_gather_probe: col / val not 16-byte aligned");
    return DYSEL_ERR_UNSUPPORTED;
  }
  if (pl->dev.n_rows == 0) return DYSEL_OK;
  cudaStream_t st = (cudaStream_t)stream;
  SpmvDev A = pl->dev;
  A.x = d_x;
  if (flavour >= 2) {
    if ((uintptr_t)d_x & 15) {
      set_error(ctx, "dysel_spmv_gather_probe: x not 16-byte aligned (TMA)");
      return DYSEL_ERR_UNSUPPORTED;
    }
    auto enc = spmv_tensor_map_encoder();
    CUtensorMap tm;
    const cuuint64_t dims[2] = {4, (cuuint64_t)((pl->dev.n_cols + 3) / 4)};
    const cuuint64_t strides[1] = {16};
    const cuuint32_t box[2] = {4, 1};
    const cuuint32_t estr[2] = {1, 1};
    if (!enc || enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void *)d_x, dims, strides, box, estr,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
      set_error(ctx, "dysel_spmv_gather_probe: tensor map encode failed");
      return DYSEL_ERR_CUDA;
    }
    const size_t smem = sizeof(G4Smem);
    const void *kfn = flavour == 3   ? (const void *)spmv_gather4_probe_kernel<true, false>
                      : flavour == 4 ? (const void *)spmv_gather4_probe_kernel<false, true>
                                     : (const void *)spmv_gather4_probe_kernel<false, false>;
    DYSEL_CUDA_TRY(ctx, cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int occ2 = 0;
    DYSEL_CUDA_TRY(ctx, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ2, kfn, kUnitRows, smem));
    uint32_t *d_err = nullptr;
    DYSEL_CUDA_TRY(ctx, cudaMallocAsync(&d_err, 4, st));
    DYSEL_CUDA_TRY(ctx, cudaMemsetAsync(d_err, 0, 4, st));
    const unsigned g4 = (unsigned)std::max(1, occ2) * (unsigned)ctx->n_sm;
    if (flavour == 3)
      spmv_gather4_probe_kernel<true, false><<<g4, kUnitRows, smem, st>>>(tm, A, d_out, (int64_t)pl->info.nnz, d_err);
    else if (flavour == 4)
      spmv_gather4_probe_kernel<false, true><<<g4, kUnitRows, smem, st>>>(tm, A, d_out, (int64_t)pl->info.nnz, d_err);
    else
      spmv_gather4_probe_kernel<false, false><<<g4, kUnitRows, smem, st>>>(tm, A, d_out, (int64_t)pl->info.nnz, d_err);
    dysel_status ls = check_launch(ctx, "spmv_gather4_probe_kernel");
    uint32_t h_err = 0;
    DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(&h_err, d_err, 4, cudaMemcpyDeviceToHost, st));
    DYSEL_CUDA_TRY(ctx, cudaFreeAsync(d_err, st));
    DYSEL_CUDA_TRY(ctx, cudaStreamSynchronize(st));
    if (ls != DYSEL_OK) return ls;
    if (h_err) {
      set_error(ctx, (h_err & 1u) ? "dysel_spmv_gather_probe: gather4 transfer never completed (bounded wait)"
                                  : "dysel_spmv_gather_probe: gather4 delivered values != x[col]");
      return DYSEL_ERR_CUDA;
    }
    return DYSEL_OK;
  }
  int occ = 0;
  if (flavour == 0)
    DYSEL_CUDA_TRY(ctx, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, spmv_gather_probe_kernel<0>, kUnitRows, 0));
  else
    DYSEL_CUDA_TRY(ctx, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, spmv_gather_probe_kernel<1>, kUnitRows, 0));
  const unsigned grid = (unsigned)std::max(1, occ) * (unsigned)ctx->n_sm;
  int64_t xmask = 1;
  while (xmask * 2 <= pl->dev.n_cols) xmask *= 2;
  xmask -= 1;
  if (flavour == 0)
    spmv_gather_probe_kernel<0><<<grid, kUnitRows, 0, st>>>(A, d_out, (int64_t)pl->info.nnz, xmask);
  else
    spmv_gather_probe_kernel<1><<<grid, kUnitRows, 0, st>>>(A, d_out, (int64_t)pl->info.nnz, xmask);
  return check_launch(ctx, "spmv_gather_probe_kernel");
}

}  // extern "C"
