// DySel transposed SpMV pool: y += A^T x over the plan's CSR,
// the scatter-add kernel whose work-groups write OVERLAPPING outputs through
// global atomics.  Such a kernel cannot be split into productive slices that
// each own part of y, so the paper's only productive option is the swap-based
// partial-productive mode (§2.2, §3.3,
// Table 1): every variant profiles the SAME slice into a private
// copy of y (initialised from y), the winner's copy is swapped in, and the
// winner runs the rest.  Variants carry DYSEL_V_ATOMICS, so AUTO resolves to
// swap and SWAP|ASYNC is rejected by the planner.
//
// Unit = 256 consecutive rows of A (= entries of x), as for dysel_spmv.
//   V0 scatter-thread  thread per row, the row's entries in CSR order
//   V1 scatter-warp    warp per row (32 rows per warp, in order), the row's
//                      entries strided over the lanes: coalesced col/val loads
//   V2 scatter-segment warp per 32-row segment: the segment's nonzeros as one
//                      flat coalesced stream, 4 x 32 entries in flight per
//                      round, each entry's row found by a 5-step shuffle search
//                      over the lanes' row ends (no per-row serial chain)
// All issue one fire-and-forget `red.global.add.f32` per nonzero
// (y[col] += val * x[row]); the order of the reductions is not fixed, so the
// result equals the fp64 oracle within fp32 rounding, not bit for bit.
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>

#include "dysel_device.cuh"
#include "spmv_plan.h"

namespace dysel {

static const char *kSpmtvSig = "dysel.spmtv";
constexpr int kSpmtvRows = 256;

struct SpmtvArgs {
  int64_t n_rows;
  const int32_t *row_ptr;
  const int32_t *col;
  const float *val;
  const float *x;
};


// No memory clobber: lets the compiler batch the next entries' loads ahead of
// earlier reductions (the kernel never reads y).
__device__ __forceinline__ void red_add_nc(float *p, float v) {
  asm volatile("red.global.add.f32 [%0], %1;" ::"l"(p), "f"(v));
}

// Dominance (reading A-32) applies to swap too: a dominated variant's
// PRIVATE copy is discarded, so its CTAs stop at the next poll; the polls are
// CTA-uniform (dysel_prof_poll holds a barrier).
template <int VID>
__global__ void __launch_bounds__(256) spmtv_kernel(SpmtvArgs a, float *__restrict__ y, dysel_slice s) {
  __shared__ dysel_prof_smem psm;
  if (!dysel_gate_open(s)) return;
  const uint32_t wa[3] = {1, 1, 1};
  const bool persistent = s.timer == nullptr && s.gate != nullptr;   // gated remainder: one wave walks the units
  const bool timed = s.timer != nullptr;
  const uint64_t n_cta = persistent ? dysel_slice_ctas(s, wa) : (uint64_t)blockIdx.x + 1;
  dysel_prof_begin(s, psm);
  uint32_t units = 0;
  bool stop = false;
  for (uint64_t cta = blockIdx.x; cta < n_cta && !stop; cta += gridDim.x) {
    uint64_t u[3];
    if (!dysel_cta_origin(s, wa, cta, u)) continue;
    ++units;
    const int64_t r0 = (int64_t)u[0] * kSpmtvRows;
    if constexpr (VID == 0) {   // thread per row, entries in CSR order
      const int64_t r = r0 + threadIdx.x;
      int k = 0, e = 0;
      float xr = 0.0f;
      if (r < a.n_rows) {
        xr = __ldg(a.x + r);
        k = __ldg(a.row_ptr + r);
        e = __ldg(a.row_ptr + r + 1);
      }
      if (!timed) {   // batch / remainder copies: no barrier in the row loop
#pragma unroll 4
        for (; k < e; ++k) red_add_nc(y + __ldg(a.col + k), __fmul_rn(__ldg(a.val + k), xr));
        continue;
      }
      for (int it = 0;; ++it) {   // profiling copy: CTA-uniform chunks so it can poll
        const int stop_k = min(e, k + 32);
        for (; k < stop_k; ++k) red_add_nc(y + __ldg(a.col + k), __fmul_rn(__ldg(a.val + k), xr));
        if (!__syncthreads_or(k < e)) break;
        if ((it & 3) == 3 && dysel_prof_poll(s, psm) && s.role == DYSEL_ROLE_PRIVATE) {
          stop = true;
          break;
        }
      }
    } else if constexpr (VID == 2) {   // warp per 32-row segment, its nonzeros as one flat stream
      const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
      const int64_t rw = r0 + w * 32;   // first row of this warp's segment
      int seg_b = 0, end_l = 0;
      float xl = 0.0f;
      if (rw < a.n_rows) {
        const int64_t rl = min(rw + lane, a.n_rows - 1);
        seg_b = __ldg(a.row_ptr + rw);
        end_l = __ldg(a.row_ptr + rl + 1);   // lanes past n_rows repeat the last row's end
        xl = rw + lane < a.n_rows ? __ldg(a.x + rw + lane) : 0.0f;
      }
      const int seg_e = __shfl_sync(0xffffffffu, end_l, 31);
      int k = seg_b + lane;
      auto step = [&](int kk) {   // entry kk of the segment: its row by a 5-step shuffle search
        int pos = 0;
#pragma unroll
        for (int st = 16; st > 0; st >>= 1) {
          const int v = __shfl_sync(0xffffffffu, end_l, pos + st - 1);
          if (v <= kk) pos += st;
        }
        const float xr = __shfl_sync(0xffffffffu, xl, pos);
        if (kk < seg_e) red_add_nc(y + __ldg(a.col + kk), __fmul_rn(__ldg(a.val + kk), xr));
      };
      if (!timed) {
        for (; __any_sync(0xffffffffu, k < seg_e); k += 128) {
#pragma unroll
          for (int u = 0; u < 4; ++u) step(k + 32 * u);
        }
        continue;
      }
      for (int it = 0;; ++it, k += 128) {   // profiling copy: CTA-uniform rounds so it can poll
        if (__any_sync(0xffffffffu, k < seg_e)) {
#pragma unroll
          for (int u = 0; u < 4; ++u) step(k + 32 * u);
        }
        if (!__syncthreads_or(k + 128 < seg_e)) break;
        if ((it & 3) == 3 && dysel_prof_poll(s, psm) && s.role == DYSEL_ROLE_PRIVATE) {
          stop = true;
          break;
        }
      }
    } else {   // warp per row (32 rows per warp, in order), entries strided over the lanes
      const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
      const int64_t rl = r0 + w * 32 + lane;   // lane l holds row l's bounds and x: one load level for all 32
      int beg_l = 0, end_l = 0;
      float x_l = 0.0f;
      if (rl < a.n_rows) {
        beg_l = __ldg(a.row_ptr + rl);
        end_l = __ldg(a.row_ptr + rl + 1);
        x_l = __ldg(a.x + rl);
      }
      for (int i = 0; i < 32; ++i) {
        {
          const int b = __shfl_sync(0xffffffffu, beg_l, i), e = __shfl_sync(0xffffffffu, end_l, i);
          const float xr = __shfl_sync(0xffffffffu, x_l, i);
#pragma unroll 4
          for (int k = b + lane; k < e; k += 32)
            red_add_nc(y + __ldg(a.col + k), __fmul_rn(__ldg(a.val + k), xr));
        }
        if (timed && (i & 7) == 7 && dysel_prof_poll(s, psm) && s.role == DYSEL_ROLE_PRIVATE) {
          stop = true;
          break;
        }
      }
    }
  }
  dysel_prof_end(s, psm, persistent ? 0u : units);
}

static uint64_t g_spmtv_wave[DYSEL_SPMTV_NVARIANTS] = {0, 0, 0};   // occupancy x #SM
static const bool g_spmtv_persistent = getenv("DYSEL_SPMTV_PERSISTENT") != nullptr;   // ablation knob

template <int VID>
static dysel_status spmtv_variant_fn(const dysel_slice *s, void *const *args, void *stream, void *) {
  const SpmtvArgs &a = *(const SpmtvArgs *)args[1];
  float *y = (float *)args[0];
  static const uint32_t WA[3] = {1, 1, 1};
  uint64_t ctas = dysel_slice_ctas(*s, WA);
  if (ctas == 0) return DYSEL_OK;
  // gated remainder: a persistent wave only when asked (DYSEL_SPMTV_PERSISTENT);
  // by default the full grid, whose CTAs the block scheduler hands out
  // dynamically — skewed rows make a static round-robin walk imbalanced
  if (g_spmtv_persistent && s->gate && !s->timer && g_spmtv_wave[VID] > 0)
    ctas = std::min<uint64_t>(ctas, g_spmtv_wave[VID]);
  spmtv_kernel<VID><<<(unsigned)ctas, 256, 0, (cudaStream_t)stream>>>(a, y, *s);
  return cudaGetLastError() == cudaSuccess ? DYSEL_OK : DYSEL_ERR_CUDA;
}

static const dysel_variant_fn kSpmtvFns[DYSEL_SPMTV_NVARIANTS] = {spmtv_variant_fn<0>, spmtv_variant_fn<1>,
                                                                   spmtv_variant_fn<2>};

dysel_status spmtv_register(dysel_ctx *ctx) {
  static const int sb[1] = {0};
  int o[3] = {0, 0, 0};
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o[0], spmtv_kernel<0>, 256, 0);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o[1], spmtv_kernel<1>, 256, 0);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o[2], spmtv_kernel<2>, 256, 0);
  cudaGetLastError();
  const uint64_t n = (uint64_t)ctx->n_sm;
  for (int i = 0; i < DYSEL_SPMTV_NVARIANTS; ++i) g_spmtv_wave[i] = (uint64_t)o[i] * n;
  dysel_variant v[DYSEL_SPMTV_NVARIANTS] = {
      {"scatter_thread", kSpmtvFns[0], {1, 1, 1}, sb, 1, DYSEL_V_ATOMICS, nullptr, (uint64_t)o[0] * n},
      {"scatter_warp", kSpmtvFns[1], {1, 1, 1}, sb, 1, DYSEL_V_ATOMICS, nullptr, (uint64_t)o[1] * n},
      {"scatter_segment", kSpmtvFns[2], {1, 1, 1}, sb, 1, DYSEL_V_ATOMICS, nullptr, (uint64_t)o[2] * n},
  };
  // initial version: the default's gated remainder is launched
  // first at high priority, so the initial version should be the variant
  // that usually wins; warp per row (coalesced entry loads)
  const int def = getenv("DYSEL_SPMTV_DEFAULT_THREAD") ? DYSEL_SPMTV_SCATTER_THREAD : DYSEL_SPMTV_SCATTER_WARP;
  return dysel_register_variants(ctx, kSpmtvSig, v, DYSEL_SPMTV_NVARIANTS, def);
}

static dysel_status spmtv_check(dysel_ctx *ctx, dysel_spmv_plan *pl, const float *x, float *y) {
  if (!pl || pl->ctx != ctx || (pl->dev.n_rows > 0 && !x) || (pl->dev.n_cols > 0 && !y)) {
    set_error(ctx, "dysel_spmtv: invalid arguments");
    return DYSEL_ERR_INVALID;
  }
  return DYSEL_OK;
}

}  // namespace dysel

using namespace dysel;

extern "C" {

dysel_status dysel_spmtv(dysel_ctx *ctx, dysel_spmv_plan *pl, const float *d_x, float *d_y, float f, uint32_t mode,
                         void *stream, dysel_report *rep) {
  if (!ctx) return DYSEL_ERR_INVALID;
  DYSEL_TRY(spmtv_check(ctx, pl, d_x, d_y));
  if (rep) rep->n_slices = 0;
  if (pl->dev.n_rows == 0 || pl->info.nnz == 0) return DYSEL_OK;   // y += 0
  SpmtvArgs a{pl->dev.n_rows, pl->dev.row_ptr, pl->dev.col, pl->dev.val, d_x};
  const uint64_t U[3] = {(uint64_t)(pl->dev.n_rows + kSpmtvRows - 1) / kSpmtvRows, 1, 1};
  void *args[2] = {d_y, &a};
  const size_t sbytes[1] = {(size_t)pl->dev.n_cols * sizeof(float)};
  const std::string key = std::string(kSpmtvSig) + "#" + pl->sig;
  return launch_keyed(ctx, kSpmtvSig, key.c_str(), U, f, mode, args, 2, sbytes, stream, rep);
}

dysel_status dysel_spmtv_variant(dysel_ctx *ctx, dysel_spmv_plan *pl, int variant_id, const float *d_x, float *d_y,
                                 void *stream) {
  if (!ctx || variant_id < 0 || variant_id >= DYSEL_SPMTV_NVARIANTS) {
    set_error(ctx, "dysel_spmtv_variant: invalid variant");
    return DYSEL_ERR_INVALID;
  }
  DYSEL_TRY(spmtv_check(ctx, pl, d_x, d_y));
  if (pl->dev.n_rows == 0 || pl->info.nnz == 0) return DYSEL_OK;
  SpmtvArgs a{pl->dev.n_rows, pl->dev.row_ptr, pl->dev.col, pl->dev.val, d_x};
  void *args[2] = {d_y, &a};
  dysel_slice s;
  memset(&s, 0, sizeof(s));
  s.g[0] = s.g[1] = s.g[2] = 1;
  s.U[0] = (uint64_t)(pl->dev.n_rows + kSpmtvRows - 1) / kSpmtvRows;
  s.U[1] = s.U[2] = 1;
  s.G[0] = (uint32_t)s.U[0];
  s.G[1] = s.G[2] = 1;
  s.granule_count = s.U[0];
  s.granule_stride = 1;
  s.role = DYSEL_ROLE_BATCH;
  s.variant = variant_id;
  DYSEL_TRY(kSpmtvFns[variant_id](&s, args, stream, nullptr));
  return check_launch(ctx, "spmtv full-grid variant");
}

}  // extern "C"
