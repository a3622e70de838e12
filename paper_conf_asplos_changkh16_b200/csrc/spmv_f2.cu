// data-placement and optimisation-combination variant pools
// of SpMV, selected at run time through the generic launcher (dysel_launch:
// the same slice planner, device timing, dominance and gated remainder as
// user-registered kernels).
//
// Case II (§4.2, "four data placement policies ... selected at
// runtime" for spmv-csr): one CSR-scalar kernel (SHOC spmv-csr, thread per
// row, CSR-order fmaf from +0) in four placements of x:
//   0 x_ldg      x through the read-only L1 path (ld.global.nc, L2 evict_last)
//   1 x_l2       x through L2 only (ld.global.cg: no L1 allocation)
//   2 x_smem     the unit's x window [min col, max col] staged into shared
//                memory by the bulk-copy engine (cp.async.bulk + mbarrier);
//                rows then gather x from shared memory (banded matrices);
//                a unit whose window exceeds kXWinMax falls back to 0
//   3 x_persist  as 0, launched with an L2 access-policy window that marks x
//                persisting (cudaLaunchAttributeAccessPolicyWindow)
// All four compute every row in the same order: bit-identical to each other
// and to the main pool's CSR-S / ELL / JDS.
//
// Case III (§4.3: Parboil spmv-jds, four GPU
// versions combining unrolling / prefetching; DySel picked the 2nd best by
// 0.8%): a GLOBAL-sort JDS (rows sorted by length over the whole matrix,
// reading A-14 keeps the main pool block-local, so this is its own pool whose
// units are 256 permuted rows) in four versions:
//   0 plain      one diagonal per iteration, dependent loads
//   1 unroll     4 diagonals per iteration (loads issued together)
//   2 prefetch   the next diagonal's jd_ptr / col / val loaded while the
//                current one is accumulated
//   3 unroll+prefetch
// Every version sums a row's entries in k order with fmaf from +0 = CSR order:
// bit-identical to each other and to CSR-S.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include <algorithm>
#include <cstring>
#include <string>
#include <vector>

#include "dysel_device.cuh"
#include "spmv_plan.h"

// ------------------------------------------------------------ global JDS plan
struct dysel_spmv_jds_plan {
  dysel_ctx *ctx = nullptr;
  int64_t n_rows = 0, n_cols = 0, nnz = 0;
  int32_t W = 0;
  int32_t *perm = nullptr;    // [n]   position -> row
  int32_t *len = nullptr;     // [n]   length of row perm[p]
  int32_t *jd_ptr = nullptr;  // [W+1]
  int32_t *col = nullptr;     // [nnz] entry (p, k) at jd_ptr[k] + p
  float *val = nullptr;
  uint64_t prep_ns = 0;
  std::string sig;
};

namespace dysel {

constexpr int kXWinMax = 12288;   // x_smem: floats of x window per unit (48 KB)
constexpr int kPlaceRows = 256;

struct PlaceArgs {
  SpmvDev A;
  const int2 *win;   // per unit [min col, max col] (x_smem)
};

__device__ __forceinline__ float ld_x_cg(const float *p) {
  float v;
  asm volatile("ld.global.cg.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
}

// x_smem staging buffer + its mbarrier (dynamic shared memory)
struct XWinSmem {
  unsigned long long bar;
  unsigned long long pad[15];   // 128-byte aligned window
  float x[kXWinMax];
};

template <int PL>
__global__ void __launch_bounds__(kPlaceRows) spmv_place_kernel(PlaceArgs a, float *__restrict__ y, dysel_slice s) {
  extern __shared__ __align__(128) unsigned char place_dsmem[];
  __shared__ dysel_prof_smem psm;
  if (!dysel_gate_open(s)) return;
  XWinSmem &W = *reinterpret_cast<XWinSmem *>(place_dsmem);
  if (PL == 2 && threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(&W.bar)) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  dysel_prof_begin(s, psm);
  const SpmvDev &A = a.A;
  const uint64_t px = policy_evict_last();
  uint32_t phase = 0;
  uint32_t units = 0;
  // one unit per CTA; the gated remainder (no timer) is one persistent wave
  const uint64_t n_cta = (s.timer == nullptr && s.gate != nullptr) ? s.granule_count : (uint64_t)blockIdx.x + 1;
  for (uint64_t b = blockIdx.x; b < n_cta; b += gridDim.x) {
    const uint32_t j = (uint32_t)(s.granule_begin + b * s.granule_stride);
    if ((uint64_t)j >= s.U[0]) continue;
    ++units;
    const int64_t r = (int64_t)j * kPlaceRows + threadIdx.x;
    int lo = 0, hi = -1;
    bool smem = false;
    if constexpr (PL == 2) {
      const int2 w = a.win[j];
      const int a0 = w.x & ~3;                                     // 16-byte aligned window start
      const int a1 = min(A.n_cols, (w.y + 4) & ~3);                // end (exclusive), rounded up in range
      // (the bulk copy needs a 16-byte aligned source: an unaligned x gathers from global memory)
      smem = w.y >= w.x && a1 - a0 <= kXWinMax && ((uintptr_t)A.x & 15) == 0;
      if (smem) {
        lo = a0;
        hi = a1;
        __syncthreads();   // the previous unit's readers are done with the window
        const int nb = (hi - lo) & ~3;   // bulk part (multiple of 16 bytes); tail by threads
        const uint32_t bar = (uint32_t)__cvta_generic_to_shared(&W.bar);
        if (threadIdx.x == 0) {
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(nb * 4) : "memory");
          if (nb > 0)
            asm volatile(
                "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                    (uint32_t)__cvta_generic_to_shared(&W.x[0])),
                "l"(A.x + lo), "r"(nb * 4), "r"(bar)
                : "memory");
        }
        for (int i = nb + threadIdx.x; i < hi - lo; i += blockDim.x) W.x[i] = __ldg(A.x + lo + i);
        uint32_t ok = 0;
        while (!ok)
          asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                       : "=r"(ok)
                       : "r"(bar), "r"(phase)
                       : "memory");
        phase ^= 1u;
        __syncthreads();   // tail entries stored
      }
    }
    if (r < A.n_rows) {
      const int kb = __ldg(A.row_ptr + r), ke = __ldg(A.row_ptr + r + 1);
      float acc = 0.0f;
      for (int k = kb; k < ke; k += 8) {
        int c[8];
        float v[8], xv[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          const bool ok = k + u < ke;
          c[u] = ok ? __ldg(A.col + k + u) : 0;
          v[u] = ok ? __ldg(A.val + k + u) : 0.0f;
        }
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          if (k + u >= ke) {
            xv[u] = 0.0f;
          } else if constexpr (PL == 1) {
            xv[u] = ld_x_cg(A.x + c[u]);
          } else if constexpr (PL == 2) {
            xv[u] = smem ? W.x[c[u] - lo] : ld_x(A.x + c[u], px);
          } else {
            xv[u] = ld_x(A.x + c[u], px);
          }
        }
#pragma unroll
        for (int u = 0; u < 8; ++u)
          if (k + u < ke) acc = __fmaf_rn(v[u], xv[u], acc);
      }
      y[r] = acc;
    }
  }
  dysel_prof_end(s, psm, units);
}

__global__ void unit_window_kernel(const int32_t *__restrict__ rp, const int32_t *__restrict__ col, int64_t n,
                                   int64_t nu, int2 *__restrict__ win) {
  const int64_t u = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (u >= nu) return;
  const int a = rp[u * kPlaceRows], b = rp[min((u + 1) * kPlaceRows, n)];
  int lo = 0x7fffffff, hi = -1;
  for (int k = a + lane; k < b; k += 32) {
    const int c = col[k];
    lo = min(lo, c);
    hi = max(hi, c);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    lo = min(lo, __shfl_xor_sync(0xffffffffu, lo, o));
    hi = max(hi, __shfl_xor_sync(0xffffffffu, hi, o));
  }
  if (lane == 0) win[u] = b > a ? make_int2(lo, hi) : make_int2(0, -1);
}

static int g_place_occ[4] = {0, 0, 0, 0};
static size_t place_smem_bytes(int pl) { return pl == 2 ? sizeof(XWinSmem) : 0; }

template <int PL>
static dysel_status place_variant_fn(const dysel_slice *s, void *const *args, void *stream, void *user) {
  dysel_spmv_plan *pl = (dysel_spmv_plan *)user;
  if (s->granule_count == 0) return DYSEL_OK;
  PlaceArgs a{pl->dev, (const int2 *)pl->xwin};
  a.A.x = (const float *)args[1];
  uint64_t grid = s->granule_count;
  if (s->timer == nullptr && s->gate != nullptr && !s->gate_full_grid && g_place_occ[PL] > 0)   // likely loser: one wave
    grid = std::min<uint64_t>(grid, (uint64_t)g_place_occ[PL] * pl->ctx->n_sm);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(kPlaceRows);
  cfg.dynamicSmemBytes = place_smem_bytes(PL);
  cfg.stream = (cudaStream_t)stream;
  cudaLaunchAttribute attr[1];
  if (PL == 3) {   // x persisting in L2 (the ctx reserved the persisting set-aside, dysel_spmv_placement)
    const size_t xb = (size_t)pl->dev.n_cols * sizeof(float);
    attr[0].id = cudaLaunchAttributeAccessPolicyWindow;
    attr[0].val.accessPolicyWindow.base_ptr = (void *)a.A.x;
    attr[0].val.accessPolicyWindow.num_bytes = std::min<size_t>(xb, pl->ctx->l2_persist_window);
    attr[0].val.accessPolicyWindow.hitRatio =
        xb ? (float)std::min<double>(1.0, (double)pl->ctx->l2_persist_bytes / (double)std::max<size_t>(xb, 1)) : 1.0f;
    attr[0].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
    attr[0].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    cfg.attrs = attr;
    cfg.numAttrs = pl->ctx->l2_persist_bytes > 0 ? 1 : 0;
  }
  return cudaLaunchKernelEx(&cfg, spmv_place_kernel<PL>, a, (float *)args[0], *s) == cudaSuccess ? DYSEL_OK
                                                                                                 : DYSEL_ERR_CUDA;
}

static const dysel_variant_fn kPlaceFns[DYSEL_SPMV_PLACE_NVARIANTS] = {place_variant_fn<0>, place_variant_fn<1>,
                                                                      place_variant_fn<2>, place_variant_fn<3>};
static const char *kPlaceNames[DYSEL_SPMV_PLACE_NVARIANTS] = {"x_ldg", "x_l2", "x_smem", "x_persist"};

static dysel_status place_init(dysel_ctx *ctx) {
  static bool done = false;
  if (done) return DYSEL_OK;
  const void *k[4] = {(const void *)spmv_place_kernel<0>, (const void *)spmv_place_kernel<1>,
                      (const void *)spmv_place_kernel<2>, (const void *)spmv_place_kernel<3>};
  for (int i = 0; i < 4; ++i) {
    if (place_smem_bytes(i) > 48 * 1024)
      DYSEL_CUDA_TRY(ctx, cudaFuncSetAttribute(k[i], cudaFuncAttributeMaxDynamicSharedMemorySize, (int)place_smem_bytes(i)));
    DYSEL_CUDA_TRY(ctx, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&g_place_occ[i], k[i], kPlaceRows, place_smem_bytes(i)));
  }
  done = true;
  return DYSEL_OK;
}

// The placement pool of a plan: per-unit x windows (built once), the L2
// persisting set-aside (once per ctx), registration under the plan's sig.
static dysel_status place_pool(dysel_ctx *ctx, dysel_spmv_plan *pl, cudaStream_t st) {
  DYSEL_TRY(place_init(ctx));
  if (!pl->place_sig.empty()) return DYSEL_OK;
  const int64_t nu = pl->n_units;
  if (nu > 0) {
    DYSEL_CUDA_TRY(ctx, cudaMalloc(&pl->xwin, nu * sizeof(int2)));
    unit_window_kernel<<<(unsigned)((nu * 32 + 255) / 256), 256, 0, st>>>(pl->dev.row_ptr, pl->dev.col,
                                                                        pl->dev.n_rows, nu, (int2 *)pl->xwin);
    DYSEL_TRY(check_launch(ctx, "unit_window_kernel"));
  }
  {   // persisting L2 set-aside for x (placement 3): a DEVICE-wide limit that
      // takes that much L2 from every other kernel (measured: a full-size
      // set-aside slowed a later L2-sized stencil 2x), so it is sized to this
      // plan's x (1 MB granules), grown only when a plan needs more, and
      // released when the ctx is destroyed
    int maxp = 0, maxw = 0;
    cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, ctx->device);
    cudaDeviceGetAttribute(&maxw, cudaDevAttrMaxAccessPolicyWindowSize, ctx->device);
    const size_t want = std::min<size_t>((size_t)std::max(maxp, 0),
                                         ((size_t)pl->dev.n_cols * sizeof(float) + (1u << 20) - 1) & ~(size_t)((1u << 20) - 1));
    if (maxw > 0 && want > ctx->l2_persist_bytes &&
        cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, want) == cudaSuccess) {
      ctx->l2_persist_bytes = want;
      ctx->l2_persist_window = (size_t)maxw;
    }
    cudaGetLastError();
  }
  static const int sb[1] = {0};
  dysel_variant vv[DYSEL_SPMV_PLACE_NVARIANTS];
  for (int i = 0; i < DYSEL_SPMV_PLACE_NVARIANTS; ++i)
    vv[i] = dysel_variant{kPlaceNames[i], kPlaceFns[i], {1, 1, 1}, sb, 1,
                          pl->info.uniform ? 0u : (uint32_t)DYSEL_V_NONUNIFORM, pl,
                          (uint64_t)std::max(1, g_place_occ[i]) * ctx->n_sm};
  const std::string sig = pl->sig + "/placement";
  DYSEL_TRY(dysel_register_variants(ctx, sig.c_str(), vv, DYSEL_SPMV_PLACE_NVARIANTS, DYSEL_SPMV_PLACE_LDG));
  mark_builtin(ctx, sig.c_str());
  pl->place_sig = sig;
  return DYSEL_OK;
}

// ------------------------------------------------------------- global JDS
struct JdsArgs {
  int64_t n;
  const int32_t *perm, *len, *jd_ptr, *col;
  const float *val, *x;
};

template <bool UNROLL, bool PREFETCH>
__global__ void __launch_bounds__(256) jds_global_kernel(JdsArgs a, float *__restrict__ y, dysel_slice s) {
  __shared__ dysel_prof_smem psm;
  if (!dysel_gate_open(s)) return;
  dysel_prof_begin(s, psm);
  uint32_t units = 0;
  const uint64_t n_cta = (s.timer == nullptr && s.gate != nullptr) ? s.granule_count : (uint64_t)blockIdx.x + 1;
  for (uint64_t b = blockIdx.x; b < n_cta; b += gridDim.x) {
    const uint64_t j = s.granule_begin + b * s.granule_stride;
    if (j >= s.U[0]) continue;
    ++units;
    const int64_t p = (int64_t)j * 256 + threadIdx.x;
    if (p >= a.n) continue;
    const int L = __ldg(a.len + p);
    float acc = 0.0f;
    if constexpr (!UNROLL && !PREFETCH) {
      for (int k = 0; k < L; ++k) {
        const int64_t e = (int64_t)__ldg(a.jd_ptr + k) + p;
        acc = __fmaf_rn(__ldg(a.val + e), __ldg(a.x + __ldg(a.col + e)), acc);
      }
    } else if constexpr (UNROLL && !PREFETCH) {
      int k = 0;
      for (; k + 4 <= L; k += 4) {
        int64_t e[4];
        int c[4];
        float v[4], xv[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) e[u] = (int64_t)__ldg(a.jd_ptr + k + u) + p;
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          c[u] = __ldg(a.col + e[u]);
          v[u] = __ldg(a.val + e[u]);
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) xv[u] = __ldg(a.x + c[u]);
#pragma unroll
        for (int u = 0; u < 4; ++u) acc = __fmaf_rn(v[u], xv[u], acc);
      }
      for (; k < L; ++k) {
        const int64_t e = (int64_t)__ldg(a.jd_ptr + k) + p;
        acc = __fmaf_rn(__ldg(a.val + e), __ldg(a.x + __ldg(a.col + e)), acc);
      }
    } else if constexpr (!UNROLL && PREFETCH) {
      if (L > 0) {
        int64_t e = (int64_t)__ldg(a.jd_ptr) + p;
        int c = __ldg(a.col + e);
        float v = __ldg(a.val + e);
        for (int k = 0; k < L; ++k) {
          int cn = 0;
          float vn = 0.0f;
          if (k + 1 < L) {   // next diagonal's entry in flight while this one is accumulated
            const int64_t en = (int64_t)__ldg(a.jd_ptr + k + 1) + p;
            cn = __ldg(a.col + en);
            vn = __ldg(a.val + en);
          }
          acc = __fmaf_rn(v, __ldg(a.x + c), acc);
          c = cn;
          v = vn;
        }
      }
    } else {   // unroll 4 + prefetch of the next group
      int cc[4];
      float vv[4];
      auto fetch = [&](int k) {
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const bool ok = k + u < L;
          const int64_t e = ok ? (int64_t)__ldg(a.jd_ptr + k + u) + p : 0;
          cc[u] = ok ? __ldg(a.col + e) : 0;
          vv[u] = ok ? __ldg(a.val + e) : 0.0f;
        }
      };
      if (L > 0) fetch(0);
      for (int k = 0; k < L; k += 4) {
        int c[4];
        float v[4], xv[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          c[u] = cc[u];
          v[u] = vv[u];
        }
        if (k + 4 < L) fetch(k + 4);
#pragma unroll
        for (int u = 0; u < 4; ++u) xv[u] = k + u < L ? __ldg(a.x + c[u]) : 0.0f;
#pragma unroll
        for (int u = 0; u < 4; ++u)
          if (k + u < L) acc = __fmaf_rn(v[u], xv[u], acc);
      }
    }
    y[__ldg(a.perm + p)] = acc;
  }
  dysel_prof_end(s, psm, units);
}

static int g_jds_occ[4] = {0, 0, 0, 0};

template <int V>
static dysel_status jds_variant_fn(const dysel_slice *s, void *const *args, void *stream, void *user) {
  const dysel_spmv_jds_plan *jp = (const dysel_spmv_jds_plan *)user;
  if (s->granule_count == 0) return DYSEL_OK;
  JdsArgs a{jp->n_rows, jp->perm, jp->len, jp->jd_ptr, jp->col, jp->val, (const float *)args[1]};
  uint64_t grid = s->granule_count;
  if (s->timer == nullptr && s->gate != nullptr && !s->gate_full_grid && g_jds_occ[V] > 0)
    grid = std::min<uint64_t>(grid, (uint64_t)g_jds_occ[V] * jp->ctx->n_sm);
  cudaStream_t st = (cudaStream_t)stream;
  float *y = (float *)args[0];
  if constexpr (V == 0) jds_global_kernel<false, false><<<(unsigned)grid, 256, 0, st>>>(a, y, *s);
  else if constexpr (V == 1) jds_global_kernel<true, false><<<(unsigned)grid, 256, 0, st>>>(a, y, *s);
  else if constexpr (V == 2) jds_global_kernel<false, true><<<(unsigned)grid, 256, 0, st>>>(a, y, *s);
  else jds_global_kernel<true, true><<<(unsigned)grid, 256, 0, st>>>(a, y, *s);
  return cudaGetLastError() == cudaSuccess ? DYSEL_OK : DYSEL_ERR_CUDA;
}

static const dysel_variant_fn kJdsFns[DYSEL_SPMV_JDS_NVARIANTS] = {jds_variant_fn<0>, jds_variant_fn<1>,
                                                                  jds_variant_fn<2>, jds_variant_fn<3>};
static const char *kJdsNames[DYSEL_SPMV_JDS_NVARIANTS] = {"jds_plain", "jds_unroll", "jds_prefetch",
                                                         "jds_unroll_prefetch"};

// global JDS construction: jd_ptr[k] = sum_{k' < k} #{p : len_p > k'}
__global__ void gjds_len_kernel(const int32_t *__restrict__ rp, int64_t n, int32_t *__restrict__ len,
                                int32_t *__restrict__ rows) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) {
    len[i] = rp[i + 1] - rp[i];
    rows[i] = (int32_t)i;
  }
}
// cnt[k] = #{p : slen_p > k} on the descending-sorted lengths
__global__ void gjds_count_kernel(const int32_t *__restrict__ slen, int64_t n, int32_t W, int32_t *__restrict__ cnt) {
  const int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= W) return;
  int64_t lo = 0, hi = n;   // first position with slen <= k (slen descending)
  while (lo < hi) {
    const int64_t m = (lo + hi) >> 1;
    if (slen[m] > k)
      lo = m + 1;
    else
      hi = m;
  }
  cnt[k] = (int32_t)lo;
}
__global__ void gjds_fill_kernel(const int32_t *__restrict__ rp, const int32_t *__restrict__ col,
                                 const float *__restrict__ val, int64_t n, const int32_t *__restrict__ perm,
                                 const int32_t *__restrict__ jd_ptr, int32_t *__restrict__ jc, float *__restrict__ jv) {
  const int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= n) return;
  const int r = perm[p];
  const int b = rp[r], e = rp[r + 1];
  for (int k = 0; k < e - b; ++k) {
    const int64_t idx = (int64_t)jd_ptr[k] + p;
    jc[idx] = col[b + k];
    jv[idx] = val[b + k];
  }
}

}  // namespace dysel

using namespace dysel;

extern "C" {

dysel_status dysel_spmv_placement(dysel_ctx *ctx, dysel_spmv_plan *pl, const float *d_x, float *d_y, float f,
                                  uint32_t mode, void *stream, dysel_report *rep) {
  if (!ctx || !pl || pl->ctx != ctx || (pl->dev.n_rows > 0 && (!d_y || (pl->dev.n_cols > 0 && !d_x)))) {
    set_error(ctx, "dysel_spmv_placement: invalid arguments");
    return DYSEL_ERR_INVALID;
  }
  if (rep) rep->n_slices = 0;
  if (pl->dev.n_rows == 0) return DYSEL_OK;
  DYSEL_TRY(place_pool(ctx, pl, (cudaStream_t)stream));
  const uint64_t U[3] = {pl->n_units, 1, 1};
  void *args[2] = {d_y, (void *)d_x};
  const size_t sb[1] = {(size_t)pl->dev.n_rows * sizeof(float)};
  return dysel_launch(ctx, pl->place_sig.c_str(), U, f, mode, args, 2, sb, stream, rep);
}

dysel_status dysel_spmv_placement_variant(dysel_ctx *ctx, dysel_spmv_plan *pl, int variant_id, const float *d_x,
                                          float *d_y, void *stream) {
  if (!ctx || !pl || pl->ctx != ctx || variant_id < 0 || variant_id >= DYSEL_SPMV_PLACE_NVARIANTS ||
      (pl->dev.n_rows > 0 && (!d_y || (pl->dev.n_cols > 0 && !d_x)))) {
    set_error(ctx, "dysel_spmv_placement_variant: invalid arguments");
    return DYSEL_ERR_INVALID;
  }
  if (pl->dev.n_rows == 0) return DYSEL_OK;
  DYSEL_TRY(place_pool(ctx, pl, (cudaStream_t)stream));
  void *args[2] = {d_y, (void *)d_x};
  dysel_slice s;
  memset(&s, 0, sizeof(s));
  s.g[0] = s.g[1] = s.g[2] = 1;
  s.U[0] = pl->n_units;
  s.U[1] = s.U[2] = 1;
  s.G[0] = pl->n_units;
  s.G[1] = s.G[2] = 1;
  s.granule_count = pl->n_units;
  s.granule_stride = 1;
  s.role = DYSEL_ROLE_BATCH;
  s.variant = variant_id;
  DYSEL_TRY(kPlaceFns[variant_id](&s, args, stream, pl));
  return check_launch(ctx, "spmv placement variant");
}

dysel_status dysel_spmv_placement_windows(const dysel_spmv_plan *pl, int32_t *h_win, size_t cap_units) {
  if (!pl || !h_win) return DYSEL_ERR_INVALID;
  if (!pl->xwin) return DYSEL_ERR_NOT_FOUND;
  const size_t n = std::min<size_t>(cap_units, pl->n_units);
  return cudaMemcpy(h_win, pl->xwin, n * sizeof(int2), cudaMemcpyDeviceToHost) == cudaSuccess ? DYSEL_OK
                                                                                             : DYSEL_ERR_CUDA;
}

dysel_status dysel_spmv_jds_prepare(dysel_ctx *ctx, int64_t n_rows, int64_t n_cols, int64_t nnz,
                                    const int32_t *d_row_ptr, const int32_t *d_col, const float *d_val, void *stream,
                                    dysel_spmv_jds_plan **out) {
  if (!ctx || !out || n_rows < 0 || n_cols < 0 || nnz < 0 || nnz >= (1ll << 31) || n_rows >= (1ll << 31) ||
      (n_rows > 0 && !d_row_ptr) || (nnz > 0 && (!d_col || !d_val))) {
    set_error(ctx, "dysel_spmv_jds_prepare: invalid arguments");
    return DYSEL_ERR_INVALID;
  }
  *out = nullptr;
  const uint64_t t0 = now_ns();
  cudaStream_t st = (cudaStream_t)stream;
  dysel_spmv_jds_plan *jp = new dysel_spmv_jds_plan();
  jp->ctx = ctx;
  jp->n_rows = n_rows;
  jp->n_cols = n_cols;
  jp->nnz = nnz;
  auto fail = [&](dysel_status s) {
    dysel_spmv_jds_plan_destroy(jp);
    return s;
  };
  if (n_rows > 0) {
    int32_t *len0 = nullptr, *rows0 = nullptr;
    void *tmp = nullptr;
    size_t tb = 0;
    if (cudaMalloc(&len0, n_rows * 4) != cudaSuccess || cudaMalloc(&rows0, n_rows * 4) != cudaSuccess ||
        cudaMalloc(&jp->len, n_rows * 4) != cudaSuccess || cudaMalloc(&jp->perm, n_rows * 4) != cudaSuccess)
      return fail(DYSEL_ERR_NOMEM);
    gjds_len_kernel<<<(unsigned)((n_rows + 255) / 256), 256, 0, st>>>(d_row_ptr, n_rows, len0, rows0);
    // stable descending sort of (length, row): ties keep row order (reading: Parboil's sort is stable)
    cub::DeviceRadixSort::SortPairsDescending(nullptr, tb, len0, jp->len, rows0, jp->perm, (int)n_rows, 0, 32, st);
    if (cudaMalloc(&tmp, std::max<size_t>(tb, 1)) != cudaSuccess) return fail(DYSEL_ERR_NOMEM);
    cub::DeviceRadixSort::SortPairsDescending(tmp, tb, len0, jp->len, rows0, jp->perm, (int)n_rows, 0, 32, st);
    int32_t W = 0;
    cudaMemcpyAsync(&W, jp->len, 4, cudaMemcpyDeviceToHost, st);
    const bool ok = cudaStreamSynchronize(st) == cudaSuccess;
    cudaFree(tmp);
    cudaFree(len0);
    cudaFree(rows0);
    if (!ok) return fail(DYSEL_ERR_CUDA);
    jp->W = W;
    int32_t *cnt = nullptr;
    if (cudaMalloc(&jp->jd_ptr, (size_t)(W + 1) * 4) != cudaSuccess || cudaMalloc(&cnt, std::max(W, 1) * 4) != cudaSuccess)
      return fail(DYSEL_ERR_NOMEM);
    if (W > 0) {
      gjds_count_kernel<<<(unsigned)((W + 255) / 256), 256, 0, st>>>(jp->len, n_rows, W, cnt);
      size_t tb2 = 0;
      void *tmp2 = nullptr;
      cudaMemsetAsync(jp->jd_ptr, 0, 4, st);
      cub::DeviceScan::InclusiveSum(nullptr, tb2, cnt, jp->jd_ptr + 1, W, st);
      if (cudaMalloc(&tmp2, std::max<size_t>(tb2, 1)) != cudaSuccess) return fail(DYSEL_ERR_NOMEM);
      cub::DeviceScan::InclusiveSum(tmp2, tb2, cnt, jp->jd_ptr + 1, W, st);
      if (cudaStreamSynchronize(st) != cudaSuccess) return fail(DYSEL_ERR_CUDA);
      cudaFree(tmp2);
    } else {
      cudaMemsetAsync(jp->jd_ptr, 0, 4, st);
    }
    cudaFree(cnt);
    if (nnz > 0) {
      if (cudaMalloc(&jp->col, nnz * 4) != cudaSuccess || cudaMalloc(&jp->val, nnz * 4) != cudaSuccess)
        return fail(DYSEL_ERR_NOMEM);
      gjds_fill_kernel<<<(unsigned)((n_rows + 255) / 256), 256, 0, st>>>(d_row_ptr, d_col, d_val, n_rows, jp->perm,
                                                                        jp->jd_ptr, jp->col, jp->val);
    }
    if (check_launch(ctx, "global JDS build") != DYSEL_OK || cudaStreamSynchronize(st) != cudaSuccess)
      return fail(DYSEL_ERR_CUDA);
  }
  for (int v = 0; v < DYSEL_SPMV_JDS_NVARIANTS; ++v) {
    if (g_jds_occ[v]) continue;
    const void *k[4] = {(const void *)jds_global_kernel<false, false>, (const void *)jds_global_kernel<true, false>,
                        (const void *)jds_global_kernel<false, true>, (const void *)jds_global_kernel<true, true>};
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&g_jds_occ[v], k[v], 256, 0);
  }
  cudaGetLastError();
  // the pool: four versions of one kernel over permuted-row units; rows sorted
  // by length make the units non-uniform unless every row has the same length
  jp->sig = "dysel.spmv.jds_global#" + std::to_string(++ctx->plan_serial);
  static const int sb[1] = {0};
  dysel_variant vv[DYSEL_SPMV_JDS_NVARIANTS];
  int32_t lmax = 0, lmin = 0;
  if (n_rows > 0) {
    cudaMemcpy(&lmax, jp->len, 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(&lmin, jp->len + n_rows - 1, 4, cudaMemcpyDeviceToHost);
  }
  const uint32_t fl = (lmax == lmin) ? 0u : (uint32_t)DYSEL_V_NONUNIFORM;
  for (int i = 0; i < DYSEL_SPMV_JDS_NVARIANTS; ++i)
    vv[i] = dysel_variant{kJdsNames[i], kJdsFns[i], {1, 1, 1}, sb, 1, fl, jp,
                          (uint64_t)std::max(1, g_jds_occ[i]) * ctx->n_sm};
  dysel_status rs = dysel_register_variants(ctx, jp->sig.c_str(), vv, DYSEL_SPMV_JDS_NVARIANTS,
                                            DYSEL_SPMV_JDS_UNROLL_PREFETCH);
  if (rs != DYSEL_OK) return fail(rs);
  mark_builtin(ctx, jp->sig.c_str());
  jp->prep_ns = now_ns() - t0;
  *out = jp;
  return DYSEL_OK;
}

dysel_status dysel_spmv_jds(dysel_ctx *ctx, dysel_spmv_jds_plan *jp, const float *d_x, float *d_y, float f,
                            uint32_t mode, void *stream, dysel_report *rep) {
  if (!ctx || !jp || jp->ctx != ctx || (jp->n_rows > 0 && (!d_y || (jp->n_cols > 0 && !d_x)))) {
    set_error(ctx, "dysel_spmv_jds: invalid arguments");
    return DYSEL_ERR_INVALID;
  }
  if (rep) rep->n_slices = 0;
  if (jp->n_rows == 0) return DYSEL_OK;
  const uint64_t U[3] = {(uint64_t)(jp->n_rows + 255) / 256, 1, 1};
  void *args[2] = {d_y, (void *)d_x};
  const size_t sb[1] = {(size_t)jp->n_rows * sizeof(float)};
  return dysel_launch(ctx, jp->sig.c_str(), U, f, mode, args, 2, sb, stream, rep);
}

dysel_status dysel_spmv_jds_variant(dysel_ctx *ctx, dysel_spmv_jds_plan *jp, int variant_id, const float *d_x,
                                    float *d_y, void *stream) {
  if (!ctx || !jp || jp->ctx != ctx || variant_id < 0 || variant_id >= DYSEL_SPMV_JDS_NVARIANTS ||
      (jp->n_rows > 0 && (!d_y || (jp->n_cols > 0 && !d_x)))) {
    set_error(ctx, "dysel_spmv_jds_variant: invalid arguments");
    return DYSEL_ERR_INVALID;
  }
  if (jp->n_rows == 0) return DYSEL_OK;
  void *args[2] = {d_y, (void *)d_x};
  dysel_slice s;
  memset(&s, 0, sizeof(s));
  s.g[0] = s.g[1] = s.g[2] = 1;
  s.U[0] = (uint64_t)(jp->n_rows + 255) / 256;
  s.U[1] = s.U[2] = 1;
  s.G[0] = (uint32_t)s.U[0];
  s.G[1] = s.G[2] = 1;
  s.granule_count = s.U[0];
  s.granule_stride = 1;
  s.role = DYSEL_ROLE_BATCH;
  s.variant = variant_id;
  DYSEL_TRY(kJdsFns[variant_id](&s, args, stream, jp));
  return check_launch(ctx, "global JDS variant");
}

dysel_status dysel_spmv_jds_copy_array(const dysel_spmv_jds_plan *jp, int which, void *dst, size_t *bytes) {
  if (!jp || !bytes) return DYSEL_ERR_INVALID;
  const void *src = nullptr;
  size_t sz = 0;
  switch (which) {
    case 0: src = jp->perm; sz = (size_t)jp->n_rows * 4; break;
    case 1: src = jp->len; sz = (size_t)jp->n_rows * 4; break;
    case 2: src = jp->jd_ptr; sz = jp->n_rows > 0 ? (size_t)(jp->W + 1) * 4 : 0; break;
    case 3: src = jp->col; sz = (size_t)jp->nnz * 4; break;
    case 4: src = jp->val; sz = (size_t)jp->nnz * 4; break;
    default: return DYSEL_ERR_INVALID;
  }
  if (!dst) {
    *bytes = sz;
    return DYSEL_OK;
  }
  if (*bytes < sz) return DYSEL_ERR_INVALID;
  *bytes = sz;
  if (sz && src && cudaMemcpy(dst, src, sz, cudaMemcpyDeviceToHost) != cudaSuccess) return DYSEL_ERR_CUDA;
  return DYSEL_OK;
}

void dysel_spmv_jds_plan_destroy(dysel_spmv_jds_plan *jp) {
  if (!jp) return;
  if (jp->ctx) {
    cudaSetDevice(jp->ctx->device);
    cudaDeviceSynchronize();
    if (!jp->sig.empty()) {
      jp->ctx->reg.erase(jp->sig);
      jp->ctx->sel_cache.erase(jp->sig);
    }
  }
  cudaFree(jp->perm);
  cudaFree(jp->len);
  cudaFree(jp->jd_ptr);
  cudaFree(jp->col);
  cudaFree(jp->val);
  cudaGetLastError();
  delete jp;
}

}  // extern "C"
