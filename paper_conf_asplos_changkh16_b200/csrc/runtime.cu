// libdysel runtime: context, slice planner, variant registry, selection cache
// and the generic dysel_launch orchestrator.
//
// Paper passages: runtime interface Fig. 6 (§3.1); GPU runtime —
// three extended copies, in-kernel timers, streams, sync / async host code
// (§3.3); safe-point / uniform / side-effect analyses
// (§3.4); orchestration (§2.4); Table 1.
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cuda.h>
#include <cudaTypedefs.h>
#include <chrono>
#include <cmath>
#include <cstring>
#include <numeric>

#include "dysel_device.cuh"
#include "internal.h"

namespace dysel {

void set_error(dysel_ctx *ctx, const std::string &msg) {
  if (ctx) ctx->last_error = msg;
}

dysel_status check_launch(dysel_ctx *ctx, const char *what) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    set_error(ctx, std::string(what) + ": " + cudaGetErrorString(e));
    return DYSEL_ERR_CUDA;
  }
  if (ctx) ctx->launches++;
  return DYSEL_OK;
}

dysel_status scratch(dysel_ctx *ctx, ScratchBuf &b, size_t bytes) {
  if (b.bytes >= bytes) return DYSEL_OK;
  if (b.ptr) {
    cudaDeviceSynchronize();
    cudaFree(b.ptr);
    b.ptr = nullptr;
    b.bytes = 0;
  }
  size_t want = std::max<size_t>(bytes, 4096);
  if (cudaMalloc(&b.ptr, want) != cudaSuccess) {
    cudaGetLastError();
    set_error(ctx, "cudaMalloc scratch failed");
    return DYSEL_ERR_NOMEM;
  }
  b.bytes = want;
  return DYSEL_OK;
}

uint64_t now_ns() {
  return (uint64_t)std::chrono::duration_cast<std::chrono::nanoseconds>(
             std::chrono::steady_clock::now().time_since_epoch())
      .count();
}

int reserve_pending_sel(dysel_ctx *ctx, uint64_t **d_slot) {
  int i = ctx->pending_head;
  PendingSel &p = ctx->pending[i];
  if (p.used) {   // ring full: retire the oldest entry first
    cudaEventSynchronize(p.ev);
    resolve_pending(ctx, nullptr);
  }
  ctx->h_pending_sel[i] = ~0ull;
  if (d_slot) *d_slot = ctx->d_pending_sel + i;
  return i;
}

dysel_status commit_pending_sel(dysel_ctx *ctx, int i, const std::string &sig, cudaStream_t st) {
  PendingSel &p = ctx->pending[i];
  DYSEL_CUDA_TRY(ctx, cudaEventRecord(p.ev, st));
  p.sig = sig;
  p.used = true;
  ctx->pending_head = (i + 1) % kPendingRing;
  return DYSEL_OK;
}

dysel_status push_pending_sel(dysel_ctx *ctx, const std::string &sig, const uint64_t *d_sel, cudaStream_t st) {
  const int i = reserve_pending_sel(ctx, nullptr);
  DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(&ctx->h_pending_sel[i], d_sel, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
  return commit_pending_sel(ctx, i, sig, st);
}

void resolve_pending(dysel_ctx *ctx, const char *block_sig) {
  // oldest first, so the latest selection of a sig wins
  for (int k = 0; k < kPendingRing; ++k) {
    int i = (ctx->pending_head + k) % kPendingRing;
    PendingSel &p = ctx->pending[i];
    if (!p.used) continue;
    if (block_sig && p.sig == block_sig) cudaEventSynchronize(p.ev);
    if (cudaEventQuery(p.ev) != cudaSuccess) continue;
    uint64_t w = ctx->h_pending_sel[i];
    if (w != ~0ull) ctx->sel_cache[p.sig] = (int)(w & 0xff);
    p.used = false;
  }
  cudaGetLastError();
}

dysel_status check_sel_timeout(dysel_ctx *ctx) {
  if (ctx && ctx->h_sel_timeout && *(volatile uint32_t *)ctx->h_sel_timeout) {
    *(volatile uint32_t *)ctx->h_sel_timeout = 0u;
    set_error(ctx, "a device-path launch timed out (5 s) waiting for its profiling slices to publish the "
                   "selection; fully/hybrid ran the remainder with the default variant, swap left the output "
                   "without the remainder");
    return DYSEL_ERR_CUDA;
  }
  return DYSEL_OK;
}

static uint64_t lcm64(uint64_t a, uint64_t b) { return a / std::gcd(a, b) * b; }

// Slice planning — a-2 / readings A-1, A-2, A-3.  Mirrors oracle/slice_plan.py
// rule for rule (tests compare the two on the same inputs).
dysel_status make_plan(dysel_ctx *ctx, const uint64_t U_in[3], const uint32_t (*wa)[3], int K, float f, int n_sm,
                       int default_variant, uint32_t mode, const uint32_t *vflags, Plan *out) {
  Plan p;
  if (K < 1 || K > DYSEL_MAX_VARIANTS || !(f >= 0.0f && f <= 1.0f) || default_variant < 0 ||
      default_variant >= K) {
    set_error(ctx, "invalid plan arguments");
    return DYSEL_ERR_INVALID;
  }
  p.K = K;
  for (int d = 0; d < 3; ++d) {
    p.U[d] = U_in[d] == 0 ? 0 : U_in[d];
    uint64_t g = 1;
    for (int v = 0; v < K; ++v) {
      if (wa[v][d] == 0) {
        set_error(ctx, "wa = 0");
        return DYSEL_ERR_INVALID;
      }
      g = lcm64(g, wa[v][d]);
    }
    if (g > 0xffffffffull) {
      set_error(ctx, "LCM of wa too large");
      return DYSEL_ERR_INVALID;
    }
    p.g[d] = (uint32_t)g;
    uint64_t G = (p.U[d] + g - 1) / g;
    if (G > 0xffffffffull) {
      set_error(ctx, "too many granules");
      return DYSEL_ERR_INVALID;
    }
    p.G[d] = (uint32_t)G;
  }
  p.Gn = (uint64_t)p.G[0] * p.G[1] * p.G[2];
  for (int v = 0; v < K; ++v)
    p.h[v] = (uint64_t)(p.g[0] / wa[v][0]) * (p.g[1] / wa[v][1]) * (p.g[2] / wa[v][2]);
  // mode resolution (A-10, A-11, A-13; programmer override wins)
  int base = (int)(mode & 3u);
  if (base == DYSEL_AUTO) {
    bool at = false, nu = false;
    for (int v = 0; v < K; ++v) {
      at |= (vflags[v] & DYSEL_V_ATOMICS) != 0;
      nu |= (vflags[v] & DYSEL_V_NONUNIFORM) != 0;
    }
    base = at ? DYSEL_SWAP : (nu ? DYSEL_HYBRID : DYSEL_FULLY);
  }
  if (base == DYSEL_SWAP && (mode & DYSEL_ASYNC)) {
    set_error(ctx, "swap-based profiling cannot run asynchronously (Table 1, P:L735-739)");
    return DYSEL_ERR_UNSUPPORTED;
  }
  p.mode = base;
  uint64_t c = (uint64_t)std::floor((double)f * (double)p.Gn / (double)K);   // A-1
  uint64_t q = (uint64_t)(n_sm / K);                                          // A-2
  if (q > 0) {
    uint64_t hmin = p.h[0];
    for (int v = 1; v < K; ++v) hmin = std::min(hmin, p.h[v]);
    uint64_t cq = q / std::gcd(q, hmin);
    if (c >= cq) c = (c / cq) * cq;
  }
  uint64_t def_ctas = 1;
  for (int d = 0; d < 3; ++d) def_ctas *= (p.U[d] + wa[default_variant][d] - 1) / wa[default_variant][d];
  bool active = !(mode & DYSEL_NO_PROFILE) && K >= 2 && p.Gn > 0;
  if (active) {
    if (mode & DYSEL_FORCE_PROFILE) {
      if (c == 0) c = (base == DYSEL_FULLY ? p.Gn >= (uint64_t)K : p.Gn >= 1) ? 1 : 0;
      active = c >= 1;
    } else {
      active = c >= 1 && def_ctas >= 128;   // P:L328-337 (A-3)
    }
  }
  p.active = active;
  p.c = active ? c : 0;
  *out = p;
  return DYSEL_OK;
}

// -------------------------------------------------------------- small kernels
__global__ void init_prof_kernel(DevProf *p, int K, int def) {
  int i = threadIdx.x;
  if (i < DYSEL_MAX_VARIANTS) {
    p->slot[i].t_start_min = ~0ull;
    p->slot[i].t_end_max = 0;
    p->slot[i].units = 0;
    p->slot[i].cycles = 0;
    p->ctas_done[i] = 0;
    p->lb[i] = 0;
    p->decided[i] = 0;
  }
  if (i == 0) {
    p->variants_done = 0;
    p->best = (((1ull << 56) - 1) << 8) | (uint64_t)def;
    p->sel = ~0ull;
    p->t_publish = 0;
    p->t_init = dysel_globaltimer();
  }
}

// Swap-mode copy-in of the winner's private output (Table 1): EVERY byte is
// gated on the selection (a losing variant's private copy may be partial —
// dominance stops it — so nothing of it may reach the output).  16-byte
// vector body when both pointers are 16-byte aligned, bytes otherwise.
__global__ void gated_copy_kernel(char *dst, const char *src, size_t bytes, const uint64_t *gate, int v) {
  if ((int)(dysel_ld_acquire_u64(gate) & 0xffu) != v) return;
  const size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x, nt = (size_t)gridDim.x * blockDim.x;
  size_t head = 0;
  if ((((uintptr_t)dst | (uintptr_t)src) & 15) == 0) {
    const size_t n16 = bytes / 16;
    for (size_t i = tid; i < n16; i += nt) reinterpret_cast<uint4 *>(dst)[i] = reinterpret_cast<const uint4 *>(src)[i];
    head = n16 * 16;
  }
  for (size_t i = head + tid; i < bytes; i += nt) dst[i] = src[i];
}

// Bounded wait for the selection (reading A-32's wait kernel) failed: flag it
// for the host (mapped pinned word, checked by the next call and by the
// report) and, where the default variant's output is usable — fully and
// hybrid, whose profiling slices are productive in place — publish the
// default so the remainder still runs; swap (private outputs) keeps the gate
// closed and the host returns an error.
__device__ __forceinline__ void selection_timeout(uint64_t *sel, uint32_t *flag, int def, int swap) {
  if (flag) *(volatile uint32_t *)flag = 1u;
  if (!swap) atomicCAS((unsigned long long *)sel, ~0ull, ((((1ull << 56) - 1)) << 8) | (uint64_t)def);
  __threadfence_system();
}

// Device path: stream-order the gated remainder behind the SELECTION rather
// than behind the profiling kernels' completion — a variant decided by
// dominance (A-32) may still be finishing productive tiles.  One thread; the
// selection is always published (every variant is decided by completion or
// dominance), so the wait ends.
__global__ void wait_selection_kernel(uint64_t *sel, uint32_t *timeout_flag, int def, int swap) {
  // bounded (5 s): a variant that never calls dysel_prof_end would otherwise
  // hang the stream; the timeout is reported, never silent (selection_timeout)
  const uint64_t t0 = dysel_globaltimer();
  for (uint32_t ns = 64; dysel_ld_acquire_u64(sel) == ~0ull; ns = ns < 2048 ? 2 * ns : ns) {
    if (dysel_globaltimer() - t0 >= 5000000000ull) {
      selection_timeout(sel, timeout_flag, def, swap);
      return;
    }
    __nanosleep(ns);
  }
}

void mark_builtin(dysel_ctx *ctx, const char *sig) {
  auto it = ctx->reg.find(sig);
  if (it != ctx->reg.end()) it->second.builtin = true;
}

// The selection gate as a stream memory operation: wait until the 64-bit
// selection word is no longer all ones (CU_STREAM_WAIT_VALUE_NOR with value 0:
// ~(*sel | 0) != 0).  Executed by the GPU front end -- unlike the one-thread
// wait kernel it needs no SM, so it opens at the publish even when the
// profiling copies and the eager wave fill every SM.
static bool gate_wait_value(cudaStream_t st, const uint64_t *sel) {
  static PFN_cuStreamWaitValue64_v11070 fn = [] {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuStreamWaitValue64", &p, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      p = nullptr;
    cudaGetLastError();
    return (PFN_cuStreamWaitValue64_v11070)p;
  }();
  return fn && fn((CUstream)st, (CUdeviceptr)sel, 0ull, CU_STREAM_WAIT_VALUE_NOR) == CUDA_SUCCESS;
}

__global__ void timer_calib_kernel(uint64_t samples, uint64_t spin_ns, uint64_t *out) {
  uint64_t prev = dysel_globaltimer(), best = ~0ull;
  for (uint64_t i = 0; i < samples; ++i) {
    uint64_t t = dysel_globaltimer();
    if (t != prev) {
      best = min(best, t - prev);
      prev = t;
    }
  }
  uint64_t t0 = dysel_globaltimer(), c0 = dysel_clock64(), t1;
  do {
    t1 = dysel_globaltimer();
  } while (t1 - t0 < spin_ns);
  uint64_t c1 = dysel_clock64();
  out[0] = best;
  out[1] = t1 - t0;
  out[2] = c1 - c0;
}

// Known-cost variant (c-8): spins cost_ns per unit, writes out[u] = v + 1.
__global__ void spin_variant_kernel(dysel_slice s, uint32_t cost_ns, uint32_t *out) {
  __shared__ dysel_prof_smem psm;
  if (!dysel_gate_open(s)) return;
  const uint32_t wa[3] = {1, 1, 1};
  dysel_prof_begin(s, psm);
  uint64_t u[3];
  bool ok = dysel_cta_origin(s, wa, blockIdx.x, u);
  if (ok && threadIdx.x == 0) {
    uint64_t t0 = dysel_globaltimer();
    while (dysel_globaltimer() - t0 < cost_ns) {
    }
    out[u[0]] = (uint32_t)s.variant + 1;
  }
  __syncthreads();
  dysel_prof_end(s, psm, ok ? 1u : 0u);
}

static dysel_status spin_fn(const dysel_slice *s, void *const *args, void *stream, void *user) {
  uint64_t ctas = s->granule_count * (uint64_t)s->g[0] * s->g[1] * s->g[2];
  if (ctas == 0) return DYSEL_OK;
  spin_variant_kernel<<<(unsigned)ctas, 32, 0, (cudaStream_t)stream>>>(*s, (uint32_t)(uintptr_t)user,
                                                                         (uint32_t *)args[0]);
  return cudaGetLastError() == cudaSuccess ? DYSEL_OK : DYSEL_ERR_CUDA;
}

// ------------------------------------------------------------ launch helpers
static dysel_slice base_slice(const Plan &p) {
  dysel_slice s;
  memset(&s, 0, sizeof(s));
  for (int d = 0; d < 3; ++d) {
    s.g[d] = p.g[d];
    s.G[d] = p.G[d];
    s.U[d] = p.U[d];
  }
  s.granule_stride = 1;
  return s;
}

// resident CTAs per SM of variant v, when every variant declares ctas_per_wave
// (the cycle-based scores need all of them), else 0 (makespan)
static uint32_t variant_occupancy(const Registered &R, int v, uint32_t mode, int n_sm) {
  if (mode & DYSEL_SCORE_MAKESPAN) return 0;
  for (const auto &x : R.v)
    if (x.ctas_per_wave == 0) return 0;
  return (uint32_t)std::max<uint64_t>(1, R.v[v].ctas_per_wave / (uint64_t)std::max(1, n_sm));
}

// Score parameters of variant v (dysel_slice score fields): cycles/unit
// (DYSEL_SCORE_CYCLES); else, when every variant declares ctas_per_wave, the
// wave-quantised full-grid prediction (reading A-34): ceil(grid CTAs / wave)
// x mean cycles per CTA; else makespan (Fig. 7b).
static void set_score_params(dysel_slice &s, const Registered &R, const Plan &P, int v, uint32_t mode, int n_sm) {
  s.score_cycles = (mode & DYSEL_SCORE_CYCLES) ? 1u : 0u;
  s.occupancy = variant_occupancy(R, v, mode, n_sm);
  if (!s.score_cycles && s.occupancy) {
    s.grid_ctas = P.Gn * P.h[v];
    s.wave_ctas = R.v[v].ctas_per_wave;
    s.units_per_cta = R.v[v].wa[0] * R.v[v].wa[1] * R.v[v].wa[2];
  }
}

// same rule as dysel_prof_end (dysel_device.cuh)
static uint64_t host_score(const dysel_timer_slot &t, const dysel_slice &sp) {
  if (sp.score_cycles || sp.occupancy) return dysel_cycle_score(sp, t.cycles, t.units);
  return std::min<uint64_t>(t.t_end_max - t.t_start_min, (1ull << 56) - 1);
}
static uint64_t host_score(const dysel_timer_slot &t, const Registered &R, const Plan &P, int v, uint32_t mode,
                           int n_sm) {
  dysel_slice sp;
  memset(&sp, 0, sizeof(sp));
  set_score_params(sp, R, P, v, mode, n_sm);
  return host_score(t, sp);
}

static void fill_report_common(dysel_report *rep, const Plan &p, int mode_used, int profiled, int selected) {
  if (!rep) return;
  rep->mode_used = mode_used;
  rep->profiled = profiled;
  rep->selected = selected;
  rep->n_variants = p.K;
  rep->c = p.c;
  rep->n_granules = p.Gn;
  rep->eager_units = 0;
  rep->tail_units = 0;
  rep->n_slices = 0;
  rep->sandbox_buffers = 0;
  rep->sandbox_bytes = 0;
  for (int v = 0; v < DYSEL_MAX_VARIANTS; ++v) {
    rep->score[v] = rep->makespan_ns[v] = rep->units[v] = rep->cycles[v] = 0;
    rep->busy_ns[v] = rep->aborted[v] = 0;
  }
}

static void add_slice_rec(dysel_report *rep, const dysel_slice &s) {
  if (!rep || !rep->slices || rep->n_slices >= rep->slices_cap) {
    if (rep) rep->n_slices++;
    return;
  }
  dysel_slice_rec &r = rep->slices[rep->n_slices++];
  r.granule_begin = s.granule_begin;
  r.granule_count = s.granule_count;
  r.granule_stride = s.granule_stride;
  r.variant = s.variant;
  r.role = s.role;
}

static void mark_units(dysel_report *rep, const dysel_slice &s) {
  if (!rep || !rep->unit_variant) return;
  for (uint64_t i = 0; i < s.granule_count; ++i) {
    uint64_t j = s.granule_begin + i * s.granule_stride;
    if (j < rep->unit_variant_cap) rep->unit_variant[j] = (uint8_t)s.variant;
  }
}

}  // namespace dysel

using namespace dysel;

// ===================================================================== C ABI
extern "C" {

const char *dysel_status_str(dysel_status s) {
  switch (s) {
    case DYSEL_OK: return "DYSEL_OK";
    case DYSEL_ERR_INVALID: return "DYSEL_ERR_INVALID";
    case DYSEL_ERR_UNSUPPORTED: return "DYSEL_ERR_UNSUPPORTED";
    case DYSEL_ERR_NOMEM: return "DYSEL_ERR_NOMEM";
    case DYSEL_ERR_CUDA: return "DYSEL_ERR_CUDA";
    case DYSEL_ERR_NOT_FOUND: return "DYSEL_ERR_NOT_FOUND";
    case DYSEL_ERR_NCCL: return "DYSEL_ERR_NCCL";
  }
  return "DYSEL_ERR_UNKNOWN";
}

const char *dysel_last_error(const dysel_ctx *ctx) { return ctx ? ctx->last_error.c_str() : "NULL ctx"; }

dysel_status dysel_create(int cuda_device, dysel_ctx **out) {
  if (!out) return DYSEL_ERR_INVALID;
  *out = nullptr;
  dysel_ctx *ctx = new (std::nothrow) dysel_ctx();
  if (!ctx) return DYSEL_ERR_NOMEM;
  ctx->device = cuda_device;
  auto fail = [&](dysel_status s) {
    dysel_destroy(ctx);
    return s;
  };
  if (cudaSetDevice(cuda_device) != cudaSuccess) {
    cudaGetLastError();
    return fail(DYSEL_ERR_CUDA);
  }
  int v = 0;
  cudaDeviceGetAttribute(&ctx->n_sm, cudaDevAttrMultiProcessorCount, cuda_device);
  cudaDeviceGetAttribute(&v, cudaDevAttrL2CacheSize, cuda_device);
  ctx->l2_bytes = (uint64_t)v;
  // profiling streams get the highest priority: profiling before eager work
  int prio_lo = 0, prio_hi = 0;
  cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
  for (int i = 0; i < DYSEL_MAX_VARIANTS; ++i) {
    if (cudaStreamCreateWithPriority(&ctx->fork[i], cudaStreamNonBlocking, prio_hi) != cudaSuccess)
      return fail(DYSEL_ERR_CUDA);
    if (cudaEventCreateWithFlags(&ctx->ev_join[i], cudaEventDisableTiming) != cudaSuccess) return fail(DYSEL_ERR_CUDA);
    if (cudaStreamCreateWithPriority(&ctx->rem[i], cudaStreamNonBlocking, prio_lo) != cudaSuccess)
      return fail(DYSEL_ERR_CUDA);
    if (cudaEventCreateWithFlags(&ctx->ev_join2[i], cudaEventDisableTiming) != cudaSuccess) return fail(DYSEL_ERR_CUDA);
  }
  if (cudaStreamCreateWithFlags(&ctx->query, cudaStreamNonBlocking) != cudaSuccess) return fail(DYSEL_ERR_CUDA);
  if (cudaStreamCreateWithPriority(&ctx->wsel, cudaStreamNonBlocking, prio_hi) != cudaSuccess)
    return fail(DYSEL_ERR_CUDA);
  if (cudaStreamCreateWithPriority(&ctx->rem_hi, cudaStreamNonBlocking, prio_hi) != cudaSuccess)
    return fail(DYSEL_ERR_CUDA);
  if (cudaEventCreateWithFlags(&ctx->ev_start, cudaEventDisableTiming) != cudaSuccess) return fail(DYSEL_ERR_CUDA);
  if (cudaEventCreateWithFlags(&ctx->ev_fork2, cudaEventDisableTiming) != cudaSuccess) return fail(DYSEL_ERR_CUDA);
  if (cudaMalloc(&ctx->d_prof, sizeof(DevProf)) != cudaSuccess) return fail(DYSEL_ERR_NOMEM);
  if (cudaMallocHost(&ctx->h_prof, sizeof(DevProf)) != cudaSuccess) return fail(DYSEL_ERR_NOMEM);
  if (cudaHostAlloc((void **)&ctx->h_pending_sel, kPendingRing * sizeof(uint64_t), cudaHostAllocMapped) != cudaSuccess ||
      cudaHostGetDevicePointer((void **)&ctx->d_pending_sel, ctx->h_pending_sel, 0) != cudaSuccess)
    return fail(DYSEL_ERR_NOMEM);
  for (int i = 0; i < kPendingRing; ++i)
    if (cudaEventCreateWithFlags(&ctx->pending[i].ev, cudaEventDisableTiming) != cudaSuccess) return fail(DYSEL_ERR_CUDA);
  if (cudaHostAlloc((void **)&ctx->h_sel_timeout, sizeof(uint32_t), cudaHostAllocMapped) != cudaSuccess ||
      cudaHostGetDevicePointer((void **)&ctx->d_sel_timeout, ctx->h_sel_timeout, 0) != cudaSuccess)
    return fail(DYSEL_ERR_NOMEM);
  *ctx->h_sel_timeout = 0u;
  if (spmv_ctx_init(ctx) != DYSEL_OK) return fail(DYSEL_ERR_CUDA);
  if (sgemm_register(ctx) != DYSEL_OK) return fail(DYSEL_ERR_CUDA);
  if (stencil_register(ctx) != DYSEL_OK) return fail(DYSEL_ERR_CUDA);
  if (spmtv_register(ctx) != DYSEL_OK) return fail(DYSEL_ERR_CUDA);
  uint64_t tick = 0;
  double cpn = 0;
  if (dysel_timer_calibrate(ctx, 1u << 16, 20000, &tick, &cpn) != DYSEL_OK) return fail(DYSEL_ERR_CUDA);
  ctx->gt_tick_ns = tick;
  *out = ctx;
  return DYSEL_OK;
}

void dysel_destroy(dysel_ctx *ctx) {
  if (!ctx) return;
  cudaSetDevice(ctx->device);
  cudaDeviceSynchronize();
  if (ctx->l2_persist_bytes > 0) {   // give the L2 set-aside of the x_persist placement back
    cudaCtxResetPersistingL2Cache();
    cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, 0);
    cudaGetLastError();
  }
  spmv_ctx_free(ctx);
  for (int i = 0; i < DYSEL_MAX_VARIANTS; ++i) {
    if (ctx->fork[i]) cudaStreamDestroy(ctx->fork[i]);
    if (ctx->ev_join[i]) cudaEventDestroy(ctx->ev_join[i]);
    if (ctx->rem[i]) cudaStreamDestroy(ctx->rem[i]);
    if (ctx->ev_join2[i]) cudaEventDestroy(ctx->ev_join2[i]);
  }
  if (ctx->query) cudaStreamDestroy(ctx->query);
  if (ctx->wsel) cudaStreamDestroy(ctx->wsel);
  if (ctx->rem_hi) cudaStreamDestroy(ctx->rem_hi);
  if (ctx->ev_start) cudaEventDestroy(ctx->ev_start);
  if (ctx->ev_fork2) cudaEventDestroy(ctx->ev_fork2);
  if (ctx->d_prof) cudaFree(ctx->d_prof);
  if (ctx->d_spmtv_state) cudaFree(ctx->d_spmtv_state);
  if (ctx->h_prof) cudaFreeHost(ctx->h_prof);
  if (ctx->h_pending_sel) cudaFreeHost(ctx->h_pending_sel);
  if (ctx->h_sel_timeout) cudaFreeHost(ctx->h_sel_timeout);
  for (int i = 0; i < kPendingRing; ++i)
    if (ctx->pending[i].ev) cudaEventDestroy(ctx->pending[i].ev);
  for (auto &b : ctx->sandbox)
    if (b.ptr) cudaFree(b.ptr);
  if (ctx->unit_variant.ptr) cudaFree(ctx->unit_variant.ptr);
  if (ctx->norm_part.ptr) cudaFree(ctx->norm_part.ptr);
  if (ctx->shard_stage.ptr) cudaFree(ctx->shard_stage.ptr);
  comm_free(ctx);
  delete ctx;
}

dysel_status dysel_device_info(const dysel_ctx *ctx, int *n_sm, uint64_t *tick, uint64_t *l2) {
  if (!ctx) return DYSEL_ERR_INVALID;
  if (n_sm) *n_sm = ctx->n_sm;
  if (tick) *tick = ctx->gt_tick_ns;
  if (l2) *l2 = ctx->l2_bytes;
  return DYSEL_OK;
}

uint64_t dysel_kernel_launches(const dysel_ctx *ctx) { return ctx ? ctx->launches : 0; }

dysel_status dysel_timer_calibrate(dysel_ctx *ctx, uint64_t samples, uint64_t spin_ns, uint64_t *tick_ns,
                                   double *cycles_per_ns) {
  if (!ctx) return DYSEL_ERR_INVALID;
  uint64_t *d = nullptr, h[3] = {0, 0, 0};
  DYSEL_CUDA_TRY(ctx, cudaMalloc(&d, 3 * sizeof(uint64_t)));
  timer_calib_kernel<<<1, 1>>>(samples, spin_ns, d);
  dysel_status st = check_launch(ctx, "timer_calib_kernel");
  if (st == DYSEL_OK && cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost) != cudaSuccess) st = DYSEL_ERR_CUDA;
  cudaFree(d);
  if (st != DYSEL_OK) return st;
  if (tick_ns) *tick_ns = h[0];
  if (cycles_per_ns) *cycles_per_ns = h[1] ? (double)h[2] / (double)h[1] : 0.0;
  return DYSEL_OK;
}

dysel_status dysel_register_variants(dysel_ctx *ctx, const char *sig, const dysel_variant *v, int n,
                                     int default_variant) {
  if (!ctx || !sig || !v || n < 1 || n > DYSEL_MAX_VARIANTS || default_variant < 0 || default_variant >= n) {
    set_error(ctx, "dysel_register_variants: invalid arguments");
    return DYSEL_ERR_INVALID;
  }
  Registered r;
  for (int i = 0; i < n; ++i) {
    if (!v[i].fn || v[i].wa[0] == 0 || v[i].wa[1] == 0 || v[i].wa[2] == 0 || v[i].n_sandbox_args < 0 ||
        (v[i].n_sandbox_args > 0 && !v[i].sandbox_args)) {
      set_error(ctx, "dysel_register_variants: bad variant descriptor");
      return DYSEL_ERR_INVALID;
    }
    r.v.push_back(v[i]);
    r.sandbox_args.emplace_back(v[i].sandbox_args, v[i].sandbox_args + v[i].n_sandbox_args);
    r.names.emplace_back(v[i].name ? v[i].name : "");
    r.v.back().sandbox_args = nullptr;
    r.v.back().name = nullptr;
  }
  r.def = default_variant;
  ctx->reg[sig] = std::move(r);
  // drop cached selections of the sig and of its shape-keyed entries (sig#...)
  const std::string pre = std::string(sig) + "#";
  for (auto c = ctx->sel_cache.begin(); c != ctx->sel_cache.end();)
    c = (c->first == sig || c->first.compare(0, pre.size(), pre) == 0) ? ctx->sel_cache.erase(c) : std::next(c);
  return DYSEL_OK;
}

dysel_status dysel_register_spin_variants(dysel_ctx *ctx, const char *sig, const uint32_t *cost_ns, int n,
                                          int default_variant) {
  if (!ctx || !cost_ns || n < 1 || n > DYSEL_MAX_VARIANTS) return DYSEL_ERR_INVALID;
  static const int sb[1] = {0};
  dysel_variant vv[DYSEL_MAX_VARIANTS];
  for (int i = 0; i < n; ++i) {
    vv[i] = dysel_variant{"spin", spin_fn, {1, 1, 1}, sb, 1, 0, (void *)(uintptr_t)cost_ns[i]};
  }
  return dysel_register_variants(ctx, sig, vv, n, default_variant);
}

dysel_status dysel_get_selection(dysel_ctx *ctx, const char *key, int *variant) {
  if (!ctx || !key || !variant) return DYSEL_ERR_INVALID;
  resolve_pending(ctx, key);
  DYSEL_TRY(check_sel_timeout(ctx));
  auto it = ctx->sel_cache.find(key);
  if (it == ctx->sel_cache.end()) return DYSEL_ERR_NOT_FOUND;
  *variant = it->second;
  return DYSEL_OK;
}

dysel_status dysel_set_selection(dysel_ctx *ctx, const char *key, int variant) {
  if (!ctx || !key || variant < 0 || variant >= DYSEL_MAX_VARIANTS) return DYSEL_ERR_INVALID;
  ctx->sel_cache[key] = variant;
  return DYSEL_OK;
}

dysel_status dysel_reset_selection(dysel_ctx *ctx, const char *key) {
  if (!ctx) return DYSEL_ERR_INVALID;
  if (!key)
    ctx->sel_cache.clear();
  else
    ctx->sel_cache.erase(key);
  return DYSEL_OK;
}

// Generic DySel launch.  Device path (default): profiling copies of all K
// variants concurrently on forked streams; the last profiling CTA publishes
// the packed selection on the device; the remainder is launched as K gated
// batch copies (only the selected one does work) — no host round trip.
// DYSEL_HOST_ORCH: the paper's host code — sync waits and reads the selection
// (P:L927-930); async polls the profiling streams and launches eager chunks of
// the best-so-far variant until all profiles are in.
dysel_status dysel_launch(dysel_ctx *ctx, const char *sig, const uint64_t ndrange_units[3], float f, uint32_t mode,
                          void *const *args, int n_args, const size_t *sandbox_bytes, void *stream_v,
                          dysel_report *rep) {
  return dysel::launch_keyed(ctx, sig, sig, ndrange_units, f, mode, args, n_args, sandbox_bytes, stream_v, rep, -1);
}

}  // extern "C"

// The selection cache (activation flag) is keyed by `key` (reading A-22):
// kernel_sig for dysel_launch, sig + problem shape for the built-in SGEMM and
// stencil pools (a selection made for one shape is not reused for another).
dysel_status dysel::launch_keyed(dysel_ctx *ctx, const char *sig, const char *key, const uint64_t ndrange_units[3],
                                 float f, uint32_t mode, void *const *args, int n_args, const size_t *sandbox_bytes,
                                 void *stream_v, dysel_report *rep, int def_override) {
  const uint64_t t_host0 = now_ns();
  if (!ctx || !sig || !ndrange_units || n_args < 0 || (n_args > 0 && !args)) {
    set_error(ctx, "dysel_launch: invalid arguments");
    return DYSEL_ERR_INVALID;
  }
  auto it = ctx->reg.find(sig);
  if (it == ctx->reg.end()) {
    set_error(ctx, std::string("dysel_launch: unknown kernel_sig ") + sig);
    return DYSEL_ERR_INVALID;
  }
  DYSEL_TRY(check_sel_timeout(ctx));   // a previous launch's selection wait timed out
  const Registered &R = it->second;
  const int K = (int)R.v.size();
  // initial ("default") version: the registered one, or a per-call choice of
  // a built-in pool (reading A-39)
  const int def = (def_override >= 0 && def_override < K) ? def_override : R.def;
  uint32_t wa[DYSEL_MAX_VARIANTS][3], vflags[DYSEL_MAX_VARIANTS];
  for (int v = 0; v < K; ++v) {
    for (int d = 0; d < 3; ++d) wa[v][d] = R.v[v].wa[d];
    vflags[v] = R.v[v].flags;
  }
  for (int v = 0; v < K; ++v)
    for (int a : R.sandbox_args[v])
      if (a < 0 || a >= n_args) {
        set_error(ctx, "dysel_launch: sandbox arg index out of range");
        return DYSEL_ERR_INVALID;
      }
  Plan P;
  DYSEL_TRY(make_plan(ctx, ndrange_units, wa, K, f, ctx->n_sm, def, mode, vflags, &P));
  resolve_pending(ctx, nullptr);
  if (P.active && !(mode & DYSEL_FORCE_PROFILE) && R.v[def].ctas_per_wave > 0) {
    // reading A-3b: the default variant's whole grid runs in one wave
    uint64_t def_ctas = 1;
    for (int d = 0; d < 3; ++d) def_ctas *= (P.U[d] + wa[def][d] - 1) / wa[def][d];
    if (def_ctas <= R.v[def].ctas_per_wave) {
      P.active = false;
      P.c = 0;
    }
  }
  cudaStream_t st = (cudaStream_t)stream_v;
  if (rep) rep->n_slices = 0;
  if (P.Gn == 0) {
    fill_report_common(rep, P, P.mode, 0, def);
    return DYSEL_OK;
  }
  std::vector<void *> base_args(args, args + n_args);
  if (!P.active) {   // activation flag off / small workload: one plain batch copy
    int v = def;
    resolve_pending(ctx, key);
    auto c = ctx->sel_cache.find(key);
    if (c != ctx->sel_cache.end() && c->second < K) v = c->second;
    dysel_slice s = base_slice(P);
    s.granule_count = P.Gn;
    s.role = DYSEL_ROLE_BATCH;
    s.variant = v;
    DYSEL_TRY(R.v[v].fn(&s, base_args.data(), st, R.v[v].user));
    DYSEL_TRY(check_launch(ctx, "variant batch"));
    fill_report_common(rep, P, P.mode | (int)(mode & DYSEL_ASYNC), 0, v);
    add_slice_rec(rep, s);
    mark_units(rep, s);
    if (rep) rep->host_ns = now_ns() - t_host0;
    return DYSEL_OK;
  }
  // generic ASYNC = the paper's host polling path: heterogeneous user kernels
  // cannot share a device-side ticket scheduler (the SpMV pool does, spmv.cu)
  // ASYNC without HOST_ORCH: device path with an eager wave of the default
  // variant beside the profiling copies (reading A-33); HOST_ORCH: the paper's
  // host polling + eager chunks
  const bool host_orch = (mode & DYSEL_HOST_ORCH) != 0;
  const bool async = (mode & DYSEL_ASYNC) != 0;
  // ---- per-variant argument vectors (sandboxes / private outputs, Table 1)
  std::vector<std::vector<void *>> vargs(K, base_args);
  int nsb_max = 0;
  for (int v = 0; v < K; ++v) nsb_max = std::max<int>(nsb_max, (int)R.sandbox_args[v].size());
  if ((P.mode == DYSEL_HYBRID || P.mode == DYSEL_SWAP) && nsb_max > 0 && !sandbox_bytes) {
    set_error(ctx, "dysel_launch: sandbox_arg_bytes required for hybrid / swap");
    return DYSEL_ERR_INVALID;
  }
  uint32_t n_sandbox = 0;   // Table 1 allocation record (dysel_report.sandbox_buffers / _bytes)
  uint64_t sandbox_total = 0;
  if (P.mode == DYSEL_HYBRID || P.mode == DYSEL_SWAP) {
    int slot = 0;
    for (int v = 0; v < K; ++v) {
      if (P.mode == DYSEL_HYBRID && v == def) continue;       // ≤ K-1 sandboxes
      for (size_t k = 0; k < R.sandbox_args[v].size(); ++k) {
        if ((size_t)slot >= sizeof(ctx->sandbox) / sizeof(ctx->sandbox[0])) {
          set_error(ctx, "too many sandbox buffers");
          return DYSEL_ERR_UNSUPPORTED;
        }
        size_t bytes = sandbox_bytes[k];
        DYSEL_TRY(scratch(ctx, ctx->sandbox[slot], bytes));
        int a = R.sandbox_args[v][k];
        if (P.mode == DYSEL_SWAP)   // private output starts as the original output
          DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(ctx->sandbox[slot].ptr, base_args[a], bytes,
                                              cudaMemcpyDeviceToDevice, st));
        vargs[v][a] = ctx->sandbox[slot].ptr;
        slot++;
        sandbox_total += bytes;
      }
    }
  }
  // ---- profiling copies, concurrently on forked streams
  // diagnostics (report requested): timing events on the launching stream,
  // the gate stream and after each phase (dysel_report.timeline_ns[2..5])
  cudaEvent_t tev[6] = {};
  if (rep)
    for (auto &e : tev) cudaEventCreate(&e);
  if (rep) cudaEventRecord(tev[0], st);
  init_prof_kernel<<<1, 32, 0, st>>>(ctx->d_prof, K, def);
  DYSEL_TRY(check_launch(ctx, "init_prof_kernel"));
  DYSEL_CUDA_TRY(ctx, cudaEventRecord(ctx->ev_start, st));
  fill_report_common(rep, P, P.mode | (async ? DYSEL_ASYNC : 0), 1, -1);
  if (rep) {   // buffers per variant redirected: one per sandbox arg (Table 1)
    for (int v = 0; v < K; ++v)
      if (!(P.mode == DYSEL_HYBRID && v == def) && P.mode != DYSEL_FULLY && !R.sandbox_args[v].empty()) n_sandbox++;
    rep->sandbox_buffers = n_sandbox;
    rep->sandbox_bytes = sandbox_total;
  }
  for (int v = 0; v < K; ++v) {
    dysel_slice s = base_slice(P);
    s.variant = v;
    s.granule_count = P.c;
    if (P.mode == DYSEL_FULLY) {
      if (mode & DYSEL_CONTIGUOUS) {
        s.granule_begin = (uint64_t)v * P.c;
      } else {
        s.granule_begin = (uint64_t)v;
        s.granule_stride = (uint64_t)K;
      }
      s.role = DYSEL_ROLE_PRODUCTIVE;
    } else if (P.mode == DYSEL_HYBRID) {
      s.role = v == def ? DYSEL_ROLE_PRODUCTIVE : DYSEL_ROLE_SANDBOX;
    } else {
      s.role = DYSEL_ROLE_PRIVATE;
    }
    s.timer = &ctx->d_prof->slot[v];
    s.ctas_done = &ctx->d_prof->ctas_done[v];
    s.ctas_total = (uint32_t)(P.c * P.h[v]);
    s.best = &ctx->d_prof->best;
    s.variants_done = &ctx->d_prof->variants_done;
    s.n_variants = (uint32_t)K;
    set_score_params(s, R, P, v, mode, ctx->n_sm);
    s.sel = &ctx->d_prof->sel;
    if (!(mode & DYSEL_NO_ABORT)) {   // reading A-32: dominance
      s.lb = &ctx->d_prof->lb[v];
      s.decided = &ctx->d_prof->decided[v];
      s.units_total = P.c * (uint64_t)P.g[0] * P.g[1] * P.g[2];
    }
    DYSEL_CUDA_TRY(ctx, cudaStreamWaitEvent(ctx->fork[v], ctx->ev_start, 0));
    DYSEL_TRY(R.v[v].fn(&s, vargs[v].data(), ctx->fork[v], R.v[v].user));
    DYSEL_TRY(check_launch(ctx, "variant profiling copy"));

    DYSEL_CUDA_TRY(ctx, cudaEventRecord(ctx->ev_join[v], ctx->fork[v]));
    add_slice_rec(rep, s);
    if (s.role == DYSEL_ROLE_PRODUCTIVE) mark_units(rep, s);
  }
  uint64_t rem_begin = P.mode == DYSEL_FULLY ? (uint64_t)K * P.c : P.c;
  const uint64_t rem_end = P.Gn;
  int selected = -1;
  uint64_t eager_units = 0;
  if (!host_orch && async && rem_begin < rem_end && R.v[def].ctas_per_wave > 0) {
    // ---- eager wave (reading A-33): the default variant fills the
    // execution slots the profiling copies leave free, on `st`, while they run
    uint64_t prof_slots = 0;   // profiling CTAs in units of the default's slots
    for (int v = 0; v < K; ++v)
      if (R.v[v].ctas_per_wave > 0)
        prof_slots += (P.c * P.h[v] * R.v[def].ctas_per_wave + R.v[v].ctas_per_wave - 1) / R.v[v].ctas_per_wave;
    const uint64_t free_slots = R.v[def].ctas_per_wave > prof_slots ? R.v[def].ctas_per_wave - prof_slots : 0;
    const uint64_t E = std::min<uint64_t>(free_slots / P.h[def], rem_end - rem_begin);
    if (E > 0) {
      dysel_slice s = base_slice(P);
      s.variant = def;
      s.role = DYSEL_ROLE_EAGER;
      s.granule_begin = rem_begin;
      s.granule_count = E;
      DYSEL_TRY(R.v[def].fn(&s, base_args.data(), st, R.v[def].user));
      DYSEL_TRY(check_launch(ctx, "variant eager wave"));
      add_slice_rec(rep, s);
      mark_units(rep, s);
      rem_begin += E;
      eager_units = E;
    }
  }
  if (!host_orch) {
    // ---- device path: gated remainder, selection never leaves the device
    // swap too (reading A-44): the winner's private copy is complete when its
    // last CTA decides it, so the copy-in and the remainder wait for the
    // selection only, not for a dominated variant's discarded private copy
    const bool dominance = !(mode & DYSEL_NO_ABORT);
    // the remainder is ordered behind the selection only — not behind the
    // eager wave (its CTAs take the slots the eager ones free) nor, with
    // dominance, behind dominated variants finishing productive tiles
    cudaStream_t gate_st = ctx->wsel;
    DYSEL_CUDA_TRY(ctx, cudaStreamWaitEvent(gate_st, ctx->ev_start, 0));
    bool wv_gate = false;   // the gate is a stream wait-value on gate_st (built-in pools)
    if (dominance) {
      wv_gate = R.builtin && gate_wait_value(gate_st, &ctx->d_prof->sel);
      if (!wv_gate) {
        wait_selection_kernel<<<1, 1, 0, gate_st>>>(&ctx->d_prof->sel, ctx->d_sel_timeout, def, P.mode == DYSEL_SWAP);
        DYSEL_TRY(check_launch(ctx, "wait_selection_kernel"));
      }
    } else {
      for (int v = 0; v < K; ++v) DYSEL_CUDA_TRY(ctx, cudaStreamWaitEvent(gate_st, ctx->ev_join[v], 0));
    }
    DYSEL_CUDA_TRY(ctx, cudaEventRecord(ctx->ev_fork2, gate_st));
    if (rep) cudaEventRecord(tev[1], gate_st);   // selection known
    if (P.mode == DYSEL_SWAP) {   // winner's private output copied in (after every private copy is complete)
      DYSEL_CUDA_TRY(ctx, cudaStreamWaitEvent(st, ctx->ev_fork2, 0));
      for (int v = 0; v < K; ++v)
        for (size_t k = 0; k < R.sandbox_args[v].size(); ++k) {
          int a = R.sandbox_args[v][k];
          gated_copy_kernel<<<2 * ctx->n_sm, 256, 0, st>>>((char *)base_args[a], (const char *)vargs[v][a],
                                                          sandbox_bytes[k], &ctx->d_prof->sel, v);
          DYSEL_TRY(check_launch(ctx, "gated_copy_kernel"));
        }
      DYSEL_CUDA_TRY(ctx, cudaEventRecord(ctx->ev_fork2, st));
    }
    if (rem_begin < rem_end) {
      // the default's gated copy goes first and on a high-priority stream: when
      // it wins (the usual case with a good initial version), the block
      // scheduler dispatches its CTAs ahead of the exiting CTAs of the losers
      // With the wait-value gate the default's copy is enqueued on the gate
      // stream itself: it starts at the publish, without the ~10 us hop of an
      // event to another stream (measured: the selection reached the other
      // streams 11-14 us after the publish)
      // (not in swap mode: there the remainder also waits for the copy-in on `st`)
      cudaStream_t def_st = (wv_gate && P.mode != DYSEL_SWAP) ? gate_st : ctx->rem_hi;
      for (int k = 0; k < K; ++k) {
        const int v = k == 0 ? def : (k <= def ? k - 1 : k);
        cudaStream_t rs = k == 0 ? def_st : ctx->rem[v];
        dysel_slice s = base_slice(P);
        s.variant = v;
        s.role = DYSEL_ROLE_BATCH;
        s.granule_begin = rem_begin;
        s.granule_count = rem_end - rem_begin;
        s.gate = &ctx->d_prof->sel;
        s.gate_full_grid = k == 0 ? 1u : 0u;
        if (!(k == 0 && def_st == gate_st)) DYSEL_CUDA_TRY(ctx, cudaStreamWaitEvent(rs, ctx->ev_fork2, 0));
        DYSEL_TRY(R.v[v].fn(&s, base_args.data(), rs, R.v[v].user));
        DYSEL_TRY(check_launch(ctx, "variant gated batch"));
        DYSEL_CUDA_TRY(ctx, cudaEventRecord(ctx->ev_join2[v], rs));

      }
      if (rep) {   // each remainder stream's completion
        cudaEventRecord(tev[2], def_st);
        for (int v = 0; v < K; ++v) cudaStreamWaitEvent(ctx->query, ctx->ev_join2[v], 0);
        cudaEventRecord(tev[3], ctx->query);
      }
      for (int v = 0; v < K; ++v) DYSEL_CUDA_TRY(ctx, cudaStreamWaitEvent(st, ctx->ev_join2[v], 0));
    }
    // the call completes with every profiling copy (stream semantics)
    if (rep) {
      for (int v = 0; v < K; ++v) cudaStreamWaitEvent(ctx->query, ctx->ev_join[v], 0);
      cudaEventRecord(tev[4], ctx->query);   // every profiling copy done
    }
    for (int v = 0; v < K; ++v) DYSEL_CUDA_TRY(ctx, cudaStreamWaitEvent(st, ctx->ev_join[v], 0));
    if (rep) cudaEventRecord(tev[5], st);
    // selection for the activation-flag cache: async D2H, resolved lazily
    DYSEL_TRY(push_pending_sel(ctx, key, &ctx->d_prof->sel, st));
    if (rep) {   // a report costs a D2H copy + sync
      DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(ctx->h_prof, ctx->d_prof, sizeof(DevProf), cudaMemcpyDeviceToHost, st));
      DYSEL_CUDA_TRY(ctx, cudaStreamSynchronize(st));
      DYSEL_TRY(check_sel_timeout(ctx));
      selected = (int)(ctx->h_prof->sel & 0xff);
      ctx->sel_cache[key] = selected;
    }
  } else if (!async) {
    // ---- paper host path, synchronous
    for (int v = 0; v < K; ++v) DYSEL_CUDA_TRY(ctx, cudaStreamWaitEvent(st, ctx->ev_join[v], 0));
    DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(ctx->h_prof, ctx->d_prof, sizeof(DevProf), cudaMemcpyDeviceToHost, st));
    DYSEL_CUDA_TRY(ctx, cudaStreamSynchronize(st));
    selected = (int)(ctx->h_prof->sel & 0xff);
  } else {
    // ---- paper host path, asynchronous: poll + eager chunks
    bool done[DYSEL_MAX_VARIANTS] = {};
    int ndone = 0;
    uint64_t best_pack = ~0ull;
    int best_v = def;
    cudaEvent_t chunk_ev = nullptr;
    cudaEventCreateWithFlags(&chunk_ev, cudaEventDisableTiming);
    bool chunk_inflight = false;
    while (ndone < K) {
      for (int v = 0; v < K; ++v) {
        if (done[v]) continue;
        cudaError_t q = cudaEventQuery(ctx->ev_join[v]);
        if (q == cudaErrorNotReady) continue;
        if (q != cudaSuccess) {
          cudaEventDestroy(chunk_ev);
          DYSEL_CUDA_TRY(ctx, q);
        }
        done[v] = true;
        ndone++;
        DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(&ctx->h_prof->slot[v], &ctx->d_prof->slot[v], sizeof(dysel_timer_slot),
                                            cudaMemcpyDeviceToHost, ctx->query));
        DYSEL_CUDA_TRY(ctx, cudaStreamSynchronize(ctx->query));
        uint64_t pk =
            (host_score(ctx->h_prof->slot[v], R, P, v, mode, ctx->n_sm) << 8) |
            (uint64_t)v;
        if (pk < best_pack) {
          best_pack = pk;
          best_v = v;
        }
      }
      if (ndone == K) break;
      if (rem_begin < rem_end && (!chunk_inflight || cudaEventQuery(chunk_ev) == cudaSuccess)) {
        uint64_t chunk = std::max<uint64_t>(1, (2ull * ctx->n_sm + P.h[best_v] - 1) / P.h[best_v]);
        chunk = std::min(chunk, rem_end - rem_begin);
        dysel_slice s = base_slice(P);
        s.variant = best_v;
        s.role = DYSEL_ROLE_EAGER;
        s.granule_begin = rem_begin;
        s.granule_count = chunk;
        DYSEL_TRY(R.v[best_v].fn(&s, base_args.data(), st, R.v[best_v].user));
        DYSEL_TRY(check_launch(ctx, "variant eager chunk"));
        cudaEventRecord(chunk_ev, st);
        chunk_inflight = true;
        add_slice_rec(rep, s);
        mark_units(rep, s);
        rem_begin += chunk;
        eager_units += chunk;
      }
    }
    cudaEventDestroy(chunk_ev);
    for (int v = 0; v < K; ++v) DYSEL_CUDA_TRY(ctx, cudaStreamWaitEvent(st, ctx->ev_join[v], 0));
    selected = (int)(best_pack & 0xff);
    ctx->h_prof->sel = best_pack;
  }
  if (host_orch) {
    if (P.mode == DYSEL_SWAP) {
      for (size_t k = 0; k < R.sandbox_args[selected].size(); ++k) {
        int a = R.sandbox_args[selected][k];
        DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(base_args[a], vargs[selected][a], sandbox_bytes[k],
                                            cudaMemcpyDeviceToDevice, st));
      }
    }
    if (rem_begin < rem_end) {
      dysel_slice s = base_slice(P);
      s.variant = selected;
      s.role = DYSEL_ROLE_BATCH;
      s.granule_begin = rem_begin;
      s.granule_count = rem_end - rem_begin;
      DYSEL_TRY(R.v[selected].fn(&s, base_args.data(), st, R.v[selected].user));
      DYSEL_TRY(check_launch(ctx, "variant batch"));
      add_slice_rec(rep, s);
      mark_units(rep, s);
    }
    ctx->sel_cache[key] = selected;
  }
  if (rep) {
    if (!host_orch && rep) {
      dysel_slice s = base_slice(P);
      s.variant = selected;
      s.role = DYSEL_ROLE_BATCH;
      s.granule_begin = rem_begin;
      s.granule_count = rem_end > rem_begin ? rem_end - rem_begin : 0;
      add_slice_rec(rep, s);
      mark_units(rep, s);
    } else {
      // host paths read slots already (sync) — refresh all for the report
      DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(ctx->h_prof->slot, ctx->d_prof->slot, sizeof(ctx->h_prof->slot),
                                          cudaMemcpyDeviceToHost, st));
      DYSEL_CUDA_TRY(ctx, cudaStreamSynchronize(st));
    }
    if (P.mode == DYSEL_SWAP) {   // winner's private prefix became the output
      for (uint64_t j = 0; j < P.c && j < rep->unit_variant_cap; ++j)
        if (rep->unit_variant) rep->unit_variant[j] = (uint8_t)selected;
    }
    rep->selected = selected;
    rep->eager_units = eager_units;
    {   // timeline, all from the call's init kernel: [0] first profiling CTA,
        // [1] selection published (device paths) -- %globaltimer; event-timed
        // (the event before the init kernel; same origin within ~1 us): [2]
        // selection known on the gate stream, [3] the default's remainder
        // done, [4] every remainder done, [5] every profiling copy done, [6]
        // the call done
      uint64_t t0 = ~0ull;
      for (int v = 0; v < K; ++v) t0 = std::min<uint64_t>(t0, ctx->h_prof->slot[v].t_start_min);
      const uint64_t ti = ctx->h_prof->t_init;
      for (int i = 0; i < 8; ++i) rep->timeline_ns[i] = ~0ull;
      if (t0 != ~0ull && t0 >= ti) {
        rep->timeline_ns[0] = t0 - ti;
        if (!host_orch && ctx->h_prof->t_publish > ti) rep->timeline_ns[1] = ctx->h_prof->t_publish - ti;
      }
      if (!host_orch) {
        cudaStreamSynchronize(st);
        for (int i = 1; i < 6; ++i) {
          float ms = 0.0f;
          if (tev[i] && cudaEventElapsedTime(&ms, tev[0], tev[i]) == cudaSuccess) rep->timeline_ns[i + 1] = (uint64_t)(ms * 1e6);
        }
        cudaGetLastError();
      }
    }
    for (int v = 0; v < K; ++v) {
      const dysel_timer_slot &t = ctx->h_prof->slot[v];
      rep->makespan_ns[v] = t.t_end_max - t.t_start_min;
      rep->units[v] = t.units;
      rep->cycles[v] = t.cycles;
      rep->score[v] = ctx->h_prof->decided[v] == 2u   // dominated (A-32): cannot win
                          ? (1ull << 56) - 1
                          : host_score(t, R, P, v, mode, ctx->n_sm);
    }
    rep->host_ns = now_ns() - t_host0;
  }
  for (auto &e : tev)
    if (e) cudaEventDestroy(e);
  return DYSEL_OK;
}
