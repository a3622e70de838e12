// DySel transposed SpMV pool: y += A^T x over the plan's CSR,
// the scatter-add kernel whose work-groups write OVERLAPPING outputs through
// global atomics.  Such a kernel cannot be split into productive slices that
// each own part of y, so the paper's only productive option is the swap-based
// partial-productive mode (§2.2, §3.3,
// Table 1): every variant profiles the SAME slice into a private
// copy of y (initialised from y), the winner's copy is swapped in, and the
// winner runs the rest.  Variants carry DYSEL_V_ATOMICS, so AUTO resolves to
// swap and SWAP|ASYNC is rejected by the planner -- except on the device path's
// additive swap (readings A-47 / A-47b below), whose final output is y itself.
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

struct NoStop {
  __device__ __forceinline__ bool operator()() const { return false; }
};

// One 256-row unit u of variant VID: y[col] += val * x[row] for its rows (one
// fire-and-forget reduction per nonzero).  stop(): checked by every thread at
// safe points (thread variant: every 32 entries; warp variants: between rows /
// rounds, warp-uniformly); a stopped unit's output is partial (private
// copies only, which are then discarded).
template <int VID, class Stop>
__device__ __forceinline__ void spmtv_unit(const SpmtvArgs &a, float *__restrict__ y, uint64_t u, const Stop &stop) {
  const int64_t r0 = (int64_t)u * kSpmtvRows;
  if constexpr (VID == 0) {   // thread per row, entries in CSR order
    const int64_t r = r0 + threadIdx.x;
    if (r >= a.n_rows) return;
    const float xr = __ldg(a.x + r);
    int k = __ldg(a.row_ptr + r);
    const int e = __ldg(a.row_ptr + r + 1);
    while (k < e) {
      const int ke = min(e, k + 32);
#pragma unroll 4
      for (; k < ke; ++k) red_add_nc(y + __ldg(a.col + k), __fmul_rn(__ldg(a.val + k), xr));
      if (k < e && stop()) return;
    }
  } else if constexpr (VID == 2) {   // warp per 32-row segment, its nonzeros as one flat stream
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t rw = r0 + w * 32;   // first row of this warp's segment
    if (rw >= a.n_rows) return;
    const int64_t rl = min(rw + lane, a.n_rows - 1);
    const int seg_b = __ldg(a.row_ptr + rw);
    const int end_l = __ldg(a.row_ptr + rl + 1);   // lanes past n_rows repeat the last row's end
    const float xl = rw + lane < a.n_rows ? __ldg(a.x + rw + lane) : 0.0f;
    const int seg_e = __shfl_sync(0xffffffffu, end_l, 31);
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
    int it = 0;
    for (int k = seg_b + lane; __any_sync(0xffffffffu, k < seg_e); k += 128, ++it) {
#pragma unroll
      for (int uu = 0; uu < 4; ++uu) step(k + 32 * uu);
      if ((it & 3) == 3 && __shfl_sync(0xffffffffu, stop() ? 1 : 0, 0)) return;
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
      const int b = __shfl_sync(0xffffffffu, beg_l, i), e = __shfl_sync(0xffffffffu, end_l, i);
      const float xr = __shfl_sync(0xffffffffu, x_l, i);
#pragma unroll 4
      for (int k = b + lane; k < e; k += 32) red_add_nc(y + __ldg(a.col + k), __fmul_rn(__ldg(a.val + k), xr));
      if ((i & 7) == 7 && __shfl_sync(0xffffffffu, stop() ? 1 : 0, 0)) return;
    }
  }
}

// Generic-launcher copies (paper host path, pure full-grid runs): one unit
// per CTA over a slice; the gated remainder (no timer) walks its slice.
template <int VID>
__global__ void __launch_bounds__(256) spmtv_kernel(SpmtvArgs a, float *__restrict__ y, dysel_slice s) {
  __shared__ dysel_prof_smem psm;
  if (!dysel_gate_open(s)) return;
  const uint32_t wa[3] = {1, 1, 1};
  const bool persistent = s.timer == nullptr && s.gate != nullptr;
  const uint64_t n_cta = persistent ? dysel_slice_ctas(s, wa) : (uint64_t)blockIdx.x + 1;
  dysel_prof_begin(s, psm);
  uint32_t units = 0;
  for (uint64_t cta = blockIdx.x; cta < n_cta; cta += gridDim.x) {
    uint64_t u[3];
    if (!dysel_cta_origin(s, wa, cta, u)) continue;
    ++units;
    spmtv_unit<VID>(a, y, u[0], NoStop());
  }
  dysel_prof_end(s, psm, persistent ? 0u : units);
}

static uint64_t g_spmtv_wave[DYSEL_SPMTV_NVARIANTS] = {0, 0, 0};   // occupancy x #SM

template <int VID>
static dysel_status spmtv_variant_fn(const dysel_slice *s, void *const *args, void *stream, void *) {
  const SpmtvArgs &a = *(const SpmtvArgs *)args[1];
  float *y = (float *)args[0];
  static const uint32_t WA[3] = {1, 1, 1};
  uint64_t ctas = dysel_slice_ctas(*s, WA);
  if (ctas == 0) return DYSEL_OK;
  // gated remainder: the full grid, whose CTAs the block scheduler hands out
  // dynamically (skewed rows make a static persistent-wave walk imbalanced)
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
  const int def = DYSEL_SPMTV_SCATTER_WARP;
  DYSEL_TRY(dysel_register_variants(ctx, kSpmtvSig, v, DYSEL_SPMTV_NVARIANTS, def));
  mark_builtin(ctx, kSpmtvSig);
  return DYSEL_OK;
}

// ---------------------------------------------------------------------------
// Swap-mode device path (reading A-47).  The generic
// launcher's swap copies y into K private outputs, profiles the NDRange
// prefix, and copies the winner's private output back before the remainder
// may start (measured +50% single shot: heavy-tailed prefix units and the
// copies).  For this scatter-add kernel the output is a commutative
// reduction (y += A^T x), so the swap is done additively:
//   1. the K private outputs start at ZERO (one memset) and each variant
//      reduces the SAME profiling units -- the plan's first light units
//      (reading A-45: no long row decides the sync latency) -- into its own;
//   2. profiling is timed per unit (busy-time score, A-6) with dominance: a
//      variant that provably cannot win is decided at once and its CTAs stop
//      (its private output is discarded); the last variant decided publishes;
//   3. the default's persistent remainder kernel (PDL, waiting for the
//      selection: SYNC, Table 1) -- or the winner's, device-launched by a
//      one-warp switch kernel when the default lost (A-42) -- claims, by
//      ticket, first the add-in chunks of the winner's private output
//      (y += private, 128-bit red.global.add: concurrent with the remainder's
//      own reductions, both are additions), then the heavy units
//      (nonzeros descending, A-40), then the other light units.
// The result equals y0 + A^T x up to the (already free) order of the fp32
// additions; Table 1's K private outputs are kept (report.sandbox_buffers).
constexpr int kSwapAddChunk = 16384;
constexpr int kSwapMaxSm = 256;
__device__ __forceinline__ uint32_t swap_smid() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r % kSwapMaxSm;
}   // floats of the winner's private output per add-in ticket

struct SwapState {
  // claim counters and the polled selection word each on its own 128-byte
  // line, away from the profiling completion chain's atomics (as SpmvState)
  alignas(128) uint32_t rem_ctr;      // tickets: add-in chunks, then heavy units
  alignas(128) uint32_t light_ctr;    // the other light units (eager phase and remainder share it, A-47b)
  alignas(128) uint32_t eager_units;  // light units done before the selection (ASYNC, A-47b)
  alignas(128) uint64_t sel;
  alignas(128) uint32_t variants_done;
  uint64_t best;
  uint64_t best_total;
  uint32_t ctas_done[DYSEL_SPMTV_NVARIANTS];
  uint32_t decided[DYSEL_SPMTV_NVARIANTS];   // 0 running, 1 completed, 2 dominated
  uint64_t busy[DYSEL_SPMTV_NVARIANTS];
  uint64_t lb[DYSEL_SPMTV_NVARIANTS];
  uint64_t max_busy[DYSEL_SPMTV_NVARIANTS];
  uint64_t aborted[DYSEL_SPMTV_NVARIANTS];
  dysel_timer_slot slot[DYSEL_SPMTV_NVARIANTS];
  uint64_t vscore[DYSEL_SPMTV_NVARIANTS];   // packed final score of each completed variant (~0: dominated / none)
  uint64_t tl[4];   // 0 first profiling CTA, 1 publish, 2 first remainder claim, 3 last remainder claim
  uint32_t prof_on_sm[kSwapMaxSm];   // profiling CTAs resident per SM (the eager phase yields there, A-47b)
};

struct SwapParams {
  SpmtvArgs a;
  float *y;          // the real output
  float *priv;       // K private outputs, `stride` floats apart (16-byte aligned)
  uint64_t stride;
  int64_t n_cols;
  uint32_t K, c, n_units, n_sm, def, n_light;
  const int32_t *seq;   // plan's unit order (A-45); nullptr = identity
  uint32_t occ[DYSEL_SPMTV_NVARIANTS];
  uint32_t add_chunks;
  uint32_t abort;
  uint32_t eager;   // ASYNC (A-47b): the default's kernel claims light units into y before the selection
  uint64_t *host_sel;
  uint64_t *tl;
};

__device__ __forceinline__ uint32_t swap_unit_at(const SwapParams &p, uint32_t i) {
  return p.seq ? (uint32_t)__ldg(p.seq + i) : i;
}
__device__ __forceinline__ uint64_t swap_ld_relaxed(const uint64_t *q) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(q) : "memory");
  return v;
}

__device__ __forceinline__ void swap_decided(SwapState *st, const SwapParams &p) {
  __threadfence();
  if (atomicAdd(&st->variants_done, 1u) + 1u != p.K) return;
  __threadfence();
  unsigned long long fin = atomicAdd((unsigned long long *)&st->best, 0ull);
  if ((uint32_t)(fin & 0xffu) != p.def) {   // switch margin (reading A-50)
    const unsigned long long ds = swap_ld_relaxed(&st->vscore[p.def]);
    if (ds != ~0ull && (fin >> 8) * 9ull > (ds >> 8) * 8ull) fin = ds;
  }
  atomicExch((unsigned long long *)&st->sel, fin);
  if (p.host_sel) *(volatile uint64_t *)p.host_sel = fin;
  if (p.tl) p.tl[1] = dysel_globaltimer();
  __threadfence();
}

// Resets the state and zeroes the K private outputs (additive swap) in one
// grid: the profiling kernel's griddepcontrol.wait sees both complete.
__global__ void spmtv_swap_init_kernel(SwapState *st, int def, float4 *priv, uint64_t n4) {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const float4 z = make_float4(0.0f, 0.0f, 0.0f, 0.0f);
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += (uint64_t)gridDim.x * blockDim.x)
    priv[i] = z;
  if (blockIdx.x != 0) return;
  const int v = threadIdx.x;
  if (v < DYSEL_SPMTV_NVARIANTS) {
    st->ctas_done[v] = 0;
    st->decided[v] = 0;
    st->busy[v] = st->lb[v] = st->max_busy[v] = st->aborted[v] = 0;
    st->vscore[v] = ~0ull;
    st->slot[v].t_start_min = ~0ull;
    st->slot[v].t_end_max = 0;
    st->slot[v].units = 0;
    st->slot[v].cycles = 0;
  }
  if (v < 4) st->tl[v] = (v == 0 || v == 2) ? ~0ull : 0ull;
  for (int i = v; i < kSwapMaxSm; i += blockDim.x) st->prof_on_sm[i] = 0;
  if (v == 0) {
    st->rem_ctr = 0;
    st->light_ctr = 0;
    st->eager_units = 0;
    st->variants_done = 0;
    st->best = (((1ull << 56) - 1) << 8) | (uint64_t)def;
    st->sel = ~0ull;
    st->best_total = ~0ull;
  }
}

// Dominance stop of a profiling unit (private output: discardable).  Any
// thread may call it at its safe points; one report per ~2 us per CTA.
struct SwapStop {
  SwapState *st;
  const SwapParams *p;
  uint32_t pv;
  uint64_t thr_den;
  unsigned long long *s_last;
  const unsigned long long *s_start;
  volatile int *s_abort;
  mutable long long next_clk = 0;
  __device__ bool operator()() const {
    if (*s_abort) return true;
    if (!p->abort) return false;
    const long long ck = clock64();
    if (ck < next_clk) return false;
    next_clk = ck + 2048;
    const unsigned long long now = dysel_globaltimer();
    const unsigned long long last = *(volatile unsigned long long *)s_last;
    if (now - last < 2000 || atomicCAS(s_last, last, now) != last) return *s_abort != 0;
    const unsigned long long l = atomicAdd((unsigned long long *)&st->lb[pv], now - last) + (now - last);
    const unsigned long long thr = l * (unsigned long long)p->n_units / thr_den;
    const unsigned long long el = now - *(volatile const unsigned long long *)s_start;
    const unsigned long long cost = thr > el ? thr : el;
    const uint32_t dec = *(volatile uint32_t *)&st->decided[pv];
    if (dec == 1u) return false;
    if (dec == 2u || cost > swap_ld_relaxed(&st->best_total)) {
      *s_abort = 1;
      if (dec != 2u && atomicCAS(&st->decided[pv], 0u, 2u) == 0u) swap_decided(st, *p);
      return true;
    }
    return false;
  }
};

__global__ void __launch_bounds__(256, 1) spmtv_swap_prof_kernel(SwapParams p, SwapState *st) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  const uint32_t sm = swap_smid();
  if (threadIdx.x == 0) {   // before the remainder kernel may launch: its eager phase yields on this SM
    atomicAdd(&st->prof_on_sm[sm], 1u);
    __threadfence();
  }
  __syncthreads();
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  __shared__ unsigned long long s_last, s_start;
  __shared__ int s_abort, s_skip;
  __shared__ unsigned long long t0s[8], t1s[8], c0s[8], c1s[8];
  const uint32_t pv = blockIdx.x % p.K, b = blockIdx.x / p.K;
  const uint32_t u = swap_unit_at(p, b);
  const int tid = threadIdx.x;
  if (tid == 0) {
    s_abort = 0;
    s_last = dysel_globaltimer();
    s_start = s_last;
    s_skip = (p.abort && *(volatile uint32_t *)&st->decided[pv] == 2u) ? 1 : 0;
    if (p.tl) atomicMin((unsigned long long *)&p.tl[0], s_last);
  }
  __syncthreads();
  const bool skipped = s_skip != 0;
  const uint64_t thr_den = (uint64_t)p.c * max(1u, p.occ[pv]) * max(1u, p.n_sm);
  if (!skipped) {
    if ((tid & 31) == 0) {
      c0s[tid >> 5] = dysel_clock64();
      t0s[tid >> 5] = dysel_globaltimer();
    }
    const SwapStop stop{st, &p, pv, thr_den, &s_last, &s_start, &s_abort};
    float *out = p.priv + (uint64_t)pv * p.stride;
    if (pv == 0) spmtv_unit<0>(p.a, out, u, stop);
    else if (pv == 1) spmtv_unit<1>(p.a, out, u, stop);
    else spmtv_unit<2>(p.a, out, u, stop);
    if ((tid & 31) == 0) {
      t1s[tid >> 5] = dysel_globaltimer();
      c1s[tid >> 5] = dysel_clock64();
    }
  }
  __syncthreads();
  if (tid == 0) atomicSub(&st->prof_on_sm[sm], 1u);
  if (tid >= 32) return;
  unsigned long long t0 = tid < 8 ? t0s[tid] : ~0ull, t1 = tid < 8 ? t1s[tid] : 0ull;
  unsigned long long c0 = tid < 8 ? c0s[tid] : ~0ull, c1 = tid < 8 ? c1s[tid] : 0ull;
#pragma unroll
  for (int o = 4; o > 0; o >>= 1) {
    t0 = min(t0, __shfl_xor_sync(0xffffffffu, t0, o));
    t1 = max(t1, __shfl_xor_sync(0xffffffffu, t1, o));
    c0 = min(c0, __shfl_xor_sync(0xffffffffu, c0, o));
    c1 = max(c1, __shfl_xor_sync(0xffffffffu, c1, o));
  }
  if (tid != 0) return;
  dysel_timer_slot *slot = &st->slot[pv];
  if (!skipped) {
    atomicMin((unsigned long long *)&slot->t_start_min, t0);
    atomicMax((unsigned long long *)&slot->t_end_max, t1);
    atomicAdd((unsigned long long *)&slot->cycles, c1 - c0);
    atomicAdd((unsigned long long *)&st->busy[pv], t1 - t0);
    atomicAdd((unsigned long long *)&st->lb[pv], t1 - s_last);
    atomicMax((unsigned long long *)&st->max_busy[pv], t1 - t0);
  }
  if (skipped || s_abort) atomicAdd((unsigned long long *)&st->aborted[pv], 1ull);
  atomicAdd((unsigned long long *)&slot->units, 1ull);
  __threadfence();
  if (atomicAdd(&st->ctas_done[pv], 1u) + 1u == p.c && atomicCAS(&st->decided[pv], 0u, 1u) == 0u) {
    __threadfence();
    const unsigned long long bz = atomicAdd((unsigned long long *)&st->busy[pv], 0ull);
    const unsigned long long mb = atomicAdd((unsigned long long *)&st->max_busy[pv], 0ull);
    const unsigned long long thr = bz * (unsigned long long)p.n_units / thr_den;
    unsigned long long pred = thr > mb ? thr : mb;
    const unsigned long long cap = (1ull << 56) - 1;
    if (pred > cap) pred = cap;
    atomicMin((unsigned long long *)&st->best_total, pred);
    st->vscore[pv] = (pred << 8) | pv;
    __threadfence();
    atomicMin((unsigned long long *)&st->best, (pred << 8) | pv);
    swap_decided(st, p);
  }
}

__device__ __forceinline__ void red_add_v4(float *q, float4 v) {
  asm volatile("red.global.add.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(q), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w)
               : "memory");
}

// Persistent remainder of variant VID (pool index = VID).  ASYNC (reading
// A-47b): the default's kernel first claims light units eagerly, straight into
// y, until the selection is published.  Then it exits unless VID won; tickets:
// add-in chunks, then heavy units, then the light units nobody claimed yet.
template <int VID>
__global__ void __launch_bounds__(256) spmtv_swap_rem_kernel(SwapParams p, SwapState *st) {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  __shared__ uint32_t s_t;
  __shared__ int s_go;
  const uint32_t L1 = max(p.c, p.n_light);
  const uint32_t n_heavy = p.n_units - L1, n_lt = L1 - p.c;
  if (p.eager && (uint32_t)VID == p.def) {
    const volatile uint32_t *on_sm = &st->prof_on_sm[swap_smid()];
    for (;;) {
      if (threadIdx.x == 0) {
        // yield while a profiling CTA shares this SM: its units are timed as
        // in the synchronous flow (per-SM contention would bias the scores)
        for (uint32_t ns = 64; *on_sm != 0u && swap_ld_relaxed(&st->sel) == ~0ull; ns = ns < 1024 ? 2 * ns : ns)
          __nanosleep(ns);
        s_t = swap_ld_relaxed(&st->sel) != ~0ull ? ~0u : atomicAdd(&st->light_ctr, 1u);
      }
      __syncthreads();
      const uint32_t t = s_t;
      __syncthreads();
      if (t >= n_lt) break;   // selected (~0u) or no light unit left
      spmtv_unit<VID>(p.a, p.y, swap_unit_at(p, p.c + t), NoStop());
      if (threadIdx.x == 0) atomicAdd(&st->eager_units, 1u);
    }
  }
  if (threadIdx.x == 0) {
    uint64_t sel = swap_ld_relaxed(&st->sel);
    for (uint32_t ns = 32; sel == ~0ull; ns = ns < 1024 ? 2 * ns : ns) {
      __nanosleep(ns);
      sel = swap_ld_relaxed(&st->sel);
    }
    s_go = (int)(sel & 0xff) == VID;
  }
  __syncthreads();
  if (!s_go) return;
  const float *pw = p.priv + (uint64_t)VID * p.stride;
  const uint32_t n_first = p.add_chunks + n_heavy;
  const bool y_vec = ((uintptr_t)p.y & 15) == 0;
  bool first = true;
  for (;;) {
    if (threadIdx.x == 0) {
      uint32_t t = atomicAdd(&st->rem_ctr, 1u);
      if (t >= n_first) {   // light units: shared counter with the eager phase
        const uint32_t l = atomicAdd(&st->light_ctr, 1u);
        t = l < n_lt ? n_first + l : ~0u;
      }
      s_t = t;
      if (p.tl && first) atomicMin((unsigned long long *)&p.tl[2], (unsigned long long)dysel_globaltimer());
    }
    first = false;
    __syncthreads();
    const uint32_t t = s_t;
    __syncthreads();
    if (t == ~0u) break;
    if (t < p.add_chunks) {   // y += the winner's private output (its profiled units' contributions)
      const int64_t i0 = (int64_t)t * kSwapAddChunk, i1 = min(i0 + (int64_t)kSwapAddChunk, (int64_t)p.n_cols);
      if (y_vec) {
        for (int64_t i = i0 + 4 * threadIdx.x; i < i1; i += 4 * blockDim.x) {
          if (i + 3 < i1) {
            const float4 v = *reinterpret_cast<const float4 *>(pw + i);
            if (v.x != 0.0f || v.y != 0.0f || v.z != 0.0f || v.w != 0.0f) red_add_v4(p.y + i, v);
          } else {
            for (int64_t q = i; q < i1; ++q)
              if (pw[q] != 0.0f) red_add_nc(p.y + q, pw[q]);
          }
        }
      } else {
        for (int64_t i = i0 + threadIdx.x; i < i1; i += blockDim.x)
          if (pw[i] != 0.0f) red_add_nc(p.y + i, pw[i]);
      }
      continue;
    }
    const uint32_t q = t - p.add_chunks;
    const uint32_t u = q < n_heavy ? swap_unit_at(p, L1 + q) : swap_unit_at(p, p.c + (q - n_heavy));
    spmtv_unit<VID>(p.a, p.y, u, NoStop());
  }
  if (p.tl && threadIdx.x == 0) atomicMax((unsigned long long *)&p.tl[3], (unsigned long long)dysel_globaltimer());
}

__global__ void spmtv_swap_switch_kernel(SwapParams p, SwapState *st) {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  if (threadIdx.x != 0) return;
  uint64_t sel = swap_ld_relaxed(&st->sel);
  for (uint32_t ns = 32; sel == ~0ull; ns = ns < 1024 ? 2 * ns : ns) {
    __nanosleep(ns);
    sel = swap_ld_relaxed(&st->sel);
  }
  const uint32_t w = (uint32_t)(sel & 0xff);
  if (w == p.def || w >= p.K) return;
  const unsigned g = p.occ[w] * p.n_sm;
  if (w == 0) spmtv_swap_rem_kernel<0><<<g, 256, 0, cudaStreamFireAndForget>>>(p, st);
  else if (w == 1) spmtv_swap_rem_kernel<1><<<g, 256, 0, cudaStreamFireAndForget>>>(p, st);
  else spmtv_swap_rem_kernel<2><<<g, 256, 0, cudaStreamFireAndForget>>>(p, st);
}

static int g_swap_occ[DYSEL_SPMTV_NVARIANTS] = {0, 0, 0};

static cudaError_t swap_launch(const void *fn, unsigned grid, unsigned block, cudaStream_t st, void **args, bool pdl) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(block);
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 1 : 0;
  return cudaLaunchKernelExC(&cfg, fn, args);
}

static dysel_status spmtv_swap_device(dysel_ctx *ctx, dysel_spmv_plan *pl, const float *d_x, float *d_y,
                                      const Plan &P, uint32_t mode, cudaStream_t st, dysel_report *rep,
                                      const std::string &key, int def) {
  const uint64_t t_host0 = now_ns();
  const int K = DYSEL_SPMTV_NVARIANTS;
  if (!g_swap_occ[0]) {
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&g_swap_occ[0], spmtv_swap_rem_kernel<0>, 256, 0);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&g_swap_occ[1], spmtv_swap_rem_kernel<1>, 256, 0);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&g_swap_occ[2], spmtv_swap_rem_kernel<2>, 256, 0);
    cudaGetLastError();
  }
  if (!ctx->d_spmtv_state) {
    DYSEL_CUDA_TRY(ctx, cudaMalloc(&ctx->d_spmtv_state, sizeof(SwapState)));
    DYSEL_CUDA_TRY(ctx, cudaMemset(ctx->d_spmtv_state, 0, sizeof(SwapState)));
  }
  SwapState *dst = (SwapState *)ctx->d_spmtv_state;
  SwapParams p;
  memset(&p, 0, sizeof(p));
  p.a = SpmtvArgs{pl->dev.n_rows, pl->dev.row_ptr, pl->dev.col, pl->dev.val, d_x};
  p.y = d_y;
  p.n_cols = pl->dev.n_cols;
  p.stride = ((uint64_t)pl->dev.n_cols + 3) / 4 * 4;
  p.K = K;
  p.c = (uint32_t)P.c;
  p.n_units = pl->n_units;
  p.n_sm = (uint32_t)ctx->n_sm;
  p.def = def;
  p.seq = pl->seq;
  p.n_light = pl->seq ? pl->n_light : pl->n_units;
  for (int i = 0; i < K; ++i) p.occ[i] = (uint32_t)std::max(1, g_swap_occ[i]);
  p.add_chunks = (uint32_t)((pl->dev.n_cols + kSwapAddChunk - 1) / kSwapAddChunk);
  p.abort = (mode & DYSEL_NO_ABORT) ? 0u : 1u;
  p.eager = (mode & DYSEL_ASYNC) ? 1u : 0u;
  const size_t priv_bytes = (size_t)K * p.stride * sizeof(float);
  DYSEL_TRY(scratch(ctx, ctx->sandbox[0], priv_bytes));
  p.priv = (float *)ctx->sandbox[0].ptr;
  if (rep) p.tl = dst->tl;
  const int pend = reserve_pending_sel(ctx, &p.host_sel);
  const uint64_t n4 = priv_bytes / sizeof(float4);   // private outputs start at 0 (additive swap)
  const unsigned init_grid = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)ctx->n_sm * 4, (n4 + 255) / 256));
  spmtv_swap_init_kernel<<<init_grid, 256, 0, st>>>(dst, def, (float4 *)p.priv, n4);
  DYSEL_TRY(check_launch(ctx, "spmtv_swap_init_kernel"));
  void *args[] = {&p, &dst};
  DYSEL_CUDA_TRY(ctx, swap_launch((const void *)spmtv_swap_prof_kernel, p.K * p.c, 256, st, args, true));
  DYSEL_TRY(check_launch(ctx, "spmtv_swap_prof_kernel"));
  const void *rem[3] = {(const void *)spmtv_swap_rem_kernel<0>, (const void *)spmtv_swap_rem_kernel<1>,
                        (const void *)spmtv_swap_rem_kernel<2>};
  DYSEL_CUDA_TRY(ctx, swap_launch(rem[def], p.occ[def] * p.n_sm, 256, st, args, true));
  DYSEL_TRY(check_launch(ctx, "spmtv_swap_rem_kernel"));
  DYSEL_CUDA_TRY(ctx, swap_launch((const void *)spmtv_swap_switch_kernel, 1, 32, st, args, true));
  DYSEL_TRY(check_launch(ctx, "spmtv_swap_switch_kernel"));
  DYSEL_TRY(commit_pending_sel(ctx, pend, key, st));
  if (rep) {
    SwapState h;
    DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(&h, dst, sizeof(h), cudaMemcpyDeviceToHost, st));
    DYSEL_CUDA_TRY(ctx, cudaStreamSynchronize(st));
    const uint64_t cap = (1ull << 56) - 1;
    rep->mode_used = DYSEL_SWAP | (p.eager ? DYSEL_ASYNC : 0);
    rep->profiled = 1;
    rep->selected = (int)(h.sel & 0xff);
    rep->n_variants = K;
    rep->c = P.c;
    rep->n_granules = P.Gn;
    rep->eager_units = h.eager_units;
    rep->tail_units = p.n_units - p.c - h.eager_units;
    rep->sandbox_buffers = (uint32_t)K;
    rep->sandbox_bytes = priv_bytes;
    for (int v = 0; v < DYSEL_MAX_VARIANTS; ++v)
      rep->score[v] = rep->makespan_ns[v] = rep->units[v] = rep->cycles[v] = rep->busy_ns[v] = rep->aborted[v] = 0;
    for (int v = 0; v < K; ++v) {
      const dysel_timer_slot &t = h.slot[v];
      rep->units[v] = t.units;
      rep->cycles[v] = t.cycles;
      rep->makespan_ns[v] = t.t_end_max > t.t_start_min ? t.t_end_max - t.t_start_min : 0;
      rep->busy_ns[v] = h.busy[v];
      rep->aborted[v] = h.aborted[v];
      rep->score[v] = h.decided[v] == 2u ? cap
                                         : std::max<uint64_t>(h.busy[v] * p.n_units /
                                                                  ((uint64_t)p.c * p.occ[v] * p.n_sm),
                                                              h.max_busy[v]);
    }
    for (int i = 0; i < 8; ++i) rep->timeline_ns[i] = ~0ull;
    if (h.tl[0] != ~0ull) {
      rep->timeline_ns[0] = 0;
      rep->timeline_ns[1] = h.tl[1] ? h.tl[1] - h.tl[0] : ~0ull;
      rep->timeline_ns[5] = h.tl[2] != ~0ull ? h.tl[2] - h.tl[0] : ~0ull;
      rep->timeline_ns[6] = h.tl[3] ? h.tl[3] - h.tl[0] : ~0ull;
    }
    if (rep->unit_variant)
      for (uint64_t j = 0; j < rep->unit_variant_cap && j < P.Gn; ++j) rep->unit_variant[j] = (uint8_t)rep->selected;
    if (rep->selected >= 0 && rep->selected < K) ctx->sel_cache[key] = rep->selected;
    rep->host_ns = now_ns() - t_host0;
  }
  return DYSEL_OK;
}

// Reading A-30d: the initial version of the SpMTV pool.  A thread per row
// issues one reduction per nonzero with no idle lanes and won every matrix
// whose longest row is short (rows of 1-48 entries, uniform or not, FEM 5x5:
// scripts/diag_spmtv_short.py, profiles/spmtv_shapes_r2.txt); a long row
// serialises it (2M-row power law, rows up to 4,096: 672 us vs scatter-warp's
// 241), so scatter-warp starts whenever some row exceeds kSpmtvThreadMaxRow.
constexpr int kSpmtvThreadMaxRow = 64;
static int spmtv_default(const dysel_spmv_plan *pl) {
  return pl->info.max_row_len <= kSpmtvThreadMaxRow ? DYSEL_SPMTV_SCATTER_THREAD : DYSEL_SPMTV_SCATTER_WARP;
}
// Reading A-3c for the SpMTV pool: a call shorter than ~2x the profiling
// latency (~25-35 us to the publish here) cannot pay for a single-shot
// profile.  dysel_spmv draws that line at 64 MiB; the scatter-add pool moves
// its bytes at about half SpMV's rate (1.5-3.3 TB/s measured: the L2
// reductions), so the same ~50 us sits at 128 MiB.
constexpr uint64_t kSpmtvMinProfBytes = 128ull << 20;

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
  if (!(mode & DYSEL_HOST_ORCH)) {   // device path: additive swap (reading A-47) when profiling is active
    auto it = ctx->reg.find(kSpmtvSig);
    if (it == ctx->reg.end()) return DYSEL_ERR_INVALID;
    uint32_t wa[DYSEL_SPMTV_NVARIANTS][3], vflags[DYSEL_SPMTV_NVARIANTS];
    for (int v = 0; v < DYSEL_SPMTV_NVARIANTS; ++v) {
      wa[v][0] = wa[v][1] = wa[v][2] = 1;
      vflags[v] = it->second.v[v].flags;
    }
    // reading A-47b: the additive swap fixes the final output space (y itself), so
    // ASYNC is accepted here; the paper's copy-back swap (HOST_ORCH, the generic
    // launcher) still rejects it (Table 1)
    const int def = spmtv_default(pl);
    Plan P;
    DYSEL_TRY(make_plan(ctx, U, wa, DYSEL_SPMTV_NVARIANTS, f, ctx->n_sm, def, mode & ~(uint32_t)DYSEL_ASYNC, vflags,
                        &P));
    if (P.mode == DYSEL_SWAP) {
      const bool forced = (mode & DYSEL_FORCE_PROFILE) != 0;
      const bool one_wave = !forced && P.Gn <= g_spmtv_wave[def];   // reading A-3b
      const uint64_t bytes = 8ull * (uint64_t)pl->info.nnz + 8ull * (uint64_t)pl->dev.n_rows + 4ull +
                             8ull * (uint64_t)pl->dev.n_cols;
      const bool small = !forced && bytes < kSpmtvMinProfBytes;    // reading A-3c
      if (P.active && !one_wave && !small)
        return spmtv_swap_device(ctx, pl, d_x, d_y, P, mode, (cudaStream_t)stream, rep, key, def);
      // unprofiled (activation flag off, A-3b, A-3c): the cached selection, else the initial version (A-30d)
      resolve_pending(ctx, key.c_str());
      int v = def;
      auto c = ctx->sel_cache.find(key);
      if (c != ctx->sel_cache.end() && c->second >= 0 && c->second < DYSEL_SPMTV_NVARIANTS) v = c->second;
      if (rep) {
        const uint64_t t0 = now_ns();
        memset(rep->score, 0, sizeof(rep->score));
        memset(rep->makespan_ns, 0, sizeof(rep->makespan_ns));
        memset(rep->units, 0, sizeof(rep->units));
        memset(rep->cycles, 0, sizeof(rep->cycles));
        memset(rep->busy_ns, 0, sizeof(rep->busy_ns));
        memset(rep->aborted, 0, sizeof(rep->aborted));
        rep->mode_used = DYSEL_SWAP;
        rep->profiled = 0;
        rep->selected = v;
        rep->n_variants = DYSEL_SPMTV_NVARIANTS;
        rep->c = 0;
        rep->n_granules = P.Gn;
        rep->eager_units = rep->tail_units = 0;
        rep->sandbox_buffers = 0;
        rep->sandbox_bytes = 0;
        for (int i = 0; i < 8; ++i) rep->timeline_ns[i] = ~0ull;
        if (rep->unit_variant)
          for (uint64_t j = 0; j < rep->unit_variant_cap && j < P.Gn; ++j) rep->unit_variant[j] = (uint8_t)v;
        rep->host_ns = now_ns() - t0;
      }
      return dysel_spmtv_variant(ctx, pl, v, d_x, d_y, stream);
    }
  }
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
