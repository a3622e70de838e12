// DySel SpMV dispatch: the B200 device protocol.
//
// One dysel_spmv call, no host round trip (the paper's GPU host polling is
// slower than micro-profiling):
//   1. init kernel: reset the ctx's device state (tickets, timer slots, scores).
//   2. K profiling kernels, one per pool variant, on high-priority forked
//      streams (profiling has priority over eager work): each is
//      the variant's own plain kernel (own registers / occupancy) over its c
//      profiling units — fully mode: units v, v+K, ... (A-24); hybrid: units
//      [0, c) for every variant, the default writing y and the others a
//      sandbox (A-4).  Every CTA is timed (Fig. 7b, B200 form); the last CTA of
//      a variant scores it (packed atomicMin, A-7/A-8), the last variant
//      publishes the selection and — CDP2 tail launch — starts the winner's
//      plain kernel over every remainder unit nobody has claimed yet.
//   3. ASYNC: an eager kernel of the default ("initial") variant
//      claims remainder units by ticket on the launching stream while the
//      profiles run; publishing the selection grabs the unclaimed tickets for
//      the tail launch, so eager work stops and the winner takes over.
// Hybrid sandbox units of a provably losing variant stop early (dominance).
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>

#include "dysel_device.cuh"
#include "spmv_plan.h"

namespace dysel {

// Scores (reading A-6): default = mean per-unit busy
// time (CTA %globaltimer end - start) divided by the variant's resident CTAs
// per SM, i.e. the time per unit per execution slot of the plain kernel that
// will run the remainder.  DYSEL_SCORE_CYCLES: sum clock64 / units.
// DYSEL_SCORE_MAKESPAN: the paper's earliest start .. latest end (Fig. 7b).
struct SpmvState {
  uint32_t ticket;          // CDP scheme: eager / remainder tickets (units)
  uint32_t c2;              // claim kernels: remainder slot tickets after the selection (slot S + c2)
  uint64_t c1;              // claim kernels: eager slot tickets (low 32 bits) | published (bit 32)
  uint64_t sw;              // claim kernels: (S << 8) | selected pool index, ~0 until published
  uint64_t pure_ctr;        // pure full-grid runs: slot tickets; the last warp of a run resets both
  uint32_t pure_done;       // pure full-grid runs: warps finished
  uint32_t variants_done;
  uint64_t best;            // (score << 8) | pool variant
  uint64_t sel;             // final packed selection, ~0 until published
  uint64_t eager_units;
  uint64_t best_total;      // min over completed variants of busy * 1024 / occ (busy score) or makespan (ns)
  uint64_t tail_begin;      // first unit of the tail launch, ~0 if none
  uint32_t ctas_done[DYSEL_MAX_VARIANTS];
  uint32_t dominated[DYSEL_MAX_VARIANTS];
  uint64_t busy[DYSEL_MAX_VARIANTS];      // sum of unit busy times (ns)
  uint64_t lb[DYSEL_MAX_VARIANTS];        // lower bound of the final busy sum (ns)
  uint64_t aborted[DYSEL_MAX_VARIANTS];   // sandbox units stopped / skipped by dominance
  uint64_t max_busy[DYSEL_MAX_VARIANTS];  // longest profiled unit (ns)
  dysel_timer_slot slot[DYSEL_MAX_VARIANTS];
  // diagnostics timeline (absolute %globaltimer ns; dysel_report.timeline_ns):
  // 0 prof start (min), 1 publish, 2 prof end (max), 3/4 eager start/end,
  // 5/6 remainder start/end, 7 longest profiling unit
  uint64_t tl[8];
};

struct ProfParams {
  uint32_t K, c, n_units, p_end;   // p_end: first remainder unit
  uint32_t n_sm;
  uint32_t hybrid, async, contiguous, score_mode, def, tail, abort;
  uint32_t eager_grid;   // ASYNC: CTAs of the eager kernel (launched by the default's first profiling CTA)
  uint64_t *host_sel;    // mapped pinned word: the publishing CTA writes the selection here (cache)
  int32_t vids[DYSEL_SPMV_NVARIANTS];
  uint32_t occ[DYSEL_SPMV_NVARIANTS];
  float *sandbox;        // (K-1) * c * 256 floats (hybrid)
  uint64_t *tl;          // SpmvState::tl when a report is requested, else nullptr (no timeline atomics)
  uint8_t *unit_variant; // optional debug map (variant id per unit)
  uint32_t pure;         // pure full-grid run of one variant (self-resetting counters, no init kernel)
  uint32_t k_claim;      // claim kernels: max slots per claim (~kClaimNnz nonzeros of work)
  uint32_t solo;         // one claim kernel (the default's) also runs the winner's remainder (A-38)
  // claim kernels, heavy-first order (A-40): tickets [0, 8 n_heavy) are the
  // slots of heavy[] (skipped if profiled: unit < p_end), the rest the
  // remainder units in order (skipped if heavy)
  uint32_t n_heavy;
  const int32_t *heavy;
  const uint32_t *heavy_bits;
};

__global__ void spmv_state_init_kernel(SpmvState *s, int K, int def) {
  // the profiling kernel behind it (PDL) may launch now; it waits for this
  // grid's completion (griddepcontrol.wait) before touching the state
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const int v = threadIdx.x;
  if (v < DYSEL_MAX_VARIANTS) {
    s->ctas_done[v] = 0;
    s->dominated[v] = 0;
    s->busy[v] = 0;
    s->lb[v] = 0;
    s->aborted[v] = 0;
    s->max_busy[v] = 0;
    s->slot[v].t_start_min = ~0ull;
    s->slot[v].t_end_max = 0;
    s->slot[v].units = 0;
    s->slot[v].cycles = 0;
  }
  if (v < 8) s->tl[v] = (v == 0 || v == 3 || v == 5) ? ~0ull : 0ull;
  if (v == 0) {
    s->ticket = 0;
    s->c2 = 0;
    s->c1 = 0;
    s->sw = ~0ull;
    s->variants_done = 0;
    s->best = (((1ull << 56) - 1) << 8) | (uint64_t)def;
    s->sel = ~0ull;
    s->eager_units = 0;
    s->best_total = ~0ull;
    s->tail_begin = ~0ull;
  }
}

__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t *p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ld_relaxed_u64(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

// Dominance abort for hybrid sandbox units: every
// ~kPollNs one thread of the CTA adds the time elapsed since the last report
// to lb[v].  lb[v] only sums time variant v's units really spent, so it is a
// lower bound of v's final busy sum; once it exceeds the busy sum of a
// COMPLETED variant (best_total) v cannot be selected any more (in hybrid mode
// every variant profiles the same c units), so its sandbox work stops and its
// remaining sandbox units are skipped: the selection is the one running them
// to completion would give.
// The comparison is made in the units of the active score: busy score ->
// lb * 1024 / occ_v vs the best completed busy * 1024 / occ; makespan score
// (sequential profiling: the variant runs alone) -> time since the variant's
// first CTA started vs the best completed makespan.
constexpr uint64_t kPollNs = 2000;
constexpr long long kPollCycles = 2048;   // ~1 us at 1.9 GHz
constexpr uint32_t kWarpPollEvery = 4;
struct SandboxPoll {
  static constexpr bool active = true;
  unsigned long long *s_last;   // smem: last report time
  const unsigned long long *s_start;   // smem: this unit's start time
  volatile int *s_abort;        // smem
  unsigned long long *lb;
  const uint64_t *best_total;
  uint32_t *dominated;
  const uint64_t *t_start;      // makespan mode: the variant's earliest CTA start
  uint64_t scale_num;           // busy mode: lower bound of the predicted time = lb * num / den
  uint64_t scale_den;
  uint32_t makespan;
  // %globaltimer reads are slow (measured: polling it every loop step doubled
  // the per-unit time of CSR-V / CSR-W sandboxes); the per-SM cycle counter
  // (CS2R) gates them to one per kPollCycles per thread.
  mutable long long next_clk = 0;
  __device__ __forceinline__ bool due() const {
    const long long c = clock64();
    if (c < next_clk) return false;
    next_clk = c + kPollCycles;
    return true;
  }
  // thread-per-row loops: every thread polls (its own loop); warp loops: warp()
  __device__ __forceinline__ bool operator()() const {
    if (*s_abort) return true;
    return due() && report();
  }
  // warp-cooperative loops: only lane 0 reads the timer (cheap for the other
  // lanes; the caller combines with __any_sync)
  // Warp loops call this once per step (~one L2 round trip of work): checking
  // only every kWarpPollEvery-th step keeps the sandbox's per-unit time close
  // to the plain kernel's (measured).
  mutable uint32_t tick = 0;
  __device__ __forceinline__ bool warp() const {
    if ((++tick & (kWarpPollEvery - 1)) != 0) return false;   // warp-uniform
    if (*s_abort) return true;
    if ((threadIdx.x & 31) != 0) return false;
    return due() && report();
  }
  // Global values read by this thread's previous report, issued without waiting
  // (a blocking global atomic / load per report stalled the polling warp for
  // ~3 L2 round trips and doubled sandbox unit times).  Stale values stay
  // safe: lb only grows (a stale lb is still a lower bound) and best_total
  // only shrinks (a stale best aborts later, never wrongly).
  mutable unsigned long long lb_seen = 0, best_seen = ~0ull, t0_seen = ~0ull;
  mutable uint32_t dom_seen = 0;
  __device__ __forceinline__ bool report() const {
    const unsigned long long now = dysel_globaltimer();
    const unsigned long long last = *(volatile unsigned long long *)s_last;
    if (now - last < kPollNs) return false;
    if (atomicCAS(s_last, last, now) != last) return *s_abort != 0;   // another thread reports
    atomicAdd(lb, now - last);   // no return value: a fire-and-forget RED
    const unsigned long long l = lb_seen + (now - last);
    unsigned long long cost;
    if (makespan) {
      cost = t0_seen == ~0ull ? 0ull : now - t0_seen;
    } else {   // predicted full-grid time >= max(throughput bound, this unit's elapsed time)
      const unsigned long long thr = l * scale_num / scale_den;
      const unsigned long long el = now - *(volatile const unsigned long long *)s_start;
      cost = thr > el ? thr : el;
    }
    if (cost > best_seen || dom_seen != 0) {
      *s_abort = 1;
      atomicExch(dominated, 1u);
      return true;
    }
    lb_seen = ld_relaxed_u64((const uint64_t *)lb);
    best_seen = ld_relaxed_u64(best_total);
    dom_seen = ld_relaxed_u32(dominated);
    if (makespan) t0_seen = ld_relaxed_u64(t_start);
    return false;
  }
};

// resident CTAs per SM each plain variant kernel is compiled for (register cap)
// (CSR-V at 6/SM spills and measured slower on D4: 1.44 vs 1.35 ms)
#ifndef DYSEL_ELL_MINB
#define DYSEL_ELL_MINB 4
#endif
#ifndef DYSEL_ELL_CLAIM_MINB
#define DYSEL_ELL_CLAIM_MINB 4
#endif
#ifndef DYSEL_SJ_MINB
#define DYSEL_SJ_MINB 8
#endif
#ifndef DYSEL_SJ_CLAIM_MINB
#define DYSEL_SJ_CLAIM_MINB 6
#endif
constexpr int kSliceMinBlocks[DYSEL_SPMV_NVARIANTS] = {DYSEL_SJ_MINB, 4, DYSEL_ELL_MINB, (DYSEL_SJ_MINB < 6 ? DYSEL_SJ_MINB : 6), 5, 3};
constexpr uint32_t kSlots = kUnitRows / 32;   // 32-row warp slots per unit
// dynamic shared memory of each variant's kernels (CSR-T's staging buffers)
__host__ __device__ constexpr size_t dyn_smem(int vid) { return vid == DYSEL_SPMV_CSR_TMA ? sizeof(TmaStageBufs) : 0; }
inline size_t pool_dyn_smem(const ProfParams &p) {
  size_t b = 0;
  for (uint32_t i = 0; i < p.K; ++i) b = std::max(b, dyn_smem(p.vids[i]));
  return b;
}
// claim kernels: CTAs per SM (CSR-S / ELL at 8 spilled ~200 B in the claim loop)
constexpr int kClaimMinBlocks[DYSEL_SPMV_NVARIANTS] = {DYSEL_SJ_CLAIM_MINB, 4, DYSEL_ELL_CLAIM_MINB, DYSEL_SJ_CLAIM_MINB, 5, 3};

// Plain kernel of one variant over a slice: the exhaustive oracle's pure
// version, the activation-flag-off path, the tail-launched remainder, the
// gated remainder (NO_TAIL) and the host path's copies (dysel_device.cuh
// timing / gating).
//
// No static shared memory: the kernel's occupancy must not depend on the
// L1 / shared-memory carveout.  Measured on D4: with the 1 KB timing buffer
// in this kernel, the smallest carveout (which device-side launches get, and
// cudaSharedmemCarveoutMaxL1 asks for) cut CSR-W's resident CTAs and ran
// 1.52 ms instead of 0.93 ms; a large carveout shrinks L1 (fewer gathers in
// flight) and ran 2.25 ms.  Timed copies (host path) use spmv_slice_timed_kernel.
// diagnostics: resident CTAs per SM (current, max) of timeline-instrumented launches
__device__ uint32_t g_resident[2][1024];

__device__ __forceinline__ uint32_t smid() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}

template <int VID>
__global__ void __launch_bounds__(kUnitRows, kSliceMinBlocks[VID])
    spmv_slice_kernel(SpmvDev A, float *__restrict__ y, dysel_slice s, uint8_t *uv, uint64_t *tl) {
  if constexpr (VID == DYSEL_SPMV_CSR_TMA) tma_stage_prologue();
  if (!dysel_gate_open(s)) return;
  if (tl && threadIdx.x == 0) {
    atomicMin((unsigned long long *)&tl[5], (unsigned long long)dysel_globaltimer());
    const uint32_t sm = smid() & 1023;
    atomicMax(&g_resident[1][sm], atomicAdd(&g_resident[0][sm], 1u) + 1u);
  }
  const uint32_t j = (uint32_t)(s.granule_begin + (uint64_t)blockIdx.x * s.granule_stride);
  run_unit<VID>(A, j, y + (size_t)j * kUnitRows);
  if (uv && threadIdx.x == 0) uv[j] = (uint8_t)VID;
  if (tl) {
    __syncthreads();
    if (threadIdx.x == 0) {
      atomicMax((unsigned long long *)&tl[6], (unsigned long long)dysel_globaltimer());
      atomicSub(&g_resident[0][smid() & 1023], 1u);
    }
  }
}

// Timed copy (generic launcher / paper host path: s.timer set, Fig. 7b).
template <int VID>
__global__ void __launch_bounds__(kUnitRows, kSliceMinBlocks[VID])
    spmv_slice_timed_kernel(SpmvDev A, float *__restrict__ y, dysel_slice s) {
  if constexpr (VID == DYSEL_SPMV_CSR_TMA) tma_stage_prologue();
  __shared__ dysel_prof_smem psm;
  if (!dysel_gate_open(s)) return;
  dysel_prof_begin(s, psm);
  const uint32_t j = (uint32_t)(s.granule_begin + (uint64_t)blockIdx.x * s.granule_stride);
  run_unit<VID>(A, j, y + (size_t)j * kUnitRows);
  dysel_prof_end(s, psm, 1u);
}

__device__ void tail_launch(int vid, const SpmvDev &A, float *y, uint64_t u0, uint64_t n_units, uint8_t *uv,
                            uint64_t *tl) {
  dysel_slice s;
  memset(&s, 0, sizeof(s));
  s.granule_begin = u0;
  s.granule_count = n_units - u0;
  s.granule_stride = 1;
  s.g[0] = s.g[1] = s.g[2] = 1;
  s.G[0] = (uint32_t)n_units;
  s.G[1] = s.G[2] = 1;
  s.U[0] = n_units;
  s.U[1] = s.U[2] = 1;
  s.role = DYSEL_ROLE_BATCH;
  s.variant = vid;
  const unsigned grid = (unsigned)(n_units - u0);
  // Fire-and-forget, not a tail launch: the remainder depends only on the
  // selection, so it starts at once, overlapping the drain of the eager CTAs
  // and of the last profiling CTAs (a tail launch would wait for the whole
  // parent grid, including its fire-and-forget eager child).  Stream order is
  // kept: a grid completes only with all its device-launched children.
  const cudaStream_t ff = cudaStreamFireAndForget;
  switch (vid) {
    case 0: spmv_slice_kernel<0><<<grid, kUnitRows, dyn_smem(0), ff>>>(A, y, s, uv, tl); break;
    case 1: spmv_slice_kernel<1><<<grid, kUnitRows, dyn_smem(1), ff>>>(A, y, s, uv, tl); break;
    case 2: spmv_slice_kernel<2><<<grid, kUnitRows, dyn_smem(2), ff>>>(A, y, s, uv, tl); break;
    case 3: spmv_slice_kernel<3><<<grid, kUnitRows, dyn_smem(3), ff>>>(A, y, s, uv, tl); break;
    case 4: spmv_slice_kernel<4><<<grid, kUnitRows, dyn_smem(4), ff>>>(A, y, s, uv, tl); break;
    default: spmv_slice_kernel<5><<<grid, kUnitRows, dyn_smem(5), ff>>>(A, y, s, uv, tl); break;
  }
}

template <int VID>
__global__ void __launch_bounds__(kUnitRows, kSliceMinBlocks[VID])
    spmv_eager_kernel(SpmvDev A, float *__restrict__ y, SpmvState *st, uint32_t p_end, uint32_t n_units, uint8_t *uv,
                      uint64_t *tl);

// Debug (dysel_debug_spmv_device_launch): one thread launches the full grid of
// a variant from the device, fire-and-forget (how = 1) or as a tail launch (2).
__global__ void spmv_device_launch_kernel(SpmvDev A, float *y, int vid, uint64_t n_units, int how, uint64_t *tl) {
  if (how == 1) {
    tail_launch(vid, A, y, 0, n_units, nullptr, tl);
    return;
  }
  dysel_slice s;
  memset(&s, 0, sizeof(s));
  s.granule_count = n_units;
  s.granule_stride = 1;
  s.g[0] = s.g[1] = s.g[2] = 1;
  s.G[0] = (uint32_t)n_units;
  s.G[1] = s.G[2] = 1;
  s.U[0] = n_units;
  s.U[1] = s.U[2] = 1;
  s.role = DYSEL_ROLE_BATCH;
  s.variant = vid;
  const unsigned grid = (unsigned)n_units;
  const cudaStream_t ts = cudaStreamTailLaunch;
  switch (vid) {
    case 0: spmv_slice_kernel<0><<<grid, kUnitRows, dyn_smem(0), ts>>>(A, y, s, nullptr, tl); break;
    case 1: spmv_slice_kernel<1><<<grid, kUnitRows, dyn_smem(1), ts>>>(A, y, s, nullptr, tl); break;
    case 2: spmv_slice_kernel<2><<<grid, kUnitRows, dyn_smem(2), ts>>>(A, y, s, nullptr, tl); break;
    case 3: spmv_slice_kernel<3><<<grid, kUnitRows, dyn_smem(3), ts>>>(A, y, s, nullptr, tl); break;
    case 4: spmv_slice_kernel<4><<<grid, kUnitRows, dyn_smem(4), ts>>>(A, y, s, nullptr, tl); break;
    default: spmv_slice_kernel<5><<<grid, kUnitRows, dyn_smem(5), ts>>>(A, y, s, nullptr, tl); break;
  }
}

// The eager grid is launched from the device (fire-and-forget child of the
// default variant's first profiling CTA), so it can only start once profiling
// CTAs are resident: a host launch becomes runnable at the same instant as the
// profiling grids when calls are queued back to back, and the persistent
// eager CTAs then take every SM first (measured: +30% step time).
__device__ void eager_launch(int vid, const SpmvDev &A, float *y, SpmvState *st, const ProfParams &p) {
  const unsigned g = p.eager_grid;
  switch (vid) {
    case 0: spmv_eager_kernel<0><<<g, kUnitRows, dyn_smem(0), cudaStreamFireAndForget>>>(A, y, st, p.p_end, p.n_units, p.unit_variant, p.tl); break;
    case 1: spmv_eager_kernel<1><<<g, kUnitRows, dyn_smem(1), cudaStreamFireAndForget>>>(A, y, st, p.p_end, p.n_units, p.unit_variant, p.tl); break;
    case 2: spmv_eager_kernel<2><<<g, kUnitRows, dyn_smem(2), cudaStreamFireAndForget>>>(A, y, st, p.p_end, p.n_units, p.unit_variant, p.tl); break;
    case 3: spmv_eager_kernel<3><<<g, kUnitRows, dyn_smem(3), cudaStreamFireAndForget>>>(A, y, st, p.p_end, p.n_units, p.unit_variant, p.tl); break;
    case 4: spmv_eager_kernel<4><<<g, kUnitRows, dyn_smem(4), cudaStreamFireAndForget>>>(A, y, st, p.p_end, p.n_units, p.unit_variant, p.tl); break;
    default: spmv_eager_kernel<5><<<g, kUnitRows, dyn_smem(5), cudaStreamFireAndForget>>>(A, y, st, p.p_end, p.n_units, p.unit_variant, p.tl); break;
  }
}

// One profiling unit of variant VID (pool index pv): the b-th unit of its slice.
// CDP: the round-1 scheme (DYSEL_DEVICE_LAUNCH) whose eager kernel and
// remainder are launched from here; the default instantiation contains no
// device-side launch (a grid that can launch children does not release
// programmatic dependents early: measured, the PDL remainder waited for it).
template <int VID, bool CDP>
__device__ __forceinline__ void prof_unit(const SpmvDev &A, float *__restrict__ y, SpmvState *st,
                                          const ProfParams &p, uint32_t pv, uint32_t b) {
  __shared__ unsigned long long s_last, s_start;
  __shared__ int s_abort, s_skip;
  __shared__ dysel_prof_smem psm;
  const uint32_t tid = threadIdx.x;
  // predicted full-grid time of a variant (A-6): max(throughput bound, longest
  // unit); throughput bound = busy_sum * G_n / (c * occupancy * #SM)
  const uint64_t thr_den = (uint64_t)p.c * max(1u, p.occ[pv]) * max(1u, p.n_sm);
  const uint32_t j = p.hybrid ? b : (p.contiguous ? pv * p.c + b : pv + p.K * b);
  // hybrid (reading A-4'): every variant runs the shared units into its own
  // sandbox and may be stopped by dominance; the winner's sandbox is copied
  // into y when the selection is published, so its profiled work is the
  // productive one (never recomputed) whichever variant wins
  const bool productive = !p.hybrid;
  const bool sandbox = !productive;
  if constexpr (CDP)
    if (tid == 0 && b == 0 && pv == p.def && p.eager_grid) eager_launch(p.vids[p.def], A, y, st, p);
  if (tid == 0) {
    s_abort = 0;
    s_last = dysel_globaltimer();
    s_start = s_last;
    s_skip =(sandbox && p.abort && ld_relaxed_u32(&st->dominated[pv]) != 0) ? 1 : 0;
    if (!s_skip) atomicMin((unsigned long long *)&st->slot[pv].t_start_min, s_last);   // variant start (makespan)
    if (p.tl) atomicMin((unsigned long long *)&p.tl[0], s_last);
  }
  __syncthreads();
  const bool skipped = s_skip != 0;
  float *out = productive ? y + (size_t)j * kUnitRows : p.sandbox + ((size_t)pv * p.c + b) * kUnitRows;
  if (!skipped) {
    if ((tid & 31) == 0) {
      psm.c0[tid >> 5] = dysel_clock64();
      psm.t0[tid >> 5] = dysel_globaltimer();
    }
    // Dominance polling only in the thread-per-row variants (a single long
    // row makes their units take milliseconds); the warp-cooperative ones
    // (CSR-V, CSR-W) finish any unit in tens of us, and polling inside their
    // loops measured +60% per-unit time on D4 (CSR-W 15 -> 24.6 us).
    constexpr bool kPolled = VID == 0 || VID == 2 || VID == 3 || VID == 5;
    if (kPolled && sandbox && p.abort)
      run_unit<VID>(A, j, out,
                    SandboxPoll{&s_last, &s_start, &s_abort, (unsigned long long *)&st->lb[pv], &st->best_total,
                                &st->dominated[pv], &st->slot[pv].t_start_min, (uint64_t)p.n_units, thr_den,
                                p.score_mode == 2 ? 1u : 0u});
    else
      run_unit<VID>(A, j, out, NoPoll());
    if ((tid & 31) == 0) {
      psm.t1[tid >> 5] = dysel_globaltimer();
      psm.c1[tid >> 5] = dysel_clock64();
    }
  }
  __syncthreads();
  if (tid >= 32) return;
  // warp-shuffle reduction of the per-warp samples (min start, max end)
  unsigned long long t0 = tid < 8 ? psm.t0[tid] : ~0ull, t1 = tid < 8 ? psm.t1[tid] : 0ull;
  unsigned long long c0 = tid < 8 ? psm.c0[tid] : ~0ull, c1 = tid < 8 ? psm.c1[tid] : 0ull;
#pragma unroll
  for (int o = 4; o > 0; o >>= 1) {
    t0 = min(t0, __shfl_xor_sync(0xffffffffu, t0, o));
    t1 = max(t1, __shfl_xor_sync(0xffffffffu, t1, o));
    c0 = min(c0, __shfl_xor_sync(0xffffffffu, c0, o));
    c1 = max(c1, __shfl_xor_sync(0xffffffffu, c1, o));
  }
  bool publish = false;
  unsigned long long fin = 0;
  if (tid == 0) {
    dysel_timer_slot *slot = &st->slot[pv];
    if (!skipped) {
      atomicMin((unsigned long long *)&slot->t_start_min, t0);
      atomicMax((unsigned long long *)&slot->t_end_max, t1);
      atomicAdd((unsigned long long *)&slot->cycles, c1 - c0);
      atomicAdd((unsigned long long *)&st->busy[pv], t1 - t0);
      atomicAdd((unsigned long long *)&st->lb[pv], t1 - s_last);   // the rest of this unit's time
      atomicMax((unsigned long long *)&st->max_busy[pv], t1 - t0);
      if (p.tl) atomicMax((unsigned long long *)&p.tl[7], t1 - t0);
    }
    if (p.tl) atomicMax((unsigned long long *)&p.tl[2], dysel_globaltimer());
    if (skipped || s_abort) atomicAdd((unsigned long long *)&st->aborted[pv], 1ull);
    atomicAdd((unsigned long long *)&slot->units, 1ull);
    if (productive && p.unit_variant) p.unit_variant[j] = (uint8_t)VID;
    __threadfence();
    const uint32_t done = atomicAdd(&st->ctas_done[pv], 1u) + 1u;
    if (done == p.c) {
      // ---- variant complete: score, packed atomicMin (A-7, A-8)
      __threadfence();
      const unsigned long long a = atomicAdd((unsigned long long *)&slot->t_start_min, 0ull);
      const unsigned long long e = atomicAdd((unsigned long long *)&slot->t_end_max, 0ull);
      const unsigned long long cy = atomicAdd((unsigned long long *)&slot->cycles, 0ull);
      const unsigned long long bz = atomicAdd((unsigned long long *)&st->busy[pv], 0ull);
      const unsigned long long mb = atomicAdd((unsigned long long *)&st->max_busy[pv], 0ull);
      const bool dom = ld_relaxed_u32(&st->dominated[pv]) != 0;
      const unsigned long long cap = (1ull << 56) - 1;
      const unsigned long long thr = bz * (unsigned long long)p.n_units / thr_den;
      const unsigned long long pred = thr > mb ? thr : mb;   // predicted full-grid time (ns)
      unsigned long long score = p.score_mode == 1 ? cy / p.c : p.score_mode == 2 ? e - a : pred;
      if (dom || score > cap) score = cap;
      if (!dom) atomicMin((unsigned long long *)&st->best_total, p.score_mode == 2 ? e - a : pred);   // dominance units
      atomicMin((unsigned long long *)&st->best, (score << 8) | pv);
      __threadfence();
      const uint32_t vd = atomicAdd(&st->variants_done, 1u) + 1u;
      if (vd == p.K) {
        // ---- last variant: publish the selection, hand the remainder to the winner
        __threadfence();
        fin = atomicAdd((unsigned long long *)&st->best, 0ull);
        publish = true;
      }
    }
  }
  publish = __shfl_sync(0xffffffffu, publish ? 1 : 0, 0) != 0;
  if (!publish) return;
  fin = __shfl_sync(0xffffffffu, fin, 0);
  const uint32_t win = (uint32_t)(fin & 0xff);
  if (p.hybrid) {   // the winner's profiled units become the productive ones (warp 0 copies)
    const size_t n = min((size_t)p.c * kUnitRows, (size_t)A.n_rows);
    const float *src = p.sandbox + (size_t)win * p.c * kUnitRows;
    const size_t n4 = n / 4;
    for (size_t q = tid; q < n4; q += 32) reinterpret_cast<float4 *>(y)[q] = reinterpret_cast<const float4 *>(src)[q];
    for (size_t q = n4 * 4 + tid; q < n; q += 32) y[q] = src[q];
    if (p.unit_variant)
      for (uint32_t u = tid; u < p.c; u += 32) p.unit_variant[u] = (uint8_t)p.vids[win];
    __syncwarp();
    __threadfence();
  }
  if (tid != 0) return;
  atomicExch((unsigned long long *)&st->sel, fin);
  {   // claim kernels: close the eager ticket range; the default keeps whole
      // units only, so the switch point S is rounded up to a unit boundary
    const uint64_t old = atomicOr((unsigned long long *)&st->c1, 1ull << 32);
    const uint64_t n_slots = (uint64_t)(p.n_units - p.p_end + p.n_heavy) * kSlots;   // claim tickets (A-40)
    const uint64_t S = min(((uint64_t)(uint32_t)old + kSlots - 1) / kSlots * kSlots, n_slots);
    atomicExch((unsigned long long *)&st->sw, (S << 8) | win);
  }
  if (p.host_sel) *(volatile uint64_t *)p.host_sel = fin;   // activation-flag cache, no D2H copy
  if (p.tl) p.tl[1] = dysel_globaltimer();
  __threadfence();
  if (CDP && p.tail) {
    const uint32_t old = p.async ? atomicAdd(&st->ticket, 1u << 30) : 0u;   // stop eager claims
    const uint64_t u0 = (uint64_t)p.p_end + old;
    if (u0 < p.n_units) {
      st->tail_begin = u0;
      if constexpr (CDP) tail_launch(p.vids[win], A, y, u0, p.n_units, p.unit_variant, p.tl);
    }
  }
}

// Profiling copy of one variant (sequential profiling: one launch per variant).
template <int VID>
__global__ void __launch_bounds__(kUnitRows, kSliceMinBlocks[VID])
    spmv_prof_kernel(SpmvDev A, float *__restrict__ y, SpmvState *st, ProfParams p, uint32_t pv) {
  if constexpr (VID == DYSEL_SPMV_CSR_TMA) tma_stage_prologue();
  prof_unit<VID, false>(A, y, st, p, pv, blockIdx.x);
}

// All K profiling slices in ONE launch (no forked streams / joins): CTA b runs
// unit b / K of pool variant b mod K (interleaved start order).  The register
// cap is generous (128 registers): each variant's code is compiled as in its
// own kernel.  A 4-CTA/SM cap (64 registers, so profiling CTAs leave more
// room to the eager claim CTAs) measured no better on D4 (+5.0-5.4% vs
// +4.2% per step, same box).  The score is normalised by the plain kernel's
// occupancy, so the cap does not bias the selection.
#ifndef DYSEL_PROF_MINB
#define DYSEL_PROF_MINB 1
#endif
template <bool CDP>
__global__ void __launch_bounds__(kUnitRows, DYSEL_PROF_MINB)
    spmv_prof_all_kernel(SpmvDev A, float *__restrict__ y, SpmvState *st, ProfParams p) {
  tma_stage_prologue();
  // launched behind the init kernel with PDL: wait for its state reset (a
  // no-op when launched without the attribute)
  asm volatile("griddepcontrol.wait;" ::: "memory");
  // programmatic dependent launch: the claim kernels queued behind this one
  // may start as soon as every profiling CTA is resident
  if constexpr (!CDP) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const uint32_t pv = blockIdx.x % p.K, b = blockIdx.x / p.K;
  switch (p.vids[pv]) {
    case 0: prof_unit<0, CDP>(A, y, st, p, pv, b); break;
    case 1: prof_unit<1, CDP>(A, y, st, p, pv, b); break;
    case 2: prof_unit<2, CDP>(A, y, st, p, pv, b); break;
    case 3: prof_unit<3, CDP>(A, y, st, p, pv, b); break;
    case 4: prof_unit<4, CDP>(A, y, st, p, pv, b); break;
    default: prof_unit<5, CDP>(A, y, st, p, pv, b); break;
  }
}

// Remainder / eager claim kernels (default device path, readings A-27/A-28).
// The HOST launches, right behind the profiling kernel and chained by
// programmatic dependent launch, one persistent kernel per pool variant —
// default first — each the variant's own code at its own occupancy.  Work is
// claimed per WARP, one 32-row slot (unit u, slot w) per ticket, with no
// CTA-wide barrier: measured on D4, a CTA-per-unit persistent loop ran CSR-W
// 1.42 ms vs 0.94 ms for the plain grid (warps idled at the per-unit barrier
// behind the unit's longest row, while a plain grid's finished warps free
// their slots for new CTAs).
//   * Eager (ASYNC, the default's kernel): slot tickets from c1
//     until the selection is published.  Publishing sets c1's bit 32; the
//     claim count T_p at that instant, rounded up to a whole unit, is the
//     switch point S: slots [0, S) belong to the default (a unit is never
//     split between two variants — JDS slots of a unit permute its rows).
//   * Remainder: the selected variant's kernel claims slots S + c2.  Every
//     other kernel exits once it sees the selection (SYNC: everyone waits
//     for it, and S = 0).
// Every slot is computed exactly once.  No device-side launch: device-launched
// grids of the same kernels measured 7% slower on D4 (0.99 vs 0.93 ms), and
// the round-1 tail launch added ~17 us of launch latency after the selection.
// lane-0 poll of the published switch word (relaxed: only the word itself is consumed)
__device__ __forceinline__ uint64_t wait_published(const uint64_t *sw_p) {
  uint64_t sw = ld_relaxed_u64(sw_p);
  for (uint32_t ns = 32; sw == ~0ull; ns = ns < 1024 ? 2 * ns : ns) {
    __nanosleep(ns);
    sw = ld_relaxed_u64(sw_p);
  }
  return sw;
}

template <int VID>
__global__ void __launch_bounds__(kUnitRows, kClaimMinBlocks[VID])
    spmv_claim_kernel(SpmvDev A, float *__restrict__ y, SpmvState *st, ProfParams p, uint32_t pv) {
  if constexpr (VID == DYSEL_SPMV_CSR_TMA) tma_stage_prologue();
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const uint32_t FULL = 0xffffffffu;
  const int lane = threadIdx.x & 31;
  const uint32_t n_hs = p.n_heavy * kSlots;
  const uint32_t n_slots = (p.n_units - p.p_end) * kSlots + n_hs;   // tickets
  const uint32_t n_warps = gridDim.x * (kUnitRows / 32);
  const uint32_t gid = blockIdx.x * (kUnitRows / 32) + (threadIdx.x >> 5);
  // Claims.  A warp's first slot of a pure run or of the remainder is static
  // (slot base + warp id: no atomic), later ones come from one global counter
  // per phase, k slots per atomic: k = min(p.k_claim, remaining / (2 x warps))
  // >= 1 (p.k_claim ~ 1024 nnz of work per claim: the counter serialises
  // claims, ~1 per ns, which capped 1-nnz rows).  Claims are made on demand:
  // issuing the next claim before running the current slots (to hide its
  // latency) measured 7% slower on D4 (a warp stuck on a long slot holds its
  // prefetched one back), and 40% slower on CSR-S.
  auto batch = [&](uint32_t rest) -> uint32_t {
    const uint32_t k = rest / (2u * n_warps);
    return k < 1u ? 1u : (k > p.k_claim ? p.k_claim : k);
  };
  // phase 0: pure run; 1: eager (default, ASYNC) from c1; 2: after the selection
  int phase = p.pure ? 0 : ((pv == p.def && p.async) ? 1 : 2);
  uint32_t S = 0, eager = 0, done = 0;
  uint32_t t = 0, e = 0;               // current claim [t, e)
  bool dyn = false;                    // dynamic claims in this phase
  auto claim = [&](uint32_t k) -> uint64_t {   // lane 0 claims k slots of this phase's counter
    uint64_t raw = 0;
    if (lane == 0)
      raw = phase == 0 ? atomicAdd((unsigned long long *)&st->pure_ctr, (unsigned long long)k)
          : phase == 1 ? atomicAdd((unsigned long long *)&st->c1, (unsigned long long)k)
                       : (uint64_t)atomicAdd(&st->c2, k);
    return __shfl_sync(FULL, raw, 0);
  };
  int rem_vid = VID;   // variant of the remainder slots (the winner; solo: any pool variant)
  // a warp's first slot of a pure run / of the remainder is static: measured
  // on D3, claiming it instead cost 30-45% (ELL 15.9 vs 11.0 us)
  const bool stat = true;
  // entering the remainder: false if another variant won
  auto enter_remainder = [&]() -> bool {
    uint64_t sw = 0;
    if (lane == 0) sw = wait_published(&st->sw);
    sw = __shfl_sync(FULL, sw, 0);
    if ((sw & 0xff) != pv && !p.solo) return false;
    rem_vid = p.vids[sw & 0xff];
    phase = 2;
    S = min((uint32_t)(sw >> 8), n_slots);
    dyn = n_slots - S > n_warps;
    t = S + gid;
    e = t < n_slots ? t + 1 : t;
    if (!stat) { dyn = true; t = e = 0; }
    return true;
  };
  if (phase == 0) {
    dyn = n_slots > n_warps;
    t = gid;
    e = gid < n_slots ? gid + 1 : gid;
    if (!stat) { dyn = true; t = e = 0; }
  } else if (phase == 2) {
    if (!enter_remainder()) return;
  } else {
    dyn = true;
  }
  for (;;) {
    if (t >= e) {   // need a claim
      if (!dyn) break;
      const uint32_t k = batch(n_slots - min(e, n_slots));
      const uint64_t r = claim(k);
      if (phase == 0) {
        const uint64_t c = (stat ? n_warps : 0u) + r;
        if (c >= n_slots) {   // each warp ends on one failed claim; the last one resets the counters
          if (lane == 0 && atomicAdd(&st->pure_done, 1u) == n_warps - 1) {
            st->pure_ctr = 0;
            st->pure_done = 0;
          }
          break;
        }
        t = (uint32_t)c;
        e = min(t + k, n_slots);
      } else if (phase == 1) {
        t = (uint32_t)r;
        uint32_t lim = n_slots;
        if (r >> 32) {   // claimed after the selection was published: only below the switch point
          uint64_t sw = 0;
          if (lane == 0) sw = wait_published(&st->sw);
          lim = (uint32_t)(__shfl_sync(FULL, sw, 0) >> 8);
        }
        if (t >= lim) {   // eager range closed: hand over to the selection
          if (!enter_remainder()) break;
          continue;
        }
        e = min(t + k, lim);
        if (p.tl && lane == 0 && eager == 0)
          atomicMin((unsigned long long *)&p.tl[3], (unsigned long long)dysel_globaltimer());
        eager += e - t;
      } else {
        t = S + (stat ? n_warps : 0u) + (uint32_t)r;
        if (t >= n_slots) break;
        e = min(t + k, n_slots);
      }
    }
    if (phase == 2) {
      if (p.tl && lane == 0 && done == 0)
        atomicMin((unsigned long long *)&p.tl[5], (unsigned long long)dysel_globaltimer());
      done += e - t;
    }
    for (uint32_t q = t; q < e; ++q) {
      uint32_t u;
      if (q < n_hs) {   // heavy-first (A-40); a profiled heavy unit is done
        u = (uint32_t)__ldg(p.heavy + q / kSlots);
        if (u < p.p_end) continue;
      } else {
        u = p.p_end + (q - n_hs) / kSlots;
        if (n_hs && ((__ldg(p.heavy_bits + (u >> 5)) >> (u & 31)) & 1u)) continue;
      }
      if (phase != 2 || rem_vid == VID)
        run_slot<VID>(A, u, (int)(q % kSlots), y + (size_t)u * kUnitRows);
      else
        run_slot_dyn(rem_vid, A, u, (int)(q % kSlots), y + (size_t)u * kUnitRows);
      if (lane == 0 && p.unit_variant && q % kSlots == 0) p.unit_variant[u] = (uint8_t)(phase == 2 ? rem_vid : VID);
    }
    t = e;
  }
  if (p.tl && lane == 0) {
    if (eager) atomicMax((unsigned long long *)&p.tl[4], (unsigned long long)dysel_globaltimer());
    if (done) atomicMax((unsigned long long *)&p.tl[6], (unsigned long long)dysel_globaltimer());
  }
}

// debug: selection preset to pool index pv with no eager range (claim kernel alone)
// eager_all: the eager range stays open (c1 unpublished) and S = n_slots, so
// the default's eager phase runs the whole grid
// Switch kernel (reading A-42, the default SpMV device path): instead of one
// host-launched claim kernel per non-default variant -- K - 1 full grids that,
// when the default wins, only drain as exiting CTAs at the end of the step --
// one 32-thread CTA queued behind the default's claim kernel waits for the
// selection and, only if another variant won, launches that variant's claim
// kernel from the device (fire-and-forget: stream order is kept, the parent
// grid completes with its child).  The child enters the remainder at the
// published switch point S like a host-launched one.
__global__ void spmv_switch_kernel(SpmvDev A, float *__restrict__ y, SpmvState *st, ProfParams p) {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  if (threadIdx.x != 0) return;
  const uint64_t sw = wait_published(&st->sw);
  const uint32_t w = (uint32_t)(sw & 0xff);
  if (w == p.def || w >= p.K || p.p_end >= p.n_units) return;
  const unsigned g = (unsigned)min((uint64_t)p.occ[w] * p.n_sm, (uint64_t)(p.n_units - p.p_end));
  const cudaStream_t ff = cudaStreamFireAndForget;
  switch (p.vids[w]) {
    case 0: spmv_claim_kernel<0><<<g, kUnitRows, dyn_smem(0), ff>>>(A, y, st, p, w); break;
    case 1: spmv_claim_kernel<1><<<g, kUnitRows, dyn_smem(1), ff>>>(A, y, st, p, w); break;
    case 2: spmv_claim_kernel<2><<<g, kUnitRows, dyn_smem(2), ff>>>(A, y, st, p, w); break;
    case 3: spmv_claim_kernel<3><<<g, kUnitRows, dyn_smem(3), ff>>>(A, y, st, p, w); break;
    case 4: spmv_claim_kernel<4><<<g, kUnitRows, dyn_smem(4), ff>>>(A, y, st, p, w); break;
    default: spmv_claim_kernel<5><<<g, kUnitRows, dyn_smem(5), ff>>>(A, y, st, p, w); break;
  }
}

__global__ void spmv_state_preset_kernel(SpmvState *s, uint32_t pv, int eager_all, uint64_t n_slots) {
  s->sel = pv;
  s->c1 = eager_all ? 0ull : 1ull << 32;
  s->sw = ((eager_all ? n_slots : 0ull) << 8) | pv;
}

// Eager copy of the default variant (ASYNC): persistent CTAs claim remainder
// units by ticket until the selection grabs the rest.
template <int VID>
__global__ void __launch_bounds__(kUnitRows, kSliceMinBlocks[VID])
    spmv_eager_kernel(SpmvDev A, float *__restrict__ y, SpmvState *st, uint32_t p_end, uint32_t n_units, uint8_t *uv,
                      uint64_t *tl) {
  if constexpr (VID == DYSEL_SPMV_CSR_TMA) tma_stage_prologue();
  __shared__ uint32_t s_t;
  if (tl && threadIdx.x == 0) atomicMin((unsigned long long *)&tl[3], (unsigned long long)dysel_globaltimer());
  if (threadIdx.x == 0) s_t = atomicAdd(&st->ticket, 1u);
  __syncthreads();
  uint32_t t = s_t, mine = 0;
  while ((uint64_t)p_end + t < n_units) {
    const uint32_t u = p_end + t;
    uint32_t next = 0;
    if (threadIdx.x == 0) next = atomicAdd(&st->ticket, 1u);
    run_unit<VID>(A, u, y + (size_t)u * kUnitRows);
    if (threadIdx.x == 0 && uv) uv[u] = (uint8_t)VID;
    ++mine;
    __syncthreads();
    if (threadIdx.x == 0) s_t = next;
    __syncthreads();
    t = s_t;
  }
  if (threadIdx.x == 0 && mine) atomicAdd((unsigned long long *)&st->eager_units, (unsigned long long)mine);
  if (tl && threadIdx.x == 0) atomicMax((unsigned long long *)&tl[4], (unsigned long long)dysel_globaltimer());
}

// ----------------------------------------------------------------- host side
template <int VID>
static dysel_status spmv_variant_fn(const dysel_slice *s, void *const *args, void *stream, void *user) {
  dysel_spmv_plan *pl = (dysel_spmv_plan *)user;
  if (s->granule_count == 0) return DYSEL_OK;
  SpmvDev A = pl->dev;
  A.x = (const float *)args[1];
  if (s->timer)
    spmv_slice_timed_kernel<VID><<<(unsigned)s->granule_count, kUnitRows, dyn_smem(VID), (cudaStream_t)stream>>>(
        A, (float *)args[0], *s);
  else
    spmv_slice_kernel<VID><<<(unsigned)s->granule_count, kUnitRows, dyn_smem(VID), (cudaStream_t)stream>>>(A, (float *)args[0], *s,
                                                                                              nullptr, nullptr);
  return cudaGetLastError() == cudaSuccess ? DYSEL_OK : DYSEL_ERR_CUDA;
}

static dysel_variant_fn kVariantFns[DYSEL_SPMV_NVARIANTS] = {spmv_variant_fn<0>, spmv_variant_fn<1>, spmv_variant_fn<2>,
                                                             spmv_variant_fn<3>, spmv_variant_fn<4>,
                                                             spmv_variant_fn<5>};
static const char *kVariantNames[DYSEL_SPMV_NVARIANTS] = {"csr_scalar", "csr_vector", "ell", "jds", "csr_stream", "csr_tma"};

struct SpmvCtxState {
  SpmvState *d_state = nullptr;
  SpmvState *h_state = nullptr;   // pinned
  int occ_slice[DYSEL_SPMV_NVARIANTS] = {};
  int occ_eager[DYSEL_SPMV_NVARIANTS] = {};
  int occ_claim[DYSEL_SPMV_NVARIANTS] = {};
};

dysel_status spmv_ctx_init(dysel_ctx *ctx) {
  SpmvCtxState *s = new SpmvCtxState();
  ctx->d_spmv_state = s;
  if (cudaMalloc(&s->d_state, sizeof(SpmvState)) != cudaSuccess) return DYSEL_ERR_NOMEM;
  if (cudaMemset(s->d_state, 0, sizeof(SpmvState)) != cudaSuccess) return DYSEL_ERR_CUDA;
  if (cudaMallocHost(&s->h_state, sizeof(SpmvState)) != cudaSuccess) return DYSEL_ERR_NOMEM;
  const void *slice[DYSEL_SPMV_NVARIANTS] = {(const void *)spmv_slice_kernel<0>, (const void *)spmv_slice_kernel<1>,
                                            (const void *)spmv_slice_kernel<2>, (const void *)spmv_slice_kernel<3>,
                                            (const void *)spmv_slice_kernel<4>,
                                            (const void *)spmv_slice_kernel<5>};
  const void *claim[DYSEL_SPMV_NVARIANTS] = {(const void *)spmv_claim_kernel<0>, (const void *)spmv_claim_kernel<1>,
                                            (const void *)spmv_claim_kernel<2>, (const void *)spmv_claim_kernel<3>,
                                            (const void *)spmv_claim_kernel<4>,
                                            (const void *)spmv_claim_kernel<5>};
  const void *eager[DYSEL_SPMV_NVARIANTS] = {(const void *)spmv_eager_kernel<0>, (const void *)spmv_eager_kernel<1>,
                                            (const void *)spmv_eager_kernel<2>, (const void *)spmv_eager_kernel<3>,
                                            (const void *)spmv_eager_kernel<4>,
                                            (const void *)spmv_eager_kernel<5>};
  {   // CSR-T's staging buffers exceed the 48 KB default dynamic limit
    const int m = (int)dyn_smem(DYSEL_SPMV_CSR_TMA);
    const void *k5[] = {(const void *)spmv_slice_kernel<5>, (const void *)spmv_slice_timed_kernel<5>,
                        (const void *)spmv_claim_kernel<5>, (const void *)spmv_eager_kernel<5>,
                        (const void *)spmv_prof_kernel<5>, (const void *)spmv_prof_all_kernel<true>,
                        (const void *)spmv_prof_all_kernel<false>};
    for (const void *k : k5)
      if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, m) != cudaSuccess) return DYSEL_ERR_CUDA;
  }
  for (int v = 0; v < DYSEL_SPMV_NVARIANTS; ++v) {
    // largest L1 for host launches (tuning knob DYSEL_SPMV_CARVEOUT = percent)
    const char *cv = getenv("DYSEL_SPMV_CARVEOUT");
    int carve = cv ? atoi(cv) : (int)cudaSharedmemCarveoutMaxL1;
    // CSR-T holds its staging buffers in static shared memory: the smallest
    // carveout that keeps the claim kernel's compiled CTAs/SM resident
    if (v == DYSEL_SPMV_CSR_TMA && !cv)
      carve = std::min(100, (int)((kClaimMinBlocks[v] * (sizeof(TmaStageBufs) + 2048) * 100 + 232447) / 232448));
    cudaFuncSetAttribute(slice[v], cudaFuncAttributePreferredSharedMemoryCarveout, carve);
    cudaFuncSetAttribute(eager[v], cudaFuncAttributePreferredSharedMemoryCarveout, carve);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&s->occ_slice[v], slice[v], kUnitRows, dyn_smem(v));
    cudaFuncSetAttribute(claim[v], cudaFuncAttributePreferredSharedMemoryCarveout, carve);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&s->occ_claim[v], claim[v], kUnitRows, dyn_smem(v));
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&s->occ_eager[v], eager[v], kUnitRows, dyn_smem(v));
  }
  return cudaGetLastError() == cudaSuccess ? DYSEL_OK : DYSEL_ERR_CUDA;
}

void spmv_ctx_free(dysel_ctx *ctx) {
  SpmvCtxState *s = (SpmvCtxState *)ctx->d_spmv_state;
  if (!s) return;
  if (s->d_state) cudaFree(s->d_state);
  if (s->h_state) cudaFreeHost(s->h_state);
  delete s;
  ctx->d_spmv_state = nullptr;
}

dysel_status spmv_register_pool(dysel_ctx *ctx, dysel_spmv_plan *pl) {
  pl->sig = "dysel.spmv#" + std::to_string(++ctx->plan_serial);
  static const int sb[1] = {0};
  dysel_variant vv[DYSEL_SPMV_NVARIANTS];
  for (int i = 0; i < pl->K; ++i)
    vv[i] = dysel_variant{kVariantNames[pl->vids[i]], kVariantFns[pl->vids[i]], {1, 1, 1}, sb, 1,
                          pl->info.uniform ? 0u : (uint32_t)DYSEL_V_NONUNIFORM, pl};
  return dysel_register_variants(ctx, pl->sig.c_str(), vv, pl->K, pl->def);
}

static dysel_slice unit_slice(uint64_t u0, uint64_t count, uint64_t n_units, int vid) {
  dysel_slice s;
  memset(&s, 0, sizeof(s));
  s.granule_begin = u0;
  s.granule_count = count;
  s.granule_stride = 1;
  s.g[0] = s.g[1] = s.g[2] = 1;
  s.G[0] = (uint32_t)n_units;
  s.G[1] = s.G[2] = 1;
  s.U[0] = n_units;
  s.U[1] = s.U[2] = 1;
  s.role = DYSEL_ROLE_BATCH;
  s.variant = vid;
  return s;
}

template <int VID>
static dysel_status launch_claim(const SpmvDev &A, float *y, SpmvState *st, const ProfParams &p, uint32_t pv,
                                 unsigned grid, cudaStream_t s, bool pdl) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kUnitRows);
  cfg.dynamicSmemBytes = dyn_smem(VID);
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, spmv_claim_kernel<VID>, A, y, st, p, pv) == cudaSuccess ? DYSEL_OK : DYSEL_ERR_CUDA;
}
typedef dysel_status (*ClaimLauncher)(const SpmvDev &, float *, SpmvState *, const ProfParams &, uint32_t, unsigned,
                                      cudaStream_t, bool);
static const ClaimLauncher kClaim[DYSEL_SPMV_NVARIANTS] = {launch_claim<0>, launch_claim<1>, launch_claim<2>,
                                                           launch_claim<3>, launch_claim<4>, launch_claim<5>};

static void set_heavy(ProfParams &p, const dysel_spmv_plan *pl) {
  p.n_heavy = pl->n_heavy;
  p.heavy = pl->heavy;
  p.heavy_bits = pl->heavy_bits;
}

// Slots per claim: about kClaimNnz nonzeros of work (at least 1, at most a unit).
constexpr int64_t kClaimNnz = 1024;
static uint32_t claim_batch(const dysel_spmv_plan *pl) {
  const int64_t slots = (int64_t)pl->n_units * kSlots;
  const int64_t per_slot = slots ? std::max<int64_t>(1, pl->info.nnz / slots) : 1;
  return (uint32_t)std::min<int64_t>(kSlots, std::max<int64_t>(1, kClaimNnz / per_slot));
}

// Pure version of one variant over the whole grid: the variant's claim kernel
// with every slot its own (the same code and occupancy that runs the DySel
// remainder, so T* and the remainder are measured on the same kernel).
static dysel_status launch_variant_full(dysel_ctx *ctx, dysel_spmv_plan *pl, int vid, const float *x, float *y,
                                        cudaStream_t st) {
  if (pl->n_units == 0) return DYSEL_OK;
  SpmvCtxState *cs = (SpmvCtxState *)ctx->d_spmv_state;
  ProfParams p;
  memset(&p, 0, sizeof(p));
  p.K = (uint32_t)pl->K;
  p.n_units = pl->n_units;
  p.pure = 1;
  p.k_claim = claim_batch(pl);
  set_heavy(p, pl);
  const uint64_t grid = std::min<uint64_t>((uint64_t)std::max(1, cs->occ_claim[vid]) * ctx->n_sm, pl->n_units);
  SpmvDev A = pl->dev;
  A.x = x;
  DYSEL_TRY(kClaim[vid](A, y, cs->d_state, p, 0, (unsigned)grid, st, false));
  return check_launch(ctx, "spmv pure claim kernel");
}

template <int VID>
static void launch_prof(const SpmvDev &A, float *y, SpmvState *st, const ProfParams &p, uint32_t pv, cudaStream_t s) {
  spmv_prof_kernel<VID><<<p.c, kUnitRows, dyn_smem(VID), s>>>(A, y, st, p, pv);
}
typedef void (*ProfLauncher)(const SpmvDev &, float *, SpmvState *, const ProfParams &, uint32_t, cudaStream_t);
static const ProfLauncher kProf[DYSEL_SPMV_NVARIANTS] = {launch_prof<0>, launch_prof<1>, launch_prof<2>, launch_prof<3>,
                                                         launch_prof<4>, launch_prof<5>};

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

dysel_status dysel_spmv_variant(dysel_ctx *ctx, dysel_spmv_plan *pl, int variant_id, const float *d_x, float *d_y,
                                void *stream) {
  if (!ctx || !pl || (pl->dev.n_rows > 0 && (!d_y || (pl->dev.n_cols > 0 && !d_x))) ||
      spmv_pool_index(pl, variant_id) < 0) {
    set_error(ctx, "dysel_spmv_variant: invalid arguments / variant not in pool");
    return DYSEL_ERR_INVALID;
  }
  return launch_variant_full(ctx, pl, variant_id, d_x, d_y, (cudaStream_t)stream);
}

dysel_status dysel_debug_spmv_device_launch(dysel_ctx *ctx, dysel_spmv_plan *pl, int variant_id, const float *d_x,
                                            float *d_y, int how, void *stream, uint32_t *h_resident_max, int n_sm) {
  if (!ctx || !pl || spmv_pool_index(pl, variant_id) < 0 || how < 0 || how > 4 || n_sm > 1024)
    return DYSEL_ERR_INVALID;
  cudaStream_t st = (cudaStream_t)stream;
  SpmvDev A = pl->dev;
  A.x = d_x;
  uint64_t *tl = nullptr;
  if (h_resident_max) {
    void *g = nullptr;
    DYSEL_CUDA_TRY(ctx, cudaGetSymbolAddress(&g, g_resident));
    DYSEL_CUDA_TRY(ctx, cudaMemsetAsync(g, 0, sizeof(g_resident), st));
    tl = ((SpmvCtxState *)ctx->d_spmv_state)->d_state->tl;
  }
  if (how == 3 || how == 4) {   // the claim kernel alone, selection preset (4: all eager)
    SpmvCtxState *cs = (SpmvCtxState *)ctx->d_spmv_state;
    const int pv = spmv_pool_index(pl, variant_id);
    spmv_state_init_kernel<<<1, 32, 0, st>>>(cs->d_state, pl->K, pv);
    spmv_state_preset_kernel<<<1, 1, 0, st>>>(cs->d_state, (uint32_t)pv, how == 4, (uint64_t)pl->n_units * kSlots);
    ProfParams p;
    memset(&p, 0, sizeof(p));
    p.K = pl->K;
    p.n_units = pl->n_units;
    p.def = pv;
    p.async = how == 4;
    p.k_claim = claim_batch(pl);
    for (int i = 0; i < pl->K; ++i) p.vids[i] = pl->vids[i];
    const uint64_t g = std::min<uint64_t>((uint64_t)std::max(1, cs->occ_claim[variant_id]) * ctx->n_sm, pl->n_units);
    DYSEL_TRY(kClaim[variant_id](A, d_y, cs->d_state, p, pv, (unsigned)g, st, false));
    DYSEL_CUDA_TRY(ctx, cudaStreamSynchronize(st));
    return check_launch(ctx, "claim");
  }
  if (how == 0) {
    dysel_slice s = unit_slice(0, pl->n_units, pl->n_units, variant_id);
    switch (variant_id) {
      case 0: spmv_slice_kernel<0><<<(unsigned)pl->n_units, kUnitRows, dyn_smem(0), st>>>(A, d_y, s, nullptr, tl); break;
      case 1: spmv_slice_kernel<1><<<(unsigned)pl->n_units, kUnitRows, dyn_smem(1), st>>>(A, d_y, s, nullptr, tl); break;
      case 2: spmv_slice_kernel<2><<<(unsigned)pl->n_units, kUnitRows, dyn_smem(2), st>>>(A, d_y, s, nullptr, tl); break;
      case 3: spmv_slice_kernel<3><<<(unsigned)pl->n_units, kUnitRows, dyn_smem(3), st>>>(A, d_y, s, nullptr, tl); break;
      case 4: spmv_slice_kernel<4><<<(unsigned)pl->n_units, kUnitRows, dyn_smem(4), st>>>(A, d_y, s, nullptr, tl); break;
    default: spmv_slice_kernel<5><<<(unsigned)pl->n_units, kUnitRows, dyn_smem(5), st>>>(A, d_y, s, nullptr, tl); break;
    }
  } else {
    spmv_device_launch_kernel<<<1, 1, 0, st>>>(A, d_y, variant_id, pl->n_units, how, tl);
  }
  DYSEL_TRY(check_launch(ctx, "spmv_device_launch_kernel"));
  if (h_resident_max) {
    void *g = nullptr;
    DYSEL_CUDA_TRY(ctx, cudaGetSymbolAddress(&g, g_resident));
    DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(h_resident_max, (uint32_t *)g + 1024, n_sm * sizeof(uint32_t),
                                        cudaMemcpyDeviceToHost, st));
    DYSEL_CUDA_TRY(ctx, cudaStreamSynchronize(st));
  }
  return DYSEL_OK;
}

dysel_status dysel_spmv(dysel_ctx *ctx, dysel_spmv_plan *pl, const float *d_x, float *d_y, float f, uint32_t mode,
                        void *stream, dysel_report *rep) {
  const uint64_t t_host0 = now_ns();
  if (!ctx || !pl || pl->ctx != ctx || (pl->dev.n_rows > 0 && (!d_y || (pl->dev.n_cols > 0 && !d_x))) ||
      !(f >= 0.0f && f <= 1.0f)) {
    set_error(ctx, "dysel_spmv: invalid arguments");
    return DYSEL_ERR_INVALID;
  }
  cudaStream_t st = (cudaStream_t)stream;
  if (rep) {
    rep->n_slices = 0;
    rep->eager_units = rep->tail_units = 0;
    for (int i = 0; i < 8; ++i) rep->timeline_ns[i] = ~0ull;
    for (int v = 0; v < DYSEL_MAX_VARIANTS; ++v)
      rep->score[v] = rep->makespan_ns[v] = rep->units[v] = rep->cycles[v] = rep->busy_ns[v] = rep->aborted[v] = 0;
  }
  if (pl->dev.n_rows == 0) return DYSEL_OK;
  if (mode & DYSEL_HOST_ORCH) {   // paper-faithful: generic launcher with the plan's registered pool
    const uint64_t U[3] = {pl->n_units, 1, 1};
    void *args[2] = {d_y, (void *)d_x};
    const size_t sb[1] = {(size_t)pl->n_units * kUnitRows * sizeof(float)};
    dysel_status s = dysel_launch(ctx, pl->sig.c_str(), U, f, mode, args, 2, sb, stream, rep);
    if (rep && s == DYSEL_OK) {   // report arrays: pool index -> DYSEL_SPMV_* id
      uint64_t sc[DYSEL_MAX_VARIANTS] = {}, ms[DYSEL_MAX_VARIANTS] = {}, un[DYSEL_MAX_VARIANTS] = {},
               cy[DYSEL_MAX_VARIANTS] = {};
      for (int i = 0; i < pl->K; ++i) {
        sc[pl->vids[i]] = rep->score[i];
        ms[pl->vids[i]] = rep->makespan_ns[i];
        un[pl->vids[i]] = rep->units[i];
        cy[pl->vids[i]] = rep->cycles[i];
      }
      memcpy(rep->score, sc, sizeof(sc));
      memcpy(rep->makespan_ns, ms, sizeof(ms));
      memcpy(rep->units, un, sizeof(un));
      memcpy(rep->cycles, cy, sizeof(cy));
      if (rep->selected >= 0 && rep->selected < pl->K) rep->selected = pl->vids[rep->selected];
      for (int i = 0; i < rep->n_slices && i < rep->slices_cap && rep->slices; ++i)
        rep->slices[i].variant = pl->vids[rep->slices[i].variant];
      if (rep->unit_variant)
        for (uint64_t j = 0; j < rep->unit_variant_cap; ++j)
          rep->unit_variant[j] = rep->unit_variant[j] < pl->K ? (uint8_t)pl->vids[rep->unit_variant[j]] : 0xff;
    }
    return s;
  }
  // ---- device path: same planning rules as the generic launcher
  uint32_t wa[DYSEL_SPMV_NVARIANTS][3], vflags[DYSEL_SPMV_NVARIANTS];
  for (int i = 0; i < pl->K; ++i) {
    wa[i][0] = wa[i][1] = wa[i][2] = 1;
    vflags[i] = pl->info.uniform ? 0u : (uint32_t)DYSEL_V_NONUNIFORM;
  }
  const uint64_t U[3] = {pl->n_units, 1, 1};
  Plan P;
  DYSEL_TRY(make_plan(ctx, U, wa, pl->K, f, ctx->n_sm, pl->def, mode, vflags, &P));
  if (P.mode == DYSEL_SWAP) {
    set_error(ctx, "dysel_spmv: swap mode needs atomics variants (NEXT f-1)");
    return DYSEL_ERR_UNSUPPORTED;
  }
  const bool async = (mode & DYSEL_ASYNC) != 0;
  SpmvCtxState *cs = (SpmvCtxState *)ctx->d_spmv_state;
  {   // reading A-3b: a grid that fits in one wave of the default variant runs
      // entirely concurrently — there is no remainder for a selection to speed up
    const uint64_t wave = (uint64_t)std::max(1, cs->occ_slice[pl->vids[pl->def]]) * ctx->n_sm;
    if (P.active && !(mode & DYSEL_FORCE_PROFILE) && P.Gn <= wave) {
      P.active = false;
      P.c = 0;
    }
  }
  if (rep) {
    rep->mode_used = P.mode | (async ? DYSEL_ASYNC : 0);
    rep->profiled = P.active ? 1 : 0;
    rep->n_variants = pl->K;
    rep->c = P.c;
    rep->n_granules = P.Gn;
  }
  uint8_t *d_uv = nullptr;
  if (rep && rep->unit_variant) {
    DYSEL_TRY(scratch(ctx, ctx->unit_variant, P.Gn));
    d_uv = (uint8_t *)ctx->unit_variant.ptr;
  }
  if (!P.active) {   // activation flag off / small workload: plain full grid of cached or default
    resolve_pending(ctx, pl->sig.c_str());
    int pv = pl->def;
    auto it = ctx->sel_cache.find(pl->sig);
    if (it != ctx->sel_cache.end() && it->second < pl->K) pv = it->second;
    DYSEL_TRY(launch_variant_full(ctx, pl, pl->vids[pv], d_x, d_y, st));
    if (rep) {
      rep->selected = pl->vids[pv];
      if (rep->unit_variant)
        for (uint64_t j = 0; j < P.Gn && j < rep->unit_variant_cap; ++j) rep->unit_variant[j] = (uint8_t)pl->vids[pv];
      rep->host_ns = now_ns() - t_host0;
    }
    return DYSEL_OK;
  }
  ProfParams p;
  memset(&p, 0, sizeof(p));
  p.K = (uint32_t)pl->K;
  p.c = (uint32_t)P.c;
  p.n_units = pl->n_units;
  p.n_sm = (uint32_t)ctx->n_sm;
  p.hybrid = P.mode == DYSEL_HYBRID;
  p.p_end = p.hybrid ? p.c : p.K * p.c;
  p.async = async;
  p.contiguous = (mode & DYSEL_CONTIGUOUS) != 0;
  const bool sequential = (mode & DYSEL_SEQUENTIAL) != 0;
  p.score_mode = (mode & DYSEL_SCORE_CYCLES) ? 1u : ((mode & DYSEL_SCORE_MAKESPAN) || sequential ? 2u : 0u);
  if (sequential) p.async = 0;   // a variant profiled alone: no eager work beside it
  p.def = (uint32_t)pl->def;
  p.k_claim = claim_batch(pl);
  set_heavy(p, pl);
  const bool cdp = (mode & DYSEL_DEVICE_LAUNCH) != 0;   // round-1 scheme: eager + remainder launched on the device
  {   // reading A-38 (opt-in): one claim kernel (the default's) runs every
      // remainder slot, whichever variant wins — not with CSR-T in the pool
      // (its staging buffers live in its own kernel's shared memory)
    bool tma = false;
    for (int i = 0; i < pl->K; ++i) tma |= pl->vids[i] == DYSEL_SPMV_CSR_TMA;
    p.solo = (!tma && (mode & DYSEL_SOLO)) ? 1u : 0u;
  }
  p.tail = (cdp && !(mode & DYSEL_NO_TAIL)) ? 1u : 0u;
  p.abort = ((mode & DYSEL_NO_ABORT) || p.score_mode == 1) ? 0u : 1u;   // dominance needs busy or makespan
  for (int i = 0; i < pl->K; ++i) {
    p.vids[i] = pl->vids[i];
    // occupancy of the kernel that will run the remainder with this variant
    p.occ[i] = (uint32_t)std::max(1, cdp ? cs->occ_slice[pl->vids[i]] : cs->occ_claim[pl->vids[i]]);
  }
  if (p.hybrid) {
    DYSEL_TRY(scratch(ctx, ctx->sandbox[0], (size_t)pl->K * P.c * kUnitRows * sizeof(float)));
    p.sandbox = (float *)ctx->sandbox[0].ptr;
  }
  p.unit_variant = d_uv;
  if (rep) p.tl = cs->d_state->tl;
  SpmvDev A = pl->dev;
  A.x = d_x;
  SpmvState *dst = cs->d_state;
  if (cdp && p.async && p.p_end < p.n_units) {
    const int dv = pl->vids[pl->def];
    p.eager_grid =
        (uint32_t)std::min<uint64_t>((uint64_t)std::max(1, cs->occ_eager[dv]) * ctx->n_sm, p.n_units - p.p_end);
    ctx->launches++;   // device-side launch
  }
  const int pend = reserve_pending_sel(ctx, &p.host_sel);
  spmv_state_init_kernel<<<1, 32, 0, st>>>(dst, pl->K, pl->def);
  DYSEL_TRY(check_launch(ctx, "spmv_state_init_kernel"));
  if (sequential) {   // one launch per variant, back to back on the stream, default first
    for (int k = 0; k < pl->K; ++k) {
      const int i = k == 0 ? pl->def : (k <= pl->def ? k - 1 : k);
      kProf[pl->vids[i]](A, d_y, dst, p, (uint32_t)i, st);
      DYSEL_TRY(check_launch(ctx, "spmv_prof_kernel"));
    }
  } else {   // all K profiling slices in one launch on the stream
    if (cdp) {
      spmv_prof_all_kernel<true><<<p.K * p.c, kUnitRows, pool_dyn_smem(p), st>>>(A, d_y, dst, p);
    } else {   // PDL behind the init kernel: launch latency overlaps the reset
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(p.K * p.c);
      cfg.blockDim = dim3(kUnitRows);
      cfg.dynamicSmemBytes = pool_dyn_smem(p);
      cfg.stream = st;
      cudaLaunchAttribute attr[1];
      attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
      attr[0].val.programmaticStreamSerializationAllowed = 1;
      cfg.attrs = attr;
#ifndef DYSEL_EXP_NO_PDL_INIT
#define DYSEL_EXP_NO_PDL_INIT 0   // experiment knob (scripts/build_exp.py): plain stream order
#endif
      cfg.numAttrs = DYSEL_EXP_NO_PDL_INIT ? 0 : 1;
      DYSEL_CUDA_TRY(ctx, cudaLaunchKernelEx(&cfg, spmv_prof_all_kernel<false>, A, d_y, dst, p));
    }
    DYSEL_TRY(check_launch(ctx, "spmv_prof_all_kernel"));
  }
  if (!cdp && p.p_end < p.n_units) {
    // host-launched claim kernels, default first; programmatic dependent
    // launch lets them start while profiling runs (not after NO_TAIL or a
    // sequential profile: then they follow in stream order)
    const bool pdl = !(mode & DYSEL_NO_TAIL) && !sequential;
    // reading A-42: the default's claim kernel + the switch kernel, unless
    // DYSEL_ALL_CLAIMS (every variant's claim kernel from the host)
    const bool sw_k = pdl && !p.solo && !(mode & DYSEL_ALL_CLAIMS) && pl->K > 1;
    for (int k = 0; k < (p.solo || sw_k ? 1 : pl->K); ++k) {
      const uint32_t i = (uint32_t)(k == 0 ? pl->def : (k <= pl->def ? k - 1 : k));
      const int v = pl->vids[i];
      const uint64_t g = std::min<uint64_t>((uint64_t)std::max(1, cs->occ_claim[v]) * ctx->n_sm,
                                            p.n_units - p.p_end);
      DYSEL_TRY(kClaim[v](A, d_y, dst, p, i, (unsigned)g, st, pdl));
      DYSEL_TRY(check_launch(ctx, "spmv_claim_kernel"));
    }
    if (sw_k) {
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(1);
      cfg.blockDim = dim3(32);
      cfg.stream = st;
      cudaLaunchAttribute attr[1];
      attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
      attr[0].val.programmaticStreamSerializationAllowed = 1;
      cfg.attrs = attr;
      cfg.numAttrs = 1;
      DYSEL_CUDA_TRY(ctx, cudaLaunchKernelEx(&cfg, spmv_switch_kernel, A, d_y, dst, p));
      DYSEL_TRY(check_launch(ctx, "spmv_switch_kernel"));
    }
  } else if (cdp && !p.tail && !p.async && p.p_end < p.n_units) {   // CDP scheme, NO_TAIL: winner via claim kernels
    for (int i = 0; i < pl->K; ++i) {
      const int v = pl->vids[i];
      const uint64_t g = std::min<uint64_t>((uint64_t)std::max(1, cs->occ_claim[v]) * ctx->n_sm,
                                            p.n_units - p.p_end);
      DYSEL_TRY(kClaim[v](A, d_y, dst, p, (uint32_t)i, (unsigned)g, st, false));
      DYSEL_TRY(check_launch(ctx, "spmv_claim_kernel"));
    }
  }
  DYSEL_TRY(commit_pending_sel(ctx, pend, pl->sig, st));
  if (rep) {
    SpmvState *h = cs->h_state;
    DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(h, dst, sizeof(SpmvState), cudaMemcpyDeviceToHost, st));
    if (d_uv && rep->unit_variant)
      DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(rep->unit_variant, d_uv, std::min<uint64_t>(P.Gn, rep->unit_variant_cap),
                                          cudaMemcpyDeviceToHost, st));
    DYSEL_CUDA_TRY(ctx, cudaStreamSynchronize(st));
    const int sel_pool = (int)(h->sel & 0xff);
    rep->selected = sel_pool < pl->K ? pl->vids[sel_pool] : -1;
    rep->eager_units = h->eager_units;
    const bool claimed = !cdp || !p.tail;   // remainder run by the claim kernels
    if (claimed) rep->eager_units = h->sw != ~0ull ? (h->sw >> 8) / kSlots : 0;
    rep->tail_units = !claimed ? (h->tail_begin != ~0ull ? pl->n_units - h->tail_begin : 0)
                          : (p.n_units - p.p_end - std::min<uint64_t>(rep->eager_units, p.n_units - p.p_end));
    const uint64_t cap = (1ull << 56) - 1;
    for (int v = 0; v < pl->K; ++v) {
      const int id = pl->vids[v];
      const dysel_timer_slot &t = h->slot[v];
      rep->busy_ns[id] = h->busy[v];
      rep->aborted[id] = h->aborted[v];
      rep->makespan_ns[id] = t.t_end_max > t.t_start_min ? t.t_end_max - t.t_start_min : 0;
      rep->units[id] = t.units;
      rep->cycles[id] = t.cycles;
      rep->score[id] = h->dominated[v] ? cap
                       : p.score_mode == 1 ? (t.units ? t.cycles / t.units : cap)
                       : p.score_mode == 2 ? rep->makespan_ns[id]
                                           : std::max<uint64_t>(h->busy[v] * p.n_units /
                                                                    ((uint64_t)p.c * p.occ[v] * p.n_sm),
                                                                h->max_busy[v]);
    }
    if (sel_pool < pl->K) ctx->sel_cache[pl->sig] = sel_pool;
    for (int i = 0; i < 7; ++i)
      rep->timeline_ns[i] = (h->tl[i] == ~0ull || h->tl[i] == 0 || h->tl[0] == ~0ull) ? ~0ull : h->tl[i] - h->tl[0];
    rep->timeline_ns[7] = h->tl[7];
    rep->host_ns = now_ns() - t_host0;
  }
  return DYSEL_OK;
}

}  // extern "C"
