// DySel SpMV dispatch: the B200 device protocol.
//
// One dysel_spmv call, no host round trip (the paper's GPU host polling is
// slower than micro-profiling):
//   1. init kernel: reset the ctx's device state (tickets, timer slots, scores).
//   2. ONE profiling kernel (PDL behind the init): CTA b runs profiled unit
//      b / K of pool variant b mod K — fully mode: a disjoint unit per
//      variant (A-24), hybrid: the same units for every variant, the default
//      writing y and the others a sandbox (A-4).  Every unit is timed (Fig. 7b,
//      B200 form); the last CTA of a variant scores it (packed atomicMin,
//      A-7/A-8); a variant that provably cannot win is decided at once
//      (dominance, A-26); the last variant decided publishes the selection and
//      the switch point.
//   3. The default ("initial") variant's claim kernel (PDL behind the
//      profiling kernel): ASYNC, its warps claim light remainder slots eagerly
//      until the selection is published; then the winner's warps
//      take the rest, heavy units first (A-40, A-45).
//   4. A one-warp switch kernel (PDL) that device-launches the winner's claim
//      kernel only when the default lost (A-42).
// The unit order (seq) and the light / heavy split come from the plan
// (spmv_prep.cu, reading A-45).
#include <algorithm>
#include <cstdlib>
#include <cstring>

#include "dysel_device.cuh"
#include "spmv_plan.h"

namespace dysel {

// Scores (reading A-6): default = predicted full-grid
// time max(busy_sum x G_n / (c x occupancy x #SM), longest unit), i.e. the
// mean per-unit busy time per execution slot of the plain kernel that will run
// the remainder.  DYSEL_SCORE_CYCLES: sum clock64 / units.
// DYSEL_SCORE_MAKESPAN: the paper's earliest start .. latest end (Fig. 7b).
struct SpmvState {
  // Hot words, each on its own 128-byte line: thousands of waiting warps poll
  // `sw` and the eager claims hammer `c1`; sharing a line (an L2 slice) with
  // the profiling completion chain's atomics queued those atomics behind the
  // traffic and delayed the publish by several us.
  alignas(128) uint64_t c1; // eager slot tickets (low 32 bits) | published (bit 32)
  alignas(128) uint64_t sw; // (S << 8) | selected pool index, ~0 until published
  alignas(128) uint32_t c2; // winner's remainder slot tickets (relative, after its static first slots)
  alignas(128) uint64_t pure_ctr;   // pure full-grid runs: slot tickets; the last warp of a run resets both
  uint32_t pure_done;       // pure full-grid runs: warps finished
  alignas(128) uint32_t variants_done;
  uint32_t pad;
  uint64_t best;            // (score << 8) | pool variant
  uint64_t sel;             // final packed selection, ~0 until published
  uint64_t best_total;      // min over completed variants of the predicted time (busy score) or makespan (ns)
  uint32_t ctas_done[DYSEL_MAX_VARIANTS];
  uint32_t decided[DYSEL_MAX_VARIANTS];   // 0 running, 1 completed, 2 dominated (set once, by CAS)
  uint64_t vscore[DYSEL_MAX_VARIANTS];    // packed final score of each completed variant (~0: dominated / none)
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
  uint32_t K, c, n_units, p_end;   // p_end: profiled prefix of the unit order (hybrid c, fully K c)
  uint32_t n_sm;
  uint32_t hybrid, async, contiguous, score_mode, def, abort;
  uint64_t *host_sel;    // mapped pinned word: the publishing CTA writes the selection here (cache)
  int32_t vids[DYSEL_SPMV_NVARIANTS];
  uint32_t occ[DYSEL_SPMV_NVARIANTS];     // claim-kernel occupancy (remainder grids)
  uint32_t occ_t[DYSEL_SPMV_NVARIANTS];   // score normalisation: the co-residency the units were timed at
                                          // (grouped profiling: min(occ, units per CTA), A-49), else occ
  float *sandbox;        // (K - 1) * c * 256 floats (hybrid: every variant but the default, A-4)
  uint64_t *tl;          // SpmvState::tl when a report is requested, else nullptr (no timeline atomics)
  uint8_t *unit_variant; // optional debug map (variant id per unit)
  uint32_t pure;         // pure full-grid run of one variant (self-resetting counters, no init kernel)
  uint32_t k_claim;      // claim kernels: max slots per claim (~kClaimNnz nonzeros of work)
  uint32_t k_min;        // ... min slots per claim (~kClaimMinNnz of work: short-row matrices)
  // unit order (reading A-45): seq[0, n_light) = light units in index order,
  // seq[n_light, n_units) = the rest, nonzeros descending (A-40); nullptr =
  // identity (every unit light).  Profiling takes seq[0, p_end); the eager
  // default only light units seq[p_end, n_light); the winner the rest first.
  const int32_t *seq;
  uint32_t n_light;
  // reading A-45: no eager execution (ASYNC behaves as SYNC) when the
  // initial version is a thread-per-row variant and the matrix has long-row
  // units -- an unproven thread-per-row default is slow on exactly the rows
  // that dominate such a matrix, and its eager work only delays the selection
  uint32_t no_eager;
  // overlapped allgather (comm.cu): count each finished 32-row slot in
  // chunk_done[unit >> chunk_shift] (nullptr = off)
  uint32_t *chunk_done;
  uint32_t chunk_shift;
  uint32_t part_first;   // grouped profiling (A-49): pool index of the first launch (it waits for the init kernel)
  uint32_t n_grp;        // ... pool indices profiled by the combined grouped kernel
  uint32_t grp_pv[DYSEL_SPMV_NVARIANTS];
};

// eager slots of the default (published switch point S is clipped to it)
__host__ __device__ __forceinline__ uint32_t eager_slots(const ProfParams &p) {
  if (p.no_eager || p.p_end >= p.n_light) return 0u;
  return (p.n_light - p.p_end) * (uint32_t)(kUnitRows / 32);
}

__global__ void spmv_state_init_kernel(SpmvState *s, int def) {
  // the profiling kernel behind it (PDL) may launch now; it waits for this
  // grid's completion (griddepcontrol.wait) before touching the state
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const int v = threadIdx.x;
  if (v < DYSEL_MAX_VARIANTS) {
    s->ctas_done[v] = 0;
    s->decided[v] = 0;
    s->vscore[v] = ~0ull;
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
    s->c2 = 0;
    s->c1 = 0;
    s->sw = ~0ull;
    s->variants_done = 0;
    s->best = (((1ull << 56) - 1) << 8) | (uint64_t)def;
    s->sel = ~0ull;
    s->best_total = ~0ull;
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

// Publishing (the last variant to be decided, by completion or dominance):
// the packed selection, the switch point S of the claim kernels (the eager
// claim count at this instant rounded up to a whole unit, clipped to the
// light range E), the activation-flag cache word.  One thread.
struct PubArgs {
  SpmvState *st;
  uint64_t *host_sel;   // mapped pinned word (selection cache), nullable
  uint64_t *tl;         // report timeline, nullable
  uint32_t K;
  uint32_t E;           // eager (light) slots
  uint32_t def;         // pool index of the initial version (switch margin, A-50)
};
constexpr uint32_t kSlots = kUnitRows / 32;   // 32-row warp slots per unit

// acq_rel counter increment: releases this thread's earlier writes / reds
// (stats, scores) and, for the thread that sees the final count, acquires
// everyone else's -- one round trip where fence + atomic + fence took three
__device__ __forceinline__ uint32_t atom_add_acq_rel(uint32_t *q, uint32_t v) {
  uint32_t old;
  asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(q), "r"(v) : "memory");
  return old;
}

__device__ __forceinline__ void decided_publish(const PubArgs a) {
  const uint32_t vd = atom_add_acq_rel(&a.st->variants_done, 1u) + 1u;
  if (vd != a.K) return;
  unsigned long long fin = atomicAdd((unsigned long long *)&a.st->best, 0ull);
  // reading A-50 (switch margin): a challenger within 1/8 of the initial
  // version's own completed score does not replace it — switching costs the
  // winner's launch and the default's drain, and closer scores are within
  // the profile's noise
  if ((uint32_t)(fin & 0xffu) != a.def) {
    const unsigned long long ds = ld_relaxed_u64(&a.st->vscore[a.def]);
    if (ds != ~0ull && (fin >> 8) * 9ull > (ds >> 8) * 8ull) fin = ds;
  }
  atomicExch((unsigned long long *)&a.st->sel, fin);
  const uint64_t old = atomicOr((unsigned long long *)&a.st->c1, 1ull << 32);   // close the eager range
  const uint64_t S = min(((uint64_t)(uint32_t)old + kSlots - 1) / kSlots * kSlots, (uint64_t)a.E);
  atomicExch((unsigned long long *)&a.st->sw, (S << 8) | (fin & 0xffull));
  if (a.host_sel) *(volatile uint64_t *)a.host_sel = fin;
  if (a.tl) a.tl[1] = dysel_globaltimer();
  __threadfence();
}

// Dominance (A-26): every ~kPollNs one thread of a profiling CTA
// adds the time elapsed since its last report to lb[v].  lb[v] only sums time
// variant v's units really spent, so it is a lower bound of v's final busy
// sum; once the prediction it implies exceeds the predicted time of a
// COMPLETED variant (best_total), v cannot be selected any more: v is DECIDED
// at once (maximal score, one CAS on decided[v]) so the selection never waits
// for its CTAs.  Its sandbox units (hybrid, non-default) stop and the rest
// are skipped; productive units (fully mode, the hybrid default) run on —
// their output is part of y (north_star: profiling slices are never
// recomputed) — and only stop polling.  The selection is the one running
// every slice to completion would give.
// The comparison is made in the units of the active score: busy score ->
// max(lb x G_n / (c x occ x #SM), this unit's elapsed time) vs the best
// completed prediction; makespan score (sequential profiling: the variant
// runs alone) -> time since the variant's first CTA started vs the best
// completed makespan.
constexpr uint64_t kPollNs = 2000;
constexpr long long kPollCycles = 2048;   // ~1 us at 1.9 GHz
constexpr uint32_t kWarpPollEvery = 4;
template <bool PRODUCTIVE>
struct ProfPoll {
  static constexpr bool active = true;
  unsigned long long *s_last;   // smem: last report time
  const unsigned long long *s_start;   // smem: this unit's start time
  volatile int *s_abort;        // smem: the variant is dominated (sandbox: stop; productive: stop polling)
  unsigned long long *lb;
  const uint64_t *best_total;
  uint32_t *decided;
  const uint64_t *t_start;      // makespan mode: the variant's earliest CTA start
  uint64_t scale_num;           // busy mode: lower bound of the predicted time = lb * num / den
  uint64_t scale_den;
  uint32_t makespan;
  PubArgs pub;
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
  // true = stop this unit (sandbox of a dominated variant)
  __device__ __forceinline__ bool operator()() const {
    if (*s_abort) return !PRODUCTIVE;
    return due() && report(true) && !PRODUCTIVE;
  }
  // warp-cooperative loops: only lane 0 reads the timer (the caller combines
  // with __any_sync); checked every kWarpPollEvery-th step only
  mutable uint32_t tick = 0;
  __device__ __forceinline__ bool warp() const {
    if ((++tick & (kWarpPollEvery - 1)) != 0) return false;   // warp-uniform
    if (*s_abort) return !PRODUCTIVE;
    if ((threadIdx.x & 31) != 0) return false;
    return due() && report(false) && !PRODUCTIVE;
  }
  // Global values read by this thread's previous report, issued without
  // waiting (a blocking global atomic / load per report stalled the polling
  // warp for ~3 L2 round trips and doubled sandbox unit times).  Stale values
  // stay safe: lb only grows (a stale lb is still a lower bound) and
  // best_total only shrinks (a stale best decides later, never wrongly).
  mutable unsigned long long lb_seen = 0, best_seen = ~0ull, t0_seen = ~0ull;
  mutable uint32_t dec_seen = 0;
  // fresh: take lb from the atomic's return (thread-per-row variants: many
  // threads of a unit poll, each rarely wins the report, so a per-thread
  // stale lb_seen lagged the variant's bound by most of its reports — D4's
  // JDS sandboxes were decided ~25 us late, delaying the selection)
  __device__ __forceinline__ bool report(bool fresh) const {
    const unsigned long long now = dysel_globaltimer();
    const unsigned long long last = *(volatile unsigned long long *)s_last;
    if (now - last < kPollNs) return false;
    if (atomicCAS(s_last, last, now) != last) return *s_abort != 0;   // another thread reports
    unsigned long long l;
    if (fresh) {
      l = atomicAdd(lb, now - last) + (now - last);
      best_seen = ld_relaxed_u64(best_total);
      dec_seen = ld_relaxed_u32(decided);
    } else {
      atomicAdd(lb, now - last);   // no return value: a fire-and-forget RED
      l = lb_seen + (now - last);
    }
    unsigned long long cost;
    if (makespan) {
      cost = t0_seen == ~0ull ? 0ull : now - t0_seen;
    } else {   // predicted full-grid time >= max(throughput bound, this unit's elapsed time)
      const unsigned long long thr = l * scale_num / scale_den;
      const unsigned long long el = now - *(volatile const unsigned long long *)s_start;
      cost = thr > el ? thr : el;
    }
    if (dec_seen == 1u) return false;   // completed (this unit's report raced its last CTA): never dominated
    if (cost > best_seen || dec_seen == 2u) {
      *s_abort = 1;
      if (dec_seen != 2u && atomicCAS(decided, 0u, 2u) == 0u) decided_publish(pub);
      return true;
    }
    lb_seen = ld_relaxed_u64((const uint64_t *)lb);
    best_seen = ld_relaxed_u64(best_total);
    dec_seen = ld_relaxed_u32(decided);
    if (makespan) t0_seen = ld_relaxed_u64(t_start);
    return false;
  }
};

// resident CTAs per SM each plain variant kernel is compiled for (register
// cap).  CSR-V at 6/SM spills and measured slower on D4 (1.44 vs 1.35 ms).
constexpr int kSliceMinBlocks[DYSEL_SPMV_NVARIANTS] = {8, 4, 4, 6, 5, 3};
// dynamic shared memory of each variant's kernels (CSR-T's staging buffers)
__host__ __device__ constexpr size_t dyn_smem(int vid) { return vid == DYSEL_SPMV_CSR_TMA ? sizeof(TmaStageBufs) : 0; }
inline size_t pool_dyn_smem(const ProfParams &p) {
  size_t b = 0;
  for (uint32_t i = 0; i < p.K; ++i) b = std::max(b, dyn_smem(p.vids[i]));
  return b;
}
// claim kernels: CTAs per SM (CSR-S / ELL at 8 spilled ~200 B in the claim loop)
constexpr int kClaimMinBlocks[DYSEL_SPMV_NVARIANTS] = {6, 4, 4, 6, 5, 3};

// Plain kernel of one variant over a slice (the paper-faithful host path's
// copies: dysel_launch with the plan's registered pool).  No static shared
// memory: the kernel's occupancy must not depend on the L1 / shared-memory
// carveout (measured on D4: 1 KB of static timing buffer with a small
// carveout cut CSR-W's resident CTAs, 1.52 vs 0.93 ms).  Timed copies use
// spmv_slice_timed_kernel.
template <int VID>
__global__ void __launch_bounds__(kUnitRows, kSliceMinBlocks[VID])
    spmv_slice_kernel(SpmvDev A, float *__restrict__ y, dysel_slice s) {
  if constexpr (VID == DYSEL_SPMV_CSR_TMA) tma_stage_prologue();
  if (!dysel_gate_open(s)) return;
  const uint32_t j = (uint32_t)(s.granule_begin + (uint64_t)blockIdx.x * s.granule_stride);
  run_unit<VID>(A, j, y + (size_t)j * kUnitRows);
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

__device__ __forceinline__ uint32_t unit_at(const ProfParams &p, uint32_t i) {
  return p.seq ? (uint32_t)__ldg(p.seq + i) : i;
}

// Shared state of one profiled unit (one per 256-thread unit group).
struct ProfUnitSmem {
  unsigned long long s_last, s_start;
  int s_abort, s_skip;
  dysel_prof_smem psm;
};
// barrier of a unit group: the whole CTA (grp 0) or named barrier grp (256 threads)
__device__ __forceinline__ void unit_sync(int grp) {
  if (grp == 0)
    __syncthreads();
  else
    asm volatile("bar.sync %0, 256;" ::"r"(grp) : "memory");
}

// One profiling unit of variant VID (pool index pv): the b-th unit of its
// slice, run by the 256 threads of unit group grp (threadIdx.x / 256).
template <int VID>
__device__ __forceinline__ void prof_unit(const SpmvDev &A, float *__restrict__ y, SpmvState *st,
                                          const ProfParams &p, uint32_t pv, uint32_t b, ProfUnitSmem &sm,
                                          int grp) {
  unsigned long long &s_last = sm.s_last, &s_start = sm.s_start;
  int &s_abort = sm.s_abort, &s_skip = sm.s_skip;
  dysel_prof_smem &psm = sm.psm;
  const uint32_t tid = threadIdx.x & (kUnitRows - 1);
  // predicted full-grid time of a variant (A-6): max(throughput bound, longest
  // unit); throughput bound = busy_sum * G_n / (c * occupancy * #SM)
  const uint64_t thr_den = (uint64_t)p.c * max(1u, p.occ_t[pv]) * max(1u, p.n_sm);
  const uint32_t jj = p.hybrid ? b : (p.contiguous ? pv * p.c + b : pv + p.K * b);   // position in seq
  const uint32_t j = unit_at(p, jj);
  // hybrid (reading A-4): every variant runs the same units; the
  // default ("first") variant writes y, the others their own sandbox
  const bool productive = !p.hybrid || pv == p.def;
  const bool sandbox = !productive;
  const PubArgs pub{st, p.host_sel, p.tl, p.K, eager_slots(p), p.def};
  if (tid == 0) {
    s_abort = 0;
    s_last = dysel_globaltimer();
    s_start = s_last;
    s_skip = (sandbox && p.abort && ld_relaxed_u32(&st->decided[pv]) == 2u) ? 1 : 0;
    if (!s_skip) atomicMin((unsigned long long *)&st->slot[pv].t_start_min, s_last);   // variant start (makespan)
    if (p.tl) atomicMin((unsigned long long *)&p.tl[0], s_last);
  }
  unit_sync(grp);
  const bool skipped = s_skip != 0;
  const uint32_t sb = pv < p.def ? pv : pv - 1;   // sandbox slot of a non-default variant (K - 1 of them)
  float *out = productive ? y + (size_t)j * kUnitRows : p.sandbox + ((size_t)sb * p.c + b) * kUnitRows;
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
    if (kPolled && p.abort && sandbox)
      run_slot<VID>(A, j, (int)(tid >> 5), out,
                    ProfPoll<false>{&s_last, &s_start, &s_abort, (unsigned long long *)&st->lb[pv], &st->best_total,
                                    &st->decided[pv], &st->slot[pv].t_start_min, (uint64_t)p.n_units, thr_den,
                                    p.score_mode == 2 ? 1u : 0u, pub});
    else if (kPolled && p.abort)
      run_slot<VID>(A, j, (int)(tid >> 5), out,
                    ProfPoll<true>{&s_last, &s_start, &s_abort, (unsigned long long *)&st->lb[pv], &st->best_total,
                                   &st->decided[pv], &st->slot[pv].t_start_min, (uint64_t)p.n_units, thr_den,
                                   p.score_mode == 2 ? 1u : 0u, pub});
    else
      run_slot<VID>(A, j, (int)(tid >> 5), out, NoPoll());
    if ((tid & 31) == 0) {
      psm.t1[tid >> 5] = dysel_globaltimer();
      psm.c1[tid >> 5] = dysel_clock64();
    }
  }
  unit_sync(grp);
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
    if (skipped || (s_abort && sandbox)) atomicAdd((unsigned long long *)&st->aborted[pv], 1ull);
    atomicAdd((unsigned long long *)&slot->units, 1ull);
    if (productive && p.unit_variant) p.unit_variant[j] = (uint8_t)VID;
    if (productive && p.chunk_done) {   // the unit's 8 slots are final (the group barrier above)
      __threadfence();
      atomicAdd(&p.chunk_done[j >> p.chunk_shift], (uint32_t)kSlots);
    }
    const uint32_t done = atom_add_acq_rel(&st->ctas_done[pv], 1u) + 1u;
    // ---- variant complete (and not already decided by dominance): score,
    // packed atomicMin (A-7, A-8); the last variant decided publishes
    if (done == p.c && atomicCAS(&st->decided[pv], 0u, 1u) == 0u) {   // (acquired by the add above)
      const unsigned long long a = atomicAdd((unsigned long long *)&slot->t_start_min, 0ull);
      const unsigned long long e = atomicAdd((unsigned long long *)&slot->t_end_max, 0ull);
      const unsigned long long cy = atomicAdd((unsigned long long *)&slot->cycles, 0ull);
      const unsigned long long bz = atomicAdd((unsigned long long *)&st->busy[pv], 0ull);
      const unsigned long long mb = atomicAdd((unsigned long long *)&st->max_busy[pv], 0ull);
      const unsigned long long cap = (1ull << 56) - 1;
      const unsigned long long thr = bz * (unsigned long long)p.n_units / thr_den;
      const unsigned long long pred = thr > mb ? thr : mb;   // predicted full-grid time (ns)
      unsigned long long score = p.score_mode == 1 ? cy / p.c : p.score_mode == 2 ? e - a : pred;
      if (score > cap) score = cap;
      atomicMin((unsigned long long *)&st->best_total, p.score_mode == 2 ? e - a : pred);   // dominance units
      st->vscore[pv] = (score << 8) | pv;   // released by decided_publish's acq_rel add
      atomicMin((unsigned long long *)&st->best, (score << 8) | pv);
      decided_publish(pub);
    }
  }
}

// Profiling copy of one variant (sequential profiling: one launch per variant).
template <int VID>
__global__ void __launch_bounds__(kUnitRows, kSliceMinBlocks[VID])
    spmv_prof_kernel(SpmvDev A, float *__restrict__ y, SpmvState *st, ProfParams p, uint32_t pv) {
  if constexpr (VID == DYSEL_SPMV_CSR_TMA) tma_stage_prologue();
  __shared__ ProfUnitSmem sm;
  prof_unit<VID>(A, y, st, p, pv, blockIdx.x, sm, 0);
}

// Grouped profiling copy of one variant (reading A-49): each CTA runs
// kProfGroups(VID) profiled units at once, one per 256-thread group (named
// barriers), so a unit is timed beside as many units of its own variant as
// the claim kernel keeps resident per SM (up to 4; CSR-T's staging buffers
// allow one) — the per-SM load of the full run (L1 / LSU / gather rate)
// instead of one unit alone on an SM, which hid CSR-S's LSU saturation on
// regular matrices.  The K launches are chained by PDL and run concurrently;
// only the first waits for the init kernel (the others start after all of
// its CTAs passed that wait).
__host__ __device__ constexpr int kProfGroups(int vid) { return vid == DYSEL_SPMV_CSR_TMA ? 3 : 4; }
// The K_g variants without staging buffers in ONE grouped launch (CTA b:
// variant grp_pv[b % K_g], its units 4 (b / K_g) .. + 3), so the PDL chain in
// front of the eager claim kernel is one or two launches, not K.
__global__ void __launch_bounds__(kUnitRows * 4, 1)
    spmv_prof_grp_all_kernel(SpmvDev A, float *__restrict__ y, SpmvState *st, ProfParams p) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  __shared__ ProfUnitSmem sm[4];
  const uint32_t pv = p.grp_pv[blockIdx.x % p.n_grp];
  const int g = (int)(threadIdx.x / kUnitRows);
  const uint32_t b = (blockIdx.x / p.n_grp) * 4 + (uint32_t)g;
  if (b >= p.c) return;
  switch (p.vids[pv]) {
    case 0: prof_unit<0>(A, y, st, p, pv, b, sm[g], g + 1); break;
    case 1: prof_unit<1>(A, y, st, p, pv, b, sm[g], g + 1); break;
    case 2: prof_unit<2>(A, y, st, p, pv, b, sm[g], g + 1); break;
    case 3: prof_unit<3>(A, y, st, p, pv, b, sm[g], g + 1); break;
    default: prof_unit<4>(A, y, st, p, pv, b, sm[g], g + 1); break;
  }
}

template <int VID>
__global__ void __launch_bounds__(kUnitRows * kProfGroups(VID), 1)
    spmv_prof_grp_kernel(SpmvDev A, float *__restrict__ y, SpmvState *st, ProfParams p, uint32_t pv) {
  constexpr int G = kProfGroups(VID);
  if constexpr (VID == DYSEL_SPMV_CSR_TMA) tma_stage_prologue();
  if (pv == p.part_first) asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  __shared__ ProfUnitSmem sm[G];
  const int g = (int)(threadIdx.x / kUnitRows);
  const uint32_t b = blockIdx.x * G + (uint32_t)g;
  if (b < p.c) prof_unit<VID>(A, y, st, p, pv, b, sm[g], G > 1 ? g + 1 : 0);
}

// All K profiling slices in ONE launch (no forked streams / joins): CTA b runs
// unit b / K of pool variant b mod K (interleaved start order).  The register
// cap is generous (128 registers): each variant's code is compiled as in its
// own kernel.  A 4-CTA/SM cap (64 registers, so profiling CTAs leave more
// room to the eager claim CTAs) measured no better on D4 (+5.0-5.4% vs
// +4.2% per step, same box).  The score is normalised by the plain kernel's
// occupancy, so the cap does not bias the selection.
__global__ void __launch_bounds__(kUnitRows, 1)
    spmv_prof_all_kernel(SpmvDev A, float *__restrict__ y, SpmvState *st, ProfParams p) {
  tma_stage_prologue();
  // launched behind the init kernel with PDL: wait for its state reset (a
  // no-op when launched without the attribute)
  asm volatile("griddepcontrol.wait;" ::: "memory");
  // programmatic dependent launch: the claim kernel queued behind this one
  // may start as soon as every profiling CTA is resident
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const uint32_t pv = blockIdx.x % p.K, b = blockIdx.x / p.K;
  __shared__ ProfUnitSmem sm;
  switch (p.vids[pv]) {
    case 0: prof_unit<0>(A, y, st, p, pv, b, sm, 0); break;
    case 1: prof_unit<1>(A, y, st, p, pv, b, sm, 0); break;
    case 2: prof_unit<2>(A, y, st, p, pv, b, sm, 0); break;
    case 3: prof_unit<3>(A, y, st, p, pv, b, sm, 0); break;
    case 4: prof_unit<4>(A, y, st, p, pv, b, sm, 0); break;
    default: prof_unit<5>(A, y, st, p, pv, b, sm, 0); break;
  }
}

// Remainder / eager claim kernel (readings A-27/A-28/A-45).  The host
// launches the DEFAULT variant's claim kernel right behind the profiling
// kernel (programmatic dependent launch), at its own occupancy; the switch
// kernel device-launches the winner's only when the default lost (A-42).
// Work is claimed per WARP, one 32-row slot per ticket, with no CTA-wide
// barrier (a CTA-per-unit persistent loop ran CSR-W 1.42 ms vs 0.94 ms for
// the plain grid: warps idled at the per-unit barrier behind the unit's
// longest row).  Ticket spaces over the plan's unit order seq (P = profiled
// prefix, L1 = max(P, n_light)):
//   * eager (ASYNC, the default's warps): slots of the light
//     units seq[P, L1), from counter c1, until the selection is published.
//     Publishing sets c1's bit 32; the claim count T_p at that instant,
//     rounded up to a whole unit, is the switch point S: the default keeps
//     eager slots [0, S) (a unit is never split between two variants — JDS
//     slots of a unit permute its rows).  An unproven default never starts a
//     heavy or long-row unit (A-45): those wait for the winner.
//   * winner: seq[L1, n) first (heavy / long-row units, nonzeros descending:
//     A-40), then the light slots from S on; a warp's first slot is static
//     (no atomic), later ones come from counter c2, k slots per atomic.
//   * pure full-grid run (the exhaustive oracle's version): the winner's
//     space with P = 0, S = 0.
// SYNC: every warp waits for the selection and S = 0.
// Every slot is computed exactly once.
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
  const uint32_t n_warps = gridDim.x * (kUnitRows / 32);
  const uint32_t gid = blockIdx.x * (kUnitRows / 32) + (threadIdx.x >> 5);
  const uint32_t P = p.pure ? 0u : p.p_end;
  const uint32_t L1 = max(P, p.n_light);
  const uint32_t n_hs = (p.n_units - L1) * kSlots;   // winner's first range: heavy / long-row slots
  const uint32_t E = (L1 - P) * kSlots;               // light slots after the profiled prefix
  const uint32_t Ee = p.pure ? 0u : eager_slots(p);   // eager ticket range
  // Claim batch: k = min(p.k_claim, remaining / (2 x warps)) >= 1 (p.k_claim
  // ~ 1024 nnz of work per claim: the counter serialises claims, ~1 per ns,
  // which capped 1-nnz rows).  Claims are made on demand: issuing the next
  // claim before running the current slots measured 7% slower on D4 (a warp
  // stuck on a long slot holds its prefetched one back).
  auto batch = [&](uint32_t rest) -> uint32_t {
    const uint32_t k = rest / (2u * n_warps);
    return k < p.k_min ? p.k_min : (k > p.k_claim ? p.k_claim : k);
  };
  // phase 0: pure run; 1: eager (default, ASYNC) from c1; 2: winner after the selection
  int phase = p.pure ? 0 : ((pv == p.def && p.async) ? 1 : 2);
  uint32_t S = 0, n_win = n_hs + E, eager = 0, done = 0;
  uint32_t t = 0, e = 0;   // current claim [t, e) in this phase's ticket space
  auto claim = [&](uint32_t k) -> uint64_t {   // lane 0 claims k slots of this phase's counter
    uint64_t raw = 0;
    if (lane == 0)
      raw = phase == 0 ? atomicAdd((unsigned long long *)&st->pure_ctr, (unsigned long long)k)
          : phase == 1 ? atomicAdd((unsigned long long *)&st->c1, (unsigned long long)k)
                       : (uint64_t)atomicAdd(&st->c2, k);
    return __shfl_sync(FULL, raw, 0);
  };
  // entering the winner's phase: false if another variant won
  auto enter_remainder = [&]() -> bool {
    uint64_t sw = 0;
    if (lane == 0) sw = wait_published(&st->sw);
    sw = __shfl_sync(FULL, sw, 0);
    if ((sw & 0xff) != pv) return false;
    phase = 2;
    S = min((uint32_t)(sw >> 8), Ee);
    n_win = n_hs + E - S;
    t = gid;   // static first slot
    e = t < n_win ? t + 1 : t;
    return true;
  };
  if (phase == 0) {
    t = gid;
    e = gid < n_win ? gid + 1 : gid;
  } else if (phase == 2) {
    if (!enter_remainder()) return;
  }
  for (;;) {
    if (t >= e) {   // need a claim
      if (phase == 1) {
        // CSR-V's warp walks its slot's 32 rows one after another (~1 us each):
        // an eager batch of several slots would hold a losing default's warps
        // (and their SM slots) for ~100 us after the selection; one slot per
        // claim bounds that drain to one slot
        // Other variants but CSR-W (whose slots take a few us): at most 2 slots
        // per eager claim, which bounds a losing default's drain to ~2 slots.
        const uint32_t k = VID == DYSEL_SPMV_CSR_VECTOR ? 1u
                           : VID == DYSEL_SPMV_CSR_STREAM ? batch(Ee - min(e, Ee))
                                                          : min(max(2u, p.k_min), batch(Ee - min(e, Ee)));
        const uint64_t r = claim(k);
        t = (uint32_t)r;
        uint32_t lim = Ee;
        if (r >> 32) {   // claimed after the selection was published: only below the switch point
          uint64_t sw = 0;
          if (lane == 0) sw = wait_published(&st->sw);
          lim = min((uint32_t)(__shfl_sync(FULL, sw, 0) >> 8), Ee);
        }
        if (t >= lim) {   // eager range closed or exhausted: hand over to the selection
          if (!enter_remainder()) break;
          continue;
        }
        e = min(t + k, lim);
        if (p.tl && lane == 0 && eager == 0)
          atomicMin((unsigned long long *)&p.tl[3], (unsigned long long)dysel_globaltimer());
        eager += e - t;
      } else {
        if (n_win <= n_warps) break;   // static slots only: no counter traffic
        const uint32_t k = batch(n_win - min(e, n_win));
        const uint64_t r = claim(k);
        const uint64_t c = (uint64_t)n_warps + r;
        if (c >= n_win) {
          // pure run: each warp ends on one failed claim; the last one resets the counters
          if (phase == 0 && lane == 0 && atomicAdd(&st->pure_done, 1u) == n_warps - 1) {
            st->pure_ctr = 0;
            st->pure_done = 0;
          }
          break;
        }
        t = (uint32_t)c;
        e = min(t + k, n_win);
      }
    }
    if (phase == 2) {
      if (p.tl && lane == 0 && done == 0)
        atomicMin((unsigned long long *)&p.tl[5], (unsigned long long)dysel_globaltimer());
      done += e - t;
    }
    for (uint32_t q = t; q < e; ++q) {
      uint32_t u, w;
      if (phase == 1) {   // eager: light slot q of seq[P, L1)
        u = unit_at(p, P + q / kSlots);
        w = q % kSlots;
      } else if (q < n_hs) {   // winner / pure: heavy-first range seq[L1, n)
        u = unit_at(p, L1 + q / kSlots);
        w = q % kSlots;
      } else {   // then the light slots from the switch point
        const uint32_t l = S + (q - n_hs);
        u = unit_at(p, P + l / kSlots);
        w = l % kSlots;
      }
      run_slot<VID>(A, u, (int)w, y + (size_t)u * kUnitRows);
      if (lane == 0 && p.unit_variant && w == 0) p.unit_variant[u] = (uint8_t)VID;
      if (p.chunk_done) {   // this slot's rows are final: release them to the chunked allgather
        __syncwarp();
        if (lane == 0) {
          __threadfence();
          atomicAdd(&p.chunk_done[u >> p.chunk_shift], 1u);
        }
      }
    }
    t = e;
  }
  if (p.tl && lane == 0) {
    if (eager) atomicMax((unsigned long long *)&p.tl[4], (unsigned long long)dysel_globaltimer());
    if (done) atomicMax((unsigned long long *)&p.tl[6], (unsigned long long)dysel_globaltimer());
  }
}

// Switch kernel (reading A-42): instead of one host-launched claim kernel per
// non-default variant -- K - 1 full grids that, when the default wins, only
// drain as exiting CTAs at the end of the step -- one 32-thread CTA queued
// behind the default's claim kernel waits for the selection and, only if
// another variant won, launches that variant's claim kernel from the device
// (fire-and-forget: stream order is kept, the parent grid completes with its
// child).  The child enters the winner's phase at the published switch point.
__global__ void spmv_switch_kernel(SpmvDev A, float *__restrict__ y, SpmvState *st, ProfParams p) {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  if (threadIdx.x != 0) return;
  const uint64_t sw = wait_published(&st->sw);
  const uint32_t w = (uint32_t)(sw & 0xff);
  if (w == p.def || w >= p.K || p.p_end >= p.n_units) return;
  // CSR-T's claim kernel is host-launched behind this one (its shared-memory
  // carveout is not applied to a device-side launch: it ran at half speed)
  if (p.vids[w] == DYSEL_SPMV_CSR_TMA) return;
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
    spmv_slice_kernel<VID><<<(unsigned)s->granule_count, kUnitRows, dyn_smem(VID), (cudaStream_t)stream>>>(
        A, (float *)args[0], *s);
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
                                            (const void *)spmv_slice_kernel<4>, (const void *)spmv_slice_kernel<5>};
  const void *claim[DYSEL_SPMV_NVARIANTS] = {(const void *)spmv_claim_kernel<0>, (const void *)spmv_claim_kernel<1>,
                                            (const void *)spmv_claim_kernel<2>, (const void *)spmv_claim_kernel<3>,
                                            (const void *)spmv_claim_kernel<4>, (const void *)spmv_claim_kernel<5>};
  const void *part[DYSEL_SPMV_NVARIANTS] = {
      (const void *)spmv_prof_grp_kernel<0>, (const void *)spmv_prof_grp_kernel<1>,
      (const void *)spmv_prof_grp_kernel<2>, (const void *)spmv_prof_grp_kernel<3>,
      (const void *)spmv_prof_grp_kernel<4>, (const void *)spmv_prof_grp_kernel<5>};
  {   // CSR-T's staging buffers exceed the 48 KB default dynamic limit
    const int m = (int)dyn_smem(DYSEL_SPMV_CSR_TMA);
    const void *k5[] = {(const void *)spmv_slice_kernel<5>, (const void *)spmv_slice_timed_kernel<5>,
                        (const void *)spmv_claim_kernel<5>, (const void *)spmv_prof_kernel<5>,
                        (const void *)spmv_prof_all_kernel, (const void *)spmv_prof_grp_kernel<5>};
    for (const void *k : k5)
      if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               k == (const void *)spmv_prof_grp_kernel<5> ? m * kProfGroups(5) : m) != cudaSuccess)
        return DYSEL_ERR_CUDA;
  }
  {   // load every kernel of the device path now (lazy module loading): a kernel's
      // first launch must not have to wait for spinning kernels of this path
    const void *pre[] = {(const void *)spmv_prof_grp_all_kernel, (const void *)spmv_switch_kernel,
                         (const void *)spmv_state_init_kernel, (const void *)spmv_prof_all_kernel};
    cudaFuncAttributes fa;
    for (const void *k : pre)
      if (cudaFuncGetAttributes(&fa, k) != cudaSuccess) return DYSEL_ERR_CUDA;
  }
  for (int v = 0; v < DYSEL_SPMV_NVARIANTS; ++v) {
    // largest L1 for the gathers; CSR-T holds its staging buffers in shared
    // memory: the smallest carveout that keeps its compiled CTAs/SM resident
    int carve = (int)cudaSharedmemCarveoutMaxL1;
    if (v == DYSEL_SPMV_CSR_TMA)
      carve = std::min(100, (int)((kClaimMinBlocks[v] * (sizeof(TmaStageBufs) + 2048) * 100 + 232447) / 232448));
    cudaFuncSetAttribute(slice[v], cudaFuncAttributePreferredSharedMemoryCarveout, carve);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&s->occ_slice[v], slice[v], kUnitRows, dyn_smem(v));
    cudaFuncSetAttribute(claim[v], cudaFuncAttributePreferredSharedMemoryCarveout, carve);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&s->occ_claim[v], claim[v], kUnitRows, dyn_smem(v));
    cudaFuncSetAttribute(part[v], cudaFuncAttributePreferredSharedMemoryCarveout, carve);
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
  DYSEL_TRY(dysel_register_variants(ctx, pl->sig.c_str(), vv, pl->K, pl->def));
  mark_builtin(ctx, pl->sig.c_str());
  return DYSEL_OK;
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

static void set_order(ProfParams &p, const dysel_spmv_plan *pl) {
  p.seq = pl->seq;
  p.n_light = pl->seq ? pl->n_light : pl->n_units;
}

// thread-per-row variants: a slot's time grows with its longest row (A-45)
static bool thread_per_row(int vid) {
  return vid == DYSEL_SPMV_CSR_SCALAR || vid == DYSEL_SPMV_ELL || vid == DYSEL_SPMV_JDS || vid == DYSEL_SPMV_CSR_TMA;
}

// Slots per claim: about kClaimNnz nonzeros of work (at least 1, at most a unit).
#ifndef DYSEL_CLAIM_NNZ
#define DYSEL_CLAIM_NNZ 4096
#endif
constexpr int64_t kClaimNnz = DYSEL_CLAIM_NNZ;
#ifndef DYSEL_GROUPED_PROFILING
#define DYSEL_GROUPED_PROFILING 1
#endif
constexpr bool kGroupedProfiling = DYSEL_GROUPED_PROFILING != 0;   // reading A-49
constexpr uint64_t kMinProfUnits = 12;   // reading A-52: three full groups of 4 units
constexpr uint64_t kMinProfBytes = 64ull << 20;   // reading A-3c: smaller matrices run unprofiled
constexpr uint64_t kMinProfFrac = 16;    // ... while K x 12 units stay within 1/16 of the matrix
#ifndef DYSEL_CLAIM_MAX_SLOTS
#define DYSEL_CLAIM_MAX_SLOTS 8
#endif
constexpr int64_t kClaimMaxSlots = DYSEL_CLAIM_MAX_SLOTS;   // one unit (32 slots measured: 2M diagonal 26 -> 45 us)
static uint32_t claim_batch(const dysel_spmv_plan *pl) {
  const int64_t slots = (int64_t)pl->n_units * kSlots;
  const int64_t per_slot = slots ? std::max<int64_t>(1, pl->info.nnz / slots) : 1;
  return (uint32_t)std::min<int64_t>(kClaimMaxSlots, std::max<int64_t>(1, kClaimNnz / per_slot));
}
// Smallest claim: ~kClaimMinNnz nonzeros of work.  The claim counter
// serialises (~1 claim per ns); on short rows a 1-2 slot claim is ~0.1 us of
// work, and the winner's phase after an eager phase claimed 2 slots at a time
// (5-point Laplacian: 4,700 units after the publish took 45 us, 2.5x the
// kernel's own rate).  Cheap slots make larger claims harmless for balance.
constexpr int64_t kClaimMinNnz = 1024;
static uint32_t claim_min(const dysel_spmv_plan *pl) {
  const int64_t slots = (int64_t)pl->n_units * kSlots;
  const int64_t per_slot = slots ? std::max<int64_t>(1, pl->info.nnz / slots) : 1;
  return (uint32_t)std::min<int64_t>(claim_batch(pl), std::max<int64_t>(1, kClaimMinNnz / per_slot));
}

// Pure version of one variant over the whole grid: the variant's claim kernel
// with every slot its own, in the winner's order (the same code, occupancy
// and order that run the DySel remainder, so T* and the remainder are
// measured on the same kernel).
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
  p.k_min = claim_min(pl);
  p.chunk_done = ctx->spmv_chunk_done;
  p.chunk_shift = ctx->spmv_chunk_shift;
  set_order(p, pl);
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
static cudaError_t launch_pdl(const void *fn, dim3 grid, dim3 block, size_t smem, cudaStream_t st, void **args);
template <int VID>
static cudaError_t launch_part(const SpmvDev &A, float *y, SpmvState *st, const ProfParams &p, uint32_t pv,
                               unsigned grid, cudaStream_t s) {
  SpmvDev a = A;
  float *yy = y;
  SpmvState *ss = st;
  ProfParams pp = p;
  uint32_t v = pv;
  void *args[] = {&a, &yy, &ss, &pp, &v};
  return launch_pdl((const void *)spmv_prof_grp_kernel<VID>, dim3(grid), dim3(kUnitRows * kProfGroups(VID)),
                    dyn_smem(VID) * kProfGroups(VID), s, args);
}
typedef cudaError_t (*PartLauncher)(const SpmvDev &, float *, SpmvState *, const ProfParams &, uint32_t, unsigned,
                                    cudaStream_t);
static const PartLauncher kPart[DYSEL_SPMV_NVARIANTS] = {launch_part<0>, launch_part<1>, launch_part<2>,
                                                         launch_part<3>, launch_part<4>, launch_part<5>};
static const ProfLauncher kProf[DYSEL_SPMV_NVARIANTS] = {launch_prof<0>, launch_prof<1>, launch_prof<2>, launch_prof<3>,
                                                         launch_prof<4>, launch_prof<5>};

static cudaError_t launch_pdl(const void *fn, dim3 grid, dim3 block, size_t smem, cudaStream_t st, void **args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelExC(&cfg, fn, args);
}

}  // namespace dysel

using namespace dysel;

extern "C" {

dysel_status dysel_spmv_variant(dysel_ctx *ctx, dysel_spmv_plan *pl, int variant_id, const float *d_x, float *d_y,
                                void *stream) {
  if (!ctx || !pl || pl->ctx != ctx || (pl->dev.n_rows > 0 && (!d_y || (pl->dev.n_cols > 0 && !d_x))) ||
      spmv_pool_index(pl, variant_id) < 0) {
    set_error(ctx, "dysel_spmv_variant: invalid arguments / variant not in pool");
    return DYSEL_ERR_INVALID;
  }
  return launch_variant_full(ctx, pl, variant_id, d_x, d_y, (cudaStream_t)stream);
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
    rep->sandbox_buffers = 0;
    rep->sandbox_bytes = 0;
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
    set_error(ctx, "dysel_spmv: swap mode needs atomics variants (dysel_spmtv)");
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
  {   // reading A-3c: a matrix of fewer than kMinProfBytes algorithmic bytes
      // runs in a few tens of us -- within ~2x the measured profiling latency
      // (~20-25 us to the publish on B200) -- so a single-shot profile cannot
      // pay for itself; the initial version runs (FORCE_PROFILE overrides)
    const uint64_t bytes = 8ull * (uint64_t)pl->info.nnz + 4ull * (uint64_t)(pl->dev.n_rows + 1) +
                           4ull * (uint64_t)pl->dev.n_cols + 4ull * (uint64_t)pl->dev.n_rows;
    if (P.active && !(mode & DYSEL_FORCE_PROFILE) && bytes < kMinProfBytes) {
      P.active = false;
      P.c = 0;
    }
  }
  // reading A-52: grouped profiling (A-49) measures a variant at the per-SM
  // load of the full run only when its slice fills several groups: with fewer
  // than kMinProfUnits units per variant, CSR-S's LSU saturation hid again
  // (regular FEM, default pool: CSR-S picked over ELL 10/10 at c = 1-4, 2/10
  // at c = 6, 0-1/10 at c = 8, 0/10 at c >= 9; +39% when it happens).  The
  // slice grows to kMinProfUnits when that keeps the profiled prefix within
  // 1/kMinProfFrac of the units.
  if (P.active && kGroupedProfiling && !(mode & DYSEL_SEQUENTIAL) && P.c < kMinProfUnits &&
      (uint64_t)pl->K * kMinProfUnits * kMinProfFrac <= P.Gn)
    P.c = kMinProfUnits;
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
  p.k_min = claim_min(pl);
  p.chunk_done = ctx->spmv_chunk_done;
  p.chunk_shift = ctx->spmv_chunk_shift;
  set_order(p, pl);
  // reading A-45: an unproven thread-per-row default gets no eager range on a
  // matrix with long-row units (measured on D4, JDS default: +12.9% with a
  // short-row eager range, +9.5% without eager work)
  p.no_eager = (pl->seq != nullptr && thread_per_row(pl->vids[pl->def])) ? 1u : 0u;
  p.abort = ((mode & DYSEL_NO_ABORT) || p.score_mode == 1) ? 0u : 1u;   // dominance needs busy or makespan
  const bool grouped = kGroupedProfiling && !sequential;
  for (int i = 0; i < pl->K; ++i) {
    p.vids[i] = pl->vids[i];
    // occupancy of the claim kernel that will run the remainder with this
    // variant (the busy-time score normalises by it, A-6)
    p.occ[i] = (uint32_t)std::max(1, cs->occ_claim[pl->vids[i]]);
    p.occ_t[i] = grouped ? std::min<uint32_t>(p.occ[i], (uint32_t)kProfGroups(pl->vids[i])) : p.occ[i];
  }
  if (p.hybrid) {   // Table 1: K - 1 slice-sized sandboxes, the default's slice is productive (A-4)
    const size_t bytes = (size_t)(pl->K - 1) * P.c * kUnitRows * sizeof(float);
    DYSEL_TRY(scratch(ctx, ctx->sandbox[0], bytes));
    p.sandbox = (float *)ctx->sandbox[0].ptr;
    if (rep) {
      rep->sandbox_buffers = (uint32_t)(pl->K - 1);
      rep->sandbox_bytes = bytes;
    }
  }
  p.unit_variant = d_uv;
  if (rep) p.tl = cs->d_state->tl;
  SpmvDev A = pl->dev;
  A.x = d_x;
  SpmvState *dst = cs->d_state;
  const int pend = reserve_pending_sel(ctx, &p.host_sel);
  spmv_state_init_kernel<<<1, 32, 0, st>>>(dst, pl->def);
  DYSEL_TRY(check_launch(ctx, "spmv_state_init_kernel"));
  if (sequential) {   // one launch per variant, back to back on the stream, default first
    for (int k = 0; k < pl->K; ++k) {
      const int i = k == 0 ? pl->def : (k <= pl->def ? k - 1 : k);
      kProf[pl->vids[i]](A, d_y, dst, p, (uint32_t)i, st);
      DYSEL_TRY(check_launch(ctx, "spmv_prof_kernel"));
    }
  } else if (grouped) {   // grouped profiling (reading A-49): one combined launch + CSR-T's, PDL-chained
    p.n_grp = 0;
    for (int i = 0; i < pl->K; ++i)
      if (pl->vids[i] != DYSEL_SPMV_CSR_TMA) p.grp_pv[p.n_grp++] = (uint32_t)i;
    p.part_first = DYSEL_SPMV_NVARIANTS;   // the combined kernel waits for the init kernel
    if (p.n_grp > 0) {
      void *args[] = {&A, &d_y, &dst, &p};
      DYSEL_CUDA_TRY(ctx, launch_pdl((const void *)spmv_prof_grp_all_kernel, dim3(p.n_grp * ((p.c + 3) / 4)),
                                     dim3(kUnitRows * 4), 0, st, args));
      DYSEL_TRY(check_launch(ctx, "spmv_prof_grp_all_kernel"));
    }
    for (int i = 0; i < pl->K; ++i) {
      if (pl->vids[i] != DYSEL_SPMV_CSR_TMA) continue;
      if (p.n_grp == 0) p.part_first = (uint32_t)i;
      const int G = kProfGroups(pl->vids[i]);
      const unsigned g = (unsigned)((p.c + G - 1) / G);
      DYSEL_CUDA_TRY(ctx, kPart[pl->vids[i]](A, d_y, dst, p, (uint32_t)i, g, st));
      DYSEL_TRY(check_launch(ctx, "spmv_prof_grp_kernel"));
    }
  } else {   // all K profiling slices in one launch, PDL behind the init kernel
    void *args[] = {&A, &d_y, &dst, &p};
    DYSEL_CUDA_TRY(ctx, launch_pdl((const void *)spmv_prof_all_kernel, dim3(p.K * p.c), dim3(kUnitRows),
                                   pool_dyn_smem(p), st, args));
    DYSEL_TRY(check_launch(ctx, "spmv_prof_all_kernel"));
  }
  if (p.p_end < p.n_units) {
    // the default's claim kernel, then the switch kernel (reading A-42); PDL
    // lets them start while profiling runs (plain stream order after a
    // sequential profile)
    const bool pdl = !sequential;
    const int v = pl->vids[pl->def];
    const uint64_t g = std::min<uint64_t>((uint64_t)std::max(1, cs->occ_claim[v]) * ctx->n_sm, p.n_units - p.p_end);
    DYSEL_TRY(kClaim[v](A, d_y, dst, p, (uint32_t)pl->def, (unsigned)g, st, pdl));
    DYSEL_TRY(check_launch(ctx, "spmv_claim_kernel"));
    if (pl->K > 1) {
      void *args[] = {&A, &d_y, &dst, &p};
      if (pdl)
        DYSEL_CUDA_TRY(ctx, launch_pdl((const void *)spmv_switch_kernel, dim3(1), dim3(32), 0, st, args));
      else
        spmv_switch_kernel<<<1, 32, 0, st>>>(A, d_y, dst, p);
      DYSEL_TRY(check_launch(ctx, "spmv_switch_kernel"));
    }
    // a non-default CSR-T: its claim kernel in plain stream order behind the
    // switch kernel (it enters the winner's phase at the published switch
    // point, or exits when another variant won)
    for (int i = 0; i < pl->K; ++i)
      if (i != pl->def && pl->vids[i] == DYSEL_SPMV_CSR_TMA) {
        const int v2 = pl->vids[i];
        const uint64_t g2 =
            std::min<uint64_t>((uint64_t)std::max(1, cs->occ_claim[v2]) * ctx->n_sm, p.n_units - p.p_end);
        DYSEL_TRY(kClaim[v2](A, d_y, dst, p, (uint32_t)i, (unsigned)g2, st, false));
        DYSEL_TRY(check_launch(ctx, "spmv_claim_kernel (CSR-T, host-gated)"));
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
    rep->eager_units = h->sw != ~0ull ? (h->sw >> 8) / kSlots : 0;
    rep->tail_units = p.n_units - p.p_end - std::min<uint64_t>(rep->eager_units, p.n_units - p.p_end);
    const uint64_t cap = (1ull << 56) - 1;
    for (int v = 0; v < pl->K; ++v) {
      const int id = pl->vids[v];
      const dysel_timer_slot &t = h->slot[v];
      rep->busy_ns[id] = h->busy[v];
      rep->aborted[id] = h->aborted[v];
      rep->makespan_ns[id] = t.t_end_max > t.t_start_min ? t.t_end_max - t.t_start_min : 0;
      rep->units[id] = t.units;
      rep->cycles[id] = t.cycles;
      rep->score[id] = h->decided[v] == 2u ? cap
                       : p.score_mode == 1 ? (t.units ? t.cycles / t.units : cap)
                       : p.score_mode == 2 ? rep->makespan_ns[id]
                                           : std::max<uint64_t>(h->busy[v] * p.n_units /
                                                                    ((uint64_t)p.c * p.occ_t[v] * p.n_sm),
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
