/*
 * dysel_device.cuh — device-side helpers for DySel variant kernels (sm_100a).
 *
 * 1. Slice mapping: the paper's profiling / eager copies shift the block index
 *    so a variant processes "a particular part of the workload"; the batch
 *    copy skips blocks already profiled (§3.3).  Here a launch
 *    covers exactly the granules of its dysel_slice (reading A-10: launch the
 *    remainder grid with an offset instead of suppressing blocks), so
 *    dysel_cta_origin() maps blockIdx -> the first unit of the CTA's tile.
 *
 * 2. Timing (Fig. 7b): the paper's thread 0 reads the 32-bit
 *    per-SM %clock, atomicMin's a global start stamp, the last block
 *    (atomicInc) computes the diff and a racy atomicMin/atomicExch picks the
 *    winner.  B200 form (readings A-6, A-7): lane 0 of every warp samples
 *    %globaltimer (ns, chip-global) and clock64 at entry and exit; warp 0
 *    reduces the per-warp samples with __shfl_xor_sync (min start, max end);
 *    thread 0 does atomicMin(t_start_min) / atomicMax(t_end_max) /
 *    atomicAdd(cycles, units) on the variant's slot, then counts its CTA.
 *    The last CTA of a variant computes the score and does ONE atomicMin on
 *    the packed word (score << 8 | v) — ties go to the lower id (A-8) — and
 *    the last variant to finish publishes the packed minimum as the
 *    selection.
 */
#ifndef DYSEL_DEVICE_CUH_
#define DYSEL_DEVICE_CUH_

#include <stdint.h>

#include "dysel.h"

__device__ __forceinline__ uint64_t dysel_globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

__device__ __forceinline__ uint64_t dysel_clock64() {
  uint64_t c;
  asm volatile("mov.u64 %0, %%clock64;" : "=l"(c));
  return c;
}

__device__ __forceinline__ uint64_t dysel_ld_acquire_u64(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

/* CTAs per granule for a variant of work-assignment factor wa. */
__host__ __device__ __forceinline__ uint64_t dysel_ctas_per_granule(const dysel_slice &s, const uint32_t wa[3]) {
  return (uint64_t)(s.g[0] / wa[0]) * (s.g[1] / wa[1]) * (s.g[2] / wa[2]);
}

__host__ __device__ __forceinline__ uint64_t dysel_slice_ctas(const dysel_slice &s, const uint32_t wa[3]) {
  return s.granule_count * dysel_ctas_per_granule(s, wa);
}

/* First unit (ux, uy, uz) of CTA `cta` of a launch over slice s; returns false
 * when that tile lies wholly outside U (edge granule). */
__host__ __device__ __forceinline__ bool dysel_cta_origin(const dysel_slice &s, const uint32_t wa[3], uint64_t cta,
                                                          uint64_t u[3]) {
  const uint32_t h0 = s.g[0] / wa[0], h1 = s.g[1] / wa[1], h2 = s.g[2] / wa[2];
  const uint64_t hper = (uint64_t)h0 * h1 * h2;
  const uint64_t gi = cta / hper, sub = cta % hper;
  const uint64_t j = s.granule_begin + gi * s.granule_stride;
  const uint64_t gx = j % s.G[0], gy = (j / s.G[0]) % s.G[1], gz = j / ((uint64_t)s.G[0] * s.G[1]);
  const uint64_t sx = sub % h0, sy = (sub / h0) % h1, sz = sub / ((uint64_t)h0 * h1);
  u[0] = gx * s.g[0] + sx * wa[0];
  u[1] = gy * s.g[1] + sy * wa[1];
  u[2] = gz * s.g[2] + sz * wa[2];
  return u[0] < s.U[0] && u[1] < s.U[1] && u[2] < s.U[2];
}

/* Gated batch copy: false => this CTA must exit (another variant was selected). */
__device__ __forceinline__ bool dysel_gate_open(const dysel_slice &s) {
  if (s.gate == nullptr) return true;
  return (int32_t)(dysel_ld_acquire_u64(s.gate) & 0xffu) == s.variant;
}

struct dysel_prof_smem {
  unsigned long long t0[32], t1[32], c0[32], c1[32];
  unsigned long long c_last;   /* thread 0: clock64 of the CTA's last dominance report */
  int dominated;               /* broadcast of the last dysel_prof_poll result */
};

/* Score from a cycle sum `cy` over `un` units (cap on un == 0): wave-quantised
 * full-grid prediction (A-34) when the slice declares its grid and wave,
 * else occupancy-normalised time per unit per slot (A-6), else cycles/unit. */
__host__ __device__ __forceinline__ unsigned long long dysel_cycle_score(const dysel_slice &s, unsigned long long cy,
                                                                         unsigned long long un) {
  const unsigned long long cap = (1ull << 56) - 1;
  if (un == 0) return cap;
  unsigned long long r;
  if (s.score_cycles)
    r = cy / un;
  else if (s.grid_ctas && s.wave_ctas && s.units_per_cta)
    r = ((s.grid_ctas + s.wave_ctas - 1) / s.wave_ctas) * (cy * (unsigned long long)s.units_per_cta / un);
  else if (s.occupancy)
    r = cy * 64ull / (un * (unsigned long long)s.occupancy);
  else
    return cap;
  return r < cap ? r : cap;
}

/* Packed selection bookkeeping shared by completion and dominance: called
 * once per variant (by whoever decided it); the last variant publishes. */
__device__ __forceinline__ void dysel_variant_decided(const dysel_slice &s) {
  __threadfence();
  const uint32_t vd = atomicAdd(s.variants_done, 1u) + 1u;
  if (vd == s.n_variants) {           /* last variant: publish the selection */
    __threadfence();
    const unsigned long long fin = atomicAdd((unsigned long long *)s.best, 0ull);
    s.sel[1] = dysel_globaltimer();   /* the library's state block keeps the publish time right after sel */
    atomicExch((unsigned long long *)s.sel, fin);
  }
}

/* Call with all threads of the CTA at kernel entry (after any early exit
 * that is uniform for the CTA).  No-op when s.timer == NULL. */
__device__ __forceinline__ void dysel_prof_begin(const dysel_slice &s, dysel_prof_smem &sm) {
  if (s.timer == nullptr) return;
  const uint32_t tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  if ((tid & 31) == 0) {
    sm.c0[tid >> 5] = dysel_clock64();
    sm.t0[tid >> 5] = dysel_globaltimer();
  }
  if (tid == 0) {
    sm.c_last = sm.c0[0];
    sm.dominated = 0;
  }
}

/* Dominance poll (reading A-32).  Call with ALL threads of the CTA (it holds
 * one __syncthreads), every few microseconds of work, between
 * dysel_prof_begin and dysel_prof_end.  Thread 0 adds the cycles elapsed
 * since its last report to the variant's running sum lb; the variant is
 * dominated once lb * 64 / (units_total * occupancy) (or lb / units_total
 * with score_cycles) exceeds the best completed score — its final score can
 * only be larger — and the first CTA to see it decides the variant (maximal
 * score).  Returns true when the variant is dominated: a SANDBOX CTA may then
 * stop (its output is discarded), a productive CTA must finish its tile. */
/* Single-thread form (no barrier), for warp-specialised kernels: the calling
 * thread (the one that ran dysel_prof_begin's thread-0 part, i.e. tid 0)
 * reports and checks; it returns the dominated flag but nothing stops the
 * CTA — it only lets the selection be published without waiting for it. */
/* Progress form (reading A-51): the caller also passes how much of its CTA's
 * work is done (done of total, uniform steps, e.g. K-slabs or z-planes).
 * Besides the strict lower bound above, thread 0 extrapolates the CTA's
 * final cycles (elapsed x total / done) to the variant's score; a projection
 * above 5/4 of the best completed score decides the variant as well.  An
 * estimate, not a bound: the 5/4 margin covers per-step variation (a GEMM
 * tile's K-slabs, a stencil column's planes are uniform work). */
__device__ __forceinline__ bool dysel_prof_poll_thread(const dysel_slice &s, dysel_prof_smem &sm, uint32_t done = 0u,
                                                       uint32_t total = 0u) {
  if (s.timer == nullptr || s.lb == nullptr) return false;
  if (!sm.dominated) {
    const unsigned long long now = dysel_clock64();
    const unsigned long long tot = atomicAdd((unsigned long long *)s.lb, now - sm.c_last) + (now - sm.c_last);
    sm.c_last = now;
    int d = *(volatile uint32_t *)s.decided == 2u;
    if (!d) {
      const unsigned long long best = *(volatile unsigned long long *)s.best >> 8;
      const unsigned long long cap = (1ull << 56) - 1;
      const unsigned long long un = s.units_total ? s.units_total : 1ull;
      /* a lower bound of the final score (tot <= final cycle sum, un >= final
       * units); makespan scores have no cycle bound */
      const bool cyc = s.score_cycles || (s.grid_ctas && s.wave_ctas && s.units_per_cta) || s.occupancy;
      unsigned long long lbs = cyc ? dysel_cycle_score(s, tot, un) : 0ull;
      if (cyc && best < cap && done > 0u && total > done && s.ctas_total > 0u) {
        const unsigned long long el = now - sm.c0[0];
        const unsigned long long proj = el / done * total * (unsigned long long)s.ctas_total;
        const unsigned long long ps = dysel_cycle_score(s, proj, un);
        if (ps > best + best / 4 && ps > lbs) lbs = ps;
      }
      if (best < cap && lbs > best) {
        d = 1;
        if (atomicCAS(s.decided, 0u, 2u) == 0u) dysel_variant_decided(s);
      }
    }
    sm.dominated = d;
  }
  return sm.dominated != 0;
}

__device__ __forceinline__ bool dysel_prof_poll(const dysel_slice &s, dysel_prof_smem &sm, uint32_t done = 0u,
                                                uint32_t total = 0u) {
  if (s.timer == nullptr || s.lb == nullptr) return false;
  const uint32_t tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  if (tid == 0) dysel_prof_poll_thread(s, sm, done, total);
  __syncthreads();
  return sm.dominated != 0;
}

/* Call with all threads at the end of the CTA's work.  `units` = units this
 * CTA processed (for cycles/unit scoring). */
__device__ __forceinline__ void dysel_prof_end(const dysel_slice &s, dysel_prof_smem &sm, uint32_t units) {
  if (s.timer == nullptr) return;
  const uint32_t tid = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  const uint32_t nw = (blockDim.x * blockDim.y * blockDim.z + 31) >> 5;
  if ((tid & 31) == 0) {
    sm.t1[tid >> 5] = dysel_globaltimer();
    sm.c1[tid >> 5] = dysel_clock64();
  }
  __syncthreads();
  if (tid < 32) {
    const uint32_t l = tid;
    unsigned long long t0 = l < nw ? sm.t0[l] : ~0ull, t1 = l < nw ? sm.t1[l] : 0ull;
    unsigned long long c0 = l < nw ? sm.c0[l] : ~0ull, c1 = l < nw ? sm.c1[l] : 0ull;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      t0 = min(t0, __shfl_xor_sync(0xffffffffu, t0, o));
      t1 = max(t1, __shfl_xor_sync(0xffffffffu, t1, o));
      c0 = min(c0, __shfl_xor_sync(0xffffffffu, c0, o));
      c1 = max(c1, __shfl_xor_sync(0xffffffffu, c1, o));
    }
    if (l == 0) {
      dysel_timer_slot *slot = s.timer;
      atomicMin((unsigned long long *)&slot->t_start_min, t0);
      atomicMax((unsigned long long *)&slot->t_end_max, t1);
      atomicAdd((unsigned long long *)&slot->cycles, c1 - c0);
      atomicAdd((unsigned long long *)&slot->units, (unsigned long long)units);
      __threadfence();
      const uint32_t done = atomicAdd(s.ctas_done, 1u) + 1u;
      /* last CTA of this variant, unless dominance decided it already */
      if (done == s.ctas_total && (s.decided == nullptr || atomicCAS(s.decided, 0u, 1u) == 0u)) {
        __threadfence();
        const unsigned long long a = atomicAdd((unsigned long long *)&slot->t_start_min, 0ull);
        const unsigned long long b = atomicAdd((unsigned long long *)&slot->t_end_max, 0ull);
        const unsigned long long cy = atomicAdd((unsigned long long *)&slot->cycles, 0ull);
        const unsigned long long un = atomicAdd((unsigned long long *)&slot->units, 0ull);
        unsigned long long score =
            s.score_cycles ? (un ? cy / un : (1ull << 56) - 1)
            : (s.occupancy || (s.grid_ctas && s.wave_ctas)) ? dysel_cycle_score(s, cy, un)
                           : (b - a);
        if (score > (1ull << 56) - 1) score = (1ull << 56) - 1;
        atomicMin((unsigned long long *)s.best, (score << 8) | (unsigned)s.variant);
        dysel_variant_decided(s);
      }
    }
  }
}

#endif /* DYSEL_DEVICE_CUH_ */
