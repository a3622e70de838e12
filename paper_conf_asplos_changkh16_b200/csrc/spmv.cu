// DySel SpMV: format preparation (a-1), the variant pool, the persistent
// ticket dispatcher (a-3..a-5 on the device) and the paper-faithful host path.
//
// Device protocol (the B200 answer to P:L1674-1691 — "querying the
// status often takes a longer latency than profiling time", so the paper's GPU
// async ≈ sync): ONE persistent launch of #SM x occupancy CTAs.  Each CTA
// claims 256-row units by ticket (atomicAdd).  Tickets [0, K*c) are the
// profiling units (claimed first = priority): fully mode gives
// unit t to variant t mod K (A-24); hybrid mode gives unit floor(t/K) to every
// variant, the default writing y and the others a sandbox (A-4).  A profiling
// unit is timed per CTA (Fig. 7b form in dysel_device.cuh); when a variant's c
// units are done its score is atomicMin'd into `best`; the last variant
// publishes `sel` and sets `release`.  Remainder units: sync mode spins on
// `release` (every profiling ticket is held by an already-running CTA, so the
// spin cannot deadlock); async mode runs the best-so-far (default until the
// first variant completes) — the paper's eager execution with one-unit chunks
// and no launch cost.  The last CTA to exit copies the state to
// the report area and resets it for the next launch (no memset launch).
#include <cub/device/device_scan.cuh>

#include <algorithm>
#include <cstring>
#include <string>

#include "dysel_device.cuh"
#include "internal.h"
#include "spmv_kernels.cuh"

namespace dysel {

// Scores (reading A-6): the dispatcher scores a variant by the
// mean busy time of its profiled units (sum over its units of the CTA's
// %globaltimer end - start, / units).  All variants run inside the same
// persistent launch with the same occupancy, so per-unit latency ranks their
// throughput; the paper's makespan (first start .. last end, Fig. 7b) is
// polluted here by ticket queueing, and stays available (DYSEL_SCORE_MAKESPAN)
// as does the clock64 sum (DYSEL_SCORE_CYCLES).
struct SpmvState {
  uint32_t ticket;
  uint32_t exited;
  uint32_t variants_done;
  uint32_t release;
  uint64_t best;          // (score << 8) | pool variant, 0xff = none yet
  uint64_t sel;           // final packed selection, ~0 until published
  uint64_t eager_units;   // remainder units started before the selection
  uint64_t best_total;    // min over completed variants of their busy sum (ns)
  uint64_t tail_begin;    // first unit handed to the tail launch (or ~0)
  uint32_t ctas_done[DYSEL_MAX_VARIANTS];
  uint32_t dominated[DYSEL_MAX_VARIANTS];
  uint64_t busy[DYSEL_MAX_VARIANTS];      // sum of unit durations (ns), completed units
  uint64_t lb[DYSEL_MAX_VARIANTS];        // lower bound of the final busy sum (ns)
  uint64_t aborted[DYSEL_MAX_VARIANTS];   // sandbox units stopped or skipped by dominance
  dysel_timer_slot slot[DYSEL_MAX_VARIANTS];
};
struct SpmvStateBlock {
  SpmvState live;
  SpmvState rep;
};

struct DispatchParams {
  uint32_t K;            // pool size
  uint32_t c;            // profiling units per variant
  uint32_t n_tickets;
  uint32_t n_units;
  uint32_t hybrid, async, contiguous, score_mode;   // score_mode 0 busy, 1 cycles, 2 makespan
  uint32_t def;          // pool index of default variant
  uint32_t tail;         // hand the remainder to the winner's plain kernel (CDP2 tail launch)
  uint32_t abort;        // dominance abort of hybrid sandbox units
  int32_t vids[DYSEL_SPMV_NVARIANTS];
  float *sandbox;        // (K-1) * c * 256 floats (hybrid)
  uint8_t *unit_variant; // optional debug map (pool index per unit)
};

__device__ __forceinline__ void reset_state(SpmvState *s) {
  s->ticket = 0;
  s->exited = 0;
  s->variants_done = 0;
  s->release = 0;
  s->best = (((1ull << 56) - 1) << 8) | 0xffull;
  s->sel = ~0ull;
  s->eager_units = 0;
  s->best_total = ~0ull;
  s->tail_begin = ~0ull;
  for (int v = 0; v < DYSEL_MAX_VARIANTS; ++v) {
    s->ctas_done[v] = 0;
    s->dominated[v] = 0;
    s->busy[v] = 0;
    s->lb[v] = 0;
    s->aborted[v] = 0;
    s->slot[v].t_start_min = ~0ull;
    s->slot[v].t_end_max = 0;
    s->slot[v].units = 0;
    s->slot[v].cycles = 0;
  }
}

__global__ void spmv_state_reset_kernel(SpmvStateBlock *b) {
  if (threadIdx.x == 0) {
    reset_state(&b->live);
    reset_state(&b->rep);
  }
}

__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t *p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
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
__device__ __forceinline__ void st_release_u32(uint32_t *p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// Dominance abort for hybrid sandbox units: every
// ~kPollNs one thread of the CTA adds the time elapsed since the last report
// to lb[v].  lb[v] only ever sums time that variant v's units have really
// spent, so it is a lower bound of v's final busy sum; once it exceeds the
// busy sum of a COMPLETED variant (best_total), v can no longer be selected
// (all variants profile the same c units in hybrid mode), so its sandbox work
// stops and its remaining sandbox units are skipped.  The selection is the one
// running them to completion would give.
constexpr uint64_t kPollNs = 2000;
struct SandboxPoll {
  static constexpr bool active = true;
  unsigned long long *s_last;   // smem: last report time
  volatile int *s_abort;        // smem
  unsigned long long *lb;
  const uint64_t *best_total;
  uint32_t *dominated;
  __device__ __forceinline__ bool operator()() const {
    if (*s_abort) return true;
    const unsigned long long now = dysel_globaltimer();
    const unsigned long long last = *(volatile unsigned long long *)s_last;
    if (now - last < kPollNs) return false;
    if (atomicCAS(s_last, last, now) != last) return *s_abort != 0;   // another thread reports
    const unsigned long long l = atomicAdd(lb, now - last) + (now - last);
    if (l > ld_relaxed_u64(best_total) || ld_relaxed_u32(dominated) != 0) {
      *s_abort = 1;
      atomicExch(dominated, 1u);
      return true;
    }
    return false;
  }
};

constexpr int kPersistMinBlocks = 4;

// resident CTAs per SM each plain variant kernel is compiled for (register cap)
constexpr int kSliceMinBlocks[DYSEL_SPMV_NVARIANTS] = {8, 4, 8, 6, 6};

template <int VID>
__global__ void __launch_bounds__(kUnitRows, kSliceMinBlocks[VID])
    spmv_slice_kernel(SpmvDev A, float *__restrict__ y, dysel_slice s, uint8_t *uv);

__device__ void tail_launch(int vid, const SpmvDev &A, float *y, uint64_t u0, uint64_t n_units, uint8_t *uv) {
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
  switch (vid) {
    case 0: spmv_slice_kernel<0><<<grid, kUnitRows, 0, cudaStreamTailLaunch>>>(A, y, s, uv); break;
    case 1: spmv_slice_kernel<1><<<grid, kUnitRows, 0, cudaStreamTailLaunch>>>(A, y, s, uv); break;
    case 2: spmv_slice_kernel<2><<<grid, kUnitRows, 0, cudaStreamTailLaunch>>>(A, y, s, uv); break;
    case 3: spmv_slice_kernel<3><<<grid, kUnitRows, 0, cudaStreamTailLaunch>>>(A, y, s, uv); break;
    default: spmv_slice_kernel<4><<<grid, kUnitRows, 0, cudaStreamTailLaunch>>>(A, y, s, uv); break;
  }
}

__global__ void __launch_bounds__(kUnitRows, kPersistMinBlocks)
    spmv_persistent_kernel(SpmvDev A, float *__restrict__ y, SpmvStateBlock *sb, DispatchParams p) {
  __shared__ uint32_t s_ticket;
  __shared__ int32_t s_v;
  __shared__ unsigned long long s_last;
  __shared__ int s_abort;
  __shared__ dysel_prof_smem psm;
  SpmvState *st = &sb->live;
  const uint32_t tid = threadIdx.x;
  const uint32_t P = p.K * p.c;
  // sync + tail: only the profiling tickets run here, the tail kernel takes [P, n)
  const uint32_t limit = (p.tail && !p.async) ? P : p.n_tickets;
  if (tid == 0) s_ticket = atomicAdd(&st->ticket, 1u);
  __syncthreads();
  uint32_t t = s_ticket;
  while (t < limit) {
    uint32_t next = 0;
    if (tid == 0) next = atomicAdd(&st->ticket, 1u);   // prefetch: latency hidden by the unit's work
    if (t < P) {
      // ---------------------------------------------------- profiling unit
      uint32_t j, pv;
      bool productive = true;
      if (p.hybrid) {
        j = t / p.K;
        pv = t % p.K;
        productive = pv == p.def;
      } else if (p.contiguous) {
        j = t;
        pv = t / p.c;
      } else {
        j = t;
        pv = t % p.K;
      }
      const bool sandbox = !productive;
      bool skipped = false;
      if (tid == 0) {
        s_abort = 0;
        s_last = dysel_globaltimer();
        skipped = sandbox && p.abort && ld_relaxed_u32(&st->dominated[pv]) != 0;
        s_v = skipped ? 1 : 0;
      }
      __syncthreads();
      skipped = s_v != 0;
      float *out = productive ? y + (size_t)j * kUnitRows
                              : p.sandbox + ((size_t)(pv < p.def ? pv : pv - 1) * p.c + j) * kUnitRows;
      if (!skipped) {
        if ((tid & 31) == 0) {
          psm.c0[tid >> 5] = dysel_clock64();
          psm.t0[tid >> 5] = dysel_globaltimer();
        }
        if (sandbox && p.abort) {
          SandboxPoll poll{&s_last, &s_abort, (unsigned long long *)&st->lb[pv], &st->best_total, &st->dominated[pv]};
          run_unit_dyn(p.vids[pv], A, j, out, poll);
        } else {
          run_unit_dyn(p.vids[pv], A, j, out, NoPoll());
        }
        if ((tid & 31) == 0) {
          psm.t1[tid >> 5] = dysel_globaltimer();
          psm.c1[tid >> 5] = dysel_clock64();
        }
      }
      __syncthreads();
      if (tid < 32) {   // warp-shuffle reduction of the per-warp samples
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
          const bool stopped = skipped || s_abort;
          if (!skipped) {
            atomicMin((unsigned long long *)&slot->t_start_min, t0);
            atomicMax((unsigned long long *)&slot->t_end_max, t1);
            atomicAdd((unsigned long long *)&slot->cycles, c1 - c0);
            atomicAdd((unsigned long long *)&st->busy[pv], t1 - t0);
            atomicAdd((unsigned long long *)&st->lb[pv], t1 - s_last);   // rest of this unit's time
          }
          if (stopped) atomicAdd((unsigned long long *)&st->aborted[pv], 1ull);
          atomicAdd((unsigned long long *)&slot->units, 1ull);
          if (productive && p.unit_variant) p.unit_variant[j] = (uint8_t)p.vids[pv];
          __threadfence();
          const uint32_t done = atomicAdd(&st->ctas_done[pv], 1u) + 1u;
          if (done == p.c) {   // variant complete: score, packed atomicMin (A-7, A-8)
            __threadfence();
            const unsigned long long a = atomicAdd((unsigned long long *)&slot->t_start_min, 0ull);
            const unsigned long long b = atomicAdd((unsigned long long *)&slot->t_end_max, 0ull);
            const unsigned long long cy = atomicAdd((unsigned long long *)&slot->cycles, 0ull);
            const unsigned long long bz = atomicAdd((unsigned long long *)&st->busy[pv], 0ull);
            const bool dom = ld_relaxed_u32(&st->dominated[pv]) != 0;
            unsigned long long score = p.score_mode == 1 ? cy / p.c : (p.score_mode == 2 ? b - a : bz / p.c);
            if (dom || score > (1ull << 56) - 1) score = (1ull << 56) - 1;
            if (!dom) atomicMin((unsigned long long *)&st->best_total, bz);
            atomicMin((unsigned long long *)&st->best, (score << 8) | pv);
            __threadfence();
            const uint32_t vd = atomicAdd(&st->variants_done, 1u) + 1u;
            if (vd == p.K) {   // last variant: publish, hand off the remainder
              __threadfence();
              const unsigned long long fin = atomicAdd((unsigned long long *)&st->best, 0ull);
              atomicExch((unsigned long long *)&st->sel, fin);
              __threadfence();
              st_release_u32(&st->release, 1u);
              if (p.tail) {
                // grab every ticket not yet claimed; dispatcher CTAs then exit
                const uint32_t old = p.async ? atomicAdd(&st->ticket, 1u << 30) : P;
                const uint64_t u0 = p.hybrid ? (uint64_t)old - (uint64_t)(p.K - 1) * p.c : old;
                if (old < p.n_tickets && u0 < p.n_units) {
                  st->tail_begin = u0;
                  tail_launch(p.vids[fin & 0xff], A, y, u0, p.n_units, p.unit_variant);
                }
              }
            }
          }
        }
      }
    } else {
      // ---------------------------------------------------- remainder unit
      const uint32_t j = p.hybrid ? t - (p.K - 1) * p.c : t;
      if (tid == 0) {
        int v;
        if (P == 0) {
          v = (int)p.def;
        } else if (!p.async) {
          uint32_t ns = 32;
          while (ld_acquire_u32(&st->release) == 0) {
            __nanosleep(ns);
            ns = min(ns * 2, 1024u);
          }
          v = (int)(ld_relaxed_u64(&st->sel) & 0xff);
        } else {
          const uint64_t b = ld_relaxed_u64(&st->best);
          v = (b & 0xff) == 0xff ? (int)p.def : (int)(b & 0xff);
          if (ld_acquire_u32(&st->release) == 0) atomicAdd((unsigned long long *)&st->eager_units, 1ull);
        }
        s_v = v;
        if (p.unit_variant) p.unit_variant[j] = (uint8_t)p.vids[v];
      }
      __syncthreads();
      run_unit_dyn(p.vids[s_v], A, j, y + (size_t)j * kUnitRows, NoPoll());
    }
    __syncthreads();
    if (tid == 0) s_ticket = next;
    __syncthreads();
    t = s_ticket;
  }
  // exit protocol: the last CTA out snapshots the state and resets it
  if (tid == 0) {
    __threadfence();
    const uint32_t e = atomicAdd(&st->exited, 1u) + 1u;
    if (e == gridDim.x) {
      __threadfence();
      volatile SpmvState *vs = st;
      SpmvState *r = &sb->rep;
      r->ticket = vs->ticket;
      r->variants_done = vs->variants_done;
      r->release = vs->release;
      r->best = vs->best;
      r->sel = vs->sel;
      r->eager_units = vs->eager_units;
      r->best_total = vs->best_total;
      r->tail_begin = vs->tail_begin;
      for (int v = 0; v < DYSEL_MAX_VARIANTS; ++v) {
        r->ctas_done[v] = vs->ctas_done[v];
        r->dominated[v] = vs->dominated[v];
        r->busy[v] = vs->busy[v];
        r->lb[v] = vs->lb[v];
        r->aborted[v] = vs->aborted[v];
        r->slot[v].t_start_min = vs->slot[v].t_start_min;
        r->slot[v].t_end_max = vs->slot[v].t_end_max;
        r->slot[v].units = vs->slot[v].units;
        r->slot[v].cycles = vs->slot[v].cycles;
      }
      reset_state(st);
      __threadfence();
    }
  }
}

// Plain full-grid / slice kernel of one variant: the exhaustive oracle's pure
// version, the activation-flag-off path, the tail-launched remainder and the
// host path's profiling / eager / batch copies (dysel_device.cuh timing).
template <int VID>
__global__ void __launch_bounds__(kUnitRows, kSliceMinBlocks[VID])
    spmv_slice_kernel(SpmvDev A, float *__restrict__ y, dysel_slice s, uint8_t *uv) {
  __shared__ dysel_prof_smem psm;
  if (!dysel_gate_open(s)) return;
  dysel_prof_begin(s, psm);
  const uint32_t j = (uint32_t)(s.granule_begin + (uint64_t)blockIdx.x * s.granule_stride);
  run_unit<VID>(A, j, y + (size_t)j * kUnitRows);
  if (uv && threadIdx.x == 0) uv[j] = (uint8_t)VID;
  dysel_prof_end(s, psm, 1u);
}

// ------------------------------------------------------ format preparation
__global__ void row_stats_kernel(const int32_t *__restrict__ rp, int64_t n, int32_t *__restrict__ max_len) {
  int m = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    m = max(m, rp[i + 1] - rp[i]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) m = max(m, __shfl_xor_sync(0xffffffffu, m, o));
  if ((threadIdx.x & 31) == 0) atomicMax(max_len, m);
}

// ELL: slot (k, i) at k * n_pad + i = k-th CSR entry of row i (pads preset to
// col = -1, val = 0 by memset).
__global__ void ell_fill_kernel(const int32_t *__restrict__ rp, const int32_t *__restrict__ col,
                                const float *__restrict__ val, int64_t n, int64_t n_pad, int32_t *__restrict__ ec,
                                float *__restrict__ ev) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  const int b = rp[i], e = rp[i + 1];
  for (int k = b; k < e; ++k) {
    ec[(int64_t)(k - b) * n_pad + i] = col[k];
    ev[(int64_t)(k - b) * n_pad + i] = val[k];
  }
}

// Block-local JDS, phase 1: per 256-row block, stable sort of the rows by
// length (descending; ties -> lower row) by rank counting; W_b.
__global__ void __launch_bounds__(kUnitRows) jds_sort_kernel(const int32_t *__restrict__ rp, int64_t n,
                                                             int32_t *__restrict__ perm,
                                                             int32_t *__restrict__ jds_len,
                                                             int64_t *__restrict__ wp1) {
  __shared__ int32_t s_len[kUnitRows];
  const int64_t r0 = (int64_t)blockIdx.x * kUnitRows;
  const int nb_rows = (int)min((int64_t)kUnitRows, n - r0);
  const int i = threadIdx.x;
  const int li = i < nb_rows ? rp[r0 + i + 1] - rp[r0 + i] : -1;
  s_len[i] = li;
  __syncthreads();
  if (i < nb_rows) {
    int rank = 0;
    for (int q = 0; q < nb_rows; ++q) {
      const int lq = s_len[q];
      rank += (lq > li) || (lq == li && q < i);
    }
    perm[r0 + rank] = (int32_t)(r0 + i);
    jds_len[r0 + rank] = li;
  }
  if (i == 0) {
    int w = 0;
    for (int q = 0; q < nb_rows; ++q) w = max(w, s_len[q]);
    wp1[blockIdx.x] = (int64_t)w + 1;   // W_b + 1 entries of jd_ptr
  }
}

// phase 2: jd_ptr_b[k] = sum_p min(len_p, k) for k = 0..W_b  (= sum of the
// diagonal counts #{p : len_p > k'} for k' < k).
__global__ void __launch_bounds__(kUnitRows) jds_ptr_kernel(const int32_t *__restrict__ jds_len, int64_t n,
                                                            const int64_t *__restrict__ jd_off,
                                                            int32_t *__restrict__ jd_ptr) {
  __shared__ int32_t s_len[kUnitRows];
  const int64_t r0 = (int64_t)blockIdx.x * kUnitRows;
  const int nb_rows = (int)min((int64_t)kUnitRows, n - r0);
  s_len[threadIdx.x] = threadIdx.x < nb_rows ? jds_len[r0 + threadIdx.x] : 0;
  __syncthreads();
  const int64_t o = jd_off[blockIdx.x];
  const int W1 = (int)(jd_off[blockIdx.x + 1] - o);
  for (int k = threadIdx.x; k < W1; k += kUnitRows) {
    int s = 0;
    for (int q = 0; q < nb_rows; ++q) s += min(s_len[q], k);
    jd_ptr[o + k] = s;
  }
}

// phase 3: scatter entries: (p, k) -> blk_off[b] + jd_ptr_b[k] + p.
__global__ void __launch_bounds__(kUnitRows) jds_fill_kernel(const int32_t *__restrict__ rp,
                                                             const int32_t *__restrict__ col,
                                                             const float *__restrict__ val, int64_t n,
                                                             const int32_t *__restrict__ perm,
                                                             const int64_t *__restrict__ jd_off,
                                                             const int32_t *__restrict__ jd_ptr,
                                                             int64_t *__restrict__ blk_off,
                                                             int32_t *__restrict__ jc, float *__restrict__ jv) {
  const int64_t r0 = (int64_t)blockIdx.x * kUnitRows;
  const int p = threadIdx.x;
  const int64_t bo = rp[r0];
  if (p == 0) blk_off[blockIdx.x] = bo;
  if (r0 + p >= n) return;
  const int g = perm[r0 + p];
  const int b = rp[g], e = rp[g + 1];
  const int32_t *jp = jd_ptr + jd_off[blockIdx.x];
  for (int k = 0; k < e - b; ++k) {
    const int64_t idx = bo + jp[k] + p;
    jc[idx] = col[b + k];
    jv[idx] = val[b + k];
  }
}

// ================================================================ host side
template <int VID>
static dysel_status spmv_variant_fn(const dysel_slice *s, void *const *args, void *stream, void *user);

}  // namespace dysel

struct dysel_spmv_plan {
  dysel_ctx *ctx = nullptr;
  dysel::SpmvDev dev{};
  dysel_spmv_plan_info info{};
  int32_t *ell_col = nullptr;
  float *ell_val = nullptr;
  int32_t *perm = nullptr, *jds_len = nullptr, *jd_ptr = nullptr, *jds_col = nullptr;
  int64_t *blk_off = nullptr, *jd_off = nullptr;
  float *jds_val = nullptr;
  int K = 0;            // pool size
  int vids[DYSEL_SPMV_NVARIANTS] = {};
  int def = 0;          // pool index of default
  uint32_t n_units = 0;
  std::string sig;      // generic-registry signature (host path)
  int persist_grid = 0;
};

namespace dysel {

template <int VID>
static dysel_status spmv_variant_fn(const dysel_slice *s, void *const *args, void *stream, void *user) {
  dysel_spmv_plan *pl = (dysel_spmv_plan *)user;
  if (s->granule_count == 0) return DYSEL_OK;
  SpmvDev A = pl->dev;
  A.x = (const float *)args[1];
  spmv_slice_kernel<VID><<<(unsigned)s->granule_count, kUnitRows, 0, (cudaStream_t)stream>>>(A, (float *)args[0], *s,
                                                                                            nullptr);
  return cudaGetLastError() == cudaSuccess ? DYSEL_OK : DYSEL_ERR_CUDA;
}

static dysel_variant_fn kVariantFns[DYSEL_SPMV_NVARIANTS] = {spmv_variant_fn<0>, spmv_variant_fn<1>, spmv_variant_fn<2>,
                                                             spmv_variant_fn<3>, spmv_variant_fn<4>};
static const char *kVariantNames[DYSEL_SPMV_NVARIANTS] = {"csr_scalar", "csr_vector", "ell", "jds", "csr_stream"};

dysel_status spmv_ctx_init(dysel_ctx *ctx) {
  if (cudaMalloc(&ctx->d_spmv_state, sizeof(SpmvStateBlock)) != cudaSuccess) return DYSEL_ERR_NOMEM;
  if (cudaMallocHost(&ctx->h_spmv_rep, sizeof(SpmvState)) != cudaSuccess) return DYSEL_ERR_NOMEM;
  spmv_state_reset_kernel<<<1, 32>>>((SpmvStateBlock *)ctx->d_spmv_state);
  if (cudaDeviceSynchronize() != cudaSuccess) return DYSEL_ERR_CUDA;
  return DYSEL_OK;
}

void spmv_ctx_free(dysel_ctx *ctx) {
  if (ctx->d_spmv_state) cudaFree(ctx->d_spmv_state);
  if (ctx->h_spmv_rep) cudaFreeHost(ctx->h_spmv_rep);
  ctx->d_spmv_state = nullptr;
  ctx->h_spmv_rep = nullptr;
}

static int pool_index(const dysel_spmv_plan *pl, int vid) {
  for (int i = 0; i < pl->K; ++i)
    if (pl->vids[i] == vid) return i;
  return -1;
}

static dysel_status launch_variant_full(dysel_ctx *ctx, dysel_spmv_plan *pl, int vid, const float *x, float *y,
                                        cudaStream_t st) {
  if (pl->n_units == 0) return DYSEL_OK;
  dysel_slice s;
  memset(&s, 0, sizeof(s));
  s.granule_count = pl->n_units;
  s.granule_stride = 1;
  s.g[0] = s.g[1] = s.g[2] = 1;
  s.G[0] = pl->n_units;
  s.G[1] = s.G[2] = 1;
  s.U[0] = pl->n_units;
  s.U[1] = s.U[2] = 1;
  s.role = DYSEL_ROLE_BATCH;
  s.variant = vid;
  void *args[2] = {y, (void *)x};
  DYSEL_TRY(kVariantFns[vid](&s, args, st, pl));
  return check_launch(ctx, "spmv full-grid variant");
}

}  // namespace dysel

using namespace dysel;

extern "C" {

dysel_status dysel_spmv_prepare(dysel_ctx *ctx, int64_t n_rows, int64_t n_cols, int64_t nnz, const int32_t *d_row_ptr,
                                const int32_t *d_col, const float *d_val, uint32_t formats_mask, int default_variant,
                                void *stream, dysel_spmv_plan **out) {
  if (!ctx || !out || n_rows < 0 || n_cols < 0 || nnz < 0 || nnz >= (1ll << 31) || n_rows >= (1ll << 31) ||
      n_cols >= (1ll << 31) || (n_rows > 0 && !d_row_ptr) || (nnz > 0 && (!d_col || !d_val)) ||
      default_variant < 0 || default_variant >= DYSEL_SPMV_NVARIANTS) {
    set_error(ctx, "dysel_spmv_prepare: invalid arguments");
    return DYSEL_ERR_INVALID;
  }
  *out = nullptr;
  cudaStream_t st = (cudaStream_t)stream;
  const uint64_t t0 = now_ns();
  dysel_spmv_plan *pl = new dysel_spmv_plan();
  pl->ctx = ctx;
  auto fail = [&](dysel_status s) {
    dysel_spmv_plan_destroy(pl);
    return s;
  };
  SpmvDev &A = pl->dev;
  A.n_rows = (int32_t)n_rows;
  A.n_cols = (int32_t)n_cols;
  A.row_ptr = d_row_ptr;
  A.col = d_col;
  A.val = d_val;
  A.vec_ok = (((uintptr_t)d_col | (uintptr_t)d_val) & 15) == 0;
  pl->n_units = (uint32_t)((n_rows + kUnitRows - 1) / kUnitRows);
  const int64_t n_pad = (int64_t)pl->n_units * kUnitRows;
  A.n_pad = n_pad;
  dysel_spmv_plan_info &I = pl->info;
  I.n_rows = n_rows;
  I.n_cols = n_cols;
  I.nnz = nnz;
  // row statistics: W, uniformity (A-13), ELL applicability (A-15)
  int32_t W = 0;
  if (n_rows > 0) {
    int32_t *d_w = nullptr;
    if (cudaMalloc(&d_w, sizeof(int32_t)) != cudaSuccess) return fail(DYSEL_ERR_NOMEM);
    cudaMemsetAsync(d_w, 0, sizeof(int32_t), st);
    row_stats_kernel<<<4 * ctx->n_sm, 256, 0, st>>>(d_row_ptr, n_rows, d_w);
    dysel_status s = check_launch(ctx, "row_stats_kernel");
    if (s == DYSEL_OK && cudaMemcpyAsync(&W, d_w, sizeof(int32_t), cudaMemcpyDeviceToHost, st) != cudaSuccess)
      s = DYSEL_ERR_CUDA;
    if (s == DYSEL_OK && cudaStreamSynchronize(st) != cudaSuccess) s = DYSEL_ERR_CUDA;
    cudaFree(d_w);
    if (s != DYSEL_OK) return fail(s);
  }
  I.max_row_len = W;
  I.uniform = (n_rows == 0 || nnz == 0) ? 1 : ((int64_t)W * n_rows <= 2 * nnz);
  const bool ell_ok = (int64_t)W * n_rows <= 4 * std::max<int64_t>(nnz, 1);
  pl->K = 0;
  pl->vids[pl->K++] = DYSEL_SPMV_CSR_SCALAR;
  pl->vids[pl->K++] = DYSEL_SPMV_CSR_VECTOR;
  if ((formats_mask & DYSEL_FMT_ELL) && ell_ok && n_rows > 0) {
    size_t slots = (size_t)W * n_pad;
    if (slots > 0) {
      if (cudaMalloc(&pl->ell_col, slots * 4) != cudaSuccess || cudaMalloc(&pl->ell_val, slots * 4) != cudaSuccess)
        return fail(DYSEL_ERR_NOMEM);
      cudaMemsetAsync(pl->ell_col, 0xff, slots * 4, st);
      cudaMemsetAsync(pl->ell_val, 0, slots * 4, st);
      ell_fill_kernel<<<(unsigned)((n_rows + 255) / 256), 256, 0, st>>>(d_row_ptr, d_col, d_val, n_rows, n_pad,
                                                                       pl->ell_col, pl->ell_val);
      if (check_launch(ctx, "ell_fill_kernel") != DYSEL_OK) return fail(DYSEL_ERR_CUDA);
    }
    A.ell_W = W;
    A.ell_col = pl->ell_col;
    A.ell_val = pl->ell_val;
    I.ell_width = W;
    I.ell_bytes = slots * 8;
    pl->vids[pl->K++] = DYSEL_SPMV_ELL;
  }
  if ((formats_mask & DYSEL_FMT_JDS) && n_rows > 0) {
    const int64_t nb = pl->n_units;
    int64_t *wp1 = nullptr;
    void *tmp = nullptr;
    size_t tmp_bytes = 0;
    if (cudaMalloc(&pl->perm, n_rows * 4) != cudaSuccess || cudaMalloc(&pl->jds_len, n_rows * 4) != cudaSuccess ||
        cudaMalloc(&pl->blk_off, (nb + 1) * 8) != cudaSuccess || cudaMalloc(&pl->jd_off, (nb + 1) * 8) != cudaSuccess ||
        cudaMalloc(&wp1, (nb + 1) * 8) != cudaSuccess)
      return fail(DYSEL_ERR_NOMEM);
    if (nnz > 0 && (cudaMalloc(&pl->jds_col, nnz * 4) != cudaSuccess || cudaMalloc(&pl->jds_val, nnz * 4) != cudaSuccess))
      return fail(DYSEL_ERR_NOMEM);
    cudaMemsetAsync(wp1 + nb, 0, 8, st);
    jds_sort_kernel<<<(unsigned)nb, kUnitRows, 0, st>>>(d_row_ptr, n_rows, pl->perm, pl->jds_len, wp1);
    if (check_launch(ctx, "jds_sort_kernel") != DYSEL_OK) return fail(DYSEL_ERR_CUDA);
    cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, wp1, pl->jd_off, nb + 1, st);
    if (cudaMalloc(&tmp, tmp_bytes) != cudaSuccess) return fail(DYSEL_ERR_NOMEM);
    cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, wp1, pl->jd_off, nb + 1, st);
    int64_t total = 0;
    cudaMemcpyAsync(&total, pl->jd_off + nb, 8, cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) {
      cudaFree(tmp);
      cudaFree(wp1);
      return fail(DYSEL_ERR_CUDA);
    }
    cudaFree(tmp);
    cudaFree(wp1);
    if (cudaMalloc(&pl->jd_ptr, std::max<int64_t>(total, 1) * 4) != cudaSuccess) return fail(DYSEL_ERR_NOMEM);
    jds_ptr_kernel<<<(unsigned)nb, kUnitRows, 0, st>>>(pl->jds_len, n_rows, pl->jd_off, pl->jd_ptr);
    if (check_launch(ctx, "jds_ptr_kernel") != DYSEL_OK) return fail(DYSEL_ERR_CUDA);
    jds_fill_kernel<<<(unsigned)nb, kUnitRows, 0, st>>>(d_row_ptr, d_col, d_val, n_rows, pl->perm, pl->jd_off,
                                                       pl->jd_ptr, pl->blk_off, pl->jds_col, pl->jds_val);
    if (check_launch(ctx, "jds_fill_kernel") != DYSEL_OK) return fail(DYSEL_ERR_CUDA);
    cudaMemcpyAsync(pl->blk_off + nb, &nnz, 8, cudaMemcpyHostToDevice, st);
    A.perm = pl->perm;
    A.jds_len = pl->jds_len;
    A.blk_off = pl->blk_off;
    A.jd_off = pl->jd_off;
    A.jd_ptr = pl->jd_ptr;
    A.jds_col = pl->jds_col;
    A.jds_val = pl->jds_val;
    I.jds_bytes = (size_t)n_rows * 8 + (size_t)(nb + 1) * 16 + (size_t)total * 4 + (size_t)nnz * 8;
    pl->vids[pl->K++] = DYSEL_SPMV_JDS;
  }
  if (formats_mask & DYSEL_FMT_STREAM) pl->vids[pl->K++] = DYSEL_SPMV_CSR_STREAM;
  if (cudaStreamSynchronize(st) != cudaSuccess) return fail(DYSEL_ERR_CUDA);
  pl->def = pool_index(pl, default_variant);
  if (pl->def < 0) {
    set_error(ctx, "dysel_spmv_prepare: default variant not in the pool (ELL inapplicable? A-15)");
    return fail(DYSEL_ERR_UNSUPPORTED);
  }
  I.n_variants = pl->K;
  for (int i = 0; i < pl->K; ++i) I.variant_ids[i] = pl->vids[i];
  I.prep_ns = now_ns() - t0;
  // register the pool for the generic (host-orchestrated) path
  pl->sig = "dysel.spmv#" + std::to_string(++ctx->plan_serial);
  static const int sb[1] = {0};
  dysel_variant vv[DYSEL_SPMV_NVARIANTS];
  for (int i = 0; i < pl->K; ++i)
    vv[i] = dysel_variant{kVariantNames[pl->vids[i]], kVariantFns[pl->vids[i]], {1, 1, 1}, sb, 1,
                          I.uniform ? 0u : (uint32_t)DYSEL_V_NONUNIFORM, pl};
  dysel_status rs = dysel_register_variants(ctx, pl->sig.c_str(), vv, pl->K, pl->def);
  if (rs != DYSEL_OK) return fail(rs);
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, spmv_persistent_kernel, kUnitRows, 0);
  pl->persist_grid = std::max(1, occ) * ctx->n_sm;
  *out = pl;
  return DYSEL_OK;
}

dysel_status dysel_spmv_plan_get_info(const dysel_spmv_plan *pl, dysel_spmv_plan_info *info) {
  if (!pl || !info) return DYSEL_ERR_INVALID;
  *info = pl->info;
  return DYSEL_OK;
}

dysel_status dysel_spmv_plan_copy_array(const dysel_spmv_plan *pl, int which, void *dst, size_t *bytes) {
  if (!pl || !bytes) return DYSEL_ERR_INVALID;
  const int64_t n = pl->info.n_rows, nnz = pl->info.nnz, nb = pl->n_units;
  const void *src = nullptr;
  size_t sz = 0;
  int64_t jd_total = 0;
  if (which == 6 && pl->jd_off) cudaMemcpy(&jd_total, pl->jd_off + nb, 8, cudaMemcpyDeviceToHost);
  switch (which) {
    case 0: src = pl->ell_col; sz = (size_t)pl->dev.ell_W * pl->dev.n_pad * 4; break;
    case 1: src = pl->ell_val; sz = (size_t)pl->dev.ell_W * pl->dev.n_pad * 4; break;
    case 2: src = pl->perm; sz = (size_t)n * 4; break;
    case 3: src = pl->jds_len; sz = (size_t)n * 4; break;
    case 4: src = pl->blk_off; sz = (size_t)(nb + 1) * 8; break;
    case 5: src = pl->jd_off; sz = (size_t)(nb + 1) * 8; break;
    case 6: src = pl->jd_ptr; sz = (size_t)jd_total * 4; break;
    case 7: src = pl->jds_col; sz = (size_t)nnz * 4; break;
    case 8: src = pl->jds_val; sz = (size_t)nnz * 4; break;
    default: return DYSEL_ERR_INVALID;
  }
  const bool has = (which <= 1) ? pl->info.ell_width > 0 || pool_index(pl, DYSEL_SPMV_ELL) >= 0
                                : pool_index(pl, DYSEL_SPMV_JDS) >= 0;
  if (!has) return DYSEL_ERR_NOT_FOUND;
  if (!dst) {
    *bytes = sz;
    return DYSEL_OK;
  }
  if (*bytes < sz) return DYSEL_ERR_INVALID;
  *bytes = sz;
  if (sz && src && cudaMemcpy(dst, src, sz, cudaMemcpyDeviceToHost) != cudaSuccess) return DYSEL_ERR_CUDA;
  return DYSEL_OK;
}

void dysel_spmv_plan_destroy(dysel_spmv_plan *pl) {
  if (!pl) return;
  if (pl->ctx) {
    cudaSetDevice(pl->ctx->device);
    cudaDeviceSynchronize();
    if (!pl->sig.empty()) {
      pl->ctx->reg.erase(pl->sig);
      pl->ctx->sel_cache.erase(pl->sig);
    }
  }
  cudaFree(pl->ell_col);
  cudaFree(pl->ell_val);
  cudaFree(pl->perm);
  cudaFree(pl->jds_len);
  cudaFree(pl->jd_ptr);
  cudaFree(pl->jds_col);
  cudaFree(pl->jds_val);
  cudaFree(pl->blk_off);
  cudaFree(pl->jd_off);
  cudaGetLastError();
  delete pl;
}

dysel_status dysel_spmv_variant(dysel_ctx *ctx, dysel_spmv_plan *pl, int variant_id, const float *d_x, float *d_y,
                                void *stream) {
  if (!ctx || !pl || (pl->dev.n_rows > 0 && (!d_y || (pl->dev.n_cols > 0 && !d_x))) || pool_index(pl, variant_id) < 0) {
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
  if (rep) rep->n_slices = 0;
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
  // device path: plan (same rules as the generic launcher) + one persistent launch
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
  if (rep) {
    rep->mode_used = P.mode | (int)(mode & DYSEL_ASYNC);
    rep->profiled = P.active ? 1 : 0;
    rep->n_variants = pl->K;
    rep->c = P.c;
    rep->n_granules = P.Gn;
    rep->eager_units = 0;
    rep->tail_units = 0;
    for (int v = 0; v < DYSEL_MAX_VARIANTS; ++v)
      rep->score[v] = rep->makespan_ns[v] = rep->units[v] = rep->cycles[v] = rep->busy_ns[v] = rep->aborted[v] = 0;
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
  DispatchParams p;
  memset(&p, 0, sizeof(p));
  p.K = (uint32_t)pl->K;
  p.c = (uint32_t)P.c;
  p.n_units = pl->n_units;
  p.hybrid = P.mode == DYSEL_HYBRID;
  p.async = (mode & DYSEL_ASYNC) != 0;
  p.contiguous = (mode & DYSEL_CONTIGUOUS) != 0;
  p.score_mode = (mode & DYSEL_SCORE_CYCLES) ? 1u : ((mode & DYSEL_SCORE_MAKESPAN) ? 2u : 0u);
  p.def = (uint32_t)pl->def;
  p.tail = (mode & DYSEL_NO_TAIL) ? 0u : 1u;
  p.abort = (mode & DYSEL_NO_ABORT) ? 0u : 1u;
  p.n_tickets = (uint32_t)(P.Gn + (p.hybrid ? (uint64_t)(pl->K - 1) * P.c : 0));
  for (int i = 0; i < pl->K; ++i) p.vids[i] = pl->vids[i];
  if (p.hybrid) {
    DYSEL_TRY(scratch(ctx, ctx->sandbox[0], (size_t)(pl->K - 1) * P.c * kUnitRows * sizeof(float)));
    p.sandbox = (float *)ctx->sandbox[0].ptr;
  }
  p.unit_variant = d_uv;
  SpmvDev A = pl->dev;
  A.x = d_x;
  // sync + tail: the dispatcher only runs the K*c profiling tickets
  const uint64_t work = (p.tail && !p.async) ? (uint64_t)p.K * p.c : p.n_tickets;
  const int grid = (int)std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)pl->persist_grid, work));
  SpmvStateBlock *sb = (SpmvStateBlock *)ctx->d_spmv_state;
  spmv_persistent_kernel<<<grid, kUnitRows, 0, st>>>(A, d_y, sb, p);
  DYSEL_TRY(check_launch(ctx, "spmv_persistent_kernel"));
  DYSEL_TRY(push_pending_sel(ctx, pl->sig, &sb->rep.sel, st));
  if (rep) {
    SpmvState *h = (SpmvState *)ctx->h_spmv_rep;
    DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(h, &sb->rep, sizeof(SpmvState), cudaMemcpyDeviceToHost, st));
    if (d_uv && rep->unit_variant)
      DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(rep->unit_variant, d_uv, std::min<uint64_t>(P.Gn, rep->unit_variant_cap),
                                          cudaMemcpyDeviceToHost, st));
    DYSEL_CUDA_TRY(ctx, cudaStreamSynchronize(st));
    const int sel_pool = (int)(h->sel & 0xff);
    rep->selected = sel_pool < pl->K ? pl->vids[sel_pool] : -1;
    rep->eager_units = h->eager_units;
    rep->tail_units = h->tail_begin != ~0ull ? pl->n_units - h->tail_begin : 0;
    for (int v = 0; v < pl->K; ++v) {
      const int id = pl->vids[v];
      const dysel_timer_slot &t = h->slot[v];
      rep->busy_ns[id] = h->busy[v];
      rep->aborted[id] = h->aborted[v];
      rep->makespan_ns[id] = t.t_end_max - t.t_start_min;
      rep->units[id] = t.units;
      rep->cycles[id] = t.cycles;
      const uint64_t cap = (1ull << 56) - 1;
      rep->score[id] = h->dominated[v] ? cap
                       : p.score_mode == 1 ? (t.units ? t.cycles / t.units : cap)
                       : p.score_mode == 2 ? rep->makespan_ns[id]
                                           : (t.units ? h->busy[v] / t.units : cap);
    }
    if (sel_pool < pl->K) ctx->sel_cache[pl->sig] = sel_pool;
    rep->host_ns = now_ns() - t_host0;
  }
  return DYSEL_OK;
}

}  // extern "C"
