/*
 * dysel.h — C ABI of libdysel.so, a B200-native (sm_100a) implementation of
 * DySel's data-parallel hot path: micro-profiled dynamic selection among
 * candidate kernel variants (Chang, Kim, Hwu, ASPLOS '16).
 *
 * Citations are PAPER.md line numbers (P:L<a>-<b>) with section / figure /
 * table.  Readings of ambiguous passages are numbered A-<n> and listed in
 * DESIGN.md §Readings.
 *
 * The method (§2.1, §2.2): K variants of one
 * data-parallel kernel each run on a small slice of the real work-groups
 * ("micro-profiling"), each slice writes its part of the final output
 * ("productive profiling"), the slices are timed on the device
 * (§3.3, Fig. 7), the fastest variant is selected and the rest of
 * the NDRange is launched with it (§2.4).
 *
 * Conventions for every call below
 *   - Pointers named d_* are DEVICE pointers, caller-owned (normally torch
 *     tensors).  The library never frees them and never keeps them after the
 *     call returns, except the CSR arrays a dysel_spmv_plan refers to (the
 *     caller must keep them alive until dysel_spmv_plan_destroy).
 *   - `stream` is a cudaStream_t passed as void*; NULL = the legacy default
 *     stream.  All device work is stream-ordered on it.  Profiling streams fork
 *     from and join back to it through events.  Device-path calls never block
 *     the host; DYSEL_HOST_ORCH calls block inside the call (as the paper's
 *     cudaDeviceSynchronize did).
 *   - Every call returns a dysel_status and never aborts or throws; CUDA /
 *     NCCL failures return DYSEL_ERR_CUDA / DYSEL_ERR_NCCL with the message in
 *     dysel_last_error(ctx).
 *   - A dysel_ctx is bound to one device and is NOT thread-safe; use one ctx
 *     per host thread, and do not run two launches of one ctx concurrently on
 *     different streams (they share the ctx's timer / ticket state).
 */
#ifndef DYSEL_H_
#define DYSEL_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ------------------------------------------------------------------ status */
typedef enum {
  DYSEL_OK = 0,
  DYSEL_ERR_INVALID = 1,     /* NULL pointer, bad size, f not in [0,1], unknown sig, n not in [1,16], wa = 0 */
  DYSEL_ERR_UNSUPPORTED = 2, /* SWAP|ASYNC (Table 1), ELL over the cap (A-15), ... */
  DYSEL_ERR_NOMEM = 3,
  DYSEL_ERR_CUDA = 4,
  DYSEL_ERR_NOT_FOUND = 5,   /* no cached selection for the key */
  DYSEL_ERR_NCCL = 6
} dysel_status;

const char *dysel_status_str(dysel_status s);

/* ------------------------------------------------------------------- modes
 * Low two bits: productive-profiling mode (§2.2, Table 1).
 *   FULLY  — each variant runs a disjoint slice and writes the final output.
 *   HYBRID — all variants run the same slice; only default_variant writes the
 *            output, the others write sandboxes (≤ K-1 extra, A-4).
 *   SWAP   — each variant writes a private full output; the winner's is
 *            swapped in; synchronous only.
 *   AUTO   — resolved from variant flags: any DYSEL_V_ATOMICS -> SWAP, any
 *            DYSEL_V_NONUNIFORM -> HYBRID, else FULLY (replaces the compiler's
 *            side-effect / uniform-workload analyses, §3.4; A-10,
 *            A-11, A-13).  Explicit bits are a programmer override
 *            (P:L974-975).
 * Orchestration (§2.4): SYNC waits for all profiling slices before
 * the remainder; ASYNC starts the remainder at once with the best variant so
 * far ("eager execution"), default_variant first.
 * Default = DYSEL_FULLY | DYSEL_ASYNC ("mode=fully_async", Fig. 6b).
 */
#define DYSEL_FULLY 0u
#define DYSEL_HYBRID 1u
#define DYSEL_SWAP 2u
#define DYSEL_AUTO 3u
#define DYSEL_SYNC 0u
#define DYSEL_ASYNC 4u
#define DYSEL_NO_PROFILE 8u     /* profiling activation flag = false: cached or default variant, plain full grid */
#define DYSEL_HOST_ORCH 16u     /* paper-faithful host orchestration: streams + host sync / polling */
#define DYSEL_FORCE_PROFILE 32u /* ignore the small-workload deactivation (< 128 CTAs); ablation */
#define DYSEL_CONTIGUOUS 64u    /* fully mode: contiguous per-variant slices instead of interleaved granules (A-24) */
#define DYSEL_SCORE_CYCLES 128u /* score = sum of per-CTA clock64 cycles / units (A-6) */
#define DYSEL_SCORE_MAKESPAN 256u /* score = latest CTA end - earliest CTA start (%globaltimer), Fig. 7b */
#define DYSEL_NO_ABORT 1024u    /* no dominance: never stop dominated sandbox units early (SpMV, A-26) nor decide
                                   a variant before its profiling CTAs finish (generic launcher, A-32) */
#define DYSEL_SEQUENTIAL 2048u  /* SpMV device path: profile the variants one after another, each alone on the
                                   GPU (default variant first), scored by makespan (reading A-23) */
/* Default score: generic launcher = makespan (variants are separate concurrent
 * grids, Fig. 7b); SpMV dispatcher = mean per-unit busy time (%globaltimer end -
 * start of each profiled unit; all variants share one launch and occupancy). */
#define DYSEL_DEFAULT_MODE (DYSEL_FULLY | DYSEL_ASYNC)

/* variant flags (replace the compiler analyses, A-10/A-11) */
#define DYSEL_V_ATOMICS 1u     /* global atomics / overlapping outputs -> SWAP */
#define DYSEL_V_NONUNIFORM 2u  /* data-dependent loop bounds -> HYBRID */

/* roles of a slice — the paper's three extended copies of each variant
 * (profiling / batch / eager, §3.3) folded into one parameter */
enum {
  DYSEL_ROLE_PRODUCTIVE = 0, /* profiling copy writing the real output */
  DYSEL_ROLE_SANDBOX = 1,    /* profiling copy writing a sandbox (hybrid) */
  DYSEL_ROLE_BATCH = 2,      /* non-profiling batch copy (remainder, or whole grid when profiling is off) */
  DYSEL_ROLE_PRIVATE = 3,    /* profiling copy writing a private output (swap) */
  DYSEL_ROLE_EAGER = 4       /* async eager chunk of the best-so-far variant */
};

#define DYSEL_MAX_VARIANTS 16

/* ------------------------------------------------------------------ context */
typedef struct dysel_ctx dysel_ctx;

/* Create a context on CUDA device `cuda_device` (calls cudaSetDevice).  Owns
 * its scratch (timer slots, selection words, tickets, sandboxes), streams and
 * events.  Queries #SM (cudaDevAttrMultiProcessorCount) and calibrates the
 * %globaltimer resolution (A-6). */
dysel_status dysel_create(int cuda_device, dysel_ctx **out);
void dysel_destroy(dysel_ctx *ctx);
const char *dysel_last_error(const dysel_ctx *ctx);
/* SM count, measured %globaltimer tick (ns) and L2 size of the ctx's device. */
dysel_status dysel_device_info(const dysel_ctx *ctx, int *n_sm, uint64_t *globaltimer_tick_ns,
                               uint64_t *l2_bytes);

/* ------------------------------------------------------------ device timing
 * One per variant, in device memory.  Written by the profiling copies
 * (Fig. 7b): earliest CTA start / latest CTA end (%globaltimer,
 * ns), profiled units, sum over CTAs of (end - start) in clock64 cycles. */
typedef struct {
  uint64_t t_start_min;
  uint64_t t_end_max;
  uint64_t units;
  uint64_t cycles;
} dysel_timer_slot;

/* What one launch of a variant must cover: `granule_count` granules starting
 * at linear granule `granule_begin`, every `granule_stride`-th (interleaved
 * fully mode, A-24).  A granule is g[0]*g[1]*g[2] units (the LCM of the
 * variants' work-assignment factors); granules are numbered x
 * fastest over G[0] x G[1] x G[2]; edge granules may be partial (clip to U).
 * A variant with wa units per CTA launches granule_count * prod(g/wa) CTAs. */
typedef struct {
  uint64_t granule_begin;
  uint64_t granule_count;
  uint64_t granule_stride;
  uint32_t g[3];
  uint32_t G[3];
  uint64_t U[3];
  int32_t role;
  int32_t variant;
  /* device-side profiling bookkeeping; NULL when the copy is untimed */
  dysel_timer_slot *timer;   /* this variant's slot */
  uint32_t *ctas_done;       /* per-variant count of finished profiling CTAs */
  uint32_t ctas_total;       /* profiling CTAs of this variant */
  uint64_t *best;            /* packed (score<<8 | v), atomicMin'd when a variant completes */
  uint32_t *variants_done;   /* completed variants; the last one copies *best into *sel */
  uint32_t n_variants;
  uint32_t score_cycles;     /* 1 => score by cycles/units */
  uint32_t occupancy;        /* resident CTAs per SM of this variant (0 = unknown); when set and
                                score_cycles == 0 the score is sum(CTA clock64 cycles) * 64 /
                                (units * occupancy): time per unit per execution slot (A-6) */
  uint64_t *sel;             /* final packed selection (~0 until profiling completes) */
  /* gated batch: when non-NULL the copy runs only if (*gate & 0xff) == variant */
  const uint64_t *gate;
  /* dominance (reading A-32; NULL = off): a running variant whose lower-bound
   * score already exceeds the best completed score cannot win, so it is
   * decided (maximal score) without waiting for its CTAs; its sandbox CTAs
   * may stop (dysel_prof_poll).  lb = running sum of the variant's CTA
   * clock64 cycles (each CTA adds its elapsed cycles when it polls);
   * decided = 0 running, 1 completed, 2 dominated (set once, by CAS);
   * units_total = units of the variant's profiling slice. */
  uint64_t *lb;
  uint32_t *decided;
  uint64_t units_total;
  /* wave-quantised score (reading A-34; used when both are non-zero and
   * score_cycles == 0): predicted full-grid time of the variant =
   * ceil(grid_ctas / wave_ctas) waves x mean cycles per full CTA
   * (= sum cycles x units_per_cta / units) */
  uint64_t grid_ctas;        /* CTAs of the variant's full grid (G_n x CTAs per granule) */
  uint64_t wave_ctas;        /* CTAs resident at once (occupancy x #SM) */
  uint32_t units_per_cta;    /* wa[0] x wa[1] x wa[2] */
  /* gated batch hint: 1 = the launcher expects this copy to win (the default
   * variant's, launched first at high priority): launch the full grid (the
   * block scheduler balances it); 0 = a variant that will most likely exit at
   * the gate: one wave of CTAs walking the slice is enough */
  uint32_t gate_full_grid;
} dysel_slice;

/* A variant = a host function that launches its kernel(s) over a slice on
 * `stream` (a cudaStream_t).  args are the dysel_launch args with sandbox /
 * private-output substitutions applied; `user` is dysel_variant.user.  Every
 * CTA of a timed launch (s->timer != NULL) must call dysel_prof_begin/end
 * exactly once, also CTAs whose tile is out of range (units = 0).
 * Device-side helpers for slice mapping and timing are in dysel_device.cuh. */
typedef dysel_status (*dysel_variant_fn)(const dysel_slice *s, void *const *args, void *stream, void *user);

typedef struct {
  const char *name;
  dysel_variant_fn fn;
  uint32_t wa[3];            /* work-assignment factor: units per CTA per dim */
  const int *sandbox_args;   /* indices into args[] of output pointers to redirect */
  int n_sandbox_args;
  uint32_t flags;            /* DYSEL_V_* */
  void *user;                /* passed to fn */
  uint64_t ctas_per_wave;    /* optional: CTAs of this variant resident at once on the device
                                (occupancy x #SM); 0 = unknown.  When the default variant's full
                                grid fits in one wave, profiling is off (reading A-3b). */
} dysel_variant;

/* Register K = n variants under kernel_sig (DySelAddKernel, Fig. 6a
 * P:L761-767).  default_variant is the "initial version" async mode starts
 * with (A-5) and the productive variant in hybrid mode (A-4).
 * Re-registering a sig replaces it and clears its cached selection. */
dysel_status dysel_register_variants(dysel_ctx *ctx, const char *kernel_sig, const dysel_variant *v,
                                     int n, int default_variant);

/* ------------------------------------------------------------------ report */
typedef struct {
  uint64_t granule_begin, granule_count, granule_stride;
  int32_t variant, role;
} dysel_slice_rec;

typedef struct {
  int32_t mode_used;        /* resolved FULLY/HYBRID/SWAP | ASYNC bit */
  int32_t profiled;         /* 1 if profiling ran */
  int32_t selected;         /* variant used for the remainder (final selection) */
  int32_t n_variants;
  uint64_t c;               /* granules per profiling slice */
  uint64_t n_granules;      /* G_n */
  uint64_t score[DYSEL_MAX_VARIANTS];   /* ns (makespan) or cycles/unit */
  uint64_t makespan_ns[DYSEL_MAX_VARIANTS];
  uint64_t units[DYSEL_MAX_VARIANTS];
  uint64_t cycles[DYSEL_MAX_VARIANTS];
  uint64_t busy_ns[DYSEL_MAX_VARIANTS];   /* sum of per-unit busy time (SpMV dispatcher) */
  uint64_t aborted[DYSEL_MAX_VARIANTS];   /* sandbox units stopped / skipped by dominance */
  uint64_t tail_units;      /* remainder units run by the tail-launched plain kernel */
  uint64_t eager_units;     /* remainder units run before the final selection (async) */
  uint64_t host_ns;         /* host time inside the call */
  dysel_slice_rec *slices;  /* optional caller array */
  int32_t slices_cap, n_slices;
  uint8_t *unit_variant;    /* optional caller HOST array, one byte per granule: variant that
                               productively computed it (debug / c-6 tests; costs a D2H copy + sync) */
  uint64_t unit_variant_cap;
  /* Filled only when a report is requested (diagnostics); ~0 = did not happen.
   * SpMV device path: ns since the first profiling CTA started -- [0] 0, [1]
   * selection published, [2] last profiling CTA ended, [3] first eager CTA
   * started, [4] last eager CTA ended, [5] first remainder CTA started, [6]
   * last remainder CTA ended, [7] longest profiling unit (ns).
   * Generic launcher (dysel_launch, SGEMM, stencil, f-2 pools): ns since the
   * call's init kernel -- [0] first profiling CTA started, [1] selection
   * published (%globaltimer); event-timed: [2] selection known on the gate
   * stream, [3] the default's gated remainder done, [4] every gated remainder
   * done, [5] every profiling copy done, [6] the call done. */
  uint64_t timeline_ns[8];
  /* Table 1 allocation record of this launch: extra output
   * buffers the profiling slices wrote instead of the real output, and their
   * bytes.  FULLY: 0.  HYBRID: K-1 slice-sized sandboxes (the default's
   * slice is productive, A-4).  SWAP: K full private outputs. */
  uint32_t sandbox_buffers;
  uint32_t pad_;
  uint64_t sandbox_bytes;
} dysel_report;

/* Launch kernel_sig over an NDRange of ndrange_units[3] units
 * (DySelLaunchKernel, Fig. 6b).  profile_fraction f in [0,1]: each
 * variant profiles c = floor(f * G_n / K) granules (A-1, rounding A-2);
 * profiling is off when c = 0, when the default variant's full grid has < 128
 * CTAs (A-3), with DYSEL_NO_PROFILE (activation flag, P:L796-804:
 * the cached selection or the default runs the whole grid), or for K = 1.
 * args[0..n_args) are passed to the variant functions (device pointers or
 * pointers to host scalars; the library only replaces sandbox entries).
 * sandbox_arg_bytes[i] gives the size of args[sandbox_args[i]] (hybrid
 * sandboxes / swap private outputs are allocated in the ctx).  On success the
 * selection is cached under kernel_sig (A-22).  rep may be NULL. */
dysel_status dysel_launch(dysel_ctx *ctx, const char *kernel_sig, const uint64_t ndrange_units[3],
                          float profile_fraction, uint32_t mode, void *const *args, int n_args,
                          const size_t *sandbox_arg_bytes, void *stream, dysel_report *rep);

/* Selection cache (profiling activation flag; key A-22). */
dysel_status dysel_get_selection(dysel_ctx *ctx, const char *key, int *variant);
dysel_status dysel_set_selection(dysel_ctx *ctx, const char *key, int variant);
dysel_status dysel_reset_selection(dysel_ctx *ctx, const char *key); /* NULL key: all */

/* ------------------------------------------------------------------- SpMV
 * y = A x (overwrite), fp32 CSR input (SHOC spmv-csr / Parboil spmv-jds,
 * P:L1128-1131).  Unit = 256 consecutive original rows.
 * Built-in variants (ids): 0 CSR-scalar (thread per row), 1 CSR-vector (warp
 * per row), 2 ELL (column-major, padded), 3 block-local JDS (A-14), 4 CSR-W
 * (warp-streaming CSR with a warp-level segmented reduction; B200 addition),
 * 5 CSR-T (CSR-S with each warp's nonzeros staged in shared memory by the
 * bulk-copy / TMA engine; data-placement variant). */
enum { DYSEL_SPMV_CSR_SCALAR = 0, DYSEL_SPMV_CSR_VECTOR = 1, DYSEL_SPMV_ELL = 2, DYSEL_SPMV_JDS = 3,
       DYSEL_SPMV_CSR_STREAM = 4, DYSEL_SPMV_CSR_TMA = 5, DYSEL_SPMV_NVARIANTS = 6 };
/* default_variant = DYSEL_SPMV_DEFAULT_AUTO: the library picks the initial
 * version from the prepare-time row statistics (reading A-30): uniform rows
 * (A-13) of fewer than 8 entries on average -> CSR-S (A-30c); other uniform
 * rows -> CSR-T when in the pool, the CSR arrays exceed the L2 size and
 * rows hold 8..32 entries (A-30b: an HBM-streaming matrix whose 32-row warp
 * slots suit one bulk copy), else ELL when in the pool; otherwise
 * CSR-W when in the pool, else CSR-V.  The choice is visible in
 * dysel_spmv_plan_info.default_variant. */
#define DYSEL_SPMV_DEFAULT_AUTO (-1)
#define DYSEL_FMT_STREAM 4u   /* include CSR-W in the pool (reads the CSR arrays directly) */
#define DYSEL_FMT_TMA 8u      /* include CSR-T in the pool (reads the CSR arrays directly) */
#define DYSEL_FMT_ELL 1u
#define DYSEL_FMT_JDS 2u

typedef struct dysel_spmv_plan dysel_spmv_plan;

typedef struct {
  int64_t n_rows, n_cols, nnz;
  int32_t n_variants;            /* variants in the pool (ELL dropped when inapplicable, A-15) */
  int32_t variant_ids[DYSEL_SPMV_NVARIANTS]; /* pool index -> DYSEL_SPMV_* id */
  int32_t ell_width;             /* W (0 if no ELL) */
  int32_t uniform;               /* max row length <= 2 * mean (A-13) */
  int32_t max_row_len;
  uint64_t prep_ns;              /* device time of format preparation (a-1) */
  uint64_t ell_bytes, jds_bytes; /* extra device memory held by the plan */
  int32_t default_variant;       /* DYSEL_SPMV_* id of the initial version (resolved when AUTO) */
  int32_t n_heavy;               /* units the winner runs first, nonzeros descending (longest-processing-time
                                    order, A-40): >= max(8192, 4 x mean) nonzeros or a row longer
                                    than max(1024, 8 x mean row) (A-45); 0 when the plan keeps index order */
  int32_t n_light;               /* the other units: the profiling sample and the eager default's range (A-45) */
} dysel_spmv_plan_info;

/* Build the variant pool for one CSR matrix: CSR -> ELL and CSR -> block JDS
 * on the device (a-1).  d_row_ptr int32 [n_rows+1], d_col int32
 * [nnz] (sorted or not), d_val fp32 [nnz]; nnz < 2^31.  formats_mask selects
 * which extra formats to build (DYSEL_FMT_*); ELL is skipped (and absent from
 * the pool) when W * n_rows > 4 * nnz.  default_variant is a DYSEL_SPMV_* id
 * (must be in the pool) or DYSEL_SPMV_DEFAULT_AUTO.  Blocks on `stream` (reads
 * back sizes). */
dysel_status dysel_spmv_prepare(dysel_ctx *ctx, int64_t n_rows, int64_t n_cols, int64_t nnz,
                                const int32_t *d_row_ptr, const int32_t *d_col, const float *d_val,
                                uint32_t formats_mask, int default_variant, void *stream,
                                dysel_spmv_plan **out);
dysel_status dysel_spmv_plan_get_info(const dysel_spmv_plan *plan, dysel_spmv_plan_info *info);
/* Test / debug: copy one of the plan's format arrays (layouts in DESIGN.md
 * §Data layout) to HOST memory, synchronously.  which: 0 ell_col (int32),
 * 1 ell_val (f32), 2 perm (int32), 3 jds_len (int32), 4 blk_off (int64),
 * 5 jd_off (int64), 6 jd_ptr (int32), 7 jds_col (int32), 8 jds_val (f32),
 * 9 unit order seq (int32 [n_units]: light units in index order, then the
 * heavy / long-row units by nonzeros descending; DYSEL_ERR_NOT_FOUND when the
 * plan keeps index order).
 * *bytes: in = capacity of dst, out = size of the array; dst NULL = query.
 * DYSEL_ERR_NOT_FOUND if the plan has no such format. */
dysel_status dysel_spmv_plan_copy_array(const dysel_spmv_plan *plan, int which, void *dst, size_t *bytes);
void dysel_spmv_plan_destroy(dysel_spmv_plan *plan);

/* One DySel SpMV launch: y = A x.  d_x fp32 [n_cols], d_y fp32 [n_rows] (any
 * 4-byte alignment).  Device path (default; SURVEY §8a device protocol):
 * an init kernel, ONE profiling kernel running all K variants' slices (the
 * units seq[0, p_end) of the plan's unit order: light units, A-45), the
 * default variant's claim kernel and a one-warp switch kernel, chained by
 * programmatic dependent launch, no host round trip.  The last profiling CTA
 * publishes the selection on the device.  SYNC: the claim kernel's warps wait
 * for it; ASYNC: they first claim light remainder slots with the default
 * variant (eager execution), then the winner's warps take the
 * heavy / long-row units first and the rest; when a non-default variant won,
 * the switch kernel launches its claim kernel from the device (reading A-42).
 * Hybrid sandbox units of a provably losing variant stop early (dominance,
 * unless DYSEL_NO_ABORT).  With DYSEL_HOST_ORCH: one kernel per variant on
 * forked streams, the host reads the selection, then the remainder kernel
 * (paper-faithful).  Mode AUTO uses the plan's uniformity flag. */
dysel_status dysel_spmv(dysel_ctx *ctx, dysel_spmv_plan *plan, const float *d_x, float *d_y,
                        float profile_fraction, uint32_t mode, void *stream, dysel_report *rep);

/* dysel_spmv with HOST buffers (serving): h_x [n_cols] is copied to the
 * caller's device staging d_x, the DySel SpMV writes d_y [n_rows], and y is
 * copied back to h_y in up to 8 chunks of whole 256-row units
 * (dysel_allgather_chunk layout), each on an internal stream as soon as the
 * SpMV kernels have counted all of its 32-row slots final (a stream
 * wait-value, no SM needed) -- the copy-out overlaps the rest of the SpMV
 * (DYSEL_HOST_ORCH: one copy after it).  h_x / h_y: caller-owned host memory,
 * pinned for asynchronous copies; d_x / d_y: caller-owned device memory.
 * Stream-ordered on `stream`: h_y is complete when `stream` is; nothing
 * blocks the host.  Errors as dysel_spmv. */
dysel_status dysel_spmv_host(dysel_ctx *ctx, dysel_spmv_plan *plan, const float *h_x, float *h_y, float *d_x,
                             float *d_y, float profile_fraction, uint32_t mode, void *stream, dysel_report *rep);

/* One full-grid run of pool variant `variant_id` (a DYSEL_SPMV_* id) with no
 * profiling: the "single pure version" the exhaustive oracle times
 * and what DYSEL_NO_PROFILE runs. */
dysel_status dysel_spmv_variant(dysel_ctx *ctx, dysel_spmv_plan *plan, int variant_id, const float *d_x,
                                float *d_y, void *stream);

/* Measurement only (not part of the method): one launch that generates the
 * memory traffic every CSR SpMV of the plan's matrix must generate -- col / val
 * streamed once (128-bit), x gathered at col (flavour 0) or read sequentially
 * (flavour 1) or gathered by the TMA unit (flavour 2: cp.async.bulk.tensor
 * tile::gather4 into shared memory; flavour 3 = 2 + a check that every
 * gathered value equals x[col], DYSEL_ERR_CUDA if not; flavour 4: a quarter of
 * the chunks through the TMA unit, the rest through the LSU; flavours 2-4 need a
 * 16-byte aligned x and synchronise `stream`), one fma per nonzero, row_ptr read and d_out [n_rows] written
 * once -- with no row structure.  Its duration is the practical floor the
 * variant kernels are judged against (SURVEY §8d roofline);
 * d_out receives meaningless values.  Grid = #SM x occupancy, stream-ordered
 * on `stream`.  DYSEL_ERR_UNSUPPORTED if col / val are not 16-byte aligned;
 * DYSEL_ERR_INVALID for a bad flavour or NULL pointers. */
dysel_status dysel_spmv_gather_probe(dysel_ctx *ctx, dysel_spmv_plan *plan, int flavour, const float *d_x,
                                     float *d_out, void *stream);

/* --------------------------------------- SpMV f-2: data placement (Case II)
 * SURVEY §8f f-2 / the paper's Case II ("four data placement policies ...
 * selected at runtime" for spmv-csr, §4.2): one CSR-scalar
 * kernel (thread per row, CSR-order fmaf from +0) in four placements of x,
 * selected by DySel through the generic launcher on the plan's 256-row units:
 *   0 x_ldg      x through the read-only L1 path (ld.global.nc)
 *   1 x_l2       x through L2 only (ld.global.cg)
 *   2 x_smem     each unit's x window [min col, max col] staged into shared
 *                memory by cp.async.bulk (banded matrices; units whose window
 *                exceeds 12,288 floats gather from global memory instead)
 *   3 x_persist  as x_ldg, launched with an L2 access-policy window marking x
 *                persisting (the ctx sets the device-wide persisting L2
 *                set-aside to the plan's x size, 1 MB granules, capped by the
 *                device maximum; grown per plan, released at dysel_destroy)
 * The four are bit-identical to each other and to CSR-S.  The pool is built
 * and registered at the plan's first placement call (x windows: one kernel).
 * d_x fp32 [n_cols], d_y fp32 [n_rows]; errors as dysel_spmv. */
enum { DYSEL_SPMV_PLACE_LDG = 0, DYSEL_SPMV_PLACE_L2 = 1, DYSEL_SPMV_PLACE_SMEM = 2, DYSEL_SPMV_PLACE_PERSIST = 3,
       DYSEL_SPMV_PLACE_NVARIANTS = 4 };
dysel_status dysel_spmv_placement(dysel_ctx *ctx, dysel_spmv_plan *plan, const float *d_x, float *d_y,
                                  float profile_fraction, uint32_t mode, void *stream, dysel_report *rep);
dysel_status dysel_spmv_placement_variant(dysel_ctx *ctx, dysel_spmv_plan *plan, int variant_id, const float *d_x,
                                          float *d_y, void *stream);
/* Test: the plan's per-unit x windows (int32 pairs [min col, max col], (0,-1)
 * for an empty unit) into HOST h_win (2 * cap_units ints); DYSEL_ERR_NOT_FOUND
 * before the first placement call. */
dysel_status dysel_spmv_placement_windows(const dysel_spmv_plan *plan, int32_t *h_win, size_t cap_units);

/* ------------------------------- SpMV f-2: global-sort JDS pool (Case III)
 * Parboil spmv-jds as the paper profiles it (P:L1424-1429, P:L1454-1461
 * §4.3): rows sorted by length over the WHOLE matrix (stable: ties keep row
 * order), entry (p, k) of permuted row p at jd_ptr[k] + p.  A standalone pool
 * (its units are 256 permuted rows, so it cannot share the block-local
 * pool's unit space, reading A-14) of four versions of the kernel:
 *   0 plain, 1 unroll (4 diagonals per iteration), 2 prefetch (next
 *   diagonal's entry in flight), 3 unroll + prefetch (initial version)
 * all summing each row in CSR order with fmaf from +0: bit-identical to each
 * other and to CSR-S.  Mode AUTO: hybrid unless every row has one length.
 * The plan owns its arrays (perm, len int32 [n]; jd_ptr int32 [W+1]; col /
 * val [nnz]) and keeps no pointer to the CSR. */
typedef struct dysel_spmv_jds_plan dysel_spmv_jds_plan;
enum { DYSEL_SPMV_JDS_PLAIN = 0, DYSEL_SPMV_JDS_UNROLL = 1, DYSEL_SPMV_JDS_PREFETCH = 2,
       DYSEL_SPMV_JDS_UNROLL_PREFETCH = 3, DYSEL_SPMV_JDS_NVARIANTS = 4 };
dysel_status dysel_spmv_jds_prepare(dysel_ctx *ctx, int64_t n_rows, int64_t n_cols, int64_t nnz,
                                    const int32_t *d_row_ptr, const int32_t *d_col, const float *d_val, void *stream,
                                    dysel_spmv_jds_plan **out);
dysel_status dysel_spmv_jds(dysel_ctx *ctx, dysel_spmv_jds_plan *plan, const float *d_x, float *d_y,
                            float profile_fraction, uint32_t mode, void *stream, dysel_report *rep);
dysel_status dysel_spmv_jds_variant(dysel_ctx *ctx, dysel_spmv_jds_plan *plan, int variant_id, const float *d_x,
                                    float *d_y, void *stream);
/* Test: copy array `which` (0 perm, 1 len, 2 jd_ptr, 3 col, 4 val) to HOST dst
 * (*bytes: in capacity, out size; dst NULL = query). */
dysel_status dysel_spmv_jds_copy_array(const dysel_spmv_jds_plan *plan, int which, void *dst, size_t *bytes);
void dysel_spmv_jds_plan_destroy(dysel_spmv_jds_plan *plan);

/* ------------------------------------------------------------------ SGEMM
 * C = alpha * A B + beta * C, fp32, row-major, no transposes (Parboil sgemm,
 * P:L1286-1294, L1427; A-17).  Unit = one 32x32 tile of C.  Built-in variants:
 * 0 S64 (SIMT FFMA 64x64), 1 S128 (SIMT 128x128), 2 T128x64 and 3 T128x128
 * (tcgen05.mma kind::tf32, 3xTF32 split in shared memory, TMEM accumulator).
 * lda >= K, ldb >= N, ldc >= N; M, N, K >= 0.  M*N = 0: no-op; K = 0: C = beta C. */
enum { DYSEL_SGEMM_S64 = 0, DYSEL_SGEMM_S128 = 1, DYSEL_SGEMM_T128x64 = 2, DYSEL_SGEMM_T128x128 = 3,
       DYSEL_SGEMM_NVARIANTS = 4 };
dysel_status dysel_sgemm(dysel_ctx *ctx, int M, int N, int K, float alpha, const float *d_A, int lda,
                         const float *d_B, int ldb, float beta, float *d_C, int ldc,
                         float profile_fraction, uint32_t mode, void *stream, dysel_report *rep);
/* Full-grid run of one SGEMM variant (exhaustive oracle timing). */
dysel_status dysel_sgemm_variant(dysel_ctx *ctx, int variant_id, int M, int N, int K, float alpha,
                                 const float *d_A, int lda, const float *d_B, int ldb, float beta,
                                 float *d_C, int ldc, void *stream);

/* ---------------------------------------------------------------- stencil
 * One 3-D 7-point Jacobi step (the paper's stencil case with
 * three versions of work-assignment factor 1, 64x and 128x):
 * fp32 arrays [nz][ny][nx] (x fastest), d_in and d_out distinct device
 * buffers of nx*ny*nz floats (caller-owned).  Interior points:
 *   out = c1 * (((((in[z-1] + in[z+1]) + in[y-1]) + in[y+1]) + in[x-1]) + in[x+1]) - c0 * in
 * (this association order, fp32, round to nearest, no contraction: all
 * variants are bit-identical); boundary points (any coordinate 0 or n-1):
 * out = in (reading A-37).  Unit = 32 x 4 x 1 points.  Built-in variants:
 * 0 base (thread per point, wa 1x1x1), 1 z-march (thread per (x, y) column
 * over 64 z-planes, wa 1x1x64), 2 TMA tile (128x8x16 points: each z-plane of
 * the tile plus its y / x halo streamed by TMA into a shared-memory ring,
 * persistent CTAs, wa 4x2x16; needs nx % 4 == 0 and 16-byte aligned buffers,
 * else the same items run the z-march column code).  nx, ny, nz >= 0 (0 volume: no-op);
 * DYSEL_ERR_INVALID for NULL or aliased buffers. */
enum { DYSEL_STENCIL_BASE = 0, DYSEL_STENCIL_ZMARCH = 1, DYSEL_STENCIL_TILED = 2, DYSEL_STENCIL_NVARIANTS = 3 };
dysel_status dysel_stencil(dysel_ctx *ctx, int nx, int ny, int nz, float c0, float c1, const float *d_in,
                           float *d_out, float profile_fraction, uint32_t mode, void *stream, dysel_report *rep);
/* Full-grid run of one stencil variant (exhaustive oracle timing). */
dysel_status dysel_stencil_variant(dysel_ctx *ctx, int variant_id, int nx, int ny, int nz, float c0, float c1,
                                   const float *d_in, float *d_out, void *stream);

/* ------------------------------------------------------------------ SpMTV
 * y += A^T x over a prepared plan's CSR (x fp32 [n_rows], y fp32 [n_cols],
 * caller-owned device memory; the plan's ELL/JDS copies are not used): the
 * scatter-add kernel whose work-groups write overlapping outputs through
 * global atomics, i.e. the paper's case for swap-based partial-productive
 * profiling (§2.2, §3.3, Table 1
 * P:L735-739).  All three built-in variants carry DYSEL_V_ATOMICS: AUTO resolves
 * to SWAP.  With DYSEL_HOST_ORCH it is the paper's copy-back swap (each
 * variant profiles the same slice into a private copy of y initialised from y;
 * the winner's copy is swapped in; the winner runs the rest) and SWAP|ASYNC
 * returns DYSEL_ERR_UNSUPPORTED (the final output space is not
 * determined until profiling ends).  Without it (default) the swap is additive
 * (DESIGN A-47): private outputs start at zero, the winner's is ADDED into y,
 * so the final output space is y itself and ASYNC is accepted (A-47b): the
 * default's kernel reduces light units straight into y until the selection
 * (report.eager_units).  Initial version (DESIGN A-30d): scatter-thread when
 * no row exceeds 64 entries, scatter-warp otherwise; below 128 MiB of
 * algorithmic bytes, one wave of the initial version, or with NO_PROFILE, the
 * call runs the cached selection or the initial version unprofiled (A-3b /
 * A-3c; FORCE_PROFILE overrides).  Unit = 256 rows of A.
 * Variants: 0 scatter-thread (thread per row), 1 scatter-warp (warp per row,
 * entries strided over lanes), 2 scatter-segment (warp per 32-row segment,
 * its nonzeros as one flat stream).  One fp32 red.global.add per nonzero, in no
 * fixed order: the result matches the fp64 oracle within fp32 rounding, not
 * bitwise.  n_rows = 0 or nnz = 0: no-op.  DYSEL_ERR_INVALID for a NULL plan
 * or buffer. */
enum { DYSEL_SPMTV_SCATTER_THREAD = 0, DYSEL_SPMTV_SCATTER_WARP = 1, DYSEL_SPMTV_SCATTER_SEGMENT = 2,
       DYSEL_SPMTV_NVARIANTS = 3 };
dysel_status dysel_spmtv(dysel_ctx *ctx, dysel_spmv_plan *plan, const float *d_x, float *d_y,
                         float profile_fraction, uint32_t mode, void *stream, dysel_report *rep);
/* Full-grid run of one SpMTV variant (exhaustive oracle timing): y += A^T x. */
dysel_status dysel_spmtv_variant(dysel_ctx *ctx, dysel_spmv_plan *plan, int variant_id, const float *d_x,
                                 float *d_y, void *stream);

/* --------------------------------------------------------------- multi-GPU
 * Row-sharded SpMV / M-sharded SGEMM over NCCL (the paper is
 * single-GPU).  nccl_unique_id points to the 128-byte
 * ncclUniqueId rank 0 created (dysel_comm_unique_id) and the caller broadcast
 * (e.g. over torch.distributed). */
dysel_status dysel_comm_unique_id(void *out_128_bytes);
dysel_status dysel_comm_init(dysel_ctx *ctx, const void *nccl_unique_id, int rank, int world);
/* nnz-balanced row partition: bounds[g] = smallest r with row_ptr[r] >= g*nnz/world, snapped down
 * to a multiple of 256 rows, bounds[0] = 0, bounds[world] = n_rows.  h_row_ptr is HOST memory. */
dysel_status dysel_partition_rows(const int32_t *h_row_ptr, int64_t n_rows, int world, int64_t *bounds);
/* y (full length, every rank) = A x where this rank's plan holds rows
 * [bounds[rank], bounds[rank+1]) with a rebased row_ptr; x full length on
 * every rank.  Local DySel launch into d_y + bounds[rank] and an in-place
 * allgatherv of y (grouped ncclBroadcast, one root per shard) OVERLAPPED with
 * it: every shard's rows go out in up to 8 chunks (dysel_allgather_chunk), a
 * chunk's broadcasts start on an internal stream as soon as the SpMV kernels
 * have counted all its 32-row slots final (device path; DYSEL_HOST_ORCH:
 * plain allgatherv after the SpMV).  Completes in stream order on `stream`.
 * The release is a stream wait-value on the chunk's counter (needs no SM;
 * it has no timeout -- the counts are exact by construction); where stream
 * memory operations are unavailable a one-thread waiter kernel releases it,
 * and a chunk it never sees complete within 2 s (a bug) fails the next call
 * with DYSEL_ERR_CUDA instead of hanging. */
dysel_status dysel_spmv_sharded(dysel_ctx *ctx, dysel_spmv_plan *local_plan, const int64_t *bounds,
                                const float *d_x, float *d_y, float profile_fraction, uint32_t mode,
                                void *stream, dysel_report *rep);
/* Chunk k (0 <= k < 8) of a shard of `rows` rows in the overlapped allgather:
 * rows [*row_begin, *row_end) relative to the shard (empty when k is past its
 * last chunk).  Chunks are whole 256-row units, 2^s units each with the
 * smallest s that needs at most 8 chunks; every rank derives every shard's
 * chunks from bounds alone.  Host function. */
dysel_status dysel_allgather_chunk(int64_t rows, int k, int64_t *row_begin, int64_t *row_end);
/* 1-GPU loopback of dysel_spmv_sharded (SURVEY §8e "testing without 8
 * GPUs"): plans[g] (g < G) holds rows [bounds[g], bounds[g+1]) with a rebased
 * row_ptr (the layout each rank's local plan has); the G shards' DySel
 * launches run one after another on this device, each selecting on its own
 * slice (a "mixed version"), each into a ctx-owned staging
 * buffer (that GPU's local y), and one cudaMemcpyAsync per shard assembles
 * d_y (full length bounds[G]) — the stand-in of the allgatherv.  d_x full
 * length.  reps: nullable array of G reports.  Stream-ordered on `stream`. */
dysel_status dysel_spmv_sharded_loopback(dysel_ctx *ctx, int G, dysel_spmv_plan *const *plans, const int64_t *bounds,
                                         const float *d_x, float *d_y, float profile_fraction, uint32_t mode,
                                         void *stream, dysel_report *reps);
/* Broadcast n floats from `root` in place (x or B distribution). */
dysel_status dysel_comm_broadcast(dysel_ctx *ctx, float *d_buf, size_t n, int root, void *stream);
/* SGEMM M-sharding: rank r owns C rows [m0, m1), blocks of
 * ceil(M / world) rounded up to 128 (one tcgen05 tile); empty for late ranks
 * when M is small. */
dysel_status dysel_sgemm_shard_rows(int M, int world, int rank, int *m0, int *m1);
/* M-sharded SGEMM: d_A_local = this rank's A_g, rows [m0, m1) of A only
 * ((m1 - m0) x K, leading dimension lda; A is never replicated), d_B the full
 * K x N matrix (replicated, e.g. by dysel_comm_broadcast), d_C the full M x N
 * matrix on every rank: C_g = alpha A_g B + beta C_g is computed in place by a
 * local DySel launch (own selection per shard), then C is allgathered. */
dysel_status dysel_sgemm_sharded(dysel_ctx *ctx, int M, int N, int K, float alpha, const float *d_A_local, int lda,
                                 const float *d_B, int ldb, float beta, float *d_C, int ldc,
                                 float profile_fraction, uint32_t mode, void *stream, dysel_report *rep);

/* --------------------------------------------------------- iterative driver */
/* Iterative use of a DySel kernel: the paper's activation
 * flag profiles an iterative kernel on its first invocation and reuses the
 * selection afterwards; §5.2 measures the per-iteration cost of
 * profiling every iteration instead.  Power iteration on a
 * square matrix, n_iter times:
 *     y_k = A x_k  (dysel_spmv),   x_{k+1} = y_k / ||y_k||_2
 * (x_{k+1} = 0 if y_k = 0).  d_x: device fp32 [n], in x_0, out x_{n_iter}
 * (overwritten every iteration); d_y: device fp32 [n], out y_{n_iter-1}.
 * profile_every: 0 = profile iteration 0 only (activation flag off
 * afterwards: cached selection), p > 0 = profile iterations 0, p, 2p, ...
 * d_norms: nullable DEVICE fp64 [n_iter], ||y_k||_2 (fp64 two-pass reduction
 * in a fixed order: deterministic).  rep: report of iteration 0.  Errors:
 * DYSEL_ERR_INVALID for a non-square plan, n_iter < 0 or profile_every < 0.
 * Stream-ordered on `stream`; blocks only where dysel_spmv's activation-flag
 * path waits for iteration 0's selection. */
dysel_status dysel_spmv_power(dysel_ctx *ctx, dysel_spmv_plan *plan, float *d_x, float *d_y, int n_iter,
                              int profile_every, float profile_fraction, uint32_t mode, void *stream,
                              double *d_norms, dysel_report *rep);
/* Row-sharded power iteration (§8e): every rank holds the full x and y
 * (n = bounds[world]); each iteration is dysel_spmv_sharded (local rows +
 * y allgather, the y -> x exchange) followed by the same deterministic
 * normalisation on every rank.  Arguments as dysel_spmv_power /
 * dysel_spmv_sharded. */
dysel_status dysel_spmv_power_sharded(dysel_ctx *ctx, dysel_spmv_plan *local_plan, const int64_t *bounds,
                                      float *d_x, float *d_y, int64_t n, int n_iter, int profile_every,
                                      float profile_fraction, uint32_t mode, void *stream, double *d_norms,
                                      dysel_report *rep);

/* ------------------------------------------------------------------- debug */
/* Number of dysel kernels launched by this ctx so far (bench.py's gpu_launches). */
uint64_t dysel_kernel_launches(const dysel_ctx *ctx);
/* Calibration microbenchmark (c-9): minimum non-zero %globaltimer delta over
 * `samples` reads and the clock64 rate (cycles per ns) over a `spin_ns` spin. */
dysel_status dysel_timer_calibrate(dysel_ctx *ctx, uint64_t samples, uint64_t spin_ns,
                                   uint64_t *tick_ns, double *cycles_per_ns);
/* Known-cost test variants (c-8): registers sig with n variants whose CTAs
 * spin cost_ns[v] per unit (wa = 1) and write out[u] = v+1 for each unit u
 * (args[0] = uint32_t* out).  Used to check selection end to end. */
dysel_status dysel_register_spin_variants(dysel_ctx *ctx, const char *sig, const uint32_t *cost_ns, int n,
                                          int default_variant);

#ifdef __cplusplus
}
#endif
#endif /* DYSEL_H_ */
