// Internal declarations of libdysel.so (not part of the C ABI).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <unordered_map>
#include <vector>

#include "dysel.h"

#define DYSEL_CUDA_TRY(ctx, expr)                                              \
  do {                                                                         \
    cudaError_t e__ = (expr);                                                  \
    if (e__ != cudaSuccess) {                                                  \
      dysel::set_error((ctx), std::string(#expr) + ": " + cudaGetErrorString(e__)); \
      return DYSEL_ERR_CUDA;                                                   \
    }                                                                          \
  } while (0)

#define DYSEL_TRY(expr)                                                        \
  do {                                                                         \
    dysel_status s__ = (expr);                                                 \
    if (s__ != DYSEL_OK) return s__;                                           \
  } while (0)

namespace dysel {

// ------------------------------------------------------------- slice plan
// C++ restatement of the planning rules (DESIGN.md §Readings A-1..A-4, A-24);
// the oracle (oracle/slice_plan.py) is an independent Python copy of the same
// rules and tests/ compare the two through dysel_launch reports.
struct Plan {
  int K = 0;
  uint32_t g[3] = {1, 1, 1};
  uint32_t G[3] = {1, 1, 1};
  uint64_t U[3] = {1, 1, 1};
  uint64_t Gn = 0;
  uint64_t h[DYSEL_MAX_VARIANTS] = {};
  uint64_t c = 0;
  bool active = false;
  int mode = DYSEL_FULLY;  // resolved FULLY/HYBRID/SWAP
};

dysel_status make_plan(dysel_ctx *ctx, const uint64_t U[3], const uint32_t (*wa)[3], int K, float f, int n_sm,
                       int default_variant, uint32_t mode, const uint32_t *vflags, Plan *out);

// ------------------------------------------------------- device prof state
// Generic (host-launched variants) profiling bookkeeping, one per ctx.
struct DevProf {
  dysel_timer_slot slot[DYSEL_MAX_VARIANTS];
  uint64_t lb[DYSEL_MAX_VARIANTS];        // dominance: running cycle sums (A-32)
  uint32_t decided[DYSEL_MAX_VARIANTS];   // 0 running, 1 completed, 2 dominated
  uint32_t ctas_done[DYSEL_MAX_VARIANTS];
  uint32_t variants_done;
  uint32_t pad;
  uint64_t best;
  uint64_t sel;
  uint64_t t_publish;   // %globaltimer when the selection was published (written at sel + 1, dysel_device.cuh)
  uint64_t t_init;      // %globaltimer of the call's init kernel (report timeline origin)
};

struct Registered {
  std::vector<dysel_variant> v;
  std::vector<std::vector<int>> sandbox_args;
  std::vector<std::string> names;
  int def = 0;
  // a built-in pool (SGEMM, stencil, SpMTV, f-2, the SpMV host path): its
  // variants always report, so the gate may be a stream wait-value with no
  // timeout (user pools keep the bounded wait kernel)
  bool builtin = false;
};

// Selection words copied D2H asynchronously after device-path launches; the
// cache is refreshed from them lazily (never blocking the launch itself).
struct PendingSel {
  std::string sig;
  cudaEvent_t ev = nullptr;
  bool used = false;
};
constexpr int kPendingRing = 32;

struct ScratchBuf {
  void *ptr = nullptr;
  size_t bytes = 0;
};

}  // namespace dysel

struct dysel_ctx {
  int device = 0;
  int n_sm = 0;
  uint64_t l2_bytes = 0;
  uint64_t gt_tick_ns = 0;
  std::string last_error;
  std::unordered_map<std::string, dysel::Registered> reg;
  std::unordered_map<std::string, int> sel_cache;
  cudaStream_t fork[DYSEL_MAX_VARIANTS] = {};
  cudaStream_t query = nullptr;
  cudaEvent_t ev_start = nullptr;
  cudaEvent_t ev_join[DYSEL_MAX_VARIANTS] = {};
  cudaEvent_t ev_fork2 = nullptr;
  cudaStream_t rem[DYSEL_MAX_VARIANTS] = {};        // gated remainder copies (device path)
  cudaStream_t wsel = nullptr;                      // wait-for-selection kernel (device path)
  cudaStream_t rem_hi = nullptr;                    // the default variant's gated remainder (high priority)
  cudaEvent_t ev_join2[DYSEL_MAX_VARIANTS] = {};
  dysel::DevProf *d_prof = nullptr;
  dysel::DevProf *h_prof = nullptr;  // pinned
  void *d_spmv_state = nullptr;      // persistent-dispatcher state (spmv.cu)
  void *d_spmtv_state = nullptr;     // swap-mode device path state (spmtv.cu)
  void *h_spmv_rep = nullptr;        // pinned copy of its report area
  dysel::ScratchBuf sandbox[2 * DYSEL_MAX_VARIANTS];
  dysel::ScratchBuf unit_variant;    // device bytes, one per granule
  dysel::ScratchBuf norm_part;       // iterate.cu: fp64 norm partials
  dysel::ScratchBuf shard_stage;     // comm.cu: loopback shard output (a GPU's local y)
  dysel::PendingSel pending[dysel::kPendingRing];
  uint64_t *h_pending_sel = nullptr;   // pinned + mapped, kPendingRing words
  uint64_t *d_pending_sel = nullptr;   // device alias of h_pending_sel
  int pending_head = 0;
  // set (mapped pinned word) by a device-path wait for the selection that
  // timed out; reported as DYSEL_ERR_CUDA by the next call / the report
  uint32_t *h_sel_timeout = nullptr;
  uint32_t *d_sel_timeout = nullptr;
  uint64_t launches = 0;
  uint64_t plan_serial = 0;
  // L2 persisting set-aside (f-2 placement pool, x_persist): bytes reserved, max window
  size_t l2_persist_bytes = 0;
  size_t l2_persist_window = 0;
  // multi-GPU
  void *nccl_comm = nullptr;
  // overlapped allgather of the row-sharded SpMV (comm.cu): while set, the
  // SpMV kernels count finished 32-row slots per chunk of 2^shift units
  uint32_t *spmv_chunk_done = nullptr;
  uint32_t spmv_chunk_shift = 0;
  cudaStream_t comm_st = nullptr;            // the chunked allgather's stream
  dysel::ScratchBuf chunk_ctr;               // per-chunk slot counters
  uint32_t *h_chunk_timeout = nullptr;       // mapped pinned flag: a chunk wait timed out
  uint32_t *d_chunk_timeout = nullptr;
  int rank = 0, world = 1;
};

namespace dysel {
void set_error(dysel_ctx *ctx, const std::string &msg);
dysel_status check_launch(dysel_ctx *ctx, const char *what);
dysel_status scratch(dysel_ctx *ctx, ScratchBuf &b, size_t bytes);
uint64_t now_ns();
// enqueue a D2H copy of *d_sel for `sig` on `st`; cache updated when it lands
dysel_status push_pending_sel(dysel_ctx *ctx, const std::string &sig, const uint64_t *d_sel, cudaStream_t st);
// device-written variant: reserve a ring slot (its mapped device pointer is
// handed to the kernel that publishes the selection), then commit after launch
int reserve_pending_sel(dysel_ctx *ctx, uint64_t **d_slot);
dysel_status commit_pending_sel(dysel_ctx *ctx, int slot, const std::string &sig, cudaStream_t st);
// DYSEL_ERR_CUDA (and clears the flag) if a device-path selection wait timed out
dysel_status check_sel_timeout(dysel_ctx *ctx);
// move landed selections into the cache; block_sig != NULL waits for that sig
void resolve_pending(dysel_ctx *ctx, const char *block_sig);
// dysel_launch with a selection-cache key distinct from the registry sig
dysel_status launch_keyed(dysel_ctx *ctx, const char *sig, const char *key, const uint64_t ndrange_units[3], float f,
                          uint32_t mode, void *const *args, int n_args, const size_t *sandbox_bytes, void *stream,
                          dysel_report *rep, int def_override = -1);
// spmv.cu
dysel_status spmv_ctx_init(dysel_ctx *ctx);
void spmv_ctx_free(dysel_ctx *ctx);
// sgemm.cu
dysel_status sgemm_register(dysel_ctx *ctx);
// stencil.cu
dysel_status stencil_register(dysel_ctx *ctx);
dysel_status spmtv_register(dysel_ctx *ctx);
// comm.cu
void comm_free(dysel_ctx *ctx);
void mark_builtin(dysel_ctx *ctx, const char *sig);
}  // namespace dysel
