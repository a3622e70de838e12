// Multi-GPU DySel: row-sharded SpMV and M-sharded SGEMM over
// NCCL (NVLink 5 / NVSwitch).  The paper is single-GPU over PCIe
// (P:L1000-1002); each shard micro-profiles and selects on its own slice, so
// different shards may run different variants — the paper's "mixed version"
// (P:L1100-1104).  The only exchange step is the allgather of the output
// (grouped ncclBroadcast, one root per shard = allgatherv, in place).
#include <dlfcn.h>
#include <nccl.h>
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstring>
#include <string>

#include "dysel_device.cuh"
#include "internal.h"

using namespace dysel;

// NCCL is resolved lazily with dlopen: no link-time dependency, and when
// torch has already loaded its libnccl.so.2 the same copy is reused (two
// NCCL versions in one process would clash).
namespace {
struct NcclApi {
  bool ok = false;
  ncclResult_t (*GetUniqueId)(ncclUniqueId *);
  ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int);
  ncclResult_t (*CommDestroy)(ncclComm_t);
  ncclResult_t (*GroupStart)();
  ncclResult_t (*GroupEnd)();
  ncclResult_t (*Broadcast)(const void *, void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t);
  const char *(*GetErrorString)(ncclResult_t);
};
NcclApi &nccl() {
  static NcclApi api = [] {
    NcclApi a{};
    void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return a;
    a.GetUniqueId = (decltype(a.GetUniqueId))dlsym(h, "ncclGetUniqueId");
    a.CommInitRank = (decltype(a.CommInitRank))dlsym(h, "ncclCommInitRank");
    a.CommDestroy = (decltype(a.CommDestroy))dlsym(h, "ncclCommDestroy");
    a.GroupStart = (decltype(a.GroupStart))dlsym(h, "ncclGroupStart");
    a.GroupEnd = (decltype(a.GroupEnd))dlsym(h, "ncclGroupEnd");
    a.Broadcast = (decltype(a.Broadcast))dlsym(h, "ncclBroadcast");
    a.GetErrorString = (decltype(a.GetErrorString))dlsym(h, "ncclGetErrorString");
    a.ok = a.GetUniqueId && a.CommInitRank && a.CommDestroy && a.GroupStart && a.GroupEnd && a.Broadcast &&
           a.GetErrorString;
    return a;
  }();
  return api;
}
}  // namespace

#define DYSEL_NCCL_TRY(ctx, expr)                                                 \
  do {                                                                            \
    ncclResult_t r__ = (expr);                                                    \
    if (r__ != ncclSuccess) {                                                     \
      set_error((ctx), std::string(#expr) + ": " + nccl().GetErrorString(r__));   \
      return DYSEL_ERR_NCCL;                                                      \
    }                                                                             \
  } while (0)

void dysel::comm_free(dysel_ctx *ctx) {
  if (ctx && ctx->nccl_comm) {
    if (nccl().ok) nccl().CommDestroy((ncclComm_t)ctx->nccl_comm);
    ctx->nccl_comm = nullptr;
  }
  if (ctx && ctx->comm_st) {
    cudaStreamDestroy(ctx->comm_st);
    ctx->comm_st = nullptr;
  }
  if (ctx && ctx->chunk_ctr.ptr) {
    cudaFree(ctx->chunk_ctr.ptr);
    ctx->chunk_ctr = ScratchBuf{};
  }
  if (ctx && ctx->h_chunk_timeout) {
    cudaFreeHost(ctx->h_chunk_timeout);
    ctx->h_chunk_timeout = ctx->d_chunk_timeout = nullptr;
  }
}

// Overlapped allgather (D4 at G = 8 is comm-bound): the shard's y
// rows go out in kAgChunks chunks of 2^shift units, each as soon as the SpMV
// kernels have counted all of its 32-row slots final (ProfParams::chunk_done),
// so the NCCL broadcasts of early chunks overlap the remainder still running.
// One waiter kernel per chunk on the comm stream (bounded spin: a missing
// count — a bug — sets the timeout flag and lets the stream go on, it never
// hangs the device).
constexpr int kAgChunks = 8;
__global__ void chunk_wait_kernel(const uint32_t *ctr, uint32_t target, uint32_t *timeout_flag, uint32_t k) {
  const uint64_t t0 = dysel_globaltimer();
  uint32_t ns = 64;
  while (*(volatile const uint32_t *)ctr < target) {
    if (dysel_globaltimer() - t0 > 2000000000ull) {   // 2 s: record chunk and count seen
      if (timeout_flag)
        *(volatile uint32_t *)timeout_flag = 0x80000000u | (k << 24) | min(*(volatile const uint32_t *)ctr, 0xffffffu);
      break;
    }
    __nanosleep(ns);
    ns = ns < 2048 ? 2 * ns : ns;
  }
  __threadfence();
}

// The chunk release itself: a stream memory operation (cuStreamWaitValue32,
// GEQ) executed by the GPU's front end -- it needs no SM.  The waiter KERNEL
// above was never scheduled before the SpMV had finished: the SpMV's claim
// kernel keeps every SM full (its grid is one wave at full occupancy and the
// shared-memory carveout is sized to it, leaving no room for even a one-thread
// CTA), so the copies of round 2's first version started only after the last
// slot (measured: first release 1,057 us into a 1,070 us call, 9M-row FEM).
// The kernel remains the fallback when stream memory operations are
// unavailable.
static PFN_cuStreamWaitValue32_v11070 wait_value_fn() {
  static PFN_cuStreamWaitValue32_v11070 fn = [] {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuStreamWaitValue32", &p, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      p = nullptr;
    cudaGetLastError();
    return (PFN_cuStreamWaitValue32_v11070)p;
  }();
  return fn;
}
static dysel_status wait_chunk(dysel_ctx *ctx, const uint32_t *ctr, uint32_t target, uint32_t k, cudaStream_t st) {
  if (auto fn = wait_value_fn())
    if (fn((CUstream)st, (CUdeviceptr)ctr, target, CU_STREAM_WAIT_VALUE_GEQ) == CUDA_SUCCESS) return DYSEL_OK;
  chunk_wait_kernel<<<1, 1, 0, st>>>(ctr, target, ctx->d_chunk_timeout, k);
  return check_launch(ctx, "chunk_wait_kernel");
}

// chunking of shard r: units_r = ceil(rows_r / 256), chunk = 2^shift units
static uint32_t ag_shift(int64_t rows) {
  const int64_t units = (rows + 255) / 256;
  uint32_t sh = 0;
  while (((units + (1ll << sh) - 1) >> sh) > kAgChunks) ++sh;
  return sh;
}

extern "C" {

dysel_status dysel_comm_unique_id(void *out) {
  if (!out) return DYSEL_ERR_INVALID;
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
  ncclUniqueId id;
  if (!nccl().ok || nccl().GetUniqueId(&id) != ncclSuccess) return DYSEL_ERR_NCCL;
  memcpy(out, &id, sizeof(id));
  return DYSEL_OK;
}

dysel_status dysel_comm_init(dysel_ctx *ctx, const void *uid, int rank, int world) {
  if (!ctx || !uid || world < 1 || rank < 0 || rank >= world) return DYSEL_ERR_INVALID;
  comm_free(ctx);
  ctx->rank = rank;
  ctx->world = world;
  // world == 1 still builds a (one-rank) communicator, so the collective
  // calls below run — and are tested — on a single GPU
  ncclUniqueId id;
  memcpy(&id, uid, sizeof(id));
  ncclComm_t comm;
  DYSEL_CUDA_TRY(ctx, cudaSetDevice(ctx->device));
  if (!nccl().ok) {
    set_error(ctx, "libnccl.so.2 could not be loaded");
    return DYSEL_ERR_NCCL;
  }
  DYSEL_NCCL_TRY(ctx, nccl().CommInitRank(&comm, world, id, rank));
  ctx->nccl_comm = comm;
  return DYSEL_OK;
}

// bounds[g] = smallest r with row_ptr[r] * world >= g * nnz, snapped down to a
// multiple of 256 rows (one SpMV unit), bounds[0] = 0, bounds[world] = n.
dysel_status dysel_partition_rows(const int32_t *rp, int64_t n, int world, int64_t *bounds) {
  if (!rp || n < 0 || world < 1 || !bounds) return DYSEL_ERR_INVALID;
  const int64_t nnz = rp[n];
  bounds[0] = 0;
  for (int g = 1; g < world; ++g) {
    const int64_t target = (int64_t)g * nnz;   // compare row_ptr[r] * world >= g * nnz (exact integers)
    int64_t lo = 0, hi = n;
    while (lo < hi) {
      const int64_t mid = (lo + hi) / 2;
      if ((int64_t)rp[mid] * world >= target)
        hi = mid;
      else
        lo = mid + 1;
    }
    bounds[g] = std::max<int64_t>(bounds[g - 1], (lo / 256) * 256);
  }
  bounds[world] = n;
  return DYSEL_OK;
}

static dysel_status allgatherv(dysel_ctx *ctx, float *buf, const int64_t *offs, const int64_t *counts,
                               cudaStream_t st) {
  if (!ctx->nccl_comm) return DYSEL_OK;
  ncclComm_t comm = (ncclComm_t)ctx->nccl_comm;
  DYSEL_NCCL_TRY(ctx, nccl().GroupStart());
  for (int r = 0; r < ctx->world; ++r)
    if (counts[r] > 0)
      DYSEL_NCCL_TRY(ctx, nccl().Broadcast(buf + offs[r], buf + offs[r], (size_t)counts[r], ncclFloat, r, comm, st));
  DYSEL_NCCL_TRY(ctx, nccl().GroupEnd());
  return DYSEL_OK;
}

dysel_status dysel_comm_broadcast(dysel_ctx *ctx, float *d_buf, size_t n, int root, void *stream) {
  if (!ctx || (n > 0 && !d_buf) || root < 0 || root >= ctx->world) return DYSEL_ERR_INVALID;
  if (!ctx->nccl_comm || n == 0) return DYSEL_OK;
  DYSEL_NCCL_TRY(ctx, nccl().Broadcast(d_buf, d_buf, n, ncclFloat, root, (ncclComm_t)ctx->nccl_comm,
                                    (cudaStream_t)stream));
  return DYSEL_OK;
}

dysel_status dysel_allgather_chunk(int64_t rows, int k, int64_t *row_begin, int64_t *row_end) {
  if (rows < 0 || k < 0 || k >= kAgChunks || !row_begin || !row_end) return DYSEL_ERR_INVALID;
  const uint32_t sh = ag_shift(rows);
  const int64_t units = (rows + 255) / 256;
  *row_begin = std::min<int64_t>(((int64_t)k << sh) * 256, rows);
  *row_end = std::min<int64_t>(std::min<int64_t>((int64_t)(k + 1) << sh, units) * 256, rows);
  if (*row_end < *row_begin) *row_end = *row_begin;
  return DYSEL_OK;
}

dysel_status dysel_spmv_sharded(dysel_ctx *ctx, dysel_spmv_plan *local, const int64_t *bounds, const float *d_x,
                                float *d_y, float f, uint32_t mode, void *stream, dysel_report *rep) {
  if (!ctx || !local || !bounds || !d_y) return DYSEL_ERR_INVALID;
  const int R = ctx->world;
  int64_t offs[1024], counts[1024];
  if (R > 1024) return DYSEL_ERR_UNSUPPORTED;
  for (int r = 0; r < R; ++r) {
    offs[r] = bounds[r];
    counts[r] = bounds[r + 1] - bounds[r];
  }
  dysel_spmv_plan_info info;
  DYSEL_TRY(dysel_spmv_plan_get_info(local, &info));
  if (info.n_rows != counts[ctx->rank]) {
    set_error(ctx, "dysel_spmv_sharded: local plan rows != bounds slice");
    return DYSEL_ERR_INVALID;
  }
  cudaStream_t st = (cudaStream_t)stream;
  // the paper-faithful host path has no slot counters: plain allgather after it
  if (!ctx->nccl_comm || (mode & DYSEL_HOST_ORCH) || counts[ctx->rank] == 0) {
    DYSEL_TRY(dysel_spmv(ctx, local, d_x, d_y + offs[ctx->rank], f, mode, stream, rep));
    return allgatherv(ctx, d_y, offs, counts, st);
  }
  if (!ctx->comm_st) {
    DYSEL_CUDA_TRY(ctx, cudaStreamCreateWithFlags(&ctx->comm_st, cudaStreamNonBlocking));
    cudaFuncAttributes fa;   // load the waiter now (lazy module loading), not while the SpMV runs
    DYSEL_CUDA_TRY(ctx, cudaFuncGetAttributes(&fa, chunk_wait_kernel));
  }
  if (!ctx->h_chunk_timeout) {
    if (cudaHostAlloc((void **)&ctx->h_chunk_timeout, sizeof(uint32_t), cudaHostAllocMapped) != cudaSuccess ||
        cudaHostGetDevicePointer((void **)&ctx->d_chunk_timeout, ctx->h_chunk_timeout, 0) != cudaSuccess)
      return DYSEL_ERR_NOMEM;
    *ctx->h_chunk_timeout = 0u;
  }
  if (const uint32_t t = *(volatile uint32_t *)ctx->h_chunk_timeout) {   // a previous call's chunk wait timed out
    *(volatile uint32_t *)ctx->h_chunk_timeout = 0u;
    set_error(ctx, "dysel_spmv_sharded: chunk " + std::to_string((t >> 24) & 0x7f) + " of the overlapped allgather "
                   "was never completed (timeout; " + std::to_string(t & 0xffffff) + " slots counted)");
    return DYSEL_ERR_CUDA;
  }
  DYSEL_TRY(scratch(ctx, ctx->chunk_ctr, kAgChunks * sizeof(uint32_t)));
  uint32_t *ctr = (uint32_t *)ctx->chunk_ctr.ptr;
  DYSEL_CUDA_TRY(ctx, cudaMemsetAsync(ctr, 0, kAgChunks * sizeof(uint32_t), st));
  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  DYSEL_CUDA_TRY(ctx, cudaEventCreateWithFlags(&ev0, cudaEventDisableTiming));
  DYSEL_CUDA_TRY(ctx, cudaEventCreateWithFlags(&ev1, cudaEventDisableTiming));
  DYSEL_CUDA_TRY(ctx, cudaEventRecord(ev0, st));   // counters zeroed
  DYSEL_CUDA_TRY(ctx, cudaStreamWaitEvent(ctx->comm_st, ev0, 0));
  // the SpMV first, then the comm stream's waiters: a spinning waiter must
  // never be resident before a kernel it waits for is loaded (with lazy module
  // loading, a kernel's first launch can wait for running kernels — measured:
  // waiters enqueued first stalled the first profiled call until they timed out)
  const uint32_t my_sh = ag_shift(counts[ctx->rank]);
  const int64_t my_units = (counts[ctx->rank] + 255) / 256;
  ctx->spmv_chunk_done = ctr;
  ctx->spmv_chunk_shift = my_sh;
  dysel_status status = dysel_spmv(ctx, local, d_x, d_y + offs[ctx->rank], f, mode, stream, rep);
  ctx->spmv_chunk_done = nullptr;
  ctx->spmv_chunk_shift = 0;
  ncclComm_t comm = (ncclComm_t)ctx->nccl_comm;
  for (int k = 0; k < kAgChunks && status == DYSEL_OK; ++k) {
    const int64_t u0 = (int64_t)k << my_sh, u1 = std::min<int64_t>((int64_t)(k + 1) << my_sh, my_units);
    if (u0 < u1) {
      status = wait_chunk(ctx, ctr + k, (uint32_t)((u1 - u0) * 8), (uint32_t)k, ctx->comm_st);
      if (status != DYSEL_OK) break;
    }
    if (nccl().GroupStart() != ncclSuccess) status = DYSEL_ERR_NCCL;
    for (int r = 0; r < R && status == DYSEL_OK; ++r) {   // chunk k of every shard (same layout on every rank)
      int64_t a = 0, e = 0;
      dysel_allgather_chunk(counts[r], k, &a, &e);
      if (e > a && nccl().Broadcast(d_y + offs[r] + a, d_y + offs[r] + a, (size_t)(e - a), ncclFloat, r, comm,
                                    ctx->comm_st) != ncclSuccess)
        status = DYSEL_ERR_NCCL;
    }
    if (nccl().GroupEnd() != ncclSuccess && status == DYSEL_OK) status = DYSEL_ERR_NCCL;
  }
  // the call completes (stream order on `st`) with the allgather
  cudaEventRecord(ev1, ctx->comm_st);
  cudaStreamWaitEvent(st, ev1, 0);
  cudaEventDestroy(ev0);
  cudaEventDestroy(ev1);
  if (status == DYSEL_ERR_NCCL) set_error(ctx, "dysel_spmv_sharded: NCCL broadcast failed");
  return status;
}

// Host buffers in and out (serving): x host -> device, the DySel SpMV, and
// y device -> host in up to kAgChunks chunks, each copied as soon as the SpMV
// kernels have counted all of its 32-row slots final -- the per-chunk
// counters and releases of the overlapped allgather, so the PCIe copy of y
// overlaps the rest of the SpMV.
dysel_status dysel_spmv_host(dysel_ctx *ctx, dysel_spmv_plan *plan, const float *h_x, float *h_y, float *d_x,
                             float *d_y, float f, uint32_t mode, void *stream, dysel_report *rep) {
  if (!ctx || !plan) return DYSEL_ERR_INVALID;
  dysel_spmv_plan_info info;
  DYSEL_TRY(dysel_spmv_plan_get_info(plan, &info));
  if ((info.n_cols > 0 && (!h_x || !d_x)) || (info.n_rows > 0 && (!h_y || !d_y))) {
    set_error(ctx, "dysel_spmv_host: invalid arguments");
    return DYSEL_ERR_INVALID;
  }
  cudaStream_t st = (cudaStream_t)stream;
  if (info.n_cols > 0)
    DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(d_x, h_x, (size_t)info.n_cols * sizeof(float), cudaMemcpyHostToDevice, st));
  if (info.n_rows == 0) return DYSEL_OK;
  const size_t ybytes = (size_t)info.n_rows * sizeof(float);
  if (mode & DYSEL_HOST_ORCH) {   // the paper-faithful host path has no slot counters
    DYSEL_TRY(dysel_spmv(ctx, plan, d_x, d_y, f, mode, stream, rep));
    DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(h_y, d_y, ybytes, cudaMemcpyDeviceToHost, st));
    return DYSEL_OK;
  }
  if (!ctx->comm_st) {
    DYSEL_CUDA_TRY(ctx, cudaStreamCreateWithFlags(&ctx->comm_st, cudaStreamNonBlocking));
    cudaFuncAttributes fa;   // load the fallback waiter now (lazy module loading), not while the SpMV runs
    DYSEL_CUDA_TRY(ctx, cudaFuncGetAttributes(&fa, chunk_wait_kernel));
  }
  if (!ctx->h_chunk_timeout) {
    if (cudaHostAlloc((void **)&ctx->h_chunk_timeout, sizeof(uint32_t), cudaHostAllocMapped) != cudaSuccess ||
        cudaHostGetDevicePointer((void **)&ctx->d_chunk_timeout, ctx->h_chunk_timeout, 0) != cudaSuccess)
      return DYSEL_ERR_NOMEM;
    *ctx->h_chunk_timeout = 0u;
  }
  if (const uint32_t t = *(volatile uint32_t *)ctx->h_chunk_timeout) {
    *(volatile uint32_t *)ctx->h_chunk_timeout = 0u;
    set_error(ctx, "dysel_spmv_host: chunk " + std::to_string((t >> 24) & 0x7f) + " of y was never completed "
                   "(timeout; " + std::to_string(t & 0xffffff) + " slots counted)");
    return DYSEL_ERR_CUDA;
  }
  DYSEL_TRY(scratch(ctx, ctx->chunk_ctr, kAgChunks * sizeof(uint32_t)));
  uint32_t *ctr = (uint32_t *)ctx->chunk_ctr.ptr;
  DYSEL_CUDA_TRY(ctx, cudaMemsetAsync(ctr, 0, kAgChunks * sizeof(uint32_t), st));
  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  DYSEL_CUDA_TRY(ctx, cudaEventCreateWithFlags(&ev0, cudaEventDisableTiming));
  DYSEL_CUDA_TRY(ctx, cudaEventCreateWithFlags(&ev1, cudaEventDisableTiming));
  DYSEL_CUDA_TRY(ctx, cudaEventRecord(ev0, st));   // x copied in, counters zeroed
  DYSEL_CUDA_TRY(ctx, cudaStreamWaitEvent(ctx->comm_st, ev0, 0));
  const uint32_t sh = ag_shift(info.n_rows);
  const int64_t units = (info.n_rows + 255) / 256;
  ctx->spmv_chunk_done = ctr;   // the SpMV first, then the releases (see dysel_spmv_sharded)
  ctx->spmv_chunk_shift = sh;
  dysel_status status = dysel_spmv(ctx, plan, d_x, d_y, f, mode, stream, rep);
  ctx->spmv_chunk_done = nullptr;
  ctx->spmv_chunk_shift = 0;
  for (int k = 0; k < kAgChunks && status == DYSEL_OK; ++k) {
    const int64_t u0 = (int64_t)k << sh, u1 = std::min<int64_t>((int64_t)(k + 1) << sh, units);
    if (u0 >= u1) continue;
    status = wait_chunk(ctx, ctr + k, (uint32_t)((u1 - u0) * 8), (uint32_t)k, ctx->comm_st);
    int64_t a = 0, e = 0;
    dysel_allgather_chunk(info.n_rows, k, &a, &e);
    if (status == DYSEL_OK && e > a &&
        cudaMemcpyAsync(h_y + a, d_y + a, (size_t)(e - a) * sizeof(float), cudaMemcpyDeviceToHost, ctx->comm_st) !=
            cudaSuccess)
      status = DYSEL_ERR_CUDA;
  }
  // the call completes (stream order on `st`) with the last chunk's copy
  cudaEventRecord(ev1, ctx->comm_st);
  cudaStreamWaitEvent(st, ev1, 0);
  cudaEventDestroy(ev0);
  cudaEventDestroy(ev1);
  if (status == DYSEL_ERR_CUDA) set_error(ctx, "dysel_spmv_host: chunked copy-out failed");
  return status;
}


dysel_status dysel_sgemm_shard_rows(int M, int world, int rank, int *m0, int *m1) {
  if (M < 0 || world < 1 || rank < 0 || rank >= world || !m0 || !m1) return DYSEL_ERR_INVALID;
  // M-blocks of ceil(M / world) rounded up to 128 rows (one tcgen05 tile)
  const int64_t per = (((int64_t)M + world - 1) / world + 127) / 128 * 128;
  *m0 = (int)std::min<int64_t>((int64_t)rank * per, M);
  *m1 = (int)std::min<int64_t>((int64_t)(rank + 1) * per, M);
  return DYSEL_OK;
}

dysel_status dysel_sgemm_sharded(dysel_ctx *ctx, int M, int N, int K, float alpha, const float *d_A_local, int lda,
                                 const float *d_B, int ldb, float beta, float *d_C, int ldc, float f, uint32_t mode,
                                 void *stream, dysel_report *rep) {
  if (!ctx || M < 0 || N < 0 || K < 0) return DYSEL_ERR_INVALID;
  const int R = ctx->world;
  if (R > 1024) return DYSEL_ERR_UNSUPPORTED;
  int64_t offs[1024], counts[1024];
  for (int r = 0; r < R; ++r) {
    int a = 0, b = 0;
    DYSEL_TRY(dysel_sgemm_shard_rows(M, R, r, &a, &b));
    offs[r] = (int64_t)a * ldc;
    counts[r] = (int64_t)(b - a) * ldc;
  }
  int m0 = 0, m1 = 0;
  DYSEL_TRY(dysel_sgemm_shard_rows(M, R, ctx->rank, &m0, &m1));
  // A_g is LOCAL (rows [m0, m1) only, row 0 = global row m0); B replicated; C_g
  // written in place inside the full C, then allgathered
  if (m1 > m0)
    DYSEL_TRY(dysel_sgemm(ctx, m1 - m0, N, K, alpha, d_A_local, lda, d_B, ldb, beta, d_C + (int64_t)m0 * ldc, ldc, f,
                          mode, stream, rep));
  return allgatherv(ctx, d_C, offs, counts, (cudaStream_t)stream);
}

// 1-GPU loopback of the row-sharded SpMV (SURVEY §8e "Testing without 8
// GPUs"): the G shards' DySel launches run one after another on this device,
// each with its own plan (rebased row_ptr) and therefore its own selection —
// the paper's "mixed version" — each into a private staging
// buffer standing in for that GPU's local y, and one cudaMemcpyAsync per
// shard stands in for its part of the allgatherv.
dysel_status dysel_spmv_sharded_loopback(dysel_ctx *ctx, int G, dysel_spmv_plan *const *plans, const int64_t *bounds,
                                         const float *d_x, float *d_y, float f, uint32_t mode, void *stream,
                                         dysel_report *reps) {
  if (!ctx || G < 1 || !plans || !bounds || (bounds[G] > 0 && (!d_y || !d_x))) {
    set_error(ctx, "dysel_spmv_sharded_loopback: invalid arguments");
    return DYSEL_ERR_INVALID;
  }
  cudaStream_t st = (cudaStream_t)stream;
  int64_t maxc = 0;
  for (int g = 0; g < G; ++g) {
    dysel_spmv_plan_info info;
    if (!plans[g] || bounds[g + 1] < bounds[g]) {
      set_error(ctx, "dysel_spmv_sharded_loopback: bad plan / bounds");
      return DYSEL_ERR_INVALID;
    }
    DYSEL_TRY(dysel_spmv_plan_get_info(plans[g], &info));
    if (info.n_rows != bounds[g + 1] - bounds[g]) {
      set_error(ctx, "dysel_spmv_sharded_loopback: plan rows != bounds slice");
      return DYSEL_ERR_INVALID;
    }
    maxc = std::max<int64_t>(maxc, info.n_rows);
  }
  DYSEL_TRY(scratch(ctx, ctx->shard_stage, (size_t)std::max<int64_t>(maxc, 1) * sizeof(float)));
  float *stage = (float *)ctx->shard_stage.ptr;
  for (int g = 0; g < G; ++g) {
    const int64_t n = bounds[g + 1] - bounds[g];
    DYSEL_TRY(dysel_spmv(ctx, plans[g], d_x, stage, f, mode, stream, reps ? reps + g : nullptr));
    if (n > 0)
      DYSEL_CUDA_TRY(ctx, cudaMemcpyAsync(d_y + bounds[g], stage, (size_t)n * sizeof(float), cudaMemcpyDeviceToDevice,
                                          st));
  }
  return DYSEL_OK;
}

}  // extern "C"

