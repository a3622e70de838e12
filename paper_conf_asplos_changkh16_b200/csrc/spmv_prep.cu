// SpMV format preparation: CSR -> ELL and CSR -> block-local
// JDS on the device, plus the plan's bookkeeping.  "Input format
// transformation may require duplication of inputs" (P:L485, P:L489-491
// §2.3).  Layouts (bit-exact contract with oracle/formats.py, DESIGN.md §Data
// layout):
//   ELL  slot (k, i) at k * n_pad + i = k-th CSR entry of row i, else col -1 / val 0.
//   JDS  per 256-row block b: rows stably sorted by length (descending, ties by
//        row), perm[b*256+p] = row, jds_len[b*256+p] = its length,
//        jd_ptr_b[k] = sum_p min(len_p, k), entry (p, k) at blk_off[b] + jd_ptr_b[k] + p.
#include <vector>
#include <cub/device/device_scan.cuh>

#include <algorithm>
#include <cstring>

#include "spmv_plan.h"

namespace dysel {

__global__ void row_stats_kernel(const int32_t *__restrict__ rp, int64_t n, int32_t *__restrict__ max_len) {
  int m = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    m = max(m, rp[i + 1] - rp[i]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) m = max(m, __shfl_xor_sync(0xffffffffu, m, o));
  if ((threadIdx.x & 31) == 0) atomicMax(max_len, m);
}

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

// per 256-row unit: nonzeros and longest row (unit order, readings A-40 / A-45);
// one warp per unit
__global__ void unit_stats_kernel(const int32_t *__restrict__ rp, int64_t n, int64_t nu, int32_t *__restrict__ nnz_u,
                                  int32_t *__restrict__ max_u) {
  const int64_t u = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (u >= nu) return;
  const int64_t r0 = u * kUnitRows, r1 = min(r0 + kUnitRows, n);
  int m = 0;
  for (int64_t r = r0 + lane; r < r1; r += 32) m = max(m, rp[r + 1] - rp[r]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) m = max(m, __shfl_xor_sync(0xffffffffu, m, o));
  if (lane == 0) {
    nnz_u[u] = rp[r1] - rp[r0];
    max_u[u] = m;
  }
}

// phase 1: per block, stable sort by length (rank counting), W_b + 1

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
    wp1[blockIdx.x] = (int64_t)w + 1;
  }
}

// phase 2: jd_ptr_b[k] = sum_p min(len_p, k), k = 0..W_b
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

// phase 3: scatter (p, k) -> blk_off[b] + jd_ptr_b[k] + p
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

int spmv_pool_index(const dysel_spmv_plan *pl, int vid) {
  for (int i = 0; i < pl->K; ++i)
    if (pl->vids[i] == vid) return i;
  return -1;
}

}  // namespace dysel

using namespace dysel;

extern "C" {

dysel_status dysel_spmv_prepare(dysel_ctx *ctx, int64_t n_rows, int64_t n_cols, int64_t nnz, const int32_t *d_row_ptr,
                                const int32_t *d_col, const float *d_val, uint32_t formats_mask, int default_variant,
                                void *stream, dysel_spmv_plan **out) {
  if (!ctx || !out || n_rows < 0 || n_cols < 0 || nnz < 0 || nnz >= (1ll << 31) || n_rows >= (1ll << 31) ||
      n_cols >= (1ll << 31) || (n_rows > 0 && !d_row_ptr) || (nnz > 0 && (!d_col || !d_val)) ||
      default_variant < DYSEL_SPMV_DEFAULT_AUTO || default_variant >= DYSEL_SPMV_NVARIANTS) {
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
  A.vec32 = (((uintptr_t)d_col | (uintptr_t)d_val) & 31) == 0;
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
    const bool ok = cudaStreamSynchronize(st) == cudaSuccess;
    cudaFree(tmp);
    cudaFree(wp1);
    if (!ok) return fail(DYSEL_ERR_CUDA);
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
  if (formats_mask & DYSEL_FMT_TMA) pl->vids[pl->K++] = DYSEL_SPMV_CSR_TMA;
  if (cudaStreamSynchronize(st) != cudaSuccess) return fail(DYSEL_ERR_CUDA);
  {   // unit order (readings A-40, A-45).  Heavy units (>= max(8192, 4 x
      // mean) nonzeros) and long-row units (a row longer than max(1024, 8 x
      // mean row)) are run FIRST by the winner, nonzeros descending
      // (longest-processing-time order: no warp starts a 10^4-entry row in the
      // last microseconds of a launch); the rest ("light" units) are sampled
      // by the profiling slices and run eagerly by the not-yet-proven default
      // variant, which therefore never starts a long row it may be slow on
      // (a thread-per-row default on a 16,384-entry row, Fig. 5(b)).
    const int64_t nu = pl->n_units;
    const int64_t mean = nu > 0 ? nnz / nu : 0;
    const int64_t thr = std::max<int64_t>(kHeavyUnitNnz, 4 * mean);
    const int64_t lcap = std::max<int64_t>(kLongRow, n_rows > 0 ? 8 * ((nnz + n_rows - 1) / n_rows) : 0);
    // (single-wave grids -- fewer than 4 units per SM -- keep the plain order:
    // every slot starts at once; measured 39 vs 41 us at 235 units)
    if (nu >= 4 * (int64_t)ctx->n_sm && (nnz >= 2 * thr || W > lcap)) {
      std::vector<int32_t> un(nu), um(nu);
      int32_t *d_st = nullptr;
      if (cudaMalloc(&d_st, 2 * nu * 4) != cudaSuccess) return fail(DYSEL_ERR_NOMEM);
      unit_stats_kernel<<<(unsigned)((nu * 32 + 255) / 256), 256, 0, st>>>(d_row_ptr, n_rows, nu, d_st, d_st + nu);
      const bool ok = cudaMemcpyAsync(un.data(), d_st, nu * 4, cudaMemcpyDeviceToHost, st) == cudaSuccess &&
                      cudaMemcpyAsync(um.data(), d_st + nu, nu * 4, cudaMemcpyDeviceToHost, st) == cudaSuccess &&
                      cudaStreamSynchronize(st) == cudaSuccess;
      cudaFree(d_st);
      if (!ok) return fail(DYSEL_ERR_CUDA);
      std::vector<int32_t> light, rest;
      for (int64_t u = 0; u < nu; ++u)
        ((int64_t)un[u] < thr && (int64_t)um[u] <= lcap ? light : rest).push_back((int32_t)u);
      std::stable_sort(rest.begin(), rest.end(), [&](int32_t a, int32_t b) { return un[a] > un[b]; });
      if (!rest.empty()) {
        std::vector<int32_t> seq(light);
        seq.insert(seq.end(), rest.begin(), rest.end());
        if (cudaMalloc(&pl->seq, nu * 4) != cudaSuccess) return fail(DYSEL_ERR_NOMEM);
        if (cudaMemcpy(pl->seq, seq.data(), nu * 4, cudaMemcpyHostToDevice) != cudaSuccess) return fail(DYSEL_ERR_CUDA);
        pl->n_light = (uint32_t)light.size();
        I.n_heavy = (int32_t)rest.size();
      }
    }
    I.n_light = pl->seq ? (int32_t)pl->n_light : (int32_t)nu;
  }
  if (default_variant == DYSEL_SPMV_DEFAULT_AUTO) {   // reading A-30: initial version from row statistics
    // A-30b: a uniform matrix whose CSR arrays exceed L2 streams from HBM --
    // CSR-T (bulk-staged col / val) when it is in the pool and its warp slots
    // suit one bulk copy each: every slot fits the staging buffer (max row
    // <= 32: 32 rows x 32 <= kTmaCap) and holds >= 256 entries (mean row >=
    // 8); otherwise (or L2-resident) ELL.  Measured (scripts/sel_sweep.py):
    // CSR-T is the best on the 25-entry FEM rows, 1.6x slower than ELL on
    // 5-entry rows, 5-13x slower where slots overflow the buffer (50 / 500).
    // A-30c: uniform rows of fewer than 8 entries -> CSR-S (thread per row):
    // 5-point Laplacian CSR-S 62 vs ELL 77 us, 2M diagonal 34 vs 43, random
    // 5-entry rows within 6% of ELL (scripts/sel_sweep.py)
    const uint64_t csr_bytes = 8ull * (uint64_t)nnz + 4ull * (uint64_t)(n_rows + 1);
    if (I.uniform && (int64_t)8 * n_rows > nnz && spmv_pool_index(pl, DYSEL_SPMV_CSR_SCALAR) >= 0)
      default_variant = DYSEL_SPMV_CSR_SCALAR;
    else if (I.uniform && csr_bytes > ctx->l2_bytes && W <= 32 && (int64_t)8 * n_rows <= nnz &&
             spmv_pool_index(pl, DYSEL_SPMV_CSR_TMA) >= 0)
      default_variant = DYSEL_SPMV_CSR_TMA;
    else if (I.uniform && spmv_pool_index(pl, DYSEL_SPMV_ELL) >= 0) default_variant = DYSEL_SPMV_ELL;
    else if (spmv_pool_index(pl, DYSEL_SPMV_CSR_STREAM) >= 0) default_variant = DYSEL_SPMV_CSR_STREAM;
    else default_variant = DYSEL_SPMV_CSR_VECTOR;
  }
  I.default_variant = default_variant;
  pl->def = spmv_pool_index(pl, default_variant);
  if (pl->def < 0) {
    set_error(ctx, "dysel_spmv_prepare: default variant not in the pool (ELL inapplicable? A-15)");
    return fail(DYSEL_ERR_UNSUPPORTED);
  }
  I.n_variants = pl->K;
  for (int i = 0; i < pl->K; ++i) I.variant_ids[i] = pl->vids[i];
  I.prep_ns = now_ns() - t0;
  dysel_status rs = spmv_register_pool(ctx, pl);
  if (rs != DYSEL_OK) return fail(rs);
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
    case 9: break;
    default: return DYSEL_ERR_INVALID;
  }
  if (which == 9) {   // unit order (A-45): identity when the plan keeps none
    src = pl->seq;
    sz = pl->seq ? (size_t)nb * 4 : 0;
    if (!pl->seq) return DYSEL_ERR_NOT_FOUND;
  }
  const bool has = which == 9 ? true
                   : (which <= 1) ? spmv_pool_index(pl, DYSEL_SPMV_ELL) >= 0
                                  : spmv_pool_index(pl, DYSEL_SPMV_JDS) >= 0;
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
    if (!pl->place_sig.empty()) {
      pl->ctx->reg.erase(pl->place_sig);
      pl->ctx->sel_cache.erase(pl->place_sig);
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
  cudaFree(pl->seq);
  cudaFree(pl->xwin);
  cudaGetLastError();
  delete pl;
}

}  // extern "C"
