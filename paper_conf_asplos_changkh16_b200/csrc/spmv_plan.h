// dysel_spmv_plan: the SpMV variant pool for one CSR matrix (shared by
// spmv_prep.cu — format preparation — and spmv.cu — dispatch).
#pragma once

#include <string>

#include "internal.h"
#include "spmv_kernels.cuh"

struct dysel_spmv_plan {
  dysel_ctx *ctx = nullptr;
  dysel::SpmvDev dev{};
  dysel_spmv_plan_info info{};
  int32_t *ell_col = nullptr;
  float *ell_val = nullptr;
  int32_t *perm = nullptr, *jds_len = nullptr, *jd_ptr = nullptr, *jds_col = nullptr;
  int64_t *blk_off = nullptr, *jd_off = nullptr;
  float *jds_val = nullptr;
  int K = 0;                          // pool size
  int vids[DYSEL_SPMV_NVARIANTS] = {};  // pool index -> DYSEL_SPMV_* id
  int def = 0;                        // pool index of the default (initial) variant
  uint32_t n_units = 0;               // 256-row units
  // unit order (readings A-40, A-45): seq[0, n_light) = light units (no row
  // longer than the long-row cap, fewer nonzeros than the heavy threshold)
  // in index order, seq[n_light, n_units) = the rest, nonzeros descending
  // (longest-processing-time first).  seq = nullptr: identity, every unit
  // light (uniform matrices, single-wave grids).
  int32_t *seq = nullptr;
  uint32_t n_light = 0;
  std::string sig;                    // generic-registry signature (host path)
  // f-2 placement pool (spmv_f2.cu): per-unit x windows (int2 [n_units]), registry sig
  void *xwin = nullptr;
  std::string place_sig;
};

namespace dysel {
constexpr int64_t kHeavyUnitNnz = 8192;   // a unit with >= max(this, 4 x mean) nonzeros is heavy (A-40)
constexpr int64_t kLongRow = 1024;        // a unit with a row longer than max(this, 8 x mean row) is long (A-45)
int spmv_pool_index(const dysel_spmv_plan *pl, int vid);
// register the plan's pool with the generic launcher (host-orchestrated path)
dysel_status spmv_register_pool(dysel_ctx *ctx, dysel_spmv_plan *pl);
}  // namespace dysel
