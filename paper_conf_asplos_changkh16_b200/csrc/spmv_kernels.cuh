// SpMV variant device functions: one 256-row unit per
// 256-thread CTA, y[rows of unit j] = A[rows] x.  Every variant's per-row
// result depends only on the row (never on CTA position), so any assignment of
// units to variants composes bit-exactly (c-6).
//
//  CSR-S  SHOC spmv-csr scalar: thread per row, sequential fma in CSR order
//         (P:L1129-1131, L1473-1480).
//  CSR-V  SHOC spmv-csr vector: warp per row ("underutilization
//         of vectors (warps)" on short rows).  B200 form: each
//         warp owns 32 rows and works on R of them at once (independent load
//         chains); rows of >= 128 entries use 128-bit col/val loads.
//  ELL    Bell & Garland [4]: column-major padded slots,
//         thread per row, coalesced; pad slots (col = -1) are skipped (A-16).
//  JDS    Parboil spmv-jds, block-local (A-14): thread per
//         permuted row of the unit, diagonal k of the block contiguous.
// CSR-S, ELL and JDS accumulate each row's products in CSR order with fmaf
// from +0, so the three are bit-identical to each other.
#pragma once

#include <stdint.h>

namespace dysel {

constexpr int kUnitRows = 256;
constexpr int kVecMin = 128;   // CSR-V: rows at least this long use 128-bit loads
constexpr int kRowBatch = 4;   // CSR-V: rows in flight per warp

struct SpmvDev {
  int32_t n_rows, n_cols;
  const int32_t *__restrict__ row_ptr;
  const int32_t *__restrict__ col;
  const float *__restrict__ val;
  // ELL (column-major, n_pad rows per slot)
  int32_t ell_W;
  int64_t n_pad;
  const int32_t *__restrict__ ell_col;
  const float *__restrict__ ell_val;
  // block-local JDS
  const int32_t *__restrict__ perm;
  const int32_t *__restrict__ jds_len;
  const int64_t *__restrict__ blk_off;
  const int64_t *__restrict__ jd_off;
  const int32_t *__restrict__ jd_ptr;
  const int32_t *__restrict__ jds_col;
  const float *__restrict__ jds_val;
  const float *__restrict__ x;
  int32_t vec_ok;   // col/val 16-byte aligned
};

// ------------------------------------------------------------ load helpers
// Streamed matrix data: read once, do not pollute L1, evict first from L2 so
// that x (re-read, gathered) stays L2-resident.
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ int ld_stream(const int32_t *p, uint64_t pol) {
  int v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ float ld_stream(const float *p, uint64_t pol) {
  float v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ int4 ld_stream4(const int32_t *p, uint64_t pol) {
  int4 v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.s32 {%0,%1,%2,%3}, [%4], %5;"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ float4 ld_stream4(const float *p, uint64_t pol) {
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "l"(p), "l"(pol));
  return v;
}
// x gather: L1-cached (banded matrices reuse it across neighbouring rows),
// kept in L2.
__device__ __forceinline__ float ld_x(const float *p, uint64_t pol) {
  float v;
  asm volatile("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
  return v;
}

// ------------------------------------------------------------------ CSR-S
__device__ __forceinline__ void unit_csr_scalar(const SpmvDev &A, uint32_t j, float *__restrict__ out) {
  const int i = threadIdx.x;
  const int64_t r = (int64_t)j * kUnitRows + i;
  if (r >= A.n_rows) return;
  const uint64_t px = policy_evict_last();
  const int b = __ldg(A.row_ptr + r), e = __ldg(A.row_ptr + r + 1);
  float s = 0.0f;
#pragma unroll 4
  for (int k = b; k < e; ++k) s = __fmaf_rn(__ldg(A.val + k), ld_x(A.x + __ldg(A.col + k), px), s);
  out[i] = s;
}

// ------------------------------------------------------------------ CSR-V
// Long row (len >= kVecMin): lane l sums, in order, the head entries
// [b, a) it owns (a = first 4-aligned index), its 4-entry groups of the body
// (chunks of 128 entries), then the tail; the 32 lane sums are xor-reduced.
__device__ __forceinline__ float csrv_long_row(const SpmvDev &A, int b, int e, int lane, uint64_t ps,
                                               uint64_t px) {
  float s = 0.0f;
  // unaligned base pointers: no head / vector body, everything in the tail loop
  const int a = A.vec_ok ? min((b + 3) & ~3, e) : b;
  if (b + lane < a) {
    const int k = b + lane;
    s = __fmaf_rn(ld_stream(A.val + k, ps), ld_x(A.x + ld_stream(A.col + k, ps), px), s);
  }
  const int body_end = A.vec_ok ? a + ((e - a) & ~3) : b;
  int base = a;
  for (; base + 256 <= body_end; base += 256) {    // two 128-entry chunks in flight
    const int k0 = base + 4 * lane, k1 = k0 + 128;
    const int4 c0 = ld_stream4(A.col + k0, ps), c1 = ld_stream4(A.col + k1, ps);
    const float4 v0 = ld_stream4(A.val + k0, ps), v1 = ld_stream4(A.val + k1, ps);
    const float x0 = ld_x(A.x + c0.x, px), x1 = ld_x(A.x + c0.y, px), x2 = ld_x(A.x + c0.z, px),
                x3 = ld_x(A.x + c0.w, px);
    const float y0 = ld_x(A.x + c1.x, px), y1 = ld_x(A.x + c1.y, px), y2 = ld_x(A.x + c1.z, px),
                y3 = ld_x(A.x + c1.w, px);
    s = __fmaf_rn(v0.x, x0, s);
    s = __fmaf_rn(v0.y, x1, s);
    s = __fmaf_rn(v0.z, x2, s);
    s = __fmaf_rn(v0.w, x3, s);
    s = __fmaf_rn(v1.x, y0, s);
    s = __fmaf_rn(v1.y, y1, s);
    s = __fmaf_rn(v1.z, y2, s);
    s = __fmaf_rn(v1.w, y3, s);
  }
  for (; base < body_end; base += 128) {
    const int k0 = base + 4 * lane;
    if (k0 < body_end) {
      const int4 c0 = ld_stream4(A.col + k0, ps);
      const float4 v0 = ld_stream4(A.val + k0, ps);
      s = __fmaf_rn(v0.x, ld_x(A.x + c0.x, px), s);
      s = __fmaf_rn(v0.y, ld_x(A.x + c0.y, px), s);
      s = __fmaf_rn(v0.z, ld_x(A.x + c0.z, px), s);
      s = __fmaf_rn(v0.w, ld_x(A.x + c0.w, px), s);
    }
  }
  for (int k = body_end + lane; k < e; k += 32)
    s = __fmaf_rn(ld_stream(A.val + k, ps), ld_x(A.x + ld_stream(A.col + k, ps), px), s);
  return s;
}

__device__ __forceinline__ void unit_csr_vector(const SpmvDev &A, uint32_t j, float *__restrict__ out) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int64_t base = (int64_t)j * kUnitRows + w * 32;
  const int nr = (int)min((int64_t)32, (int64_t)A.n_rows - base);
  if (nr <= 0) return;
  const uint64_t ps = policy_evict_first(), px = policy_evict_last();
  const int rb = lane < nr ? __ldg(A.row_ptr + base + lane) : 0;
  const int re = lane < nr ? __ldg(A.row_ptr + base + lane + 1) : 0;
  float mine = 0.0f;
  for (int i0 = 0; i0 < nr; i0 += kRowBatch) {
    int b[kRowBatch], e[kRowBatch];
    float s[kRowBatch];
#pragma unroll
    for (int r = 0; r < kRowBatch; ++r) {
      b[r] = __shfl_sync(0xffffffffu, rb, (i0 + r) & 31);
      e[r] = __shfl_sync(0xffffffffu, re, (i0 + r) & 31);
      if (i0 + r >= nr) b[r] = e[r] = 0;
    }
    // first pass of every short row: all loads of the batch issued together
    int c[kRowBatch];
    float v[kRowBatch];
#pragma unroll
    for (int r = 0; r < kRowBatch; ++r) {
      const int k = b[r] + lane;
      const bool ok = (e[r] - b[r] < kVecMin) && k < e[r];
      c[r] = ok ? ld_stream(A.col + k, ps) : -1;
      v[r] = ok ? ld_stream(A.val + k, ps) : 0.0f;
    }
#pragma unroll
    for (int r = 0; r < kRowBatch; ++r) s[r] = c[r] >= 0 ? __fmaf_rn(v[r], ld_x(A.x + c[r], px), 0.0f) : 0.0f;
#pragma unroll
    for (int r = 0; r < kRowBatch; ++r) {
      const int len = e[r] - b[r];
      if (len < kVecMin) {
        for (int k = b[r] + lane + 32; k < e[r]; k += 32)
          s[r] = __fmaf_rn(ld_stream(A.val + k, ps), ld_x(A.x + ld_stream(A.col + k, ps), px), s[r]);
      } else {
        s[r] = csrv_long_row(A, b[r], e[r], lane, ps, px);
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1)
#pragma unroll
      for (int r = 0; r < kRowBatch; ++r) s[r] += __shfl_xor_sync(0xffffffffu, s[r], o);
#pragma unroll
    for (int r = 0; r < kRowBatch; ++r)
      if (lane == i0 + r) mine = s[r];
  }
  if (lane < nr) out[w * 32 + lane] = mine;
}

// -------------------------------------------------------------------- ELL
__device__ __forceinline__ void unit_ell(const SpmvDev &A, uint32_t j, float *__restrict__ out) {
  const int i = threadIdx.x;
  const int64_t r = (int64_t)j * kUnitRows + i;
  if (r >= A.n_rows) return;
  const uint64_t ps = policy_evict_first(), px = policy_evict_last();
  const int32_t *cp = A.ell_col + r;
  const float *vp = A.ell_val + r;
  float s = 0.0f;
  int k = 0;
  bool live = true;   // pads (col = -1) only follow a row's entries
  for (; k + 2 <= A.ell_W; k += 2) {
    const int c0 = ld_stream(cp + (int64_t)k * A.n_pad, ps);
    const int c1 = ld_stream(cp + (int64_t)(k + 1) * A.n_pad, ps);
    const float v0 = ld_stream(vp + (int64_t)k * A.n_pad, ps);
    const float v1 = ld_stream(vp + (int64_t)(k + 1) * A.n_pad, ps);
    if (c0 < 0) {
      live = false;
      break;
    }
    s = __fmaf_rn(v0, ld_x(A.x + c0, px), s);
    if (c1 < 0) {
      live = false;
      break;
    }
    s = __fmaf_rn(v1, ld_x(A.x + c1, px), s);
  }
  if (live && k < A.ell_W) {
    const int c0 = ld_stream(cp + (int64_t)k * A.n_pad, ps);
    if (c0 >= 0) s = __fmaf_rn(ld_stream(vp + (int64_t)k * A.n_pad, ps), ld_x(A.x + c0, px), s);
  }
  out[i] = s;
}

// -------------------------------------------------------------------- JDS
__device__ __forceinline__ void unit_jds(const SpmvDev &A, uint32_t j, float *__restrict__ out) {
  const int p = threadIdx.x;
  const int64_t q = (int64_t)j * kUnitRows + p;
  if (q >= A.n_rows) return;
  const uint64_t ps = policy_evict_first(), px = policy_evict_last();
  const int len = __ldg(A.jds_len + q);
  const int32_t *jp = A.jd_ptr + __ldg(A.jd_off + j);
  const int64_t base = __ldg(A.blk_off + j) + p;
  float s = 0.0f;
#pragma unroll 4
  for (int k = 0; k < len; ++k) {
    const int64_t idx = base + __ldg(jp + k);
    s = __fmaf_rn(ld_stream(A.jds_val + idx, ps), ld_x(A.x + ld_stream(A.jds_col + idx, ps), px), s);
  }
  out[__ldg(A.perm + q) - (int64_t)j * kUnitRows] = s;
}

template <int VID>
__device__ __forceinline__ void run_unit(const SpmvDev &A, uint32_t j, float *out) {
  if constexpr (VID == 0) unit_csr_scalar(A, j, out);
  else if constexpr (VID == 1) unit_csr_vector(A, j, out);
  else if constexpr (VID == 2) unit_ell(A, j, out);
  else unit_jds(A, j, out);
}

__device__ __forceinline__ void run_unit_dyn(int vid, const SpmvDev &A, uint32_t j, float *out) {
  switch (vid) {
    case 0: unit_csr_scalar(A, j, out); break;
    case 1: unit_csr_vector(A, j, out); break;
    case 2: unit_ell(A, j, out); break;
    default: unit_jds(A, j, out); break;
  }
}

}  // namespace dysel
