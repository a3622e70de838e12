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
//  CSR-W  (B200-native addition) warp-streaming CSR: each
//         warp streams the contiguous nonzeros of its 32-row group with fully
//         coalesced loads and forms the row sums with a warp-level segmented
//         reduction (head flags from __reduce_or_sync, Hillis-Steele scan with
//         __shfl_up_sync); chunks wholly inside one row skip the scan.
// CSR-S, ELL and JDS accumulate each row's products in CSR order with fmaf
// from +0, so the three are bit-identical to each other.
//
// Poll: the persistent dispatcher passes a SandboxPoll to hybrid-mode sandbox
// runs so a provably-losing variant can stop early (spmv.cu, dominance rule);
// NoPoll compiles to nothing.
#pragma once

#include <stdint.h>

namespace dysel {

constexpr int kUnitRows = 256;
constexpr int kVecMin = 128;   // CSR-V: rows at least this long use 128-bit loads
constexpr int kRowBatch = 4;   // CSR-V: rows in flight per warp
#ifndef DYSEL_CHUNK
#define DYSEL_CHUNK 8
#endif
constexpr int kChunk = DYSEL_CHUNK;   // CSR-S / JDS: entries per thread in flight
#ifndef DYSEL_ELL_CHUNK
#define DYSEL_ELL_CHUNK 16
#endif
constexpr int kEllChunk = DYSEL_ELL_CHUNK;   // ELL: slots per thread in flight
constexpr int kStreamUnroll = 4;   // CSR-W: 32-entry chunks in flight per warp
#ifndef DYSEL_STREAM_LONG
#define DYSEL_STREAM_LONG 512
#endif
constexpr int kStreamLong = DYSEL_STREAM_LONG;   // CSR-W: open-row stretch that switches to the 256-entry loop

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
  int32_t vec32;    // col/val 32-byte aligned (256-bit loads)
};

struct NoPoll {
  static constexpr bool active = false;
  __device__ __forceinline__ bool operator()() const { return false; }
  __device__ __forceinline__ bool warp() const { return false; }
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
// 256-bit loads (sm_100: LDG.E.256): one full 32-byte sector per lane
__device__ __forceinline__ void ld_stream8(const int32_t *p, uint64_t pol, int (&v)[8]) {
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
               : "l"(p), "l"(pol));
}
__device__ __forceinline__ void ld_stream8(const float *p, uint64_t pol, float (&v)[8]) {
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
               : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]), "=f"(v[7])
               : "l"(p), "l"(pol));
}
__device__ __forceinline__ float4 ld_stream4(const float *p, uint64_t pol) {
  float4 v;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "l"(p), "l"(pol));
  return v;
}
// x gather: L1-cached (banded matrices reuse it across neighbouring rows),
// kept in L2.  (D4 CSR-W, cold: 0.815 ms; with L1::no_allocate 0.811-0.813,
// through L2 only (.cg) 0.813 -- within noise: the gathers are bound by the
// L1TEX request rate either way.)
__device__ __forceinline__ float ld_x(const float *p, uint64_t pol) {
  float v;
  asm volatile("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
  return v;
}

// ------------------------------------------------------------------ CSR-S
// The row is walked in chunks of kChunk entries: the chunk's col/val loads,
// then its x gathers, are all issued before the first fma, so a thread has
// kChunk independent loads in flight instead of one dependent chain per entry.
// The fmas still run one by one in CSR order (same bits as the plain loop).
template <class Poll>
__device__ __forceinline__ void unit_csr_scalar(const SpmvDev &A, uint32_t j, int w, float *__restrict__ out,
                                                const Poll &poll) {
  const int i = w * 32 + (threadIdx.x & 31);
  const int64_t r = (int64_t)j * kUnitRows + i;
  if (r >= A.n_rows) return;
  const uint64_t px = policy_evict_last();
  const int b = __ldg(A.row_ptr + r), e = __ldg(A.row_ptr + r + 1);
  float s = 0.0f;
  for (int k = b; k < e; k += kChunk) {
    int c[kChunk];
    float v[kChunk], xv[kChunk];
#pragma unroll
    for (int u = 0; u < kChunk; ++u) {
      const bool ok = k + u < e;
      c[u] = ok ? __ldg(A.col + k + u) : 0;
      v[u] = ok ? __ldg(A.val + k + u) : 0.0f;
    }
#pragma unroll
    for (int u = 0; u < kChunk; ++u) xv[u] = k + u < e ? ld_x(A.x + c[u], px) : 0.0f;
#pragma unroll
    for (int u = 0; u < kChunk; ++u)
      if (k + u < e) s = __fmaf_rn(v[u], xv[u], s);
    if (Poll::active && ((k - b) & 63) >= 64 - kChunk && poll()) break;
  }
  out[i] = s;
}

// ------------------------------------------------------------------ CSR-V
// Long row (len >= kVecMin): lane l sums, in order, the head entries
// [b, a) it owns (a = first 4-aligned index), its 4-entry groups of the body
// (chunks of 128 entries), then the tail; the 32 lane sums are xor-reduced.
template <class Poll>
__device__ __forceinline__ float csrv_long_row(const SpmvDev &A, int b, int e, int lane, uint64_t ps, uint64_t px,
                                               const Poll &poll) {
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
    if (Poll::active && __any_sync(0xffffffffu, poll.warp())) return s;   // warp-uniform exit
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

template <class Poll>
__device__ __forceinline__ void unit_csr_vector(const SpmvDev &A, uint32_t j, int w, float *__restrict__ out,
                                                const Poll &poll) {
  const int lane = threadIdx.x & 31;
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
        s[r] = csrv_long_row(A, b[r], e[r], lane, ps, px, poll);
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1)
#pragma unroll
      for (int r = 0; r < kRowBatch; ++r) s[r] += __shfl_xor_sync(0xffffffffu, s[r], o);
#pragma unroll
    for (int r = 0; r < kRowBatch; ++r)
      if (lane == i0 + r) mine = s[r];
    if (Poll::active && __any_sync(0xffffffffu, poll.warp())) break;   // warp-uniform exit
  }
  if (lane < nr) out[w * 32 + lane] = mine;
}

// -------------------------------------------------------------------- ELL
// Chunks of kChunk slots: loads first, then the gathers of the live slots,
// then the fmas in slot order.  Pads only follow a row's entries, so a chunk
// ending in a pad ends the row.
template <class Poll>
__device__ __forceinline__ void unit_ell(const SpmvDev &A, uint32_t j, int w, float *__restrict__ out, const Poll &poll) {
  const int i = w * 32 + (threadIdx.x & 31);
  const int64_t r = (int64_t)j * kUnitRows + i;
  if (r >= A.n_rows) return;
  const uint64_t ps = policy_evict_first(), px = policy_evict_last();
  const int32_t *cp = A.ell_col + r;
  const float *vp = A.ell_val + r;
  const int W = A.ell_W;
  float s = 0.0f;
  for (int k = 0; k < W; k += kEllChunk) {
    int c[kEllChunk];
    float v[kEllChunk], xv[kEllChunk];
#pragma unroll
    for (int u = 0; u < kEllChunk; ++u) {
      const bool ok = k + u < W;
      c[u] = ok ? ld_stream(cp + (int64_t)(k + u) * A.n_pad, ps) : -1;
      v[u] = ok ? ld_stream(vp + (int64_t)(k + u) * A.n_pad, ps) : 0.0f;
    }
#pragma unroll
    for (int u = 0; u < kEllChunk; ++u) xv[u] = c[u] >= 0 ? ld_x(A.x + c[u], px) : 0.0f;
#pragma unroll
    for (int u = 0; u < kEllChunk; ++u)
      if (c[u] >= 0) s = __fmaf_rn(v[u], xv[u], s);
    if (c[kEllChunk - 1] < 0) break;
    if (Poll::active && (k & 63) >= 64 - kEllChunk && poll()) break;
  }
  out[i] = s;
}

// -------------------------------------------------------------------- JDS
// Chunks of kChunk diagonals; the jd_ptr offsets of the next chunk (the same
// for every thread of the block: broadcast loads) are fetched while the
// current chunk's col/val loads and gathers are in flight.
template <class Poll>
__device__ __forceinline__ void unit_jds(const SpmvDev &A, uint32_t j, int w, float *__restrict__ out, const Poll &poll) {
  const int p = w * 32 + (threadIdx.x & 31);
  const int64_t q = (int64_t)j * kUnitRows + p;
  if (q >= A.n_rows) return;
  const uint64_t ps = policy_evict_first(), px = policy_evict_last();
  const int len = __ldg(A.jds_len + q);
  const int32_t *jp = A.jd_ptr + __ldg(A.jd_off + j);
  const int64_t base = __ldg(A.blk_off + j) + p;
  float s = 0.0f;
  int off[kChunk];
#pragma unroll
  for (int u = 0; u < kChunk; ++u) off[u] = u < len ? __ldg(jp + u) : 0;
  for (int k = 0; k < len; k += kChunk) {
    int c[kChunk];
    float v[kChunk], xv[kChunk];
#pragma unroll
    for (int u = 0; u < kChunk; ++u) {
      const bool ok = k + u < len;
      c[u] = ok ? ld_stream(A.jds_col + base + off[u], ps) : 0;
      v[u] = ok ? ld_stream(A.jds_val + base + off[u], ps) : 0.0f;
    }
#pragma unroll
    for (int u = 0; u < kChunk; ++u) off[u] = k + kChunk + u < len ? __ldg(jp + k + kChunk + u) : 0;
#pragma unroll
    for (int u = 0; u < kChunk; ++u) xv[u] = k + u < len ? ld_x(A.x + c[u], px) : 0.0f;
#pragma unroll
    for (int u = 0; u < kChunk; ++u)
      if (k + u < len) s = __fmaf_rn(v[u], xv[u], s);
    if (Poll::active && (k & 63) >= 64 - kChunk && poll()) break;
  }
  out[__ldg(A.perm + q) - (int64_t)j * kUnitRows] = s;
}

// ------------------------------------------------------------------ CSR-W
// Warp-streaming CSR.  Lane i owns row i of the warp's 32-row group
// (accumulator acc).  The group's nonzeros [s, e) are walked in 32-entry
// chunks, entry k = cb + lane per lane (coalesced 128-byte col / val loads).
// Chunk wholly inside the open row: per-lane partial `part += p`.  Otherwise:
// fold `part` into the open row (butterfly), then a segmented inclusive scan
// of the products (heads = row starts in the chunk, bit 0 always set); row i
// takes the scan value at the last lane of its segment.  The per-row order
// depends only on the row's offset inside its group: deterministic (c-6).
template <class Poll>
__device__ __forceinline__ void unit_csr_stream_s(const SpmvDev &A, uint32_t j, int w, float *__restrict__ out,
                                                  const Poll &poll) {
  const uint32_t FULL = 0xffffffffu;
  const int lane = threadIdx.x & 31;
  const int64_t base = (int64_t)j * kUnitRows + w * 32;
  const int nr = (int)min((int64_t)32, (int64_t)A.n_rows - base);
  if (nr <= 0) return;
  const uint64_t ps = policy_evict_first(), px = policy_evict_last();
  const int gend = __ldg(A.row_ptr + base + nr);
  const int re = lane < nr ? __ldg(A.row_ptr + base + lane + 1) : gend;
  const int rs = lane < nr ? __ldg(A.row_ptr + base + lane) : gend;
  const int s = __shfl_sync(FULL, rs, 0);
  const int e = gend;
  float acc = 0.0f, part = 0.0f;
  // open row at chunk start: the non-empty row containing entry cb
  auto open_row = [&](int cb) -> int {
    const uint32_t m = __ballot_sync(FULL, rs <= cb && cb < re);
    return m ? __ffs(m) - 1 : -1;
  };
  int o = open_row(s);
  int oe = o >= 0 ? __shfl_sync(FULL, re, o) : e;
  const uint32_t lane_mask_le = (lane == 31) ? FULL : ((2u << lane) - 1u);
  for (int c0 = s; c0 < e; c0 += 32 * kStreamUnroll) {
    // long stretch of the open row ahead: 128-bit loads, 256 entries per step
    // (o, oe unchanged: the stretch ends inside the open row)
    if (A.vec_ok && oe - c0 >= kStreamLong) {
      const int a = (c0 + 3) & ~3;
      if (c0 + lane < a) part += ld_stream(A.val + c0 + lane, ps) * ld_x(A.x + ld_stream(A.col + c0 + lane, ps), px);
      const int body_end = a + ((oe - a) & ~255);
      bool stop = false;
      for (int base = a; base < body_end; base += 256) {
        const int k0 = base + 4 * lane, k1 = k0 + 128;
        const int4 q0 = ld_stream4(A.col + k0, ps), q1 = ld_stream4(A.col + k1, ps);
        const float4 v0 = ld_stream4(A.val + k0, ps), v1 = ld_stream4(A.val + k1, ps);
        const float x0 = ld_x(A.x + q0.x, px), x1 = ld_x(A.x + q0.y, px), x2 = ld_x(A.x + q0.z, px),
                    x3 = ld_x(A.x + q0.w, px);
        const float z0 = ld_x(A.x + q1.x, px), z1 = ld_x(A.x + q1.y, px), z2 = ld_x(A.x + q1.z, px),
                    z3 = ld_x(A.x + q1.w, px);
        part = __fmaf_rn(v0.x, x0, part);
        part = __fmaf_rn(v0.y, x1, part);
        part = __fmaf_rn(v0.z, x2, part);
        part = __fmaf_rn(v0.w, x3, part);
        part = __fmaf_rn(v1.x, z0, part);
        part = __fmaf_rn(v1.y, z1, part);
        part = __fmaf_rn(v1.z, z2, part);
        part = __fmaf_rn(v1.w, z3, part);
        if (Poll::active && __any_sync(FULL, poll.warp())) {
          stop = true;
          break;
        }
      }
      if (stop) break;
      c0 = body_end;
      if (c0 >= e) break;
    }
    int cc[kStreamUnroll];
    float vv[kStreamUnroll], pp[kStreamUnroll];
#pragma unroll
    for (int u = 0; u < kStreamUnroll; ++u) {
      const int k = c0 + 32 * u + lane;
      const bool ok = k < e;
      cc[u] = ok ? ld_stream(A.col + k, ps) : -1;
      vv[u] = ok ? ld_stream(A.val + k, ps) : 0.0f;
    }
#pragma unroll
    for (int u = 0; u < kStreamUnroll; ++u) pp[u] = cc[u] >= 0 ? vv[u] * ld_x(A.x + cc[u], px) : 0.0f;
#pragma unroll
    for (int u = 0; u < kStreamUnroll; ++u) {
      const int cb = c0 + 32 * u;
      if (cb >= e) break;
      if (oe >= cb + 32) {   // whole chunk inside the open row
        part += pp[u];
        continue;
      }
      // fold the open row's per-lane partials
      float P = part;
#pragma unroll
      for (int d = 16; d > 0; d >>= 1) P += __shfl_xor_sync(FULL, P, d);
      if (lane == o) acc += P;
      part = 0.0f;
      // segmented inclusive scan over the chunk
      const uint32_t bit = (rs >= cb && rs < cb + 32 && rs < re) ? (1u << (rs - cb)) : 0u;
      const uint32_t H = __reduce_or_sync(FULL, bit) | 1u;
      const int seg_start = 31 - __clz(H & lane_mask_le);
      float v = pp[u];
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const float t = __shfl_up_sync(FULL, v, d);
        if (lane - d >= seg_start) v += t;
      }
      const int lo = max(rs, cb), hi = min(re, cb + 32);
      const bool has = lo < hi;
      const float got = __shfl_sync(FULL, v, has ? hi - 1 - cb : 0);
      if (has) acc += got;
      const int nb = cb + 32;
      o = open_row(nb);
      oe = o >= 0 ? __shfl_sync(FULL, re, o) : e;
    }
    if (Poll::active && __any_sync(FULL, poll.warp())) break;   // warp-uniform exit
  }
  float P = part;
#pragma unroll
  for (int d = 16; d > 0; d >>= 1) P += __shfl_xor_sync(FULL, P, d);
  if (lane == o) acc += P;
  if (lane < nr) out[w * 32 + lane] = acc;
}

// CSR-W, 128-bit form (col / val 16-byte aligned, vec_ok): the group's
// nonzeros are walked from a = s & ~3 in 128-entry chunks, lane l loading
// entries cb + 4l .. cb + 4l + 3 with one 128-bit col and one 128-bit val load
// (4x fewer load requests than 32-bit chunks; the x gathers are the same).
// Entries outside [s, e) contribute +0.  A chunk wholly inside the open row
// adds its 4 products to the lane partial; otherwise the row sums come from a
// two-level segmented scan: sequential within the lane's 4 entries, then a
// Hillis-Steele scan of the lane totals (segment starts = lanes holding a row
// start, from a ballot); the open row's lane partials are folded (butterfly)
// only when some chunk since the last fold added to them.  The order of every
// row's additions depends only on the row's offset inside its group and on
// s mod 4: deterministic (c-6).
// (Measured alternative, A-41b: lanes owning 8 contiguous entries
// with lane-local row sums and direct row writes issued 1.8x the instructions
// and ran 12% slower on D4.)
#ifndef DYSEL_STREAM_VEC
#define DYSEL_STREAM_VEC 2
#endif
constexpr int kStreamVec = DYSEL_STREAM_VEC;   // 128-entry chunks in flight per warp (8 x gathers per lane; D4 cold: 2 -> 0.816 ms, 3 -> 0.844, 4 -> 0.872)
template <class Poll>
__device__ __forceinline__ void unit_csr_stream(const SpmvDev &A, uint32_t j, int w, float *__restrict__ out,
                                                const Poll &poll) {
  if (!A.vec_ok) {
    unit_csr_stream_s(A, j, w, out, poll);
    return;
  }
  const uint32_t FULL = 0xffffffffu;
  const int lane = threadIdx.x & 31;
  const int64_t base = (int64_t)j * kUnitRows + w * 32;
  const int nr = (int)min((int64_t)32, (int64_t)A.n_rows - base);
  if (nr <= 0) return;
  const uint64_t ps = policy_evict_first(), px = policy_evict_last();
  const int gend = __ldg(A.row_ptr + base + nr);
  const int re = lane < nr ? __ldg(A.row_ptr + base + lane + 1) : gend;
  const int rs = lane < nr ? __ldg(A.row_ptr + base + lane) : gend;
  const int s = __shfl_sync(FULL, rs, 0);
  const int e = gend;
  float acc = 0.0f, part = 0.0f;
  auto open_row = [&](int cb) -> int {
    const uint32_t m = __ballot_sync(FULL, rs <= cb && cb < re);
    return m ? __ffs(m) - 1 : -1;
  };
  int o = open_row(s);
  int oe = o >= 0 ? __shfl_sync(FULL, re, o) : e;
  const uint32_t lane_mask_le = (lane == 31) ? FULL : ((2u << lane) - 1u);
  const bool starts = rs < re;   // this lane's row is non-empty
  bool pend = false;             // some lane partial added since the last fold (warp-uniform)
  for (int c0 = s & ~3; c0 < e; c0 += 128 * kStreamVec) {
    // long stretch of the open row ahead (c0 >= s: no foreign entries)
    if (c0 >= s && oe - c0 >= kStreamLong) {
      const int a = c0;   // 16-byte aligned here
      const int body_end = a + ((oe - a) & ~255);
      bool stop = false;
      pend = true;
      for (int b0 = a; b0 < body_end; b0 += 256) {
        const int k0 = b0 + 4 * lane, k1 = k0 + 128;
        const int4 q0 = ld_stream4(A.col + k0, ps), q1 = ld_stream4(A.col + k1, ps);
        const float4 v0 = ld_stream4(A.val + k0, ps), v1 = ld_stream4(A.val + k1, ps);
        const float x0 = ld_x(A.x + q0.x, px), x1 = ld_x(A.x + q0.y, px), x2 = ld_x(A.x + q0.z, px),
                    x3 = ld_x(A.x + q0.w, px);
        const float z0 = ld_x(A.x + q1.x, px), z1 = ld_x(A.x + q1.y, px), z2 = ld_x(A.x + q1.z, px),
                    z3 = ld_x(A.x + q1.w, px);
        part = __fmaf_rn(v0.x, x0, part);
        part = __fmaf_rn(v0.y, x1, part);
        part = __fmaf_rn(v0.z, x2, part);
        part = __fmaf_rn(v0.w, x3, part);
        part = __fmaf_rn(v1.x, z0, part);
        part = __fmaf_rn(v1.y, z1, part);
        part = __fmaf_rn(v1.z, z2, part);
        part = __fmaf_rn(v1.w, z3, part);
        if (Poll::active && __any_sync(FULL, poll.warp())) {
          stop = true;
          break;
        }
      }
      if (stop) break;
      c0 = body_end;
      if (c0 >= e) break;
    }
    float p[kStreamVec][4];
#pragma unroll
    for (int u = 0; u < kStreamVec; ++u) {
      const int k = c0 + 128 * u + 4 * lane;
      int cc[4] = {-1, -1, -1, -1};
      float vv[4] = {0.0f, 0.0f, 0.0f, 0.0f};
      if (k + 3 < e) {
        const int4 q = ld_stream4(A.col + k, ps);
        const float4 v = ld_stream4(A.val + k, ps);
        cc[0] = q.x; cc[1] = q.y; cc[2] = q.z; cc[3] = q.w;
        vv[0] = v.x; vv[1] = v.y; vv[2] = v.z; vv[3] = v.w;
      } else {
#pragma unroll
        for (int i = 0; i < 4; ++i)
          if (k + i < e) {
            cc[i] = ld_stream(A.col + k + i, ps);
            vv[i] = ld_stream(A.val + k + i, ps);
          }
      }
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const bool ok = k + i >= s && k + i < e;
        p[u][i] = ok ? vv[i] * ld_x(A.x + cc[i], px) : 0.0f;
      }
    }
#pragma unroll
    for (int u = 0; u < kStreamVec; ++u) {
      const int cb = c0 + 128 * u;
      if (cb >= e) break;
      if (oe >= cb + 128) {   // whole chunk inside the open row
        part += (p[u][0] + p[u][1]) + (p[u][2] + p[u][3]);
        pend = true;
        continue;
      }
      if (pend) {   // fold the open row's per-lane partials
        float P = part;
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) P += __shfl_xor_sync(FULL, P, d);
        if (lane == o) acc += P;
        part = 0.0f;
        pend = false;
      }
      // head bits of the chunk's 128 entries (word q: entries 32q .. 32q+31);
      // entry 0 always starts a segment
      const int off = rs - cb;
      const bool in = starts && off >= 0 && off < 128;
      uint32_t hw[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) hw[q] = __reduce_or_sync(FULL, (in && (off >> 5) == q) ? 1u << (off & 31) : 0u);
      hw[0] |= 1u;
      const uint32_t word = lane < 8 ? hw[0] : lane < 16 ? hw[1] : lane < 24 ? hw[2] : hw[3];
      const uint32_t h = (word >> ((4 * lane) & 31)) & 0xfu;
      // level 1: sequential segmented sums within the lane's 4 entries
      float v0 = p[u][0];
      float v1 = (h & 2u) ? p[u][1] : v0 + p[u][1];
      float v2 = (h & 4u) ? p[u][2] : v1 + p[u][2];
      float v3 = (h & 8u) ? p[u][3] : v2 + p[u][3];
      // level 2: segmented inclusive scan of the lane totals
      const uint32_t H = __ballot_sync(FULL, h != 0u) | 1u;
      const int seg_start = 31 - __clz(H & lane_mask_le);
      float c = v3;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const float t = __shfl_up_sync(FULL, c, d);
        if (lane - d >= seg_start) c += t;
      }
      float cin = __shfl_up_sync(FULL, c, 1);
      if (lane == 0) cin = 0.0f;
      if (!(h & 1u)) v0 += cin;
      if (!(h & 3u)) v1 += cin;
      if (!(h & 7u)) v2 += cin;
      if (!(h & 15u)) v3 += cin;
      // each row takes the value at its last entry inside the chunk
      const int lo = max(rs, cb), hi = min(re, cb + 128);
      const bool has = lo < hi;
      const int src = has ? hi - 1 - cb : 0;
      const float g0 = __shfl_sync(FULL, v0, src >> 2), g1 = __shfl_sync(FULL, v1, src >> 2),
                  g2 = __shfl_sync(FULL, v2, src >> 2), g3 = __shfl_sync(FULL, v3, src >> 2);
      const int si = src & 3;
      if (has) acc += si == 0 ? g0 : si == 1 ? g1 : si == 2 ? g2 : g3;
      o = open_row(cb + 128);
      oe = o >= 0 ? __shfl_sync(FULL, re, o) : e;
    }
    if (Poll::active && __any_sync(FULL, poll.warp())) break;   // warp-uniform exit
  }
  if (pend) {
    float P = part;
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) P += __shfl_xor_sync(FULL, P, d);
    if (lane == o) acc += P;
  }
  if (lane < nr) out[w * 32 + lane] = acc;
}


// ------------------------------------------------------------------ CSR-T
// Bulk-staged CSR (B200 data-placement variant; north_star
// "TMA or shared-memory staging"): the nonzeros of the warp's 32-row group
// are moved into shared memory by the bulk-copy (TMA) engine in ONE request
// per array (cp.async.bulk + mbarrier complete_tx), instead of one dependent
// col/val load chain per thread; each lane then walks its row from shared
// memory with kTmaGather x gathers in flight.  Compute is CSR-S's: lane i owns
// row i and fmas its entries in CSR order from +0, so CSR-T is bit-identical
// to CSR-S / ELL / JDS.  A group of more than kTmaCap nonzeros (heavy rows),
// or unaligned col / val (vec_ok = 0), runs the CSR-S code.
constexpr int kTmaCap = 1024;     // entries staged per warp (4 KB col + 4 KB val)
constexpr int kTmaGather = 16;    // x gathers in flight per lane
constexpr int kTmaWarps = kUnitRows / 32;
struct TmaStageBufs {
  int32_t col[kTmaWarps][kTmaCap];
  float val[kTmaWarps][kTmaCap];
  unsigned long long bar[kTmaWarps];   // one mbarrier per warp, initialised once per CTA
  uint32_t phase[kTmaWarps];           // its current phase parity
};

// dynamic shared memory (kernels that can run CSR-T are launched with
// sizeof(TmaStageBufs) bytes of it per 256-thread unit group, spmv.cu dyn_smem):
// group threadIdx.x / 256 uses the group-th set (grouped profiling, A-49)
__device__ __forceinline__ TmaStageBufs &tma_stage_bufs() {
  extern __shared__ __align__(128) unsigned char spmv_dyn_smem[];
  return *reinterpret_cast<TmaStageBufs *>(spmv_dyn_smem + (threadIdx.x / kUnitRows) * sizeof(TmaStageBufs));
}

__device__ __forceinline__ uint32_t spmv_smem_u32(const void *p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}

// CTA prologue of every kernel that may run CSR-T: initialise the per-warp
// mbarriers once (re-initialising a live mbarrier is undefined).  A no-op in a
// launch without the staging buffers (%dynamic_smem_size too small).
__device__ __forceinline__ void tma_stage_prologue() {
  uint32_t dyn;
  asm("mov.u32 %0, %%dynamic_smem_size;" : "=r"(dyn));
  if (dyn < (threadIdx.x / kUnitRows + 1) * sizeof(TmaStageBufs)) return;   // (uniform per CTA in practice)
  TmaStageBufs &t = tma_stage_bufs();
  const uint32_t i = threadIdx.x % kUnitRows;
  if (i < kTmaWarps) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(spmv_smem_u32(&t.bar[i])) : "memory");
    t.phase[i] = 0;
  }
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncthreads();
}

template <class Poll>
__device__ __forceinline__ void unit_csr_tma(const SpmvDev &A, uint32_t j, int w, float *__restrict__ out,
                                             const Poll &poll) {
  const uint32_t FULL = 0xffffffffu;
  const int lane = threadIdx.x & 31;
  const int64_t base = (int64_t)j * kUnitRows + w * 32;
  const int nr = (int)min((int64_t)32, (int64_t)A.n_rows - base);
  if (nr <= 0) return;
  const int rb = lane < nr ? __ldg(A.row_ptr + base + lane) : 0;
  const int re = lane < nr ? __ldg(A.row_ptr + base + lane + 1) : 0;
  const int s = __shfl_sync(FULL, rb, 0);
  const int e = __shfl_sync(FULL, re, nr - 1);
  const int a = s & ~3;   // 16-byte aligned start (entries [a, s) are loaded, never used)
  if (!A.vec_ok || e - a > kTmaCap) {
    unit_csr_scalar(A, j, w, out, poll);
    return;
  }
  TmaStageBufs &tsm = tma_stage_bufs();
  const int wl = (threadIdx.x >> 5) & (kTmaWarps - 1);   // this warp's buffers (any slot w may run here)
  const uint64_t px = policy_evict_last();
  const int nb = (e - a) & ~3;   // bulk part; the < 4 tail entries by lanes 0..2
  const uint32_t bar = spmv_smem_u32(&tsm.bar[wl]);
  __syncwarp();   // the previous slot's reads of the buffers and its phase flip are done
  const uint32_t par = tsm.phase[wl];
  __syncwarp();
  if (lane == 0) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(nb * 8) : "memory");
    if (nb > 0) {
      const uint64_t pst = policy_evict_first();
      asm volatile(
          "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
              spmv_smem_u32(&tsm.col[wl][0])),
          "l"(A.col + a), "r"(nb * 4), "r"(bar), "l"(pst)
          : "memory");
      asm volatile(
          "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
              spmv_smem_u32(&tsm.val[wl][0])),
          "l"(A.val + a), "r"(nb * 4), "r"(bar), "l"(pst)
          : "memory");
    }
  }
  if (lane < (e - a) - nb) {
    tsm.col[wl][nb + lane] = __ldg(A.col + a + nb + lane);
    tsm.val[wl][nb + lane] = __ldg(A.val + a + nb + lane);
  }
  {
    uint32_t ok = 0;
    while (!ok)
      asm volatile(
          "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
          : "=r"(ok)
          : "r"(bar), "r"(par)
          : "memory");
  }
  __syncwarp();   // tail entries stored by lanes; every lane has seen the phase complete
  if (lane == 0) tsm.phase[wl] = par ^ 1u;
  const int32_t *cs = tsm.col[wl] - a;
  const float *vs = tsm.val[wl] - a;
  float acc = 0.0f;
  for (int k = rb; k < re; k += kTmaGather) {
    float v[kTmaGather], xv[kTmaGather];
#pragma unroll
    for (int u = 0; u < kTmaGather; ++u) {
      const bool ok = k + u < re;
      v[u] = ok ? vs[k + u] : 0.0f;
      xv[u] = ok ? ld_x(A.x + cs[k + u], px) : 0.0f;
    }
#pragma unroll
    for (int u = 0; u < kTmaGather; ++u)
      if (k + u < re) acc = __fmaf_rn(v[u], xv[u], acc);
    if (Poll::active && ((k - rb) & 127) >= 128 - kTmaGather && poll()) break;
  }
  if (lane < nr) out[w * 32 + lane] = acc;
}

// One 32-row warp slot w (0..7) of unit j: rows 256 j + 32 w + lane (JDS:
// permuted positions 32 w + lane of block j, whose rows lie anywhere in the
// unit).  The 8 slots of a unit, run by the same variant in any order and by
// any warps, compute the whole unit; the per-row arithmetic does not depend on
// which warp runs it.
template <int VID, class Poll = NoPoll>
__device__ __forceinline__ void run_slot(const SpmvDev &A, uint32_t j, int w, float *out, const Poll &poll = Poll()) {
  if constexpr (VID == 0) unit_csr_scalar(A, j, w, out, poll);
  else if constexpr (VID == 1) unit_csr_vector(A, j, w, out, poll);
  else if constexpr (VID == 2) unit_ell(A, j, w, out, poll);
  else if constexpr (VID == 3) unit_jds(A, j, w, out, poll);
  else if constexpr (VID == 4) unit_csr_stream(A, j, w, out, poll);
  else unit_csr_tma(A, j, w, out, poll);
}

// Whole unit by a 256-thread CTA: warp w runs slot w.
template <int VID, class Poll = NoPoll>
__device__ __forceinline__ void run_unit(const SpmvDev &A, uint32_t j, float *out, const Poll &poll = Poll()) {
  run_slot<VID, Poll>(A, j, (int)(threadIdx.x >> 5), out, poll);
}

// One warp slot of any pool variant but CSR-T (which needs the staging
// buffers): the solo claim kernel's remainder when the winner is not the
// kernel's own variant (reading A-38).
static __device__ __noinline__ void run_slot_dyn(int vid, const SpmvDev &A, uint32_t j, int w, float *out) {
  switch (vid) {
    case 0: run_slot<0>(A, j, w, out); break;
    case 1: run_slot<1>(A, j, w, out); break;
    case 2: run_slot<2>(A, j, w, out); break;
    case 3: run_slot<3>(A, j, w, out); break;
    default: run_slot<4>(A, j, w, out); break;
  }
}

template <class Poll>
__device__ __forceinline__ void run_unit_dyn(int vid, const SpmvDev &A, uint32_t j, float *out, const Poll &poll) {
  switch (vid) {
    case 0: run_unit<0>(A, j, out, poll); break;
    case 1: run_unit<1>(A, j, out, poll); break;
    case 2: run_unit<2>(A, j, out, poll); break;
    case 3: run_unit<3>(A, j, out, poll); break;
    case 4: run_unit<4>(A, j, out, poll); break;
    default: run_unit<5>(A, j, out, poll); break;
  }
}

}  // namespace dysel
