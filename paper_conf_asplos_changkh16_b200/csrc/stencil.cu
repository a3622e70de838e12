// DySel stencil pool: the paper's third GPU case with
// "three versions and work assignment factors relative to the base version
// of 64x and 128x" combining tiling, coarsening and scratchpad data placement
// (§4.3; Fig. 10b discussion P:L1462-1465).
//
// 3-D 7-point Jacobi step (reading A-37), fp32, x fastest, [nz][ny][nx]:
//   interior  out = c1 * (((((in[z-1] + in[z+1]) + in[y-1]) + in[y+1]) + in[x-1]) + in[x+1]) - c0 * in
//   boundary  out = in
// Every variant evaluates exactly this expression order with rn intrinsics
// (no contraction), so the three are bit-identical to each other (c-6).
//
// Unit = 32 (x) x 4 (y) x 1 (z) points.  Work assignment (units per CTA):
//   V0 base        wa (1, 1, 1)    thread per point
//   V1 z-march     wa (1, 1, 64)   thread per (x, y) column, 64 z-planes, z +-1 in registers
//   V2 TMA tile    wa (4, 2, 16)   128 x 8 x 16 item, planes streamed into a shared-
//                                  memory ring by TMA (scratchpad placement, 128x)
// The LCM granule is (4, 2, 64) units: the slice planner's safe point.
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstring>
#include <string>

#include "dysel_device.cuh"
#include "internal.h"

namespace dysel {

static const char *kStencilSig = "dysel.stencil";

struct StencilArgs {
  int nx, ny, nz;
  float c0, c1;
  const float *in;
};

__device__ __forceinline__ float st_point(float c, float zm, float zp, float ym, float yp, float xm, float xp, float c0,
                                          float c1) {
  float s = __fadd_rn(zm, zp);
  s = __fadd_rn(s, ym);
  s = __fadd_rn(s, yp);
  s = __fadd_rn(s, xm);
  s = __fadd_rn(s, xp);
  return __fsub_rn(__fmul_rn(c1, s), __fmul_rn(c0, c));
}

__device__ __forceinline__ bool st_interior(const StencilArgs &g, int x, int y, int z) {
  return x > 0 && y > 0 && z > 0 && x < g.nx - 1 && y < g.ny - 1 && z < g.nz - 1;
}

// ------------------------------------------------------------------- V0
__global__ void __launch_bounds__(128) stencil_base_kernel(StencilArgs g, float *__restrict__ out, dysel_slice s) {
  __shared__ dysel_prof_smem psm;
  if (!dysel_gate_open(s)) return;
  const uint32_t wa[3] = {1, 1, 1};
  const bool persistent = s.timer == nullptr && s.gate != nullptr;   // gated remainder: one wave walks the tiles
  const uint64_t n_cta = persistent ? dysel_slice_ctas(s, wa) : (uint64_t)blockIdx.x + 1;
  dysel_prof_begin(s, psm);
  bool ok = false;
  for (uint64_t cta = blockIdx.x; cta < n_cta; cta += gridDim.x) {
  uint64_t u[3];
  ok = dysel_cta_origin(s, wa, cta, u);
  if (ok) {
    const int x = (int)u[0] * 32 + (threadIdx.x & 31), y = (int)u[1] * 4 + (threadIdx.x >> 5), z = (int)u[2];
    if (x < g.nx && y < g.ny) {
      const size_t sx = 1, sy = (size_t)g.nx, sz = (size_t)g.nx * g.ny;
      const size_t i = (size_t)z * sz + (size_t)y * sy + x;
      const float c = __ldg(g.in + i);
      out[i] = st_interior(g, x, y, z)
                   ? st_point(c, __ldg(g.in + i - sz), __ldg(g.in + i + sz), __ldg(g.in + i - sy), __ldg(g.in + i + sy),
                              __ldg(g.in + i - sx), __ldg(g.in + i + sx), g.c0, g.c1)
                   : c;
    }
  }
  }
  dysel_prof_end(s, psm, ok ? 1u : 0u);
}

// ------------------------------------------------------------------- V1
// z-march in chunks of kZq planes: all loads of a chunk (the next kZq centre
// values and the 4 in-plane neighbours of each plane) are issued before its
// first point is computed, so a thread waits once per chunk, not once per
// plane.  kZq = 2 fits the 32-register budget of 16 CTAs/SM without spills
// (512 x 512 x 64: 43 us at 16/SM vs 50 us with kZq = 4 at 10/SM and 60 us
// with kZq = 4 squeezed to 32 registers).
constexpr int kZq = 2;
// poll(): called by all threads every 16 planes (A-32 dominance; productive
// copies only report, sandbox copies stop when it returns true)
template <class Poll>
__device__ __forceinline__ void zmarch_column(const StencilArgs &g, float *__restrict__ out, int x, int y, int z0,
                                              int z1, const Poll &poll) {
  const bool col = x < g.nx && y < g.ny;
  const bool inner_xy = col && x > 0 && y > 0 && x < g.nx - 1 && y < g.ny - 1;
  const int sy = g.nx;
  const size_t sz = (size_t)g.nx * g.ny;
  // running pointers at plane z (64-bit adds only; neighbour offsets are 32-bit)
  const size_t off0 = (size_t)z0 * sz + (col ? (size_t)y * sy + x : 0);
  const float *pin = g.in + off0;
  float *pout = out + off0;
  float zm = (col && z0 > 0) ? __ldg(pin - sz) : 0.0f;
  float c = col ? __ldg(pin) : 0.0f;
  for (int z = z0; z < z1; z += kZq) {
    if (((z - z0) & 15) == 15 - (kZq - 1) && poll(z - z0 + kZq, z1 - z0)) return;
    float up[kZq], ym[kZq], yp[kZq], xm[kZq], xp[kZq];
#pragma unroll
    for (int q = 0; q < kZq; ++q) {
      const int zz = z + q;
      const float *pq = pin + (size_t)q * sz;
      up[q] = (col && zz < z1 && zz + 1 < g.nz) ? __ldg(pq + sz) : 0.0f;
      const bool in = inner_xy && zz < z1 && zz > 0 && zz < g.nz - 1;
      ym[q] = in ? __ldg(pq - sy) : 0.0f;
      yp[q] = in ? __ldg(pq + sy) : 0.0f;
      xm[q] = in ? __ldg(pq - 1) : 0.0f;
      xp[q] = in ? __ldg(pq + 1) : 0.0f;
    }
#pragma unroll
    for (int q = 0; q < kZq; ++q) {
      const int zz = z + q;
      if (col && zz < z1) {
        pout[(size_t)q * sz] = (inner_xy && zz > 0 && zz < g.nz - 1)
                                   ? st_point(c, zm, up[q], ym[q], yp[q], xm[q], xp[q], g.c0, g.c1)
                                   : c;
        zm = c;
        c = up[q];
      }
    }
    pin += kZq * sz;
    pout += kZq * sz;
  }
}

// Untimed launches (full grid, gated remainder) use a lean instantiation with
// no timing / dominance code and a 16-CTA/SM register cap, so a 2,048-CTA grid
// (512 x 512 x 64) is resident in one wave; timed (profiling) copies keep the
// timing code.
template <bool TIMED>
__global__ void __launch_bounds__(128, TIMED ? 1 : 16)
    stencil_zmarch_kernel(StencilArgs g, float *__restrict__ out, dysel_slice s) {
  __shared__ dysel_prof_smem psm;
  if (!dysel_gate_open(s)) return;
  const uint32_t wa[3] = {1, 1, 64};
  const bool persistent = !TIMED && s.gate != nullptr;   // gated remainder: one wave walks the tiles
  const uint64_t n_cta = persistent ? dysel_slice_ctas(s, wa) : (uint64_t)blockIdx.x + 1;
  if constexpr (TIMED) dysel_prof_begin(s, psm);
  uint32_t units = 0;
  for (uint64_t cta = blockIdx.x; cta < n_cta; cta += gridDim.x) {
  uint64_t u[3];
  const bool ok = dysel_cta_origin(s, wa, cta, u);
  if (ok) {
    const int x = (int)u[0] * 32 + (threadIdx.x & 31), y = (int)u[1] * 4 + (threadIdx.x >> 5);
    const int z0 = (int)u[2], z1 = min(z0 + 64, g.nz);
    if constexpr (TIMED)
      zmarch_column(g, out, x, y, z0, z1,
                    [&](int done, int total) {
                      return dysel_prof_poll(s, psm, (uint32_t)done, (uint32_t)total) &&
                             s.role == DYSEL_ROLE_SANDBOX;
                    });
    else
      zmarch_column(g, out, x, y, z0, z1, [](int, int) { return false; });
    units = (uint32_t)(z1 - z0);
  }
  }
  if constexpr (TIMED) dysel_prof_end(s, psm, units);
}

// ------------------------------------------------------------------- V2
// TMA-staged tile (scratchpad data placement, the paper's 128x version):
// item = 128 (x) x 8 (y) x 16 (z) points = wa (4, 2, 16) units.  Warp 0's
// elected lane is a producer that streams the item's planes z0-1 .. z0+16 as
// one 3-D TMA box each ({128, 10, 1}: the 8 tile rows and their y halo) plus
// two {4, 8, 1} x-halo boxes, into a kStNS-deep ring of shared-memory stages
// (mbarrier full / empty pairs; the ring runs on across items, so a CTA keeps
// ~5 planes = 26 KB in flight).  Warps 1..8 (tile row r = warp - 1, lane owns
// 4 consecutive x) compute plane z from stages z-1, z, z+1 with 128-bit shared
// loads (x +-1 by shuffles, tile edges from the halo boxes) and 128-bit
// coalesced stores, then release stage z-1.  Persistent: one wave of CTAs
// walks the slice's items (x fastest, then y, then z chunk, so concurrently
// running CTAs share their y / z halo planes in L2).  Needs nx % 4 == 0 and
// 16-byte aligned in / out (TMA row pitch, 128-bit stores); otherwise the same
// items run the z-march column code (same expression, bit-identical).
#ifndef DYSEL_ST_NS
#define DYSEL_ST_NS 8
#endif
#ifndef DYSEL_ST_TZ
#define DYSEL_ST_TZ 16
#endif
constexpr int kStTX = 128, kStTY = 8, kStTZ = DYSEL_ST_TZ, kStNS = DYSEL_ST_NS;
constexpr int kStRows = kStTY + 3;                          // y0-1 .. y0+9 (a y0 == 0 box lands one row down)
constexpr int kStPlaneBytes = kStRows * kStTX * 4;          // 5632
constexpr int kStStage = kStPlaneBytes + 2 * kStTY * 4 * 4;  // + x-halo boxes: 5888 = 46 x 128
constexpr int kStDynSmem = kStNS * kStStage + 128;          // + 128 B alignment slack
constexpr int kStThreads = 32 * (kStTY + 1);
#ifndef DYSEL_ST_PROF_ITEMS
#define DYSEL_ST_PROF_ITEMS 4
#endif
constexpr int kStProfItems = DYSEL_ST_PROF_ITEMS;   // items per CTA of a timed (profiling) copy

__device__ __forceinline__ uint32_t st_smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void st_mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "W_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra W_%=;\n\t}" ::"r"(bar),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void st_tma_3d(uint32_t dst, const CUtensorMap *tm, int c0, int c1, int c2, uint32_t bar) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(
          dst),
      "l"((uint64_t)tm), "r"(c0), "r"(c1), "r"(c2), "r"(bar)
      : "memory");
}

struct StPos {   // a ring position: stage and mbarrier phase parity
  uint32_t st, ph;
  __device__ __forceinline__ void inc() {
    if (++st == (uint32_t)kStNS) {
      st = 0;
      ph ^= 1u;
    }
  }
};

struct StItem {
  int x0, y0, z0, z1;   // tile origin, output planes [z0, z1)
  uint32_t ux, uy;      // units of the tile inside U (x, y)
};
__device__ __forceinline__ bool st_item(const dysel_slice &s, const StencilArgs &g, uint64_t it, StItem &o) {
  const uint32_t wa[3] = {4, 2, kStTZ};
  uint64_t u[3];
  if (!dysel_cta_origin(s, wa, it, u)) return false;
  o.x0 = (int)u[0] * 32;
  o.y0 = (int)u[1] * 4;
  o.z0 = (int)u[2];
  o.z1 = min(o.z0 + kStTZ, g.nz);
  o.ux = (uint32_t)(s.U[0] - u[0] < 4 ? s.U[0] - u[0] : 4);
  o.uy = (uint32_t)(s.U[1] - u[1] < 2 ? s.U[1] - u[1] : 2);
  return true;
}

// A CTA's share of the slice: whole items round-robin (item b, b + G, ...;
// concurrently running CTAs then work on neighbouring tiles of the same z
// band, in z lockstep, so the y / x / z halo planes one CTA loads are L2 hits
// for its neighbours), except the last, partial round: its item-planes are
// split evenly over all G CTAs as contiguous z pieces (2.3 items per CTA on
// 512x512x64 otherwise left the last round to a third of the machine).
// z-adjacent pieces of one tile are merged into one run (one ring fill).
struct StRun {
  int x0, y0, zs, ze;   // output planes [zs, ze) of tile (x0, y0)
  uint32_t units;
};
struct StRuns {
  uint64_t it, it_end, p, pb;
  __device__ __forceinline__ bool next(const dysel_slice &s, const StencilArgs &g, StRun &r) {
    while (it < it_end) {   // whole items, round-robin
      StItem I;
      const bool ok = st_item(s, g, it, I);
      it += gridDim.x;
      if (!ok) continue;
      r.x0 = I.x0;
      r.y0 = I.y0;
      r.zs = I.z0;
      r.ze = I.z1;
      r.units = (uint32_t)(I.z1 - I.z0) * I.ux * I.uy;
      return true;
    }
    while (p < pb) {        // the last round's plane range
      uint64_t it = p / kStTZ;
      StItem I;
      if (!st_item(s, g, it, I) || I.z0 + (int)(p - it * kStTZ) >= I.z1) {
        p = (it + 1) * kStTZ;
        continue;
      }
      r.x0 = I.x0;
      r.y0 = I.y0;
      r.zs = I.z0 + (int)(p - it * kStTZ);
      const uint64_t left = pb - it * kStTZ;
      r.ze = min(I.z0 + (int)(left < kStTZ ? left : kStTZ), I.z1);
      p = r.ze == I.z1 ? (it + 1) * kStTZ : it * kStTZ + (uint64_t)(r.ze - I.z0);
      uint64_t un = (uint64_t)(r.ze - r.zs);
      while (p < pb && p == (it + 1) * kStTZ) {   // merge the tile's next z-chunk
        StItem J;
        if (!st_item(s, g, it + 1, J) || J.x0 != r.x0 || J.y0 != r.y0 || J.z0 != r.ze) break;
        ++it;
        const uint64_t lj = pb - it * kStTZ;
        const int ze = min(J.z0 + (int)(lj < kStTZ ? lj : kStTZ), J.z1);
        un += (uint64_t)(ze - r.ze);
        r.ze = ze;
        p = ze == J.z1 ? (it + 1) * kStTZ : it * kStTZ + (uint64_t)(ze - J.z0);
      }
      r.units = (uint32_t)(un * I.ux * I.uy);
      return true;
    }
    return false;
  }
};
__device__ __forceinline__ StRuns st_runs(uint64_t n_items) {
  const uint64_t G = gridDim.x, full = n_items / G * G, P = (n_items - full) * kStTZ;
  return StRuns{blockIdx.x, full, full * kStTZ + P * blockIdx.x / G, full * kStTZ + P * (blockIdx.x + 1) / G};
}

template <bool TIMED, bool TMA>
__global__ void __launch_bounds__(kStThreads, 3)
    stencil_tma_kernel(const __grid_constant__ CUtensorMap tmP, const __grid_constant__ CUtensorMap tmH,
                       StencilArgs g, float *__restrict__ out, dysel_slice s) {
  extern __shared__ __align__(128) unsigned char st_dsmem[];
  __shared__ __align__(8) uint64_t full[kStNS], empty_[kStNS];
  __shared__ dysel_prof_smem psm;
  if (!dysel_gate_open(s)) return;
  const uint32_t wa[3] = {4, 2, kStTZ};
  const uint64_t n_items = dysel_slice_ctas(s, wa);
  if constexpr (TIMED) dysel_prof_begin(s, psm);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const uint32_t sbase = (st_smem_u32(st_dsmem) + 127u) & ~127u;
  const unsigned char *gbase = st_dsmem + (sbase - st_smem_u32(st_dsmem));
  uint32_t units = 0;
  if constexpr (!TMA) {   // fallback: the z-march column code over the same items
    StRuns R = st_runs(n_items);
    StRun I;
    while (R.next(s, g, I)) {
      if (warp > 0)
#pragma unroll 1
        for (int e = 0; e < 4; ++e)
          zmarch_column(g, out, I.x0 + 4 * lane + e, I.y0 + warp - 1, I.zs, I.ze, [](int, int) { return false; });
      units += I.units;
    }
    if constexpr (TIMED) dysel_prof_end(s, psm, units);
    return;
  }
  if (tid == 0) {
    for (int i = 0; i < kStNS; ++i) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(st_smem_u32(&full[i])));
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(st_smem_u32(&empty_[i])), "r"(kStTY));
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmP) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"((uint64_t)&tmH) : "memory");
  }
  __syncthreads();
  if (warp == 0) {
    if (lane == 0) {   // ------------------------------------- TMA producer
      uint32_t seq = 0, wst = 0, wph = 0;
      StRuns R = st_runs(n_items);
      StRun I;
      while (R.next(s, g, I)) {
        if constexpr (TIMED) dysel_prof_poll_thread(s, psm);   // dominance report only (no abort in the ring)
        const int ps = max(I.zs - 1, 0), pe = min(I.ze, g.nz - 1);
        const bool hl = I.x0 > 0, hr = I.x0 + kStTX < g.nx;
        const uint32_t bytes = (uint32_t)kStPlaneBytes - kStTX * 4 + (hl ? 128u : 0u) + (hr ? 128u : 0u);
        for (int p = ps; p <= pe; ++p, ++seq) {
          const uint32_t st = wst;
          if (seq >= (uint32_t)kStNS) st_mbar_wait(st_smem_u32(&empty_[st]), wph ^ 1u);
          if (++wst == (uint32_t)kStNS) {   // ring position (stage, phase) of the next plane
            wst = 0;
            wph ^= 1u;
          }
          const uint32_t fb = st_smem_u32(&full[st]), dst = sbase + st * kStStage;
          asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(fb), "r"(bytes) : "memory");
          // the y0 == 0 box starts at row 0 and lands one stage row down (a
          // negative box start is avoided; row y0 - 1 is not read there)
          st_tma_3d(dst + (I.y0 == 0 ? kStTX * 4 : 0), &tmP, I.x0, I.y0 == 0 ? 0 : I.y0 - 1, p, fb);
          if (hl) st_tma_3d(dst + kStPlaneBytes, &tmH, I.x0 - 4, I.y0, p, fb);
          if (hr) st_tma_3d(dst + kStPlaneBytes + kStTY * 16, &tmH, I.x0 + kStTX, I.y0, p, fb);
        }
        units += I.units;
      }
    }
  } else {   // ------------------------------------------------ consumers
    const int r = warp - 1;
    // this lane's 16 bytes of tile row r (stage row r + 1) in stage 0; x halo words
    const uint32_t lane_row = sbase + (uint32_t)(r + 1) * (kStTX * 4) + lane * 16;
    const uint32_t halo_w = sbase + kStPlaneBytes + (lane == 0 ? r * 16 + 12 : kStTY * 16 + r * 16);
    const uint32_t full0 = st_smem_u32(&full[0]), empty0 = st_smem_u32(&empty_[0]);
    const size_t sz = (size_t)g.nx * g.ny;
    uint32_t seq0 = 0;
    StRuns R = st_runs(n_items);
    StRun I;
    while (R.next(s, g, I)) {
      const int ps = max(I.zs - 1, 0), pe = min(I.ze, g.nz - 1);
      const int y = I.y0 + r, xb = I.x0 + 4 * lane;
      const bool st_ok = y < g.ny && xb < g.nx;
      const bool y_in = y > 0 && y < g.ny - 1, ex = xb > 0, ew = xb + 3 < g.nx - 1;
      const bool edge = (lane == 0 && I.x0 > 0) || (lane == 31 && I.x0 + kStTX < g.nx);
      // ring position (stage, phase) of a plane: the run's first loaded plane
      // ps sits at seq0; positions advance incrementally (no division)
      StPos prev{seq0 % kStNS, (seq0 / kStNS) & 1u}, cur = prev;
      auto wait_at = [&](const StPos &q) { st_mbar_wait(full0 + q.st * 8, q.ph); };
      auto release_at = [&](const StPos &q) {
        __syncwarp();
        if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(empty0 + q.st * 8) : "memory");
      };
      auto lds4 = [&](uint32_t addr) {
        float4 v;
        asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(addr));
        return v;
      };
      float4 zm = make_float4(0.f, 0.f, 0.f, 0.f), c;
      if (ps < I.zs) {
        wait_at(prev);
        zm = lds4(lane_row + prev.st * kStStage);
        cur.inc();
      }
      wait_at(cur);
      c = lds4(lane_row + cur.st * kStStage);
      float *orow = out + ((size_t)I.zs * g.ny + (size_t)(st_ok ? y : 0)) * g.nx + (st_ok ? xb : 0);
      for (int z = I.zs; z < I.ze; ++z) {
        StPos nxt = cur;
        nxt.inc();
        float4 zp = make_float4(0.f, 0.f, 0.f, 0.f);
        if (z + 1 <= pe) {
          wait_at(nxt);
          zp = lds4(lane_row + nxt.st * kStStage);
        }
        const uint32_t so = cur.st * kStStage;
        const float4 ym = lds4(lane_row + so - kStTX * 4), yp = lds4(lane_row + so + kStTX * 4);
        float xl = __shfl_up_sync(0xffffffffu, c.w, 1), xr = __shfl_down_sync(0xffffffffu, c.x, 1);
        if (edge) {
          float h;
          asm volatile("ld.shared.f32 %0, [%1];" : "=f"(h) : "r"(halo_w + so));
          if (lane == 0) xl = h; else xr = h;
        }
        // all four points computed branch-free, boundary points select the centre
        const bool in_yz = y_in && z > 0 && z < g.nz - 1;
        const float vx = st_point(c.x, zm.x, zp.x, ym.x, yp.x, xl, c.y, g.c0, g.c1);
        const float vy = st_point(c.y, zm.y, zp.y, ym.y, yp.y, c.x, c.z, g.c0, g.c1);
        const float vz = st_point(c.z, zm.z, zp.z, ym.z, yp.z, c.y, c.w, g.c0, g.c1);
        const float vw = st_point(c.w, zm.w, zp.w, ym.w, yp.w, c.z, xr, g.c0, g.c1);
        float4 o;
        o.x = (in_yz && ex) ? vx : c.x;
        o.y = in_yz ? vy : c.y;
        o.z = in_yz ? vz : c.z;
        o.w = (in_yz && ew) ? vw : c.w;
        if (st_ok) *reinterpret_cast<float4 *>(orow) = o;
        if (z - 1 >= ps) release_at(prev);
        prev = cur;
        cur = nxt;
        zm = c;
        c = zp;
        orow += sz;
      }
      // cur = plane ze, prev = plane ze - 1: release both (ze if it was loaded)
      release_at(prev);
      if (pe == I.ze) release_at(cur);
      seq0 += (uint32_t)(pe - ps + 1);
    }
  }
  if constexpr (TIMED) dysel_prof_end(s, psm, units);
}

static uint64_t g_stencil_wave[DYSEL_STENCIL_NVARIANTS] = {0, 0, 0};   // occupancy x #SM

static PFN_cuTensorMapEncodeTiled_v12000 st_encoder() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (PFN_cuTensorMapEncodeTiled_v12000)p;
    cudaGetLastError();
  }
  return fn;
}

// V2's two 3-D maps over `in` ([nz][ny][nx] fp32): the {128, 10, 1} plane box
// and the {4, 8, 1} x-halo box; zero fill out of bounds.  False when the
// layout does not allow TMA (nx % 4, alignment) -> the column fallback.
static bool stencil_maps(const StencilArgs &g, const float *out, CUtensorMap *mp, CUtensorMap *mh) {
  if (g.nx % 4 != 0 || ((uintptr_t)g.in & 15) != 0 || ((uintptr_t)out & 15) != 0) return false;
  auto enc = st_encoder();
  if (!enc) return false;
  const cuuint64_t dims[3] = {(cuuint64_t)g.nx, (cuuint64_t)g.ny, (cuuint64_t)g.nz};
  const cuuint64_t strides[2] = {(cuuint64_t)g.nx * 4, (cuuint64_t)g.nx * g.ny * 4};
  const cuuint32_t es[3] = {1, 1, 1};
  const cuuint32_t bp[3] = {kStTX, kStTY + 2, 1}, bh[3] = {4, kStTY, 1};
  void *base = const_cast<float *>(g.in);
  return enc(mp, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, base, dims, strides, bp, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
             CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS &&
         enc(mh, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, base, dims, strides, bh, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
             CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

template <bool TIMED, bool TMA>
static void launch_tma_tile(const StencilArgs &g, float *out, const dysel_slice &s, uint64_t ctas, cudaStream_t st,
                            const CUtensorMap &mp, const CUtensorMap &mh) {
  static bool attr = false;   // > 48 KB of dynamic shared memory needs the opt-in once
  if (!attr) {
    cudaFuncSetAttribute(stencil_tma_kernel<TIMED, TMA>, cudaFuncAttributeMaxDynamicSharedMemorySize, kStDynSmem);
    attr = true;
  }
  stencil_tma_kernel<TIMED, TMA><<<(unsigned)ctas, kStThreads, TMA ? kStDynSmem : 0, st>>>(mp, mh, g, out, s);
}

template <int VID>
static dysel_status stencil_variant_fn(const dysel_slice *s, void *const *args, void *stream, void *) {
  const StencilArgs &g = *(const StencilArgs *)args[1];
  float *out = (float *)args[0];
  cudaStream_t st = (cudaStream_t)stream;
  static const uint32_t WA[3][3] = {{1, 1, 1}, {1, 1, 64}, {4, 2, kStTZ}};
  uint64_t ctas = dysel_slice_ctas(*s, WA[VID]);
  if (ctas == 0) return DYSEL_OK;
  // gated remainder: one persistent wave (a variant that lost the selection
  // then costs one wave of exiting CTAs instead of one per tile: 130K for base)
  if (s->gate && !s->timer && !s->gate_full_grid && g_stencil_wave[VID] > 0)
    ctas = std::min<uint64_t>(ctas, g_stencil_wave[VID]);
  if constexpr (VID == DYSEL_STENCIL_BASE)
    stencil_base_kernel<<<(unsigned)ctas, 128, 0, st>>>(g, out, *s);
  else if constexpr (VID == DYSEL_STENCIL_ZMARCH) {
    if (s->timer)
      stencil_zmarch_kernel<true><<<(unsigned)ctas, 128, 0, st>>>(g, out, *s);
    else
      stencil_zmarch_kernel<false><<<(unsigned)ctas, 128, 0, st>>>(g, out, *s);
  } else {
    // V2 is persistent in every launch: untimed, one wave (each CTA an equal
    // plane range, >= 4 planes); a timed (profiling) copy runs kStProfItems
    // items per CTA so its cycles include the ring's steady state, not one
    // cold fill per item (ctas_total follows its grid)
    dysel_slice sl = *s;
    if (s->timer) {
      ctas = (ctas + kStProfItems - 1) / kStProfItems;
      sl.ctas_total = (uint32_t)ctas;
    } else if (g_stencil_wave[VID] > 0) {
      ctas = std::min<uint64_t>((ctas * kStTZ + 3) / 4, g_stencil_wave[VID]);
    }
    CUtensorMap mp, mh;
    memset(&mp, 0, sizeof(mp));
    memset(&mh, 0, sizeof(mh));
    const bool tma = stencil_maps(g, out, &mp, &mh);
    if (s->timer)
      tma ? launch_tma_tile<true, true>(g, out, sl, ctas, st, mp, mh)
          : launch_tma_tile<true, false>(g, out, sl, ctas, st, mp, mh);
    else
      tma ? launch_tma_tile<false, true>(g, out, sl, ctas, st, mp, mh)
          : launch_tma_tile<false, false>(g, out, sl, ctas, st, mp, mh);
  }
  return cudaGetLastError() == cudaSuccess ? DYSEL_OK : DYSEL_ERR_CUDA;
}

static const dysel_variant_fn kStencilFns[DYSEL_STENCIL_NVARIANTS] = {
    stencil_variant_fn<0>, stencil_variant_fn<1>, stencil_variant_fn<2>};

dysel_status stencil_register(dysel_ctx *ctx) {
  static const int sb[1] = {0};
  int o[3] = {0, 0, 0};
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o[0], stencil_base_kernel, 128, 0);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o[1], stencil_zmarch_kernel<false>, 128, 0);
  cudaFuncSetAttribute(stencil_tma_kernel<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, kStDynSmem);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o[2], stencil_tma_kernel<false, true>, kStThreads, kStDynSmem);
  cudaGetLastError();
  const uint64_t n = (uint64_t)ctx->n_sm;
  for (int i = 0; i < DYSEL_STENCIL_NVARIANTS; ++i) g_stencil_wave[i] = (uint64_t)o[i] * n;
  dysel_variant v[DYSEL_STENCIL_NVARIANTS] = {
      {"base", kStencilFns[0], {1, 1, 1}, sb, 1, 0, nullptr, (uint64_t)o[0] * n},
      {"zmarch64", kStencilFns[1], {1, 1, 64}, sb, 1, 0, nullptr, (uint64_t)o[1] * n},
      {"tma128x8x16", kStencilFns[2], {4, 2, kStTZ}, sb, 1, 0, nullptr, (uint64_t)o[2] * n},
  };
  // initial version (A-5): the TMA tile (the B200-first design:
  // planes streamed into shared memory, the fastest on grids larger than L2).
  // A grid whose items fit in one wave of it is not profiled (reading A-3b).
  DYSEL_TRY(dysel_register_variants(ctx, kStencilSig, v, DYSEL_STENCIL_NVARIANTS, DYSEL_STENCIL_TILED));
  mark_builtin(ctx, kStencilSig);
  return DYSEL_OK;
}

static dysel_status stencil_check(dysel_ctx *ctx, int nx, int ny, int nz, const float *in, float *out) {
  if (nx < 0 || ny < 0 || nz < 0 || ((int64_t)nx * ny * nz > 0 && (!in || !out)) || in == out) {
    set_error(ctx, "dysel_stencil: invalid arguments (in and out must not alias)");
    return DYSEL_ERR_INVALID;
  }
  return DYSEL_OK;
}

}  // namespace dysel

using namespace dysel;

extern "C" {

constexpr uint64_t kStencilMinProfBytes = 650ull * 1000 * 1000;   // 2 x 50 us x 6.5 TB/s (reading A-3c)

dysel_status dysel_stencil(dysel_ctx *ctx, int nx, int ny, int nz, float c0, float c1, const float *d_in,
                           float *d_out, float f, uint32_t mode, void *stream, dysel_report *rep) {
  if (!ctx) return DYSEL_ERR_INVALID;
  DYSEL_TRY(stencil_check(ctx, nx, ny, nz, d_in, d_out));
  if (rep) rep->n_slices = 0;
  if ((int64_t)nx * ny * nz == 0) return DYSEL_OK;
  StencilArgs g{nx, ny, nz, c0, c1, d_in};
  const uint64_t U[3] = {(uint64_t)(nx + 31) / 32, (uint64_t)(ny + 3) / 4, (uint64_t)nz};
  void *args[2] = {d_out, &g};
  const size_t sbytes[1] = {(size_t)nx * ny * nz * sizeof(float)};
  const std::string key = std::string(kStencilSig) + "#" + std::to_string(nx) + "x" + std::to_string(ny) + "x" +
                          std::to_string(nz);
  // reading A-3c for the stencil pool: the selection is published ~45-50 us
  // into a profiled call (each profiling CTA streams 4 items); a sweep whose
  // in + out bytes take less than twice that at HBM speed (~650 MB) cannot
  // recover it in one call -- run the cached / initial version (FORCE_PROFILE
  // overrides; iterated sweeps amortise one profile with the activation flag)
  if (!(mode & DYSEL_FORCE_PROFILE) && 2ull * sbytes[0] < kStencilMinProfBytes) mode |= DYSEL_NO_PROFILE;
  return launch_keyed(ctx, kStencilSig, key.c_str(), U, f, mode, args, 2, sbytes, stream, rep);
}

dysel_status dysel_stencil_variant(dysel_ctx *ctx, int variant_id, int nx, int ny, int nz, float c0, float c1,
                                   const float *d_in, float *d_out, void *stream) {
  if (!ctx || variant_id < 0 || variant_id >= DYSEL_STENCIL_NVARIANTS) {
    set_error(ctx, "dysel_stencil_variant: invalid variant");
    return DYSEL_ERR_INVALID;
  }
  DYSEL_TRY(stencil_check(ctx, nx, ny, nz, d_in, d_out));
  if ((int64_t)nx * ny * nz == 0) return DYSEL_OK;
  StencilArgs g{nx, ny, nz, c0, c1, d_in};
  void *args[2] = {d_out, &g};
  dysel_slice s;
  memset(&s, 0, sizeof(s));
  const uint32_t gg[3] = {4, 2, 64};
  const uint64_t U[3] = {(uint64_t)(nx + 31) / 32, (uint64_t)(ny + 3) / 4, (uint64_t)nz};
  for (int d = 0; d < 3; ++d) {
    s.g[d] = gg[d];
    s.U[d] = U[d];
    s.G[d] = (uint32_t)((U[d] + gg[d] - 1) / gg[d]);
  }
  s.granule_count = (uint64_t)s.G[0] * s.G[1] * s.G[2];
  s.granule_stride = 1;
  s.role = DYSEL_ROLE_BATCH;
  s.variant = variant_id;
  DYSEL_TRY(kStencilFns[variant_id](&s, args, stream, nullptr));
  return check_launch(ctx, "stencil full-grid variant");
}

}  // extern "C"
