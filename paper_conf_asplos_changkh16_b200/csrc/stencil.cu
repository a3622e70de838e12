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
//   V2 smem-tiled  wa (2, 1, 64)   64 x 4 tile, 2 points per thread along x, z-march,
//                                  the plane's x / y neighbours staged in shared memory
// The LCM granule is (2, 1, 64) units: the slice planner's safe point.
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
    if (((z - z0) & 15) == 15 - (kZq - 1) && poll()) return;
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
                    [&]() { return dysel_prof_poll(s, psm) && s.role == DYSEL_ROLE_SANDBOX; });
    else
      zmarch_column(g, out, x, y, z0, z1, []() { return false; });
    units = (uint32_t)(z1 - z0);
  }
  }
  if constexpr (TIMED) dysel_prof_end(s, psm, units);
}

// ------------------------------------------------------------------- V2
// 64 x 4 tile, thread (tx, ty) owns x = x0 + tx and x0 + 32 + tx.  Each
// z-plane: stage the (64+2) x (4+2) plane (with halo) in shared memory, then
// every point reads its 4 in-plane neighbours from it; z +-1 stay in registers.
__global__ void __launch_bounds__(128) stencil_tiled_kernel(StencilArgs g, float *__restrict__ out, dysel_slice s) {
  __shared__ dysel_prof_smem psm;
  __shared__ float pl[4 + 2][64 + 2 + 2];   // +2 padding columns (bank spread)
  if (!dysel_gate_open(s)) return;
  const uint32_t wa[3] = {2, 1, 64};
  const bool persistent = s.timer == nullptr && s.gate != nullptr;   // gated remainder: one wave walks the tiles
  const uint64_t n_cta = persistent ? dysel_slice_ctas(s, wa) : (uint64_t)blockIdx.x + 1;
  dysel_prof_begin(s, psm);
  uint32_t units = 0;
  for (uint64_t cta = blockIdx.x; cta < n_cta; cta += gridDim.x) {
  uint64_t u[3];
  const bool ok = dysel_cta_origin(s, wa, cta, u);
  if (ok) {
    const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
    const int x0 = (int)u[0] * 32, y0 = (int)u[1] * 4;
    const int z0 = (int)u[2], z1 = min(z0 + 64, g.nz);
    const size_t sy = (size_t)g.nx, sz = (size_t)g.nx * g.ny;
    const int y = y0 + ty;
    int xs[2] = {x0 + tx, x0 + 32 + tx};
    bool colv[2], inner[2];
    float zm[2], c[2];
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      colv[h] = xs[h] < g.nx && y < g.ny;
      inner[h] = colv[h] && xs[h] > 0 && y > 0 && xs[h] < g.nx - 1 && y < g.ny - 1;
      const size_t i = (size_t)z0 * sz + (size_t)y * sy + xs[h];
      zm[h] = (colv[h] && z0 > 0) ? __ldg(g.in + i - sz) : 0.0f;
      c[h] = colv[h] ? __ldg(g.in + i) : 0.0f;
    }
    for (int z = z0; z < z1; ++z) {
      if (((z - z0) & 15) == 15 && dysel_prof_poll(s, psm) && s.role == DYSEL_ROLE_SANDBOX) break;
      // stage plane z: interior of the tile from registers, halo from global
      __syncthreads();   // previous plane's readers are done
#pragma unroll
      for (int h = 0; h < 2; ++h) pl[ty + 1][h * 32 + tx + 1] = c[h];
      const size_t pz = (size_t)z * sz;
      if (ty == 0 || ty == 3) {   // y halo rows (64 wide)
        const int yy = ty == 0 ? y0 - 1 : y0 + 4;
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int xx = x0 + h * 32 + tx;
          pl[ty == 0 ? 0 : 5][h * 32 + tx + 1] =
              (yy >= 0 && yy < g.ny && xx < g.nx) ? __ldg(g.in + pz + (size_t)yy * sy + xx) : 0.0f;
        }
      }
      if (tx == 0) {   // x halo columns of row ty
        const int xl = x0 - 1, xr = x0 + 64;
        pl[ty + 1][0] = (xl >= 0 && y < g.ny) ? __ldg(g.in + pz + (size_t)y * sy + xl) : 0.0f;
        pl[ty + 1][65] = (xr < g.nx && y < g.ny) ? __ldg(g.in + pz + (size_t)y * sy + xr) : 0.0f;
      }
      __syncthreads();
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const size_t i = pz + (size_t)y * sy + xs[h];
        const float zp = (colv[h] && z + 1 < g.nz) ? __ldg(g.in + i + sz) : 0.0f;
        if (colv[h]) {
          const int lx = h * 32 + tx + 1;
          out[i] = (inner[h] && z > 0 && z < g.nz - 1)
                       ? st_point(c[h], zm[h], zp, pl[ty][lx], pl[ty + 2][lx], pl[ty + 1][lx - 1], pl[ty + 1][lx + 1],
                                  g.c0, g.c1)
                       : c[h];
        }
        zm[h] = c[h];
        c[h] = zp;
      }
    }
    units = (uint32_t)((z1 - z0) * ((x0 + 32 < g.nx) ? 2 : 1));
  }
  __syncthreads();   // the plane buffer is reused by the next tile
  }
  dysel_prof_end(s, psm, units);
}

static uint64_t g_stencil_wave[DYSEL_STENCIL_NVARIANTS] = {0, 0, 0};   // occupancy x #SM
template <int VID>
static dysel_status stencil_variant_fn(const dysel_slice *s, void *const *args, void *stream, void *) {
  const StencilArgs &g = *(const StencilArgs *)args[1];
  float *out = (float *)args[0];
  cudaStream_t st = (cudaStream_t)stream;
  static const uint32_t WA[3][3] = {{1, 1, 1}, {1, 1, 64}, {2, 1, 64}};
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
  }
  else
    stencil_tiled_kernel<<<(unsigned)ctas, 128, 0, st>>>(g, out, *s);
  return cudaGetLastError() == cudaSuccess ? DYSEL_OK : DYSEL_ERR_CUDA;
}

static const dysel_variant_fn kStencilFns[DYSEL_STENCIL_NVARIANTS] = {
    stencil_variant_fn<0>, stencil_variant_fn<1>, stencil_variant_fn<2>};

dysel_status stencil_register(dysel_ctx *ctx) {
  static const int sb[1] = {0};
  int o[3] = {0, 0, 0};
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o[0], stencil_base_kernel, 128, 0);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o[1], stencil_zmarch_kernel<false>, 128, 0);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o[2], stencil_tiled_kernel, 128, 0);
  cudaGetLastError();
  const uint64_t n = (uint64_t)ctx->n_sm;
  for (int i = 0; i < DYSEL_STENCIL_NVARIANTS; ++i) g_stencil_wave[i] = (uint64_t)o[i] * n;
  dysel_variant v[DYSEL_STENCIL_NVARIANTS] = {
      {"base", kStencilFns[0], {1, 1, 1}, sb, 1, 0, nullptr, (uint64_t)o[0] * n},
      {"zmarch64", kStencilFns[1], {1, 1, 64}, sb, 1, 0, nullptr, (uint64_t)o[1] * n},
      {"tiled64x4_zmarch64", kStencilFns[2], {2, 1, 64}, sb, 1, 0, nullptr, (uint64_t)o[2] * n},
  };
  // initial version (A-5): the z-march (2.5-D blocking, the
  // standard first choice for a 3-D stencil on a GPU).  A grid of it that
  // fits in one wave is not profiled (reading A-3b).
  return dysel_register_variants(ctx, kStencilSig, v, DYSEL_STENCIL_NVARIANTS, DYSEL_STENCIL_ZMARCH);
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
  const uint32_t gg[3] = {2, 1, 64};
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
