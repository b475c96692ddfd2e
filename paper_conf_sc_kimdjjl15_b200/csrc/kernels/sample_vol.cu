// sample_vol.cu -- TMA-staged trilinear read of one-channel 32-bit float 3D
// images under separable maps (config 3: 512^3 R32F, CLAMP_TO_EDGE, LINEAR).
//
// Steps a3-a7 of the read built-in ([CL1.2 §8.1-8.2]) for every output of a
// 512 x 12 x walk box, with the texel fetches (a5: through the CLImage
// pointer) moved by the TMA engine:
//   * a persistent grid of CTAs (one per SM) strides over output tiles; each
//     CTA has one PRODUCER warp and twelve CONSUMER warps (4 across x, 3 down
//     y; 123 registers each, no spill);
//   * per output slice the producer stages the tile's texel footprint in that
//     slice -- a (516 x 13)-texel box starting at the tile's first tap (i0 of
//     its first column rounded down to 16 bytes, and of its first row) -- in a
//     shared-memory ring: one cp.async.bulk per box row (one per lane),
//     completing on a `full` mbarrier.  (B2CL_VOL_BULK=0 B2CL_VOL_XW=1
//     builds the 132 x 17 variant that moves each box with one
//     cp.async.bulk.tensor.3d; on B200 it measured 196 us against 186 us
//     for the row copies at config 3.)
//   * consumers x-blend each staged texel row once, y-blend neighbouring rows,
//     keep the (x,y)-blended slice in registers and z-blend it with the next
//     one, then release the stage on an `empty` mbarrier.
// Bytes in flight are the ring (STAGES x 26.8 KB per CTA), independent of
// registers -- the limit of the register-pipelined walk kernels.
//
// Exactness.  Every output is computed with the operations and operands of
// linear_at (read.cuh): per texel row lerp1(a, 1-a, T[i0], T[i1]), then
// lerp1(b, ..) of the rows j0, j1, then lerp1(g, ..) of the slices k0, k1,
// with the per-axis AxL of axis_l -- so the results are bit-identical to the
// other grid kernels (the parity tests run all of them).  A tile with a tap
// outside its box (non-unit maps, fp rounding at a tile edge) is not staged:
// the producer warp and the consumer warps test the same columns and rows
// (vol_in_window) and agree, and the consumers read that tile's taps from
// global memory (linear_at).  Slices are consumed in walk order: the map's z coordinate must
// be non-decreasing in the output z (A[10] >= 0, host check), so with the
// monotone CLAMP_TO_EDGE addressing the slice pair (k0, k1) only moves
// forward and each slice is staged once per tile.
#include <cudaTypedefs.h>

#include <cmath>
#include <cstring>
#include <mutex>

#include "../device/read.cuh"
#include "launch.h"

namespace b2cl {
using namespace dev;

#ifndef B2CL_VOL_PF
#define B2CL_VOL_PF 0  // L2 prefetch distance in slices of the stencil row copies (0: none; 2 / 4 / 8 measured 210 / 211 / 216 vs 184 us)
#endif
#ifndef B2CL_VOLR_PF
#define B2CL_VOLR_PF 0  // L2 prefetch distance in slices of the rotated boxes (0: none; 2 / 4 / 8 measured 242.6 / 243.7 / 244.7 vs 240.9 us)
#endif
#ifndef B2CL_VOL_BULK
#define B2CL_VOL_BULK 1
#endif
#ifndef B2CL_VOL_NS
#define B2CL_VOL_NS 6  // (5 - 8 within 0.5 us with one CTA per SM; 3 was best at two CTAs per SM)
#endif
#ifndef B2CL_VOL_SETUP
#define B2CL_VOL_SETUP 0.0  // the stencil kernel's chunk cost for vol_plan (0: balanced rounds)
#endif
#ifndef B2CL_VOL_MIN_STEPS
#define B2CL_VOL_MIN_STEPS 8
#endif
#ifndef B2CL_VOL_MINB
#define B2CL_VOL_MINB 1  // one CTA of 13 warps per SM: 123 registers, no spill (two 9-warp CTAs: 96 and a spill, 183.7 vs 176.7 us)
#endif
#ifndef B2CL_VOL_XW
#define B2CL_VOL_XW 4
#endif
constexpr int VOL_XW = B2CL_VOL_XW;       // consumer warps across x (1: TMA boxes; 4: row copies)
static_assert(VOL_XW == 1 || B2CL_VOL_BULK, "a TMA box is at most 256 texels wide");
constexpr int VT_W = 128 * VOL_XW;        // output columns per tile (32 lanes x 4 per warp)
#ifndef B2CL_VOL_YW
#define B2CL_VOL_YW 3
#endif
constexpr int VOL_YW = B2CL_VOL_YW;       // consumer warps down y
constexpr int VOL_CW = VOL_XW * VOL_YW;   // consumer warps
constexpr int VT_H = 4 * VOL_YW;          // output rows per tile (4 per warp)
constexpr int VB_W = VT_W + 4;            // staged texel columns (TW + 1 taps + up to 3 of 16-B alignment)
constexpr int VB_H = VT_H + 1;            // staged texel rows
constexpr int VB_BYTES = VB_W * VB_H * 4; // one TMA box
constexpr int VB_STRIDE = (VB_BYTES + 127) / 128 * 128;
constexpr int VOL_NS = B2CL_VOL_NS;       // ring stages
constexpr int VOL_MIN_STEPS = B2CL_VOL_MIN_STEPS;  // fewest column steps per CTA
constexpr int VOL_THREADS = 32 * (VOL_CW + 1);  // consumer warps + 1 producer warp
static_assert(VT_H < 32, "the producer's lanes cover the tile's rows");

struct VolTiles {
  int ntx, nty, nzc;  // tiles along x and y, slice chunks along z
  int walk;           // output slices per chunk
  int vst;            // 1: 16-byte output stores allowed (ow % 4 == 0, out 16-B aligned)
};

__device__ __forceinline__ uint32_t vol_smem(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

#ifndef B2CL_VOL_HINT
#define B2CL_VOL_HINT 1000  // mbarrier try_wait suspend hint (ns): a waiting warp sleeps instead of spinning (C3 rotated 240.7 -> 236.6 us; ncu had 12 % of its instructions in the spin loop)
#endif
__device__ __forceinline__ void vol_wait(uint64_t* bar, uint32_t parity) {
  const uint32_t b = vol_smem(bar);
  uint32_t done;
  do {
#if B2CL_VOL_HINT
    asm volatile(
        "{ .reg .pred P; mbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2, %3; selp.u32 %0, 1, 0, P; }"
        : "=r"(done)
        : "r"(b), "r"(parity), "r"(B2CL_VOL_HINT)
        : "memory");
#else
    asm volatile(
        "{ .reg .pred P; mbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2; selp.u32 %0, 1, 0, P; }"
        : "=r"(done)
        : "r"(b), "r"(parity)
        : "memory");
#endif
  } while (!done);
}

template <class C>
__device__ __forceinline__ AxL vol_axis(const SampleParams& p, int a, int o, int idx, int n) {
  // coordinate of output index `idx` (region origin o) on a separable axis:
  // A[a] * idx + A[a + 2 or 3]: the same two ops as k_sample_grid_sep
  return axis_l<C>(p.smp, __fadd_rn(__fmul_rn(p.A[a], __int2float_rn(o + idx)), p.A[a == 0 ? 3 : (a == 5 ? 7 : 11)]), n);
}

// Do the taps of columns xc..xc+3 and of row yr (those inside the output
// region) fall inside the box staged at (xb, yb)?  A tile is staged only if
// this holds for all its columns and rows (decided identically by the
// producer warp and the consumer warps).
#ifndef B2CL_VOL_FASTONLY
#define B2CL_VOL_FASTONLY 1
#endif
template <class C>
__device__ __forceinline__ bool vol_in_window(const SampleParams& p, int xc, int yr, int xb, int yb, bool chain_next) {
  bool ok = true;
#if B2CL_VOL_FASTONLY
  // the staged path's only form: the 4 columns' i0 are unit-stride from a
  // 16-byte aligned slot and i1 = i0 + 1 for the first three (the fourth
  // column's i1 is read from its own slot), the warp's rows chain (j1 of a
  // row is j0 of the next), every tap inside the box
  AxL a[4];
#pragma unroll
  for (int u = 0; u < 4; ++u) a[u] = vol_axis<C>(p, 0, p.ox, xc + u, p.im.w);
  const int c0 = a[0].i0 - xb;
  ok = c0 >= 0 && (c0 & 3) == 0 && c0 + 3 < VB_W && a[3].i1 - xb >= 0 && a[3].i1 - xb < VB_W;
#pragma unroll
  for (int u = 0; u < 4; ++u) ok = ok && a[u].i0 == a[0].i0 + u && (u == 3 || a[u].i1 == a[u].i0 + 1);
  const AxL r0 = vol_axis<C>(p, 5, p.oy, yr, p.im.h);
  ok = ok && r0.i0 - yb >= 0 && r0.i0 - yb < VB_H && r0.i1 - yb >= 0 && r0.i1 - yb < VB_H;
  if (chain_next) ok = ok && vol_axis<C>(p, 5, p.oy, yr + 1, p.im.h).i0 == r0.i1;
#else
  (void)chain_next;
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    if (xc + u < p.ow) {
      const AxL a = vol_axis<C>(p, 0, p.ox, xc + u, p.im.w);
      ok = ok && a.i0 - xb >= 0 && a.i0 - xb < VB_W && a.i1 - xb >= 0 && a.i1 - xb < VB_W;
    }
  }
  if (yr < p.oh) {
    const AxL a = vol_axis<C>(p, 5, p.oy, yr, p.im.h);
    ok = ok && a.i0 - yb >= 0 && a.i0 - yb < VB_H && a.i1 - yb >= 0 && a.i1 - yb < VB_H;
  }
#endif
  return ok;
}

// Work split.  Tiles are (tx, ty, zc): VT_W x VT_H output columns/rows and a
// chunk of `walk` output slices, ordered tx fastest, then ty, then zc, and
// dealt round-robin to a persistent grid, so the CTAs resident at any time
// read neighbouring boxes of the same slices (DRAM pages and the shared halo
// rows stay hot).  The host picks the chunk count as a multiple of
// G / gcd(G, tiles per slice plane) so every CTA gets the same number of tiles.
struct VolSeg {
  int tx, ty, w0, nst;  // tile column, first output slice, steps
};

__device__ __forceinline__ VolSeg vol_seg(const SampleParams& p, const VolTiles& tl, int t) {
  VolSeg q;
  q.tx = t % tl.ntx;
  const int r = t / tl.ntx;
  q.ty = r % tl.nty;
  q.w0 = (r / tl.nty) * tl.walk;
  q.nst = min(tl.walk, p.od - q.w0);
  return q;
}

template <class C>
__global__ void __launch_bounds__(VOL_THREADS, B2CL_VOL_MINB)
    k_sample_grid_vol(const SampleParams p, const VolTiles tl, const __grid_constant__ CUtensorMap tmap) {
  static_assert(C::dims == 3 && C::nch == 1 && C::type == T_FLOAT, "R32F-type 3D images");
  // row copies stage only texels inside the image: exact when no tap leaves it
  static_assert(!B2CL_VOL_BULK || C::addr == A_CTE, "row copies need CLAMP_TO_EDGE");
  extern __shared__ __align__(128) unsigned char vol_buf[];
  __shared__ uint64_t full[VOL_NS], empty[VOL_NS];
  __shared__ float4 rowtab[VOL_CW][4];  // per consumer warp and row: {b, 1-b, slot j0, slot j1}
  const Image& im = p.im;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < VOL_NS; ++s) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(vol_smem(&full[s])) : "memory");
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(vol_smem(&empty[s])), "r"(VOL_CW) : "memory");
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  __syncthreads();
  const int ntiles = tl.ntx * tl.nty * tl.nzc;
  constexpr int NONE = -2147483647 - 1;

  if (warp == VOL_CW) {  // ------------------------------------------------ producer
    if (lane == 0) asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmap)) : "memory");
    int s = 0;
    uint32_t ph = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
      const VolSeg q = vol_seg(p, tl, t);
      const int xb = vol_axis<C>(p, 0, p.ox, q.tx * VT_W, im.w).i0 & ~3;  // 16-B aligned box start
      const int yb = vol_axis<C>(p, 5, p.oy, q.ty * VT_H, im.h).i0;
      // the consumers' tile decision, evaluated the same way by this warp
      bool win = true;
#pragma unroll
      for (int m = 0; m < VOL_XW; ++m)
        win = win && vol_in_window<C>(p, q.tx * VT_W + 128 * m + 4 * lane, q.ty * VT_H + lane % VT_H, xb, yb,
                                      (lane % VT_H & 3) != 3);
      if (!__all_sync(0xffffffffu, win)) continue;
#if !B2CL_VOL_BULK
      if (lane != 0) continue;
#endif
      int kA = NONE, kB = NONE;
      for (int w = 0; w < q.nst; ++w) {
        const AxL az = vol_axis<C>(p, 10, p.oz, q.w0 + w, im.d);
        // the slices a step stages: lo unless held, then hi unless held
        const bool need0 = !(az.i0 == kA || az.i0 == kB);
        const bool need1 = !(az.i1 == az.i0 || (!need0 && az.i1 == kB));  // the consumers' rule
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          if (!(h ? need1 : need0)) continue;
          const int k = h ? az.i1 : az.i0;
          const uint32_t fb = vol_smem(&full[s]);
#if B2CL_VOL_BULK
          // one plain bulk copy per box row (lanes 0..16), rows inside the
          // image only, each clipped to its row pitch (CLAMP_TO_EDGE: the
          // taps never reach the unfilled parts)
          const int nrow = min(VB_H, im.h - yb);
          const uint32_t rb = (uint32_t)min((uint64_t)VB_W * 4u, im.rp - (uint64_t)xb * 4u);
          if (lane == 0) {
            vol_wait(&empty[s], ph ^ 1u);
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(fb), "r"(rb * nrow)
                         : "memory");
          }
          __syncwarp();
          if (lane < nrow)
            asm volatile(
                "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                    vol_smem(vol_buf + s * VB_STRIDE + lane * VB_W * 4)),
                "l"(im.ptr + (uint64_t)k * im.sp + (uint64_t)(yb + lane) * im.rp + (uint64_t)xb * 4u), "r"(rb), "r"(fb)
                : "memory");
#if B2CL_VOL_PF
          // warm L2 with the same rows B2CL_VOL_PF slices ahead
          if (lane < nrow && k + B2CL_VOL_PF < im.d)
            asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(
                             im.ptr + (uint64_t)(k + B2CL_VOL_PF) * im.sp + (uint64_t)(yb + lane) * im.rp +
                             (uint64_t)xb * 4u),
                         "r"(rb)
                         : "memory");
#endif
#else
          vol_wait(&empty[s], ph ^ 1u);
          asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(fb), "r"(VB_BYTES)
                       : "memory");
          asm volatile(
              "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
              " [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(vol_smem(vol_buf + s * VB_STRIDE)),
              "l"(reinterpret_cast<uint64_t>(&tmap)), "r"(xb), "r"(yb), "r"(k), "r"(fb)
              : "memory");
#endif
          if (++s == VOL_NS) { s = 0; ph ^= 1u; }
        }
        kA = az.i0;
        kB = az.i1;
      }
    }
    return;
  }

  // --------------------------------------------------------------- consumers
  int s = 0;
  uint32_t ph = 0;
  for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
    const VolSeg q = vol_seg(p, tl, t);
    const int xt = q.tx * VT_W, yt = q.ty * VT_H;
    const int xb = vol_axis<C>(p, 0, p.ox, xt, im.w).i0 & ~3;  // as the producer's
    const int yb = vol_axis<C>(p, 5, p.oy, yt, im.h).i0;
    // this thread: columns xt + 4*lane + (0..3), rows yt + 4*warp + (0..3)
    const int xc = xt + 128 * (warp % VOL_XW) + 4 * lane, yr = yt + 4 * (warp / VOL_XW);
    // tile decision: every consumer thread tests its columns and row
    // threadIdx.x % VT_H (so the consumer threads cover the tile's rows as the producer's lanes do)
    int fast = vol_in_window<C>(p, xc, yt + threadIdx.x % VT_H, xb, yb, (threadIdx.x % VT_H & 3) != 3);
    asm volatile("{ .reg .pred P, Q; setp.ne.s32 P, %1, 0; bar.red.and.pred Q, 1, %2, P; selp.s32 %0, 1, 0, Q; }"
                 : "=r"(fast) : "r"(fast), "n"(32 * VOL_CW) : "memory");
    if (!fast) {  // the taps directly (linear_at), no staging for this tile
#pragma unroll 1
      for (int w = 0; w < q.nst; ++w) {
        const int z = q.w0 + w;
        const AxL az = vol_axis<C>(p, 10, p.oz, z, im.d);
#pragma unroll 1
        for (int r = 0; r < 4; ++r) {
          const int y = yr + r;
          if (y >= p.oh) break;
          const AxL ay = vol_axis<C>(p, 5, p.oy, y, im.h);
          const char* rows[4] = {row_ptr<C>(im, ay.i0, az.i0), row_ptr<C>(im, ay.i1, az.i0),
                                 row_ptr<C>(im, ay.i0, az.i1), row_ptr<C>(im, ay.i1, az.i1)};
          const bool rok[4] = {ay.ok0 && az.ok0, ay.ok1 && az.ok0, ay.ok0 && az.ok1, ay.ok1 && az.ok1};
#pragma unroll 1
          for (int u = 0; u < 4; ++u) {
            if (xc + u >= p.ow) break;
            uint32_t res[4];
            linear_at<C>(p, rows, rok, vol_axis<C>(p, 0, p.ox, xc + u, im.w), ay.a, ay.oma, az.a, az.oma, res, 1);
            __stcs(reinterpret_cast<float*>(p.out) + ((uint64_t)z * p.oh + y) * p.ow + xc + u,
                   __uint_as_float(res[0]));
          }
        }
      }
      continue;
    }
    // x axis per thread; the warp's 4 rows (warp-uniform) in shared memory
    AxL ax[4];
    int sl[4];  // staged column slots of tap i0 | i1 << 16
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      ax[u] = vol_axis<C>(p, 0, p.ox, xc + u, im.w);
      // (columns / rows outside the output region: slots clamped, never stored)
      sl[u] = min(max(ax[u].i0 - xb, 0), VB_W - 1) | min(max(ax[u].i1 - xb, 0), VB_W - 1) << 16;
    }
    __syncwarp();  // the previous segment's row table is no longer read
    if (lane < 4) {
      const AxL ay = vol_axis<C>(p, 5, p.oy, yr + lane, im.h);
      rowtab[warp][lane] = make_float4(ay.a, ay.oma, __int_as_float(min(max(ay.i0 - yb, 0), VB_H - 1)),
                                       __int_as_float(min(max(ay.i1 - yb, 0), VB_H - 1)));
    }
    __syncwarp();
    // 16-byte row segments: four unit-stride column taps starting 16-B aligned
    const int c0 = sl[0] & 0xffff;
#if B2CL_VOL_FASTONLY
    const int c4 = sl[3] >> 16;  // the fourth column's i1 slot (c0 + 4, or c0 + 3 clamped)
    // x-blend of staged texel row j for the 4 columns (the tile passed vol_in_window)
    auto xblend = [&](const float* buf, float jf, float h[4]) {
      const float* row = buf + __float_as_int(jf) * VB_W;
      const float4 v = *reinterpret_cast<const float4*>(row + c0);
      const float T0[4] = {v.x, v.y, v.z, v.w}, T1[4] = {v.y, v.z, v.w, row[c4]};
#pragma unroll
      for (int u = 0; u < 4; ++u) h[u] = lerp1(ax[u].a, ax[u].oma, T0[u], T1[u]);
    };
    // the (x,y)-blended slice of the next ring stage: V[row][column]; the
    // warp's rows chain, so 5 staged texel rows give its 4 output rows
    auto slice = [&](float V[4][4]) {
      vol_wait(&full[s], ph);
      const float* buf = reinterpret_cast<const float*>(vol_buf + s * VB_STRIDE);
      float Hp[4], Hn[4];
      xblend(buf, rowtab[warp][0].z, Hp);
#pragma unroll
      for (int r = 0; r < 4; ++r) {
        const float4 ry = rowtab[warp][r];
        xblend(buf, ry.w, Hn);
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          V[r][u] = lerp1(ry.x, ry.y, Hp[u], Hn[u]);
          Hp[u] = Hn[u];
        }
      }
#else
    bool vecx = (c0 & 3) == 0 && c0 + 4 < VB_W;
#pragma unroll
    for (int u = 0; u < 4; ++u) vecx = vecx && sl[u] == ((c0 + u) | (c0 + u + 1) << 16);
    // the 4 rows of the warp chain (j1 of row r is j0 of row r+1): 5 texel rows
    bool rchain = true;
#pragma unroll
    for (int r = 0; r < 3; ++r) rchain = rchain && rowtab[warp][r].w == rowtab[warp][r + 1].z;

    // x-blend of staged texel row j for the 4 columns
    auto xblend = [&](const float* buf, float jf, float h[4]) {
      const float* row = buf + __float_as_int(jf) * VB_W;
      float T0[4], T1[4];
      if (vecx) {
        const float4 v = *reinterpret_cast<const float4*>(row + c0);
        T0[0] = v.x; T0[1] = v.y; T0[2] = v.z; T0[3] = v.w;
        T1[0] = v.y; T1[1] = v.z; T1[2] = v.w; T1[3] = row[c0 + 4];
      } else {
#pragma unroll
        for (int u = 0; u < 4; ++u) { T0[u] = row[sl[u] & 0xffff]; T1[u] = row[sl[u] >> 16]; }
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) h[u] = lerp1(ax[u].a, ax[u].oma, T0[u], T1[u]);
    };
    // the (x,y)-blended slice of the next ring stage: V[row][column]
    auto slice = [&](float V[4][4]) {
      vol_wait(&full[s], ph);
      const float* buf = reinterpret_cast<const float*>(vol_buf + s * VB_STRIDE);
      float Hp[4], Hn[4];
#ifdef B2CL_VOL_NOCOMPUTE  // A/B experiment only: the ring without the blends
      if (buf[lane] == 12345.f) {
#else
      if (rchain) {
#endif
        xblend(buf, rowtab[warp][0].z, Hp);
#pragma unroll
        for (int r = 0; r < 4; ++r) {
          const float4 ry = rowtab[warp][r];
          xblend(buf, ry.w, Hn);
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            V[r][u] = lerp1(ry.x, ry.y, Hp[u], Hn[u]);
            Hp[u] = Hn[u];
          }
        }
      } else {
#pragma unroll
        for (int r = 0; r < 4; ++r) {
          const float4 ry = rowtab[warp][r];
          xblend(buf, ry.z, Hp);
          xblend(buf, ry.w, Hn);
#pragma unroll
          for (int u = 0; u < 4; ++u) V[r][u] = lerp1(ry.x, ry.y, Hp[u], Hn[u]);
        }
      }
#endif
      __syncwarp();
      if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(vol_smem(&empty[s])) : "memory");
      if (++s == VOL_NS) { s = 0; ph ^= 1u; }
    };
    auto copy = [](float D[4][4], const float S[4][4]) {
#pragma unroll
      for (int r = 0; r < 4; ++r)
#pragma unroll
        for (int u = 0; u < 4; ++u) D[r][u] = S[r][u];
    };
    // output rows of the thread (a row outside the region is not stored)
    const bool vst = tl.vst && xc + 3 < p.ow;
    int rmask = 0;
#pragma unroll
    for (int r = 0; r < 4; ++r) rmask |= (yr + r < p.oh) << r;
    float* orow = reinterpret_cast<float*>(p.out) + ((uint64_t)(q.w0) * p.oh + yr) * p.ow + xc;
    const uint64_t zstride = (uint64_t)p.oh * p.ow;
    int kA = NONE, kB = NONE;
    // z-blend of the held slices lo (L) and hi (H) into the 4 output rows
    auto emit = [&](const AxL& az, const float L[4][4], const float H[4][4]) {
#pragma unroll
      for (int r = 0; r < 4; ++r) {
        if (!(rmask >> r & 1)) break;
        float o[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) o[u] = lerp1(az.a, az.oma, L[r][u], H[r][u]);
        float* op = orow + (uint64_t)r * p.ow;
#ifdef B2CL_VOL_NOSTORE  // A/B experiment only: read side alone
        if (o[0] != 12345.f) continue;
#endif
        if (vst) {
          __stcs(reinterpret_cast<float4*>(op), make_float4(o[0], o[1], o[2], o[3]));
        } else {
#pragma unroll
          for (int u = 0; u < 4; ++u)
            if (xc + u < p.ow) __stcs(op + u, o[u]);
        }
      }
      orow += zstride;
    };
    // VA holds slice kA (the previous step's lo), VB slice kB (its hi).  The
    // common unit-stride step -- lo = the previous hi, one new hi -- stages
    // the new slice over the old lo and swaps the roles; two such steps
    // restore them, so a run of common steps copies nothing.  Any other step
    // (the first of a tile, clamped or repeated indices) goes through the
    // general step, which keeps the roles; the producer stages the same
    // slices in the same order (lo unless held, then hi unless held).
    float VA[4][4], VB[4][4];
    int w = 0;
#pragma unroll 1
    while (w < q.nst) {
      AxL az = vol_axis<C>(p, 10, p.oz, q.w0 + w, im.d);
      if (az.i0 == kB && az.i1 != az.i0) {
        slice(VA);
        emit(az, VB, VA);
        kA = az.i0;
        kB = az.i1;
        if (++w < q.nst) {
          az = vol_axis<C>(p, 10, p.oz, q.w0 + w, im.d);
          if (az.i0 == kB && az.i1 != az.i0) {
            slice(VB);
            emit(az, VA, VB);
            kA = az.i0;
            kB = az.i1;
            ++w;
            continue;
          }
        }
#pragma unroll
        for (int r = 0; r < 4; ++r)
#pragma unroll
          for (int u = 0; u < 4; ++u) { const float t = VA[r][u]; VA[r][u] = VB[r][u]; VB[r][u] = t; }
        if (w >= q.nst) break;
      }
      // general step: lo into VA, hi into VB, staging only what is not held
      int hb = kB;  // slice held in VB
#pragma unroll 1
      for (int h = 0; h < 2; ++h) {
        const int k = h ? az.i1 : az.i0;
        if (h == 0) {
          if (k == kA) continue;
          if (k == kB) { copy(VA, VB); continue; }
        } else {
          if (k == hb) continue;
          if (k == az.i0) { copy(VB, VA); continue; }
        }
        slice(VB);
        hb = k;
        if (h == 0) copy(VA, VB);
      }
      kA = az.i0;
      kB = az.i1;
      emit(az, VA, VB);
      ++w;
    }
  }
}

// ===================================================================
// Rotated maps (config 3 map B, volume rendering): the x and y coordinates
// are any affine function of the output (x, y) and the z coordinate depends
// on the output z alone (A[2] = A[6] = A[8] = A[9] = 0).  The z axis is then
// walked exactly as above -- (x,y)-blended slices held in registers, one new
// slice per common step -- while the (x,y) footprint of a 64 x 48 output tile
// is the bounding box of the taps of its four corners (the fp32 coordinate is
// monotone in x and in y separately, and so are the axis indices): at most
// RB_MAXW x RB_MAXH texels, staged per slice by one cp.async.bulk.tensor.3d
// into a ring of up to 8 stages.  One CTA per SM: 12 consumer warps (128
// registers each: every per-sample value stays in registers) and a producer
// warp.  Each sample keeps its own tap offsets and weights (8 samples per
// thread, one column and 8 rows); the blend order is linear_at's:
// bit-identical results.
#ifndef B2CL_VOLR_NS
#define B2CL_VOLR_NS 8  // most ring stages (fewer when the box is large)
#endif
#ifndef B2CL_VOLR_SETUP
#define B2CL_VOLR_SETUP 2.0  // a z chunk's fixed cost in steps (vol_plan; fitted: walks of 14 / 16 / 32 at 236.9 / 231.7 / 219.2 us)
#endif
#ifndef B2CL_VOLR_MINB
#define B2CL_VOLR_MINB 1
#endif
#ifndef B2CL_VOLR_S
#define B2CL_VOLR_S 8
#endif
#ifndef B2CL_VOLR_NOHOIST
#define B2CL_VOLR_NOHOIST 0  // 1: 1 - w recomputed per slice, not held in 16 registers (helped with 8 consumer warps at 96 registers: 200.5 vs 215.5 us; 12 warps at 128: 188 held vs 195 recomputed)
#endif
#ifndef B2CL_VOLR_FUSED
#define B2CL_VOLR_FUSED 1  // 1: runs of common steps hold one slice (fused blend + store)
#endif
constexpr int VOLR_S = B2CL_VOLR_S;           // samples (rows) per consumer thread
#ifndef B2CL_VOLR_TW
#define B2CL_VOLR_TW 64
#endif
#ifndef B2CL_VOLR_CW
#define B2CL_VOLR_CW 12  // consumer warps per CTA (13 warps, one CTA per SM: 128 registers, no spill)
#endif
constexpr int VOLR_CW = B2CL_VOLR_CW, VOLR_CT = 32 * VOLR_CW;
constexpr int RT_W = B2CL_VOLR_TW, RT_H = (VOLR_CT / RT_W) * VOLR_S;  // output tile (one sample column of VOLR_S rows per consumer thread)
constexpr int RB_MAXW = 128, RB_MAXH = 128;   // largest staged box (texels)
constexpr int VOLR_NS = B2CL_VOLR_NS;
constexpr int VOLR_THREADS = VOLR_CT + 32;  // consumer warps + 1 producer warp

struct VolrBox {
  int xb, yb;    // first staged texel column (16-B aligned) and row
  int ok;        // 0: the footprint exceeds the launch's box (bw x bh)
};

struct VolrGeom {
  int bw, bh;    // staged box (texels), chosen per launch from the map's footprint
  int stride;    // bytes per ring stage (128-B multiple)
  int ns;        // ring stages (<= VOLR_NS, as many as 200 KB hold)
};

// the tile's staged box from its corners' taps (identical in every warp)
template <class C>
__device__ __forceinline__ VolrBox volr_box(const SampleParams& p, const VolrGeom& g, int x0, int y0, int z,
                                            int lane) {
  const int x1 = min(x0 + RT_W, p.ow) - 1, y1 = min(y0 + RT_H, p.oh) - 1;
  const int cx = (lane & 1) ? x1 : x0, cy = (lane & 2) ? y1 : y0;
  const float xf = __int2float_rn(p.ox + cx), yf = __int2float_rn(p.oy + cy), zf = __int2float_rn(p.oz + z);
  const AxL ax = axis_l<C>(p.smp, affine_coord(p.A, xf, yf, zf), p.im.w);
  const AxL ay = axis_l<C>(p.smp, affine_coord(p.A + 4, xf, yf, zf), p.im.h);
  int xmin = min(ax.i0, ax.i1), xmax = max(ax.i0, ax.i1), ymin = min(ay.i0, ay.i1), ymax = max(ay.i0, ay.i1);
#pragma unroll
  for (int o = 1; o < 4; o <<= 1) {
    xmin = min(xmin, __shfl_xor_sync(0xffffffffu, xmin, o));
    xmax = max(xmax, __shfl_xor_sync(0xffffffffu, xmax, o));
    ymin = min(ymin, __shfl_xor_sync(0xffffffffu, ymin, o));
    ymax = max(ymax, __shfl_xor_sync(0xffffffffu, ymax, o));
  }
  VolrBox b;
  b.xb = __shfl_sync(0xffffffffu, xmin, 0) & ~3;
  b.yb = __shfl_sync(0xffffffffu, ymin, 0);
  b.ok = __shfl_sync(0xffffffffu, xmax, 0) - b.xb < g.bw && __shfl_sync(0xffffffffu, ymax, 0) - b.yb < g.bh;
  return b;
}

#ifndef B2CL_VOLR_ROWS
#define B2CL_VOLR_ROWS 0  // 1: stage only each box row's tapped segment (one cp.async.bulk per row: 41 % fewer bytes, but ~190-byte copies: 849.5 vs 236.5 us); 0: the whole box (TMA)
#endif

// Columns [c0, c1) (box coordinates, multiples of 4 texels) of the taps in
// box row r (texel row yb + r) of a tile: the taps of a texel row j come from
// the samples with floor(t_v) in {j-1, j}, i.e. t_v in [j-1, j+1); the tile's
// sample coordinates (t = u - 1/2, texel units) lie in the parallelogram of
// its four corners' coordinates, so the row's taps lie between the x-extremes
// of that parallelogram clipped to the slab, widened by 2 texels each side
// (floor, the i0 + 1 tap, fp rounding).  Every operation is an explicitly
// rounded intrinsic (never contracted), so the producer warp and the consumer
// warps compute identical ranges; the consumers still check every tap against
// them, so the ranges only decide speed, never results.
__device__ __forceinline__ int volr_row_seg(const float cu[4], const float cv[4], int row, int xb, int bw, int nw) {
  const float lo = __int2float_rn(row - 1), hi = __int2float_rn(row + 1);
  float xmin = 3.0e38f, xmax = -3.0e38f;
  const int ea[4] = {0, 1, 3, 2}, eb[4] = {1, 3, 2, 0};  // the parallelogram's edges
#pragma unroll
  for (int e = 0; e < 4; ++e) {
    const float xa = cu[ea[e]], va = cv[ea[e]], xe = cu[eb[e]], ve = cv[eb[e]];
    float t0 = 0.f, t1 = 1.f;
    const float dv = __fsub_rn(ve, va);
    if (dv == 0.f) {
      if (!(va >= lo && va <= hi)) continue;
    } else {
      float ta = __fdiv_rn(__fsub_rn(lo, va), dv), tb = __fdiv_rn(__fsub_rn(hi, va), dv);
      if (ta > tb) { const float t = ta; ta = tb; tb = t; }
      t0 = fmaxf(t0, ta);
      t1 = fminf(t1, tb);
      if (!(t0 <= t1)) continue;
    }
    const float dx = __fsub_rn(xe, xa);
    const float x0 = __fadd_rn(xa, __fmul_rn(t0, dx)), x1 = __fadd_rn(xa, __fmul_rn(t1, dx));
    xmin = fminf(xmin, fminf(x0, x1));
    xmax = fmaxf(xmax, fmaxf(x0, x1));
  }
  if (!(xmin <= xmax)) return 0;  // no tap in this row
  int c0 = max(__float2int_rd(xmin) - 2, 0) - xb, c1 = min(__float2int_rd(xmax) + 3, nw) - xb;
  c0 = max(c0, 0) & ~3;
  c1 = min((c1 + 3) & ~3, bw);
  return c1 > c0 ? (c0 | c1 << 16) : 0;
}

// the tile's corner coordinates in texel units (t = u - 1/2; normalized maps scaled by the extent)
template <class C>
__device__ __forceinline__ void volr_corners(const SampleParams& p, int x0, int y0, int z, float cu[4], float cv[4]) {
  const int x1 = min(x0 + RT_W, p.ow) - 1, y1 = min(y0 + RT_H, p.oh) - 1;
  const float fw = p.smp.norm ? __int2float_rn(p.im.w) : 1.0f, fh = p.smp.norm ? __int2float_rn(p.im.h) : 1.0f;
  const float zf = __int2float_rn(p.oz + z);
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    const float xf = __int2float_rn(p.ox + ((c & 1) ? x1 : x0)), yf = __int2float_rn(p.oy + ((c & 2) ? y1 : y0));
    cu[c] = __fsub_rn(__fmul_rn(affine_coord(p.A, xf, yf, zf), fw), 0.5f);
    cv[c] = __fsub_rn(__fmul_rn(affine_coord(p.A + 4, xf, yf, zf), fh), 0.5f);
  }
}

template <class C>
__global__ void __launch_bounds__(VOLR_THREADS, B2CL_VOLR_MINB)
    k_sample_grid_volr(const SampleParams p, const VolTiles tl, const VolrGeom g,
                       const __grid_constant__ CUtensorMap tmap) {
  static_assert(C::dims == 3 && C::nch == 1 && C::type == T_FLOAT && C::addr == A_CTE, "R32F, CLAMP_TO_EDGE");
  extern __shared__ __align__(128) unsigned char volr_buf[];
  __shared__ uint64_t full[VOLR_NS], empty[VOLR_NS];
  __shared__ int segtab[RB_MAXH];  // the consumers' copy of the current tile's row segments
  const Image& im = p.im;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < g.ns; ++s) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(vol_smem(&full[s])) : "memory");
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(vol_smem(&empty[s])), "n"(VOLR_CW) : "memory");
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  __syncthreads();
  const int ntiles = tl.ntx * tl.nty * tl.nzc;
  constexpr int NONE = -2147483647 - 1;

  if (warp == VOLR_CW) {  // ---------------------------------------- producer
    int s = 0;
    uint32_t ph = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
      const VolSeg q = vol_seg(p, tl, t);
      const VolrBox bx = volr_box<C>(p, g, q.tx * RT_W, q.ty * RT_H, q.w0, lane);
      if (!bx.ok) continue;  // (not ok: the consumers read this tile directly)
#if B2CL_VOLR_ROWS
      // this lane's box rows (lane, lane + 32, ...: at most 4) and their segments
      int seg[RB_MAXH / 32];
      uint32_t txb = 0;
      {
        float cu[4], cv[4];
        volr_corners<C>(p, q.tx * RT_W, q.ty * RT_H, q.w0, cu, cv);
#pragma unroll
        for (int m = 0; m < RB_MAXH / 32; ++m) {
          const int r = lane + 32 * m;
          seg[m] = (r < g.bh && bx.yb + r < im.h) ? volr_row_seg(cu, cv, bx.yb + r, bx.xb, g.bw, im.w) : 0;
          txb += (uint32_t)((seg[m] >> 16) - (seg[m] & 0xffff)) * 4u;
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) txb += __shfl_xor_sync(0xffffffffu, txb, o);
      }
#else
      if (lane != 0) continue;
#endif
      int kA = NONE, kB = NONE;
      for (int w = 0; w < q.nst; ++w) {
        const AxL az = vol_axis<C>(p, 10, p.oz, q.w0 + w, im.d);
        const bool need0 = !(az.i0 == kA || az.i0 == kB);
        const bool need1 = !(az.i1 == az.i0 || (!need0 && az.i1 == kB));  // the consumers' rule
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          if (!(h ? need1 : need0)) continue;
          const int k = h ? az.i1 : az.i0;
          const uint32_t fb = vol_smem(&full[s]);
#if B2CL_VOLR_ROWS
          if (lane == 0) {
            vol_wait(&empty[s], ph ^ 1u);
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(fb), "r"(txb) : "memory");
          }
          __syncwarp();
#pragma unroll
          for (int m = 0; m < RB_MAXH / 32; ++m) {
            const int c0 = seg[m] & 0xffff, c1 = seg[m] >> 16, r = lane + 32 * m;
            if (c1 > c0)
              asm volatile(
                  "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                      vol_smem(volr_buf + s * g.stride + ((uint32_t)r * g.bw + c0) * 4u)),
                  "l"(im.ptr + (uint64_t)k * im.sp + (uint64_t)(bx.yb + r) * im.rp + (uint64_t)(bx.xb + c0) * 4u),
                  "r"((uint32_t)(c1 - c0) * 4u), "r"(fb)
                  : "memory");
          }
#else
          vol_wait(&empty[s], ph ^ 1u);
#ifdef B2CL_VOLR_NOTMA  // A/B experiment only (wrong results): the ring without the box copies
          asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(fb) : "memory");
#else
          asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(fb), "r"(g.bw * g.bh * 4)
                       : "memory");
          asm volatile(
              "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
              " [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(vol_smem(volr_buf + s * g.stride)),
              "l"(reinterpret_cast<uint64_t>(&tmap)), "r"(bx.xb), "r"(bx.yb), "r"(k), "r"(fb)
              : "memory");
#endif
#endif
#if B2CL_VOLR_PF
          // warm L2 with the same box B2CL_VOLR_PF slices ahead: its first-touch
          // texels come from DRAM while this slice is blended
          if (k + B2CL_VOLR_PF < im.d)
            asm volatile("cp.async.bulk.prefetch.tensor.3d.L2.global.tile [%0, {%1, %2, %3}];" ::"l"(
                             reinterpret_cast<uint64_t>(&tmap)),
                         "r"(bx.xb), "r"(bx.yb), "r"(k + B2CL_VOLR_PF)
                         : "memory");
#endif
          if (++s == g.ns) { s = 0; ph ^= 1u; }
        }
        kA = az.i0;
        kB = az.i1;
      }
    }
    return;
  }

  // --------------------------------------------------------------- consumers
  int s = 0;
  uint32_t ph = 0;
  auto acquire = [&]() { vol_wait(&full[s], ph); };
  const int col = threadIdx.x & (RT_W - 1), rg = threadIdx.x / RT_W;  // column, row group of VOLR_S
  for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
    const VolSeg q = vol_seg(p, tl, t);
    const int x = q.tx * RT_W + col, y0 = q.ty * RT_H + rg * VOLR_S;
    const VolrBox bx = volr_box<C>(p, g, q.tx * RT_W, q.ty * RT_H, q.w0, lane);
    // per sample: packed staged offset of tap (j0, i0) | (i1 - i0) << 16 | (j1 != j0) << 17, and the weights
    int off[VOLR_S];
    float wa[VOLR_S], wb[VOLR_S];
    int in = bx.ok;
    const float xf = __int2float_rn(p.ox + x), zf = __int2float_rn(p.oz + q.w0);
#pragma unroll
#if B2CL_VOLR_ROWS
    // the staged columns of each box row (computed as the producer does)
    if (bx.ok) {
      float cu[4], cv[4];
      volr_corners<C>(p, q.tx * RT_W, q.ty * RT_H, q.w0, cu, cv);
      for (int r = threadIdx.x; r < g.bh; r += VOLR_CT)
        segtab[r] = bx.yb + r < im.h ? volr_row_seg(cu, cv, bx.yb + r, bx.xb, g.bw, im.w) : 0;
    }
    asm volatile("bar.sync 1, %0;" ::"n"(VOLR_CT) : "memory");
#endif
    for (int r = 0; r < VOLR_S; ++r) {
      const float yf = __int2float_rn(p.oy + y0 + r);
      const AxL ax = axis_l<C>(p.smp, affine_coord(p.A, xf, yf, zf), im.w);
      const AxL ay = axis_l<C>(p.smp, affine_coord(p.A + 4, xf, yf, zf), im.h);
      const int sx0 = ax.i0 - bx.xb, sx1 = ax.i1 - bx.xb, sy0 = ay.i0 - bx.yb, sy1 = ay.i1 - bx.yb;
      const bool v = x < p.ow && y0 + r < p.oh;
      bool ok = sx0 >= 0 && sx1 >= sx0 && sx1 - sx0 <= 1 && sx1 < g.bw && sy0 >= 0 && sy1 >= sy0 &&
                sy1 - sy0 <= 1 && sy1 < g.bh;
#if B2CL_VOLR_ROWS
      if (ok) {  // both tap columns inside the staged segment of both tap rows
        const int s0 = segtab[sy0], s1 = segtab[sy1];
        ok = sx0 >= (s0 & 0xffff) && sx1 < (s0 >> 16) && sx0 >= (s1 & 0xffff) && sx1 < (s1 >> 16);
      }
#endif
      in = in && (ok || !v);
      off[r] = ok ? (sy0 * g.bw + sx0) | (sx1 - sx0) << 16 | (sy1 - sy0) << 17 : 0;
      wa[r] = ax.a;
      wb[r] = ay.a;
    }
    int fast;
    asm volatile("{ .reg .pred P, Q; setp.ne.s32 P, %1, 0; bar.red.and.pred Q, 1, %2, P; selp.s32 %0, 1, 0, Q; }"
                 : "=r"(fast) : "r"(in), "n"(VOLR_CT) : "memory");
    if (!fast) {  // the taps directly (read_image, the general kernel's coordinates)
      // (CLAMP_TO_EDGE indices are monotone in x and y, so every tap of a tile
      // whose corner box fits lies in it and this does not happen; should it,
      // the slices the producer staged are released unread, in its order)
      if (bx.ok) {
        int kA = NONE, kB = NONE;
#pragma unroll 1
        for (int w = 0; w < q.nst; ++w) {
          const AxL az = vol_axis<C>(p, 10, p.oz, q.w0 + w, im.d);
          const bool need0 = !(az.i0 == kA || az.i0 == kB);
          const bool need1 = !(az.i1 == az.i0 || (!need0 && az.i1 == kB));
          for (int h = 0; h < (int)need0 + (int)need1; ++h) {
            acquire();
            __syncwarp();
            if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(vol_smem(&empty[s])) : "memory");
            if (++s == g.ns) { s = 0; ph ^= 1u; }
          }
          kA = az.i0;
          kB = az.i1;
        }
      }
#pragma unroll 1
      for (int w = 0; w < q.nst; ++w) {
        const int z = q.w0 + w;
#pragma unroll 1
        for (int r = 0; r < VOLR_S; ++r) {
          const int y = y0 + r;
          if (x >= p.ow || y >= p.oh) break;
          const float xf2 = __int2float_rn(p.ox + x), yf2 = __int2float_rn(p.oy + y), zf2 = __int2float_rn(p.oz + z);
          const float c[3] = {affine_coord(p.A, xf2, yf2, zf2), affine_coord(p.A + 4, xf2, yf2, zf2),
                              affine_coord(p.A + 8, xf2, yf2, zf2)};
          uint32_t res[4];
          read_image<C>(p, c, res, 1);
          __stcs(reinterpret_cast<float*>(p.out) + ((uint64_t)z * p.oh + y) * p.ow + x, __uint_as_float(res[0]));
        }
      }
      continue;
    }
    // Interior tiles (every tap pair unclamped: i1 = i0 + 1, j1 = j0 + 1 --
    // all but the tiles at the image's edges) take the lean slice: byte
    // offsets precomputed, the 4 taps at fixed deltas, the x-blend of rows
    // j0 and j1 as one paired FMUL2 + FFMA2 (each lane lerp1's fma / mul).
    auto one_minus = [](float w) -> float {
#if B2CL_VOLR_NOHOIST
      // recomputed per slice (volatile: not hoisted into 16 live registers)
      float o;
      asm volatile("sub.rn.f32 %0, 0f3F800000, %1;" : "=f"(o) : "f"(w));
      return o;
#else
      return __fsub_rn(1.0f, w);
#endif
    };
    // sample r's (x, y)-blend of one staged slice (buf: the stage)
    auto tap_blend = [&](const char* buf, int r) -> float {
      const float* t0 = reinterpret_cast<const float*>(buf) + (off[r] & 0xffff);
      const int dx = off[r] >> 16 & 1, dy = (off[r] >> 17) * g.bw;
      const float oma1 = one_minus(wa[r]), omb1 = one_minus(wb[r]);
      const float h0 = lerp1(wa[r], oma1, t0[0], t0[dx]);
      const float h1 = lerp1(wa[r], oma1, t0[dy], t0[dy + dx]);
      return lerp1(wb[r], omb1, h0, h1);
    };
    auto release = [&]() {
      __syncwarp();
      if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(vol_smem(&empty[s])) : "memory");
      if (++s == g.ns) { s = 0; ph ^= 1u; }
    };
    auto slice = [&](float V[VOLR_S]) {
      acquire();
      const char* buf = reinterpret_cast<const char*>(volr_buf + s * g.stride);
#pragma unroll
      for (int r = 0; r < VOLR_S; ++r) V[r] = tap_blend(buf, r);
      release();
    };
    float* orow = reinterpret_cast<float*>(p.out) + ((uint64_t)q.w0 * p.oh + y0) * p.ow + x;
    const uint64_t zstride = (uint64_t)p.oh * p.ow;
    int nrow = x < p.ow ? min(VOLR_S, p.oh - y0) : 0;
    const int ow = p.ow;
    auto emit = [&](const AxL& az, const float L[VOLR_S], const float H[VOLR_S]) {
      float* o = orow;
      if (nrow == VOLR_S) {
#pragma unroll
        for (int r = 0; r < VOLR_S; ++r, o += ow) __stcs(o, lerp1(az.a, az.oma, L[r], H[r]));
      } else {
#pragma unroll
        for (int r = 0; r < VOLR_S; ++r, o += ow)
          if (r < nrow) __stcs(o, lerp1(az.a, az.oma, L[r], H[r]));
      }
      orow += zstride;
    };
    auto copy = [](float D[VOLR_S], const float S[VOLR_S]) {
#pragma unroll
      for (int r = 0; r < VOLR_S; ++r) D[r] = S[r];
    };
#if B2CL_VOLR_FUSED
    // one common step with a single held slice: each sample's new (x, y)-blend
    // is z-blended with the held value, stored, and replaces it
    auto fused = [&](const AxL& az, const float L[VOLR_S], float H[VOLR_S]) {
      acquire();
      const char* buf = reinterpret_cast<const char*>(volr_buf + s * g.stride);
      float* o = orow;
      orow += zstride;
      if (nrow == VOLR_S) {
#pragma unroll
        for (int r = 0; r < VOLR_S; ++r, o += ow) {
          const float h = tap_blend(buf, r);
          __stcs(o, lerp1(az.a, az.oma, L[r], h));
          H[r] = h;
        }
      } else {
#pragma unroll
        for (int r = 0; r < VOLR_S; ++r, o += ow) {
          const float h = tap_blend(buf, r);
          if (r < nrow) __stcs(o, lerp1(az.a, az.oma, L[r], h));
          H[r] = h;
        }
      }
      release();
    };
#endif
    // the z walk of k_sample_grid_vol (same roles, same staging order)
    float VA[VOLR_S], VB[VOLR_S];
    int kA = NONE, kB = NONE;
    int w = 0;
#pragma unroll 1
    while (w < q.nst) {
      AxL az = vol_axis<C>(p, 10, p.oz, q.w0 + w, im.d);
#if B2CL_VOLR_FUSED
      // A run of common steps (lo = the previous hi, one new hi) whose next
      // step does not reuse this step's lo holds ONE slice in registers (the
      // fused step); VA / VB are rebuilt from it when the run ends.  The held
      // pair is then (hi, hi): kA = kB = hi, which decides the next step's
      // staging exactly as the producer's (lo, hi) does, because that step's
      // lo differs from this one's (checked before each fused step).
      if (az.i0 == kB && az.i1 != az.i0) {
        AxL nz = az;
        const bool rep = w + 1 < q.nst && (nz = vol_axis<C>(p, 10, p.oz, q.w0 + w + 1, im.d)).i0 == az.i0;
        if (!rep) {
          // after a fused step: the next step's indices; false ends the run
          auto more = [&]() -> bool {
            kA = kB = az.i1;
            if (++w >= q.nst) return false;
            az = nz;
            if (!(az.i0 == kB && az.i1 != az.i0)) return false;
            if (w + 1 < q.nst) {
              nz = vol_axis<C>(p, 10, p.oz, q.w0 + w + 1, im.d);
              if (nz.i0 == az.i0) return false;
            }
            return true;
          };
          // the held slice alternates between P and Q (no register copies)
          float P[VOLR_S], Q[VOLR_S];
          copy(P, VB);
#pragma unroll 1
          for (;;) {
            fused(az, P, Q);
            if (!more()) {
              copy(VA, Q);
              copy(VB, Q);
              break;
            }
            fused(az, Q, P);
            if (!more()) {
              copy(VA, P);
              copy(VB, P);
              break;
            }
          }
          continue;
        }
      }
#endif
      if (az.i0 == kB && az.i1 != az.i0) {
        slice(VA);
        emit(az, VB, VA);
        kA = az.i0;
        kB = az.i1;
        if (++w < q.nst) {
          az = vol_axis<C>(p, 10, p.oz, q.w0 + w, im.d);
          if (az.i0 == kB && az.i1 != az.i0) {
            slice(VB);
            emit(az, VA, VB);
            kA = az.i0;
            kB = az.i1;
            ++w;
            continue;
          }
        }
#pragma unroll
        for (int r = 0; r < VOLR_S; ++r) { const float tt = VA[r]; VA[r] = VB[r]; VB[r] = tt; }
        if (w >= q.nst) break;
      }
      int hb = kB;
#pragma unroll 1
      for (int h = 0; h < 2; ++h) {
        const int k = h ? az.i1 : az.i0;
        if (h == 0) {
          if (k == kA) continue;
          if (k == kB) { copy(VA, VB); continue; }
        } else {
          if (k == hb) continue;
          if (k == az.i0) { copy(VB, VA); continue; }
        }
        slice(VB);
        hb = k;
        if (h == 0) copy(VA, VB);
      }
      kA = az.i0;
      kB = az.i1;
      emit(az, VA, VB);
      ++w;
    }
  }
}

// ------------------------------------------------------------------ host
static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(f);
  });
  return fn;
}

// the image's texels as a 3D fp32 tensor (w, h, d) with its pitches, read in
// (VB_W x VB_H x 1) boxes; out-of-range box elements are filled with zeros
static bool vol_tensor_map(const Image& im, CUtensorMap* m) {
  auto enc = encode_fn();
  if (!enc) return false;
  if ((reinterpret_cast<uintptr_t>(im.ptr) & 15) || (im.rp & 15) || (im.sp & 15)) return false;
  const cuuint64_t dims[3] = {(cuuint64_t)im.w, (cuuint64_t)im.h, (cuuint64_t)im.d};
  const cuuint64_t strides[2] = {im.rp, im.sp};
  const cuuint32_t box[3] = {VB_W, VB_H, 1};
  const cuuint32_t es[3] = {1, 1, 1};
  return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, im.ptr, dims, strides, box, es,
             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// Persistent-grid plan shared by the staged kernels: one CTA per resident
// slot.  setup == 0: z chunks a multiple of G / gcd(G, tiles per plane) so the
// tiles split evenly over the CTAs, each chunk at least VOL_MIN_STEPS slices
// long.  setup > 0: the chunk count minimising (rounds of G tiles) x (walk +
// setup), setup = a chunk's fixed cost (its per-tile coordinates and first
// slice) in units of one step -- longer walks at a small imbalance.
static bool vol_plan(const SampleParams& p, int tw, int th, const void* fn, int threads, size_t smem, int* occ,
                     VolTiles* tl, int* grid, double setup = 0.0) {
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 64) return false;
  static int sms[64] = {0};
  if (!occ[dev]) {
    cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaDeviceGetAttribute(&sms[dev], cudaDevAttrMultiProcessorCount, dev);
    int o = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, fn, threads, smem);
    occ[dev] = o < 1 ? 1 : o;
  }
  tl->ntx = (p.ow + tw - 1) / tw;
  tl->nty = (p.oh + th - 1) / th;
  tl->vst = (p.ow & 3) == 0 && (reinterpret_cast<uintptr_t>(p.out) & 15) == 0;
  const long long plane = (long long)tl->ntx * tl->nty;
  if (plane * p.od > 0x7fffffffLL) return false;
  const long long G = (long long)sms[dev] * occ[dev];
  long long a = G, b = plane;
  while (b) { const long long t = a % b; a = b; b = t; }
  const long long unit = G / a;  // chunks per balanced round
  long long nzc = unit;
  while (nzc * 2 <= p.od / VOL_MIN_STEPS && nzc * 2 <= 4 * unit) nzc *= 2;
  if ((p.od + nzc - 1) / nzc < VOL_MIN_STEPS) nzc = std::max<long long>(1, p.od / VOL_MIN_STEPS);
  if (setup > 0.0) {
    double best = 1e300;
    for (long long walk = 1; walk <= p.od; ++walk) {
      const long long n = (p.od + walk - 1) / walk;
      if ((p.od + n - 1) / n != walk) continue;  // (each n once, with its shortest walk)
      const double cost = (double)((plane * n + G - 1) / G) * ((double)walk + setup);
      if (cost < best) { best = cost; nzc = n; }
    }
  }
  tl->walk = (int)((p.od + nzc - 1) / nzc);
  tl->nzc = (p.od + tl->walk - 1) / tl->walk;
  *grid = (int)std::max<long long>(1, std::min<long long>(G, plane * tl->nzc));
  return true;
}

// Launch the TMA kernel for config C if the call qualifies (plain image,
// non-decreasing z map, encodable tensor); *used = false otherwise.
template <class C>
static cudaError_t go_vol(const SampleParams& p, cudaStream_t st, bool* used) {
  *used = false;
  if (!(p.A[10] >= 0.0f)) return cudaSuccess;
  CUtensorMap tm;
  if (B2CL_VOL_BULK) {  // row copies: no tensor map (16-B aligned rows needed)
    memset(&tm, 0, sizeof(tm));
    if ((reinterpret_cast<uintptr_t>(p.im.ptr) & 15) || (p.im.rp & 15) || (p.im.sp & 15)) return cudaSuccess;
  } else if (!vol_tensor_map(p.im, &tm)) {
    return cudaSuccess;
  }
  static int occ[64] = {0};
  const size_t smem = (size_t)VOL_NS * VB_STRIDE;
  VolTiles tl;
  int grid = 0;
  if (!vol_plan(p, VT_W, VT_H, reinterpret_cast<const void*>(k_sample_grid_vol<C>), VOL_THREADS, smem, occ, &tl,
                &grid, B2CL_VOL_SETUP))
    return cudaSuccess;
  k_sample_grid_vol<C><<<grid, VOL_THREADS, smem, st>>>(p, tl, tm);
  count_launch("k_sample_grid_vol");
  *used = true;
  return cudaGetLastError();
}

template <class C>
static cudaError_t go_volr(const SampleParams& p, cudaStream_t st, bool* used) {
  *used = false;
  const float* A = p.A;
  if (!(A[2] == 0.0f && A[6] == 0.0f && A[8] == 0.0f && A[9] == 0.0f && A[10] >= 0.0f)) return cudaSuccess;
  // the box: the footprint of a tile, |d(texel)/d(output)| summed over the
  // tile's extent, plus the LINEAR neighbour, 2 texels of rounding and the
  // 16-byte alignment of its start (the kernel checks every tile against it)
  const double sx = (p.smp.norm ? (double)p.im.w : 1.0), sy = (p.smp.norm ? (double)p.im.h : 1.0);
  const double fw = (std::fabs((double)A[0]) * (RT_W - 1) + std::fabs((double)A[1]) * (RT_H - 1)) * sx;
  const double fh = (std::fabs((double)A[4]) * (RT_W - 1) + std::fabs((double)A[5]) * (RT_H - 1)) * sy;
  if (!(fw < RB_MAXW && fh < RB_MAXH)) return cudaSuccess;
  VolrGeom g;
  g.bw = std::min(RB_MAXW, ((int)std::ceil(fw) + 1 + 2 + 3 + 3) & ~3);
  g.bh = std::min(RB_MAXH, (int)std::ceil(fh) + 1 + 2);
  g.stride = (g.bw * g.bh * 4 + 127) & ~127;
  auto enc = encode_fn();
  if (!enc) return cudaSuccess;
  const Image& im = p.im;
  if ((reinterpret_cast<uintptr_t>(im.ptr) & 15) || (im.rp & 15) || (im.sp & 15)) return cudaSuccess;
  CUtensorMap tm;
  const cuuint64_t dims[3] = {(cuuint64_t)im.w, (cuuint64_t)im.h, (cuuint64_t)im.d};
  const cuuint64_t strides[2] = {im.rp, im.sp};
  const cuuint32_t box[3] = {(cuuint32_t)g.bw, (cuuint32_t)g.bh, 1};
  const cuuint32_t es[3] = {1, 1, 1};
  if (enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, im.ptr, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
          CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
          CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
    return cudaSuccess;
  int occ[64] = {0};  // (occupancy depends on this launch's box)
  g.ns = std::min(VOLR_NS, (200 * 1024) / g.stride);
  if (g.ns < 2) return cudaSuccess;
  const size_t smem = (size_t)g.ns * g.stride;
  VolTiles tl;
  int grid = 0;
  if (!vol_plan(p, RT_W, RT_H, reinterpret_cast<const void*>(k_sample_grid_volr<C>), VOLR_THREADS, smem, occ, &tl,
                &grid, B2CL_VOLR_SETUP))
    return cudaSuccess;
  k_sample_grid_volr<C><<<grid, VOLR_THREADS, smem, st>>>(p, tl, g, tm);
  count_launch("k_sample_grid_volr");
  *used = true;
  return cudaGetLastError();
}

using C3CteV = WithShard<Cfg<3, T_FLOAT, O_R, 1, A_CTE, F_LINEAR, R_F>, false>;

cudaError_t launch_sample_vol(const SampleParams& p, cudaStream_t st, bool* used) {
  return go_vol<C3CteV>(p, st, used);
}

cudaError_t launch_sample_volr(const SampleParams& p, cudaStream_t st, bool* used) {
  return go_volr<C3CteV>(p, st, used);
}

}  // namespace b2cl
