// sample_box.cu -- TMA-staged LINEAR read of 2D RGBA32F images under ANY
// affine coordinate map (config 2 map (B): a 30 degree rotation at unit
// scale), steps a3-a7 of read_imagef ([CL1.2 §8.1-8.2]).
//
// The general one-thread-per-sample kernel (sample.cu k_sample_grid) gathers
// 4 x 16 B per sample straight from global memory.  Under a rotation a
// quarter-warp's 8 samples (one 128-B output line) tap texels spread over
// several rows, so each 16-B gather costs ~12 L1 wavefronts instead of 4:
// ncu showed the L1 data pipe at 93 % with DRAM at 53 % (profiles/r01/
// ncu_full_c2_mapb_s5.md).  Here each 32 x 32 output tile's footprint --
// the index bounding box of its taps -- is moved into shared memory by ONE
// cp.async.bulk.tensor.2d (the TMA engine: no LSU instructions), and the
// 4 taps of every sample are read from there (LDS.128).
//
// The box.  Per axis the fp32 coordinate ((A0*x + A1*y) + A2*z) + A3 is
// monotone in x and in y separately (every step is a rounded multiply or add
// of a monotone argument), so over the rectangular tile its extremes are at
// the tile's corners; each addressing mode is monotone between integer
// coordinates, so the corner taps bound the tile's taps unless the
// coordinate range crosses an integer: REPEAT then has a wrap seam inside
// the tile (not staged), MIRRORED_REPEAT a fold whose extreme index (0 for
// an even integer, n-1 for an odd one) joins the box.  Every sample still
// checks its 4 taps against the box and a sample with a tap outside it is
// read directly (read_image, global memory), so the result never depends on
// the box being right.
//
// Exactness: per sample the coordinates, AxL (axis_l) and the blend
// (x within rows j0, j1 with lerp1, then y) are linear_at's operations in
// linear_at's order -- bit-identical to every other grid kernel.  Taps
// outside the image under CLAMP read TMA's out-of-bounds zero fill, which is
// the border colour of CL_RGBA (the channel map of a zero texel, reading A8).
#include <cmath>
#include <cstring>

#include "../device/read.cuh"
#include "launch.h"
#include "tma.h"

namespace b2cl {
using namespace dev;

#ifndef B2CL_BOX_TH
#define B2CL_BOX_TH 32
#endif
constexpr int BX_W = 32, BX_H = B2CL_BOX_TH;  // output tile
#ifndef B2CL_BOX_PERSIST
#define B2CL_BOX_PERSIST 0
#endif
#ifndef B2CL_BOX_CW
#define B2CL_BOX_CW 4
#endif
#ifndef B2CL_BOX_NS
#define B2CL_BOX_NS 2
#endif
#ifndef B2CL_BOX_STAGE
#define B2CL_BOX_STAGE 0  // 0: tensor TMA box, 1: bulk copy per row, 2: 16-B cp.async by all threads
#endif
#ifndef B2CL_BOX_PF
#define B2CL_BOX_PF 592  // L2 prefetch distance in tiles (0: none): 148 SMs x 4 (measured 148 / 296 / 444 / 592 / 888 / 1776: 96.6 / 92.6 / 90.9 / 90.5 / 91.8 / 114.1 us, none 100.2)
#endif
#ifndef B2CL_BOX_L2PROMO
#define B2CL_BOX_L2PROMO 3  // CU_TENSOR_MAP_L2_PROMOTION_L2_256B
#endif
#ifndef B2CL_BOX_UNROLL
#define B2CL_BOX_UNROLL 2
#endif
#ifndef B2CL_BOX_MINB
#define B2CL_BOX_MINB 4
#endif
constexpr int kBoxUnroll = B2CL_BOX_UNROLL;  // rows of a warp in flight together
constexpr int BX_CW = B2CL_BOX_CW;  // blending warps: warp w takes rows w, w + CW, ...
constexpr int BX_NS = B2CL_BOX_PERSIST ? B2CL_BOX_NS : 1;  // ring stages (boxes in flight per CTA)
constexpr int BX_THREADS = 32 * (BX_CW + (B2CL_BOX_PERSIST ? 1 : 0));  // (+ 1 producer warp)
constexpr int BX_MAXW = 64;                   // TMA box: <= 256 fp32 elements per row = 64 texels

struct BoxGeom {
  int bw, bh;      // staged box (texels), fixed per launch from the map's footprint
  int stride;      // bytes per ring stage (128-byte multiple)
  int ntx, ntiles; // output tiles along x, in total (x fastest, then y, then z)
};

// One sample's two axes: axis_linear's operations (scalar: ptxas fuses a
// paired mul.rn.f32x2 feeding an add.rn.f32x2 into one FFMA2 -- a single
// rounding -- even under -fmad=false, so the address math never uses the
// paired forms).  Returns the floor index b of t = u - 1/2 per axis and the
// weight a = t - floor(t).
template <class C>
__device__ __forceinline__ void box_axis1(float s, float fn, int& b, float& a) {
  float u;
  if (C::addr == A_REPEAT) {
    u = __fmul_rn(__fsub_rn(s, floorf(s)), fn);
  } else if (C::addr == A_MIRROR) {
    const float sp = fabsf(__fsub_rn(s, __fmul_rn(2.0f, rintf(__fmul_rn(0.5f, s)))));
    u = __fmul_rn(sp, fn);
  } else {  // CLAMP_TO_EDGE, normalized
    u = __fmul_rn(s, fn);
  }
  const float t = __fsub_rn(u, 0.5f);
  b = ifloor(t);
  a = __fsub_rn(t, floorf(t));
}

// the LINEAR tap indices of axis_linear from b (n = image size on the axis)
template <class C>
__device__ __forceinline__ void box_taps(int b, int n, int& i0, int& i1) {
  if (C::addr == A_REPEAT) {
    i0 = b < 0 ? b + n : b;
    i1 = b + 1 > n - 1 ? b + 1 - n : b + 1;
  } else if (C::addr == A_MIRROR) {
    i0 = max(b, 0);
    i1 = min(b + 1, n - 1);
  } else {
    i0 = min(max(b, 0), n - 1);
    i1 = min(max(min(b, 0x7ffffffe) + 1, 0), n - 1);
  }
}

// lerp1 on channel pairs: fma(a, x1, (1 - a) * x0) per lane
__device__ __forceinline__ float2 lerp2(float2 a, float2 oma, float2 x0, float2 x1) {
  return __ffma2_rn(a, x1, __fmul2_rn(oma, x0));
}

// One output sample of a tile: the coordinate, the LINEAR taps, the blend
// from the staged box (or the built-in on global memory when a tap falls
// outside it), the 16-byte streaming store.
struct BoxCol {  // per thread: the terms of one output column
  float cx0, cx1, cz0, cz1, fnw, fnh;
  float4* out;
};

template <class C>
__device__ __forceinline__ void box_sample(const SampleParams& p, const BoxGeom& g, const BoxCol& k, int y,
                                           const char* bbase, int xb, int yb, int staged) {
  const Image& im = p.im;
  const float yf = __int2float_rn(p.oy + y);
  // affine_coord's operands and order: ((A0*x + A1*y) + A2*z) + A3
  const float2 c = make_float2(__fadd_rn(__fadd_rn(__fadd_rn(k.cx0, __fmul_rn(p.A[1], yf)), k.cz0), p.A[3]),
                               __fadd_rn(__fadd_rn(__fadd_rn(k.cx1, __fmul_rn(p.A[5], yf)), k.cz1), p.A[7]));
  int2 b;
  float2 a;
  box_axis1<C>(c.x, k.fnw, b.x, a.x);
  box_axis1<C>(c.y, k.fnh, b.y, a.y);
  int i0, i1, j0, j1;
  box_taps<C>(b.x, im.w, i0, i1);
  box_taps<C>(b.y, im.h, j0, j1);
  const int sx0 = i0 - xb, sx1 = i1 - xb, sy0 = j0 - yb, sy1 = j1 - yb;
  const bool in = staged && (unsigned)sx0 < (unsigned)g.bw && (unsigned)sx1 < (unsigned)g.bw &&
                  (unsigned)sy0 < (unsigned)g.bh && (unsigned)sy1 < (unsigned)g.bh;
  float4 o;
  if (in) {
    const uint32_t rowb = (uint32_t)g.bw * 16u;
    const char* r0 = bbase + (uint32_t)sy0 * rowb;
    const char* r1 = bbase + (uint32_t)sy1 * rowb;
    const float4 t00 = *reinterpret_cast<const float4*>(r0 + (uint32_t)sx0 * 16u);
    const float4 t10 = *reinterpret_cast<const float4*>(r0 + (uint32_t)sx1 * 16u);
    const float4 t01 = *reinterpret_cast<const float4*>(r1 + (uint32_t)sx0 * 16u);
    const float4 t11 = *reinterpret_cast<const float4*>(r1 + (uint32_t)sx1 * 16u);
    // linear_at: x-blend of row j0 and of row j1, then the y-blend (paired
    // forms: each lane one fma / mul, as lerp1)
    const float2 ax2 = make_float2(a.x, a.x), ay2 = make_float2(a.y, a.y);
    const float2 oma = __fadd2_rn(make_float2(1.0f, 1.0f), make_float2(-a.x, -a.x));
    const float2 omb = __fadd2_rn(make_float2(1.0f, 1.0f), make_float2(-a.y, -a.y));
    const float2 h0a = lerp2(ax2, oma, make_float2(t00.x, t00.y), make_float2(t10.x, t10.y));
    const float2 h0b = lerp2(ax2, oma, make_float2(t00.z, t00.w), make_float2(t10.z, t10.w));
    const float2 h1a = lerp2(ax2, oma, make_float2(t01.x, t01.y), make_float2(t11.x, t11.y));
    const float2 h1b = lerp2(ax2, oma, make_float2(t01.z, t01.w), make_float2(t11.z, t11.w));
    const float2 va = lerp2(ay2, omb, h0a, h1a), vb = lerp2(ay2, omb, h0b, h1b);
    o = make_float4(va.x, va.y, vb.x, vb.y);
  } else {  // a tap outside the box: the built-in on global memory
    const float cc[3] = {c.x, c.y, 0.f};
    uint32_t res[4];
    read_image<C>(p, cc, res, 4);
    o = make_float4(__uint_as_float(res[0]), __uint_as_float(res[1]), __uint_as_float(res[2]),
                    __uint_as_float(res[3]));
  }
  __stcs(k.out + (uint64_t)y * p.ow, o);
}

template <class C>
__device__ __forceinline__ BoxCol box_col(const SampleParams& p, int x, int z) {
  BoxCol k;
  const float xf = __int2float_rn(p.ox + x), zf = __int2float_rn(p.oz + z);
  k.cx0 = __fmul_rn(p.A[0], xf);
  k.cx1 = __fmul_rn(p.A[4], xf);
  k.cz0 = __fmul_rn(p.A[2], zf);
  k.cz1 = __fmul_rn(p.A[6], zf);
  k.fnw = __int2float_rn(p.im.w);
  k.fnh = __int2float_rn(p.im.h);
  k.out = reinterpret_cast<float4*>(p.out) + ((uint64_t)z * p.oh) * p.ow + x;
  return k;
}

// The tile's box from its corners, evaluated by lanes 0..7 of the calling
// warp at once (lane & 3 = the corner, lane >> 2 = the axis: u, v) and
// combined by shuffles (the rules of box_axis); every lane returns the result.
template <class C>
__device__ __forceinline__ bool tile_box(const SampleParams& p, const BoxGeom& g, int x0, int y0, int z, int lane,
                                         int& xlo, int& ylo) {
  const int x1 = min(x0 + BX_W, p.ow) - 1, y1 = min(y0 + BX_H, p.oh) - 1;
  const int cx = (lane & 1) ? x1 : x0, cy = (lane & 2) ? y1 : y0;
  const bool vax = (lane >> 2) & 1;
  const float xf = __int2float_rn(p.ox + cx), yf = __int2float_rn(p.oy + cy), zf = __int2float_rn(p.oz + z);
  const float sc = affine_coord(vax ? p.A + 4 : p.A, xf, yf, zf);
  const int n = vax ? p.im.h : p.im.w;
  const AxL a = axis_l<C>(p.smp, sc, n);
  int lo = min(a.i0, a.i1), hi = max(a.i0, a.i1);
  int chained = a.i1 == a.i0 + 1;
  float smin = sc, smax = sc;
#pragma unroll
  for (int o = 1; o < 4; o <<= 1) {
    lo = min(lo, __shfl_xor_sync(0xffffffffu, lo, o));
    hi = max(hi, __shfl_xor_sync(0xffffffffu, hi, o));
    chained &= __shfl_xor_sync(0xffffffffu, chained, o);
    smin = fminf(smin, __shfl_xor_sync(0xffffffffu, smin, o));
    smax = fmaxf(smax, __shfl_xor_sync(0xffffffffu, smax, o));
  }
  bool ok = fabsf(smin) < 1e7f && fabsf(smax) < 1e7f;  // (false for NaN, inf, huge)
  const float f0 = floorf(smin), f1 = floorf(smax);
  if (C::addr == A_REPEAT) {
    // a seam inside the tile, or corners whose taps wrap (texel n-1 next to 0)
    ok = ok && f0 == f1 && chained;
  } else if (C::addr == A_MIRROR) {
    if (f1 - f0 >= 2.0f) {
      lo = 0;
      hi = n - 1;
    } else if (f1 != f0) {  // one fold inside: at an even integer u -> 0, odd -> n
      if (fmodf(f1, 2.0f) == 0.0f) lo = 0;
      else hi = n - 1;
    }
  }
  ok = ok && hi - lo < (vax ? g.bh : g.bw);
  xlo = __shfl_sync(0xffffffffu, lo, 0);
  ylo = __shfl_sync(0xffffffffu, lo, 4);
  return __shfl_sync(0xffffffffu, (int)ok, 0) && __shfl_sync(0xffffffffu, (int)ok, 4);
}

#if !B2CL_BOX_PERSIST
// One CTA per output tile: warp 0 computes the box and issues its TMA copy,
// then all BX_CW warps blend the tile's rows from it (several CTAs per SM
// overlap one CTA's copy with the others' blending).
template <class C>
__global__ void __launch_bounds__(BX_THREADS, B2CL_BOX_MINB)
    k_sample_grid_box(const SampleParams p, const BoxGeom g, const __grid_constant__ CUtensorMap tmap) {
  static_assert(C::dims == 2 && C::type == T_FLOAT && C::order == O_RGBA && C::filt == F_LINEAR, "2D RGBA32F");
  extern __shared__ __align__(128) unsigned char box_buf[];
  __shared__ uint64_t full;
  __shared__ int bx[3];  // box origin (texels) and "staged"
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int x0 = blockIdx.x * BX_W, y0 = blockIdx.y * BX_H, z = blockIdx.z;
  if (warp == 0) {
    int xlo, ylo;
    const bool ok = tile_box<C>(p, g, x0, y0, z, lane, xlo, ylo);
    if (lane == 0) {
      bx[0] = xlo;
      bx[1] = ylo;
      bx[2] = ok;
    }
#if B2CL_BOX_STAGE == 0  // one tensor box (TMA)
    if (lane == 0 && ok) {
      mbar_init(&full, 1);
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      mbar_expect_tx(&full, (uint32_t)(g.bw * g.bh * 16));
      tma_load_2d(box_buf, &tmap, 4 * xlo, ylo, &full);
    }
#if B2CL_BOX_PF
    // warm L2 with the box of the tile B2CL_BOX_PF launch positions ahead (the
    // one that starts about when this wave of CTAs retires): its first-touch
    // texels come from DRAM now, so that tile's own copy hits L2
    {
      const long long nx = gridDim.x, ny = gridDim.y;
      const long long t = blockIdx.x + nx * (blockIdx.y + ny * (long long)blockIdx.z) + B2CL_BOX_PF;
      if (t < nx * ny * (long long)gridDim.z) {
        const int fz = (int)(t / (nx * ny)), fy = (int)((t / nx) % ny), fx = (int)(t % nx);
        int pxl, pyl;
        const bool pok = tile_box<C>(p, g, fx * BX_W, fy * BX_H, fz, lane, pxl, pyl);
        if (lane == 0 && pok)
          asm volatile("cp.async.bulk.prefetch.tensor.2d.L2.global.tile [%0, {%1, %2}];" ::"l"(
                           reinterpret_cast<uint64_t>(&tmap)),
                       "r"(4 * pxl), "r"(pyl)
                       : "memory");
      }
    }
#endif
#elif B2CL_BOX_STAGE == 1  // one plain bulk copy per box row, rows spread over the lanes
    if (ok) {
      // the taps of REPEAT / MIRRORED_REPEAT / CLAMP_TO_EDGE never leave the
      // image, so the rows and columns past its edge are not copied
      const Image& im = p.im;
      const int nrow = min(g.bh, im.h - ylo);
      const uint32_t rb = (uint32_t)min(g.bw, im.w - xlo) * 16u;
      if (lane == 0) {
        mbar_init(&full, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_expect_tx(&full, rb * (uint32_t)nrow);
      }
      __syncwarp();
      for (int r = lane; r < nrow; r += 32)
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                smem_u32(box_buf + (uint32_t)r * (uint32_t)g.bw * 16u)),
            "l"(im.ptr + (uint64_t)(ylo + r) * im.rp + (uint64_t)xlo * 16u), "r"(rb), "r"(smem_u32(&full))
            : "memory");
    }
#endif
  }
#if B2CL_BOX_STAGE == 2  // 16-byte cp.async copies by every thread
  __syncthreads();
  if (bx[2]) {
    const Image& im = p.im;
    const int xlo = bx[0], ylo = bx[1];
    const int nrow = min(g.bh, im.h - ylo), ncol = min(g.bw, im.w - xlo);
    for (int e = tid; e < nrow * ncol; e += BX_THREADS) {
      const int r = e / ncol, c = e - r * ncol;
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(box_buf + ((uint32_t)r * g.bw + c) * 16u)),
                   "l"(im.ptr + (uint64_t)(ylo + r) * im.rp + (uint64_t)(xlo + c) * 16u)
                   : "memory");
    }
    asm volatile("cp.async.wait_all;" ::: "memory");
  }
#endif
  __syncthreads();
  const int xb = bx[0], yb = bx[1], staged = bx[2];
  const int x = x0 + lane;
  // (a thread must not leave while the copy is in flight: it waits first)
  if (B2CL_BOX_STAGE != 2 && staged) mbar_wait(&full, 0);
  if (x >= p.ow) return;
  const BoxCol k = box_col<C>(p, x, z);
  const int nr = min(BX_H, p.oh - y0);
#pragma unroll kBoxUnroll
  for (int r = warp; r < nr; r += BX_CW) box_sample<C>(p, g, k, y0 + r, reinterpret_cast<const char*>(box_buf), xb, yb, staged);
}
#else
// Persistent CTAs (B2CL_BOX_PERSIST=1; measured slower at config 2 map (B):
// 105.7 vs 101.3 us): one PRODUCER warp computes each tile's box and moves it
// into a ring of BX_NS stages (one TMA box each, on the stage's `full`
// mbarrier; origin and "staged" ride along in `meta`); BX_CW CONSUMER warps
// blend the tile from the stage and release it on `empty`.
template <class C>
__global__ void __launch_bounds__(BX_THREADS, B2CL_BOX_MINB)
    k_sample_grid_box(const SampleParams p, const BoxGeom g, const __grid_constant__ CUtensorMap tmap) {
  static_assert(C::dims == 2 && C::type == T_FLOAT && C::order == O_RGBA && C::filt == F_LINEAR, "2D RGBA32F");
  extern __shared__ __align__(128) unsigned char box_buf[];
  __shared__ uint64_t full[BX_NS], empty[BX_NS];
  __shared__ int meta[BX_NS][4];  // box origin (texels), staged
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) {
    for (int s = 0; s < BX_NS; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], BX_CW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  __syncthreads();
  const int tpl = g.ntx * ((p.oh + BX_H - 1) / BX_H);  // tiles per output slice
  if (warp == BX_CW) {  // -------------------------------------------- producer
    int s = 0;
    uint32_t ph = 0;
    for (int t = blockIdx.x; t < g.ntiles; t += gridDim.x) {
      const int z = t / tpl, r = t - z * tpl;
      int xlo, ylo;
      const bool ok = tile_box<C>(p, g, (r % g.ntx) * BX_W, (r / g.ntx) * BX_H, z, lane, xlo, ylo);
      if (lane == 0) {
        mbar_wait(&empty[s], ph ^ 1u);
        meta[s][0] = xlo;
        meta[s][1] = ylo;
        meta[s][2] = ok;
        if (ok) {
          mbar_expect_tx(&full[s], (uint32_t)(g.bw * g.bh * 16));
          tma_load_2d(box_buf + s * g.stride, &tmap, 4 * xlo, ylo, &full[s]);
        } else {
          asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&full[s])) : "memory");
        }
      }
      __syncwarp();
      if (++s == BX_NS) { s = 0; ph ^= 1u; }
    }
    return;
  }
  int s = 0;  // ------------------------------------------------------- consumers
  uint32_t ph = 0;
  for (int t = blockIdx.x; t < g.ntiles; t += gridDim.x) {
    const int z = t / tpl, rr = t - z * tpl;
    const int x0 = (rr % g.ntx) * BX_W, y0 = (rr / g.ntx) * BX_H;
    const int x = x0 + lane;
    const BoxCol k = box_col<C>(p, x, z);
    const int nr = x < p.ow ? min(BX_H, p.oh - y0) : 0;
    mbar_wait(&full[s], ph);
    const int xb = meta[s][0], yb = meta[s][1], staged = meta[s][2];
    const char* bbase = reinterpret_cast<const char*>(box_buf + s * g.stride);
#pragma unroll 2
    for (int r = warp; r < nr; r += BX_CW) box_sample<C>(p, g, k, y0 + r, bbase, xb, yb, staged);
    __syncwarp();
    if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&empty[s])) : "memory");
    if (++s == BX_NS) { s = 0; ph ^= 1u; }
  }
}
#endif

// ------------------------------------------------------------------ host
// Row width of the staged box (texels, >= bw_min): a sample's 4 taps are 4
// LDS.128, and the 8 lanes of a quarter-warp (8 consecutive outputs along x,
// one 128-byte output line) hit shared memory at texel offsets
// j * BW + i whose 16-byte bank group (offset mod 8) collides when the map
// steps them by (1, 1) texels and BW = -1 (mod 8), etc.  The padding whose
// bank groups spread best is picked by counting the wavefronts of a quarter
// warp at 64 sub-texel phases, for the map's texel step per output column
// (dx, dy) (ncu, C2 map B: 46 texels = 15 wavefronts per LDS.128, 48 = 6).
static int pick_box_width(double dx, double dy, int bw_min, int bw_max) {
  int best = bw_min;
  long best_cost = -1;
  for (int bw = bw_min; bw <= std::min(bw_max, bw_min + 7); ++bw) {
    long cost = 0;
    for (int px = 0; px < 8; ++px)
      for (int py = 0; py < 8; ++py) {
        long addr[8];
        for (int k = 0; k < 8; ++k) {
          const long i = (long)std::floor(px / 8.0 + k * dx), j = (long)std::floor(py / 8.0 + k * dy);
          addr[k] = j * bw + i;
        }
        int worst = 0;
        for (int g = 0; g < 8; ++g) {  // distinct 16-byte addresses in bank group g
          int m = 0;
          for (int k = 0; k < 8; ++k) {
            if ((((addr[k] % 8) + 8) % 8) != g) continue;
            bool dup = false;
            for (int l = 0; l < k; ++l) dup = dup || addr[l] == addr[k];
            m += !dup;
          }
          worst = std::max(worst, m);
        }
        cost += worst;
      }
    if (best_cost < 0 || cost < best_cost) {
      best_cost = cost;
      best = bw;
    }
  }
  return best;
}

template <class C>
static cudaError_t go_box(const SampleParams& p, cudaStream_t st, bool* used) {
  *used = false;
  const Image& im = p.im;
  if ((reinterpret_cast<uintptr_t>(im.ptr) & 15) || (im.rp & 15) || p.outc != 4) return cudaSuccess;
  if ((reinterpret_cast<uintptr_t>(p.out) & 15)) return cudaSuccess;
  const double sx = p.smp.norm ? (double)im.w : 1.0, sy = p.smp.norm ? (double)im.h : 1.0;
  const double fw = (std::fabs((double)p.A[0]) * (BX_W - 1) + std::fabs((double)p.A[1]) * (BX_H - 1)) * sx;
  const double fh = (std::fabs((double)p.A[4]) * (BX_W - 1) + std::fabs((double)p.A[5]) * (BX_H - 1)) * sy;
  if (!(fw < BX_MAXW && fh < 200.0)) return cudaSuccess;
  BoxGeom g;
  // taps span floor(u - 1/2) .. floor(u - 1/2) + 1 over a coordinate range of
  // fw texels: ceil(fw) + 2 columns, + 1 for the rounding of the coordinate
  const int bw_min = std::min(BX_MAXW, (int)std::ceil(fw) + 3);
  g.bw = pick_box_width(std::fabs((double)p.A[0]) * sx, std::fabs((double)p.A[4]) * sy, bw_min, BX_MAXW);
  g.bh = (int)std::ceil(fh) + 3;
  g.stride = (g.bw * g.bh * 16 + 127) & ~127;
  const size_t smem = (size_t)BX_NS * g.stride;
  if (smem > 110 * 1024) return cudaSuccess;
  auto enc = tma_encode_fn();
  if (!enc) return cudaSuccess;
  CUtensorMap tm;
  const cuuint64_t dims[2] = {(cuuint64_t)im.w * 4, (cuuint64_t)im.h};
  const cuuint64_t strides[1] = {im.rp};
  const cuuint32_t box[2] = {(cuuint32_t)(4 * g.bw), (cuuint32_t)g.bh};
  const cuuint32_t es[2] = {1, 1};
  if (enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, im.ptr, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
          CU_TENSOR_MAP_SWIZZLE_NONE, (CUtensorMapL2promotion)B2CL_BOX_L2PROMO,
          CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
    return cudaSuccess;
  static bool attr_set = false;
  if (!attr_set) {
    cudaFuncSetAttribute(reinterpret_cast<const void*>(k_sample_grid_box<C>),
                         cudaFuncAttributeMaxDynamicSharedMemorySize, 110 * 1024);
    attr_set = true;
  }
  g.ntx = (p.ow + BX_W - 1) / BX_W;
  const long long nt = (long long)g.ntx * ((p.oh + BX_H - 1) / BX_H) * p.od;
  if (nt > 0x7fffffffLL) return cudaSuccess;
  g.ntiles = (int)nt;
#if B2CL_BOX_PERSIST
  int dev = 0;
  cudaGetDevice(&dev);
  static int sms[64] = {0};
  if (dev < 0 || dev >= 64) return cudaSuccess;
  if (!sms[dev]) cudaDeviceGetAttribute(&sms[dev], cudaDevAttrMultiProcessorCount, dev);
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, reinterpret_cast<const void*>(k_sample_grid_box<C>),
                                                BX_THREADS, smem);
  const int grid = (int)std::min<long long>(nt, (long long)sms[dev] * std::max(occ, 1));
  k_sample_grid_box<C><<<grid, BX_THREADS, smem, st>>>(p, g, tm);
#else
  dim3 grd(g.ntx, (p.oh + BX_H - 1) / BX_H, p.od);
  k_sample_grid_box<C><<<grd, BX_THREADS, smem, st>>>(p, g, tm);
#endif
  count_launch("k_sample_grid_box");
  *used = true;
  return cudaGetLastError();
}

using C2RepeatB = WithShard<Cfg<2, T_FLOAT, O_RGBA, 1, A_REPEAT, F_LINEAR, R_F>, false>;
using C2MirrorB = WithShard<Cfg<2, T_FLOAT, O_RGBA, 1, A_MIRROR, F_LINEAR, R_F>, false>;
using C2CteB = WithShard<Cfg<2, T_FLOAT, O_RGBA, 1, A_CTE, F_LINEAR, R_F>, false>;

cudaError_t launch_sample_box(const SampleParams& p, cudaStream_t st, bool* used) {
  *used = false;
  if (p.dims != 2 || p.arr || p.im.type != T_FLOAT || p.im.order != O_RGBA || p.smp.filt != F_LINEAR ||
      !p.smp.norm || p.rclass != R_F)
    return cudaSuccess;
  switch (p.smp.addr) {
    case A_REPEAT: return go_box<C2RepeatB>(p, st, used);
    case A_MIRROR: return go_box<C2MirrorB>(p, st, used);
    case A_CTE: return go_box<C2CteB>(p, st, used);
    default: return cudaSuccess;
  }
}

}  // namespace b2cl
