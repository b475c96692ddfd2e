// sample.cu -- read_imagef / read_imagei / read_imageui kernels (steps a3-a7).
//
// Per sample: coordinates (affine grid or list) -> per-axis addressing
// ([CL1.2 §8.2]) -> texel fetch through the CLImage pointer with one
// vector load per texel (16 B for RGBA32F) -> conversion and channel map
// ([CL1.2 §8.3]) -> LINEAR blend in the separable FMA form.
//
// Grid kernels:
//  * k_sample_grid      one thread per output sample, any affine map;
//  * k_sample_grid_walk separable maps, compile-time format: register reuse
//    of texel rows along the outermost axis (see its comment);
//  * k_sample_grid_sep  separable maps (every off-diagonal coefficient 0):
//    the x-axis addressing of XPT columns is computed once per thread and
//    reused down RPW rows, the y/z-axis addressing and the texel row
//    pointers once per row.  The coordinates it evaluates differ from the
//    general form ((A0*x + A1*y) + A2*z) + A3 only by additions of a signed
//    zero, which can change nothing but the sign of a zero coordinate, and
//    every addressing mode maps +0 and -0 to the same indices and weights --
//    so both kernels return identical bits (the parity tests run both).
// Every template argument may be `RT` (decided from the parameters at run
// time): the fully run-time instance covers every format x sampler; the
// compile-time instances are the hot configurations of BASELINE.json.
#include <atomic>
#include <cmath>
#include <type_traits>

#include "../device/read.cuh"
#include "launch.h"
#include "tma.h"

namespace b2cl {
using namespace dev;

template <int OUTC>
__device__ __forceinline__ void store_out(const SampleParams& p, uint64_t idx, const uint32_t r[4]) {
  const int outc = OUTC == RT ? p.outc : OUTC;
  if (outc == 4) {
    __stcs(reinterpret_cast<uint4*>(p.out) + idx, make_uint4(r[0], r[1], r[2], r[3]));
  } else if (outc == 1) {
    __stcs(reinterpret_cast<unsigned int*>(p.out) + idx, r[0]);
  } else if (outc == 2) {
    __stcs(reinterpret_cast<uint2*>(p.out) + idx, make_uint2(r[0], r[1]));
  } else {
    unsigned int* o = reinterpret_cast<unsigned int*>(p.out) + idx * 3;
    o[0] = r[0]; o[1] = r[1]; o[2] = r[2];
  }
}

template <class C, int OUTC>
__global__ void __launch_bounds__(256) k_sample_grid(const SampleParams p) {
#ifndef B2CL_GRID_PATCH
#define B2CL_GRID_PATCH 1
#endif
#if B2CL_GRID_PATCH
  // block = 32 x 8 outputs; each warp takes an 8 x 4 patch of them (not one
  // 32-wide row), so under rotations and other non-axis-aligned maps a
  // warp's taps fall in a compact texel region: fewer cache lines per load
#ifndef B2CL_GRID_PW
#define B2CL_GRID_PW 8
#endif
  constexpr int PW = B2CL_GRID_PW, PH = 32 / PW;  // warp patch (PW x PH outputs)
  const int lane = threadIdx.x, w = threadIdx.y;
#ifndef B2CL_GRID_QW
#define B2CL_GRID_QW 0
#endif
#if B2CL_GRID_QW && B2CL_GRID_PW == 8
  // each quarter-warp (8 lanes: one L1 wavefront group of 16-B loads) takes a
  // QW x (8/QW) block of the 8 x 4 patch instead of one 8-wide row
  constexpr int QW = B2CL_GRID_QW, QH = 8 / QW;
  const int qq = lane >> 3, qr = lane & 7;
  const int lx = (qq % (PW / QW)) * QW + qr % QW, ly = (qq / (PW / QW)) * QH + qr / QW;
#else
  const int lx = lane % PW, ly = lane / PW;
#endif
  const int x = blockIdx.x * 32 + (w % (32 / PW)) * PW + lx;
  const int y = blockIdx.y * 8 + (w / (32 / PW)) * PH + ly;
#else
  const int x = blockIdx.x * blockDim.x + threadIdx.x;
  const int y = blockIdx.y * blockDim.y + threadIdx.y;
#endif
  const int z = blockIdx.z;
  if (x >= p.ow || y >= p.oh) return;
  const float xf = __int2float_rn(p.ox + x), yf = __int2float_rn(p.oy + y),
              zf = __int2float_rn(p.oz + z);
  float c[3];
  c[0] = affine_coord(p.A, xf, yf, zf);
  c[1] = C::cdims > 1 ? affine_coord(p.A + 4, xf, yf, zf) : 0.f;
  c[2] = C::cdims > 2 ? affine_coord(p.A + 8, xf, yf, zf) : 0.f;
  uint32_t r[4];
  read_image<C>(p, c, r, OUTC == RT ? p.outc : OUTC);
  store_out<OUTC>(p, ((uint64_t)z * p.oh + y) * p.ow + x, r);
}

#ifndef B2CL_SEP_UNROLL
#define B2CL_SEP_UNROLL 1
#endif
constexpr int kSepUnroll = B2CL_SEP_UNROLL;  // rows of a thread in flight together

// Separable maps: block = 32 x 4 threads; tile = (32*XPT) columns x (4*RPW) rows
// of one output slice.  Lane -> columns lane + 32*t, warp -> RPW consecutive rows.
template <class C, int OUTC, int XPT, int RPW>
#ifndef B2CL_SEP_MINB
#define B2CL_SEP_MINB 11
#endif
__global__ void __launch_bounds__(128, (C::type == RT ? 1 : B2CL_SEP_MINB)) k_sample_grid_sep(const SampleParams p) {
  const Image& im = p.im;
  const int z = blockIdx.z;
  const int x0 = blockIdx.x * (32 * XPT) + threadIdx.x;
  // MIRRORED_REPEAT folds output rows onto shared texel rows symmetrically
  // about the mirror axis; taking row tiles alternately from both ends keeps
  // those texel rows in L2 between their two uses (a traversal order only)
  int ty = blockIdx.y;
  if (C::addr == A_MIRROR) ty = (ty & 1) ? gridDim.y - 1 - (ty >> 1) : (ty >> 1);
  const int y0 = ty * (4 * RPW) + threadIdx.y * RPW;
  const bool lin = filt_of<C>(p) == F_LINEAR;
  // x axis: once per column
  AxL ax[XPT];
  AxN nx[XPT];
#pragma unroll
  for (int t = 0; t < XPT; ++t) {
    const float s = __fadd_rn(__fmul_rn(p.A[0], __int2float_rn(p.ox + x0 + 32 * t)), p.A[3]);
    if (lin) ax[t] = axis_l<C>(p.smp, s, im.w);
    else nx[t] = axis_n<C>(p.smp, s, im.w);
  }
  // z axis: once per block
  AxL az{0, 0, 0.f, 1.f, true, true};
  AxN nz{0, true};
  if (C::dims > 2) {
    const float s = __fadd_rn(__fmul_rn(p.A[10], __int2float_rn(p.oz + z)), p.A[11]);
    if (lin) az = axis_l<C>(p.smp, s, im.d);
    else nz = axis_n<C>(p.smp, s, im.d);
  }
#pragma unroll kSepUnroll
  for (int r = 0; r < RPW; ++r) {
    const int y = y0 + r;
    if (y >= p.oh) break;
    const uint64_t obase = ((uint64_t)z * p.oh + y) * p.ow;
    if (lin) {
      AxL ay{0, 0, 0.f, 1.f, true, true};
      if (C::dims > 1)
        ay = axis_l<C>(p.smp, __fadd_rn(__fmul_rn(p.A[5], __int2float_rn(p.oy + y)), p.A[7]), im.h);
      const char* rows[4] = {row_ptr<C>(im, ay.i0, az.i0), row_ptr<C>(im, ay.i1, az.i0),
                             row_ptr<C>(im, ay.i0, az.i1), row_ptr<C>(im, ay.i1, az.i1)};
      const bool rok[4] = {ay.ok0 && az.ok0, ay.ok1 && az.ok0, ay.ok0 && az.ok1, ay.ok1 && az.ok1};
#pragma unroll
      for (int t = 0; t < XPT; ++t) {
        const int x = x0 + 32 * t;
        if (x < p.ow) {
          uint32_t res[4];
          linear_at<C>(p, rows, rok, ax[t], ay.a, ay.oma, az.a, az.oma, res,
                       OUTC == RT ? p.outc : OUTC);
          store_out<OUTC>(p, obase + x, res);
        }
      }
    } else {
      AxN ny{0, true};
      if (C::dims > 1)
        ny = axis_n<C>(p.smp, __fadd_rn(__fmul_rn(p.A[5], __int2float_rn(p.oy + y)), p.A[7]), im.h);
      const char* row = row_ptr<C>(im, ny.i, nz.i);
#pragma unroll
      for (int t = 0; t < XPT; ++t) {
        const int x = x0 + 32 * t;
        if (x < p.ow) {
          uint32_t res[4];
          nearest_at<C>(p, row, nx[t], ny.ok && nz.ok, res);
          store_out<OUTC>(p, obase + x, res);
        }
      }
    }
  }
}

// Separable map, LINEAR, compile-time format: register reuse along a walk.
// Each warp walks consecutive outputs along the outermost image axis (y for
// 2D, z for 3D) with lanes across x.  The blend is separable -- x, then y,
// then z, as linear_at -- and every partial result before the walk-axis
// blend depends only on the texel row(s) at one walk index and on the fixed
// x (and 3D: y) weights.  So a step keeps, per column and channel, ONE value
// for each of the two walk indices it blends (lo, hi):
//   2D: the x-blended row            lerp(a, T[j][i0], T[j][i1])
//   3D: the x- then y-blended slice   lerp(b, lerp(a, T[j0][k][i0..]), lerp(a, T[j1][k][i0..]))
// and blends them along the walk axis.  When step w+1's lo index equals step
// w's hi (warp-uniform test) that value is reused from registers, so a
// sample costs half the taps in global loads and half the x/y blends.  The
// next hi is loaded and pre-blended before this step is finished (software
// pipelining).  The operations and their order are exactly linear_at's, so
// the results are bit-identical to the other kernels.
//   2D: block = 32 x 4 threads, tile = (32*XPT) columns x (4*WALK) rows;
//       warp w walks rows [y0 + w*WALK, +WALK).
//   3D: tile = (32*XPT) columns x 4 rows x WALK slices; warp w owns one row
//       and walks slices [z0, z0 + WALK).
template <class C, int XPT>
struct WalkVals {  // pre-blended values at one walk index: [column][channel]
  float v[XPT][C::nch];
};

template <class C, int XPT>
__device__ __forceinline__ void walk_load(const Image& im, const AxL (&ax)[XPT], const AxL& afix,
                                          int widx, bool wok, WalkVals<C, XPT>& out) {
  constexpr bool D3 = C::dims == 3;
  constexpr int NJ = D3 ? 2 : 1;  // texel rows per walk index
  uint32_t m0[NJ][XPT][4], m1[NJ][XPT][4];
#pragma unroll
  for (int js = 0; js < NJ; ++js) {
    const int j = D3 ? (js ? afix.i1 : afix.i0) : widx;
    const int k = D3 ? widx : 0;
    const bool rok = wok && (!D3 || (js ? afix.ok1 : afix.ok0));
    const char* row = row_ptr<C>(im, j, k);
#pragma unroll
    for (int t = 0; t < XPT; ++t) {
      fetch<C>(im, row, ax[t].i0, rok && ax[t].ok0, R_F, m0[js][t]);
      fetch<C>(im, row, ax[t].i1, rok && ax[t].ok1, R_F, m1[js][t]);
    }
  }
#pragma unroll
  for (int t = 0; t < XPT; ++t)
#pragma unroll
    for (int ch = 0; ch < C::nch; ++ch) {
      const float r0 = lerp1(ax[t].a, ax[t].oma, __uint_as_float(m0[0][t][ch]),
                             __uint_as_float(m1[0][t][ch]));
      if constexpr (D3) {
        const float r1 = lerp1(ax[t].a, ax[t].oma, __uint_as_float(m0[NJ - 1][t][ch]),
                               __uint_as_float(m1[NJ - 1][t][ch]));
        out.v[t][ch] = lerp1(afix.a, afix.oma, r0, r1);
      } else {
        out.v[t][ch] = r0;
      }
    }
}

template <class C, int OUTC, int XPT, int WALK>
__global__ void __launch_bounds__(128) k_sample_grid_walk(const SampleParams p) {
  static_assert(C::nch != RT && C::type != RT && C::order != RT, "compile-time format");
  static_assert(C::dims >= 2, "walk needs a second axis");
  constexpr int NCH = C::nch;
  constexpr bool D3 = C::dims == 3;
  using Vals = WalkVals<C, XPT>;
  const Image& im = p.im;
  // 3D: the 4 warps of a block split x (one texel row per block, wide DRAM bursts)
  const int x0 = D3 ? blockIdx.x * (128 * XPT) + threadIdx.y * (32 * XPT) + threadIdx.x
                    : blockIdx.x * (32 * XPT) + threadIdx.x;
  AxL ax[XPT];
#pragma unroll
  for (int t = 0; t < XPT; ++t)
    ax[t] = axis_l<C>(p.smp, __fadd_rn(__fmul_rn(p.A[0], __int2float_rn(p.ox + x0 + 32 * t)), p.A[3]),
                      im.w);
  // the fixed axis (3D: y) and the walk range
  int yfix = 0, zfix = 0, w0;
  AxL afix{0, 0, 0.f, 1.f, true, true};
  if (D3) {
    yfix = blockIdx.y;
    if (yfix >= p.oh) return;  // warp-uniform
    w0 = blockIdx.z * WALK;
    afix = axis_l<C>(p.smp, __fadd_rn(__fmul_rn(p.A[5], __int2float_rn(p.oy + yfix)), p.A[7]), im.h);
  } else {
    zfix = blockIdx.z;
    w0 = blockIdx.y * (4 * WALK) + threadIdx.y * WALK;
  }
  const int wlen = D3 ? p.od : p.oh;
  if (w0 >= wlen) return;
  const float awc = D3 ? p.A[10] : p.A[5], awo = D3 ? p.A[11] : p.A[7];
  const int nw = D3 ? im.d : im.h;
  const int wor = D3 ? p.oz : p.oy;  // origin of the output region along the walk
  auto walk_axis = [&](int wv) {
    return axis_l<C>(p.smp, __fadd_rn(__fmul_rn(awc, __int2float_rn(wor + wv)), awo), nw);
  };
  AxL aw = walk_axis(w0);
  // Three value buffers in fixed rotating roles (lo, hi, next-hi): no
  // register copies between steps.  A step loads the next hi, blends
  // (lo, hi), and -- only when the next lo is not this hi (no reuse) --
  // reloads it into the hi buffer after the blend, which becomes the next lo.
  Vals B0, B1, B2;
  walk_load<C, XPT>(im, ax, afix, aw.i0, aw.ok0, B0);
  walk_load<C, XPT>(im, ax, afix, aw.i1, aw.ok1, B1);
  const float fa = D3 ? afix.a : 0.f;  // 3D: the fixed y weight (NaN test of A26)
  // one step with (lo, hi, nx) = values at aw; returns false after the last step
  auto step = [&](int w, Vals& lo, Vals& hi, Vals& nx) -> bool {
    const int wv = w0 + w;
    const bool next = w + 1 < WALK && wv + 1 < wlen;
    AxL an = aw;
    if (next) {
      an = walk_axis(wv + 1);
      walk_load<C, XPT>(im, ax, afix, an.i1, an.ok1, nx);
    }
    const int y = D3 ? yfix : wv, z = D3 ? wv : zfix;
    const uint64_t obase = ((uint64_t)z * p.oh + y) * p.ow;
#pragma unroll
    for (int t = 0; t < XPT; ++t) {
      const int x = x0 + 32 * t;
      uint32_t m[4] = {0u, 0u, 0u, 0u};
#pragma unroll
      for (int ch = 0; ch < NCH; ++ch)
        m[ch] = __float_as_uint(lerp1(aw.a, aw.oma, lo.v[t][ch], hi.v[t][ch]));
      uint32_t res[4];
      map_order(C::order, m, 0x3f800000u, res);
      if (const_in_output(C::order, OUTC) && (ax[t].a != ax[t].a || aw.a != aw.a || fa != fa))
        res[0] = res[1] = res[2] = res[3] = 0x7fffffffu;
      if (x < p.ow) store_out<OUTC>(p, obase + x, res);
    }
    if (!next) return false;
    // the next step's lo is this step's hi unless the walk skips
    if (!(an.i0 == aw.i1 && an.ok0 == aw.ok1)) walk_load<C, XPT>(im, ax, afix, an.i0, an.ok0, hi);
    aw = an;
    return true;
  };
#pragma unroll 1
  for (int w = 0; w < WALK; w += 3) {
    if (!step(w, B0, B1, B2)) break;
    if (!step(w + 1, B1, B2, B0)) break;
    if (!step(w + 2, B2, B0, B1)) break;
  }
}

// 3D walk for one-channel 32-bit float images (config 3: R32F trilinear),
// four CONSECUTIVE columns per thread (a warp covers 128 columns).  When the
// x axis is a unit-stride stencil over the warp -- column x+t taps
// (i0 + t, i0 + t + 1), all in range, i0 16-byte aligned, the next lane
// starting 4 texels further (warp-uniform vote, once per thread) -- a texel
// row costs one 16-byte load plus one shuffle for the fifth texel, instead
// of eight scalar loads, and the four outputs leave in one 16-byte store.
// Otherwise (image edges, other maps) the same columns load texel by texel.
// Blend order and operands are walk_load's and linear_at's: bit-identical.
template <class C>
struct Walk4 {
  float v[4];  // x- then y-blended value of this slice for the 4 columns
};

template <class C>
__device__ __forceinline__ void walk4_load(const Image& im, const AxL (&ax)[4], const AxL& afix,
                                           int k, bool kok, bool vec, Walk4<C>& out) {
  float r[2][4];
#pragma unroll
  for (int js = 0; js < 2; ++js) {
    const int j = js ? afix.i1 : afix.i0;
    const bool rok = kok && (js ? afix.ok1 : afix.ok0);
    const char* row = row_ptr<C>(im, j, k);
    float T0[4], T1[4];
    if (vec) {
      float4 q = make_float4(0.f, 0.f, 0.f, 0.f);
      if (rok) q = __ldg(reinterpret_cast<const float4*>(row + (uint64_t)(unsigned)ax[0].i0 * 4u));
      float e = __shfl_down_sync(0xffffffffu, q.x, 1);
      if ((threadIdx.x & 31) == 31)
        e = rok ? __ldg(reinterpret_cast<const float*>(row + (uint64_t)(unsigned)ax[3].i1 * 4u)) : 0.f;
      T0[0] = q.x; T0[1] = q.y; T0[2] = q.z; T0[3] = q.w;
      T1[0] = q.y; T1[1] = q.z; T1[2] = q.w; T1[3] = e;
    } else {
#pragma unroll
      for (int t = 0; t < 4; ++t) {
        uint32_t m0[4], m1[4];
        fetch<C>(im, row, ax[t].i0, rok && ax[t].ok0, R_F, m0);
        fetch<C>(im, row, ax[t].i1, rok && ax[t].ok1, R_F, m1);
        T0[t] = __uint_as_float(m0[0]);
        T1[t] = __uint_as_float(m1[0]);
      }
    }
#pragma unroll
    for (int t = 0; t < 4; ++t) r[js][t] = lerp1(ax[t].a, ax[t].oma, T0[t], T1[t]);
  }
#pragma unroll
  for (int t = 0; t < 4; ++t) out.v[t] = lerp1(afix.a, afix.oma, r[0][t], r[1][t]);
}

// the walk of one thread (VEC: the 16-byte row loads; else texel by texel)
template <class C, int WALK, bool VEC>
__device__ __forceinline__ void walk4_run(const SampleParams& p, const AxL (&ax)[4], int x0,
                                          int yfix, int w0, bool vst) {
  const Image& im = p.im;
  const AxL afix =
      axis_l<C>(p.smp, __fadd_rn(__fmul_rn(p.A[5], __int2float_rn(p.oy + yfix)), p.A[7]), im.h);
  auto walk_axis = [&](int wv) {
    return axis_l<C>(p.smp, __fadd_rn(__fmul_rn(p.A[10], __int2float_rn(p.oz + wv)), p.A[11]), im.d);
  };
  AxL aw = walk_axis(w0);
  Walk4<C> B0, B1, B2;
  walk4_load<C>(im, ax, afix, aw.i0, aw.ok0, VEC, B0);
  walk4_load<C>(im, ax, afix, aw.i1, aw.ok1, VEC, B1);
  float* obase = reinterpret_cast<float*>(p.out) + (uint64_t)yfix * p.ow + x0;
  const uint64_t zstride = (uint64_t)p.oh * p.ow;
  auto step = [&](int w, Walk4<C>& lo, Walk4<C>& hi, Walk4<C>& nx) -> bool {
    const int wv = w0 + w;
    const bool next = w + 1 < WALK && wv + 1 < p.od;
    AxL an = aw;
    if (next) {
      an = walk_axis(wv + 1);
      walk4_load<C>(im, ax, afix, an.i1, an.ok1, VEC, nx);
    }
    float o[4];
#pragma unroll
    for (int t = 0; t < 4; ++t) o[t] = lerp1(aw.a, aw.oma, lo.v[t], hi.v[t]);
    float* orow = obase + (uint64_t)wv * zstride;
    if (vst) {
      __stcs(reinterpret_cast<float4*>(orow), make_float4(o[0], o[1], o[2], o[3]));
    } else {
#pragma unroll
      for (int t = 0; t < 4; ++t)
        if (x0 + t < p.ow) __stcs(orow + t, o[t]);
    }
    if (!next) return false;
    if (!(an.i0 == aw.i1 && an.ok0 == aw.ok1)) walk4_load<C>(im, ax, afix, an.i0, an.ok0, VEC, hi);
    aw = an;
    return true;
  };
#pragma unroll 1
  for (int w = 0; w < WALK; w += 3) {
    if (!step(w, B0, B1, B2)) break;
    if (!step(w + 1, B1, B2, B0)) break;
    if (!step(w + 2, B2, B0, B1)) break;
  }
}

#ifndef B2CL_W4_MINB
#define B2CL_W4_MINB 12
#endif
template <class C, int WALK>
__global__ void __launch_bounds__(128, B2CL_W4_MINB) k_sample_grid_walk4(const SampleParams p) {
  static_assert(C::dims == 3 && C::nch == 1 && C::type == T_FLOAT, "R32F-type 3D images");
  const Image& im = p.im;
  const int lane = threadIdx.x & 31;
  const int x0 = blockIdx.x * 512 + threadIdx.y * 128 + lane * 4;
  AxL ax[4];
#pragma unroll
  for (int t = 0; t < 4; ++t)
    ax[t] = axis_l<C>(p.smp, __fadd_rn(__fmul_rn(p.A[0], __int2float_rn(p.ox + x0 + t)), p.A[3]),
                      im.w);
  bool ok = (ax[0].i0 & 3) == 0 && x0 + 3 < p.ow;
#pragma unroll
  for (int t = 0; t < 4; ++t)
    ok = ok && ax[t].ok0 && ax[t].ok1 && ax[t].i0 == ax[0].i0 + t && ax[t].i1 == ax[t].i0 + 1;
  const int nb = __shfl_down_sync(0xffffffffu, ax[0].i0, 1);
  if (lane < 31) ok = ok && nb == ax[0].i0 + 4;
  const bool vec = __all_sync(0xffffffffu, ok);
  const bool vst = (p.ow & 3) == 0 && x0 + 3 < p.ow;  // 16-byte output stores
  const int yfix = blockIdx.y;
  const int w0 = blockIdx.z * WALK;
  if (yfix >= p.oh || w0 >= p.od) return;  // block-uniform
  if (vec) walk4_run<C, WALK, true>(p, ax, x0, yfix, w0, vst);
  else walk4_run<C, WALK, false>(p, ax, x0, yfix, w0, vst);
}

// Separable LINEAR maps of 2D RGBA32F images under REPEAT / MIRRORED_REPEAT
// (every tap in range): the filter footprint of a TW x TH output tile is
// staged in shared memory once, so L2 serves each texel about once per tile
// instead of once per tap (the direct kernels issue 4 x 16-byte gathers per
// sample, and their L1 catches only part of the reuse).
//   Per axis the taps of consecutive outputs CHAIN upward (i1(x) = i0(x+1):
//   unit-scale maps, wrap seams included) or downward (i0(x) = i1(x+1): the
//   reflected half of MIRRORED_REPEAT).  Upward, slot k < TW holds texel
//   column i0(x0+k) and slot TW holds i1(x0+TW-1): output column t blends
//   slots (t, t+1).  Downward, slot k holds i1(x0+k), slot TW holds
//   i0(x0+TW-1): column t blends slots (t+1, t).  Rows likewise.  A tile whose
//   taps chain neither way on some axis (it contains a mirror fold, or the map
//   has another scale) reads its taps directly.
//   Block = 4 warps: warp w takes columns (w & 1)*32 + lane and walks rows
//   (w >> 1)*TH/2 .. +TH/2, blending x once per row and y from the previous
//   row's x-blend.  Operations, operands and order are linear_at's: the
//   results are bit-identical to the other kernels.
template <class C, int TW, int TH>
__global__ void __launch_bounds__(128) k_sample_grid_tile(const SampleParams p) {
  static_assert(C::type == T_FLOAT && C::order == O_RGBA && C::dims == 2 && TW == 64, "2D RGBA32F");
  static_assert(C::addr == A_REPEAT || C::addr == A_MIRROR, "taps always in range");
  constexpr int RPW = TH / 2;
  __shared__ __align__(16) float4 tile[TH + 1][TW + 1];
  __shared__ int colI0[TW], colI1[TW], rowJ0[TH], rowJ1[TH];
  __shared__ float colA[TW], colOma[TW], rowA[TH], rowOma[TH];
  __shared__ float2 rowW[TH];  // (b, 1 - b) of each row, for the staged walk
  __shared__ int chain[4];  // columns up, columns down, rows up, rows down
  const Image& im = p.im;
  const int tid = threadIdx.x;
  int ty = blockIdx.y;  // MIRRORED: row tiles alternately from both ends (as k_sample_grid_sep)
  if (C::addr == A_MIRROR) ty = (ty & 1) ? gridDim.y - 1 - (ty >> 1) : (ty >> 1);
  const int x0 = blockIdx.x * TW, y0 = ty * TH;
  const uint64_t zoff = (uint64_t)blockIdx.z * p.oh;  // 2D slices of the output repeat (A[2] = 0)
  // per-axis addressing: threads [0, TW) take the columns, [TW, TW + TH) the rows
  if (tid < 4) chain[tid] = 1;
  if (tid < TW) {
    const AxL ax =
        axis_l<C>(p.smp, __fadd_rn(__fmul_rn(p.A[0], __int2float_rn(p.ox + x0 + tid)), p.A[3]), im.w);
    colI0[tid] = ax.i0;
    colI1[tid] = ax.i1;
    colA[tid] = ax.a;
    colOma[tid] = ax.oma;
  } else if (tid < TW + TH) {
    const int r = tid - TW;
    const AxL ay =
        axis_l<C>(p.smp, __fadd_rn(__fmul_rn(p.A[5], __int2float_rn(p.oy + y0 + r)), p.A[7]), im.h);
    rowJ0[r] = ay.i0;
    rowJ1[r] = ay.i1;
    rowA[r] = ay.a;
    rowOma[r] = ay.oma;
    rowW[r] = make_float2(ay.a, ay.oma);
  }
  __syncthreads();
  if (tid < TW - 1) {
    if (colI1[tid] != colI0[tid + 1]) chain[0] = 0;
    if (colI0[tid] != colI1[tid + 1]) chain[1] = 0;
  } else if (tid >= TW && tid < TW + TH - 1) {
    const int r = tid - TW;
    if (rowJ1[r] != rowJ0[r + 1]) chain[2] = 0;
    if (rowJ0[r] != rowJ1[r + 1]) chain[3] = 0;
  }
  __syncthreads();
  const bool cup = chain[0], cdn = !cup && chain[1], rup = chain[2], rdn = !rup && chain[3];
  const int warp = tid >> 5, lane = tid & 31;
  const int c = (warp & 1) * 32 + lane, r0 = (warp >> 1) * RPW, x = x0 + c;
  const float a = colA[c], oma = colOma[c];
  float4* out = reinterpret_cast<float4*>(p.out);
  if (!(cup || cdn) || !(rup || rdn)) {  // the taps directly (same operations as linear_at)
    const AxL ax{colI0[c], colI1[c], a, oma, true, true};
#pragma unroll 1
    for (int r = r0; r < r0 + RPW; ++r) {
      const int y = y0 + r;
      if (y >= p.oh) break;
      const char* rows[4] = {row_ptr<C>(im, rowJ0[r], 0), row_ptr<C>(im, rowJ1[r], 0), nullptr, nullptr};
      const bool rok[4] = {true, true, false, false};
      uint32_t res[4];
      linear_at<C>(p, rows, rok, ax, rowA[r], rowOma[r], 0.f, 1.f, res, 4);
      if (x < p.ow)
        __stcs(out + ((zoff + y) * p.ow + x), make_float4(__uint_as_float(res[0]), __uint_as_float(res[1]),
                                                           __uint_as_float(res[2]), __uint_as_float(res[3])));
    }
    return;
  }
  // stage the (TH+1) x (TW+1) footprint with 16-byte async copies (no
  // register round trip): warp w takes slot rows w, w+4, ...; lane l the slot
  // columns l and l+32 (lane 0 also slot TW), whose byte offsets are fixed
  // for the tile -- a copy costs an address add, not an index computation
  {
    const int iA = cup ? colI0[lane] : colI1[lane], iB = cup ? colI0[lane + 32] : colI1[lane + 32];
    const int iC = cup ? colI1[TW - 1] : colI0[TW - 1];
    const uint64_t oA = (uint64_t)(unsigned)iA * 16u, oB = (uint64_t)(unsigned)iB * 16u,
                   oC = (uint64_t)(unsigned)iC * 16u;
    uint32_t dst = static_cast<uint32_t>(__cvta_generic_to_shared(&tile[warp][lane]));
    for (int r = warp; r <= TH; r += 4, dst += 4 * (TW + 1) * 16) {
      const int j = r < TH ? (rup ? rowJ0[r] : rowJ1[r]) : (rup ? rowJ1[TH - 1] : rowJ0[TH - 1]);
      const char* rp = row_ptr<C>(im, j, 0);
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(rp + oA) : "memory");
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst + 32 * 16), "l"(rp + oB) : "memory");
      if (lane == 0)
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst + TW * 16), "l"(rp + oC) : "memory");
    }
  }
  asm volatile("cp.async.wait_all;" ::: "memory");
  __syncthreads();
  // slots of tap i0 / i1 of this column; the row taps are slot rows r, r + 1
  // (upward chain: j0 = r; downward: j1 = r).  One instance of the row walk
  // per chain direction, so no per-sample selects.
  const int ci0 = cup ? c : c + 1, ci1 = cup ? c + 1 : c;
  const int nrow = x < p.ow ? min(RPW, p.oh - (y0 + r0)) : 0;
  float4* orow = out + ((zoff + y0 + r0) * p.ow + x);
  auto walk = [&](auto up) {
    constexpr bool UP = decltype(up)::value;
    const float4* trow = &tile[r0][0];
    auto xblend = [&](const float4* t, float h[4]) {
      const float4 t0 = t[ci0], t1 = t[ci1];
      h[0] = lerp1(a, oma, t0.x, t1.x);
      h[1] = lerp1(a, oma, t0.y, t1.y);
      h[2] = lerp1(a, oma, t0.z, t1.z);
      h[3] = lerp1(a, oma, t0.w, t1.w);
    };
    float hr[4], hn[4];  // x-blends of slot rows r and r + 1
    xblend(trow, hr);
#pragma unroll 4
    for (int r = 0; r < RPW; ++r) {
      trow += TW + 1;
      xblend(trow, hn);
      const float2 bw = rowW[r0 + r];  // (b, 1 - b)
      const float* v0 = UP ? hr : hn;  // the x-blend of row j0
      const float* v1 = UP ? hn : hr;  // ... and of row j1
      if (r < nrow)
        __stcs(orow, make_float4(lerp1(bw.x, bw.y, v0[0], v1[0]), lerp1(bw.x, bw.y, v0[1], v1[1]),
                                 lerp1(bw.x, bw.y, v0[2], v1[2]), lerp1(bw.x, bw.y, v0[3], v1[3])));
      orow += p.ow;
#pragma unroll
      for (int ch = 0; ch < 4; ++ch) hr[ch] = hn[ch];
    }
  };
  if (rup) walk(std::true_type{});
  else walk(std::false_type{});
}

// MIRRORED_REPEAT folds: an output column x and its mirror image Mx - x tap
// (nearly) the same texel columns, and likewise rows.  k_sample_grid_fold
// stages ONE texel box per block -- the union of the taps of a 64 x 16 tile
// of "primary" outputs and of its three mirror images -- and blends all four
// output tiles from it: a quarter of the staging of k_sample_grid_tile per
// output.  The pairing (Mx, My) is the host's guess; every tap is checked
// against the staged box and a tile that does not fit reads its taps
// directly, so results are always linear_at's (bit-identical).
//   Primary columns: xp in [0, Px) maps to x = xp for xp < Ax, else
//   Mx + 1 + (xp - Ax) (the columns whose mirror image is outside the
//   output); column x's partner Mx - x is used when inside [0, ow) and != x.
// Once the box origin is known, each row's two texel rows are turned into
// shared-memory addresses and its output row into a global row pointer, so
// the blend loop addresses a tap with one add and a store with one 64-bit add.
#ifndef B2CL_FOLD_UNROLL
#define B2CL_FOLD_UNROLL 1
#endif
constexpr int kFoldUnroll = B2CL_FOLD_UNROLL;  // output tiles of a block in flight together
#ifndef B2CL_FOLD_WALK_UNROLL
#define B2CL_FOLD_WALK_UNROLL 8
#endif
constexpr int kFoldWalkUnroll = B2CL_FOLD_WALK_UNROLL;  // rows of the walk unrolled

struct FoldMap {
  int Mx, Ax, Px;  // columns
  int My, Ay, Py;  // rows
  int gx, gy, gz;  // tiles along x, y, z
};

__device__ __forceinline__ int fold_prim(int pi, int M, int A) { return pi < A ? pi : M + 1 + (pi - A); }

#ifndef B2CL_FOLD_MINB
#define B2CL_FOLD_MINB 5  // 5 CTAs of 4 warps per SM: at most 96 registers (1: 104 registers, 4 CTAs; 6 / 7: 80 / 72 -- 59.6 / 58.6 / 59.2 vs 57.8 us)
#endif
#ifndef B2CL_FOLD_CTAS
#define B2CL_FOLD_CTAS 0  // persistent CTAs per SM for the fold kernel (0: one CTA per tile)
#endif
#ifndef B2CL_FOLD_PF
#define B2CL_FOLD_PF 0  // L2 prefetch distance in tiles of the fold kernel (0: none; 148 / 444 / 740 measured 61.5 / 61.9 / 61.8 vs 57.7 us)
#endif
#ifndef B2CL_FOLD_TMA
#define B2CL_FOLD_TMA 0  // 1: stage the union box with one cp.async.bulk.tensor.3d (measured 61.5 vs 58.2 us for the 16-B cp.async)
#endif
#ifndef B2CL_FOLD_PAD
#define B2CL_FOLD_PAD 6  // (4 / 5 / 8 within 0.3 us)
#endif
// the staged box: the tile's taps plus room for the mirror images' offsets
#ifndef B2CL_FOLD_TH
#define B2CL_FOLD_TH 16  // primary rows per tile (16 or 32; 32 measured 58.4-60.2 vs 57.7 us)
#endif
constexpr int FOLD_TW = 64, FOLD_TH = B2CL_FOLD_TH, FOLD_BW = FOLD_TW + B2CL_FOLD_PAD, FOLD_BH = FOLD_TH + B2CL_FOLD_PAD;

// one tile's tables: [0] primary, [1] partner; x / y = -1 marks an absent output
struct FoldTables {
  float4 rT[2][FOLD_TH];  // per row: {b, 1 - b, j0, j1} -- j as int bits, or (staged tiles, after
                          // fold_rows_addr) the shared addresses of box rows j0, j1
  uint64_t rO[2][FOLD_TH];  // per row (staged tiles): the output row's address
  int cI0[2][FOLD_TW], cI1[2][FOLD_TW], cX[2][FOLD_TW];
  float cA[2][FOLD_TW], cOma[2][FOLD_TW];
  int rY[2][FOLD_TH];
  int rflag[2][FOLD_TH / 8];  // per row set and 8-row block: 1 chained up, 2 down, 0 neither / absent rows
};

// column c of table h of the tile whose primary columns start at xp0; the
// tap range joins [lo, hi]
template <class C>
__device__ __forceinline__ void fold_col(const SampleParams& p, const FoldMap& fm, FoldTables& T, int h, int c,
                                         int xp0, int& lo, int& hi) {
  const int xp = xp0 + c;
  int x = xp < fm.Px ? fold_prim(xp, fm.Mx, fm.Ax) : -1;
  if (h == 1 && x >= 0) {
    const int xm = fm.Mx - x;
    x = (xm >= 0 && xm < p.ow && xm != x) ? xm : -1;
  }
  T.cX[h][c] = x;
  if (x >= 0) {
    const AxL ax = axis_l<C>(p.smp, __fadd_rn(__fmul_rn(p.A[0], __int2float_rn(p.ox + x)), p.A[3]), p.im.w);
    T.cI0[h][c] = ax.i0; T.cI1[h][c] = ax.i1; T.cA[h][c] = ax.a; T.cOma[h][c] = ax.oma;
    lo = min(lo, min(ax.i0, ax.i1));
    hi = max(hi, max(ax.i0, ax.i1));
  } else {
    T.cI0[h][c] = T.cI1[h][c] = 0x3fffffff;  // (never staged, never stored)
    T.cA[h][c] = 0.f; T.cOma[h][c] = 1.f;
  }
}

// the rows of the tile whose primary rows start at yp0: called by 2 * FOLD_TH
// threads (full warps), idx = hr * FOLD_TH + r computes row r of table hr and (warp ballots) the
// walk direction of each 8-row block of each row set -- all rows present and
// chained UP (j1 of a row = j0 of the next) or DOWN (j0 = j1 of the next)
template <class C>
__device__ __forceinline__ void fold_rows(const SampleParams& p, const FoldMap& fm, FoldTables& T, int idx,
                                          int yp0, int& lo, int& hi) {
  const int hr = idx / FOLD_TH, r = idx % FOLD_TH, lane = idx & 31;
  const int yp = yp0 + r;
  int y = yp < fm.Py ? fold_prim(yp, fm.My, fm.Ay) : -1;
  if (hr == 1 && y >= 0) {
    const int ym = fm.My - y;
    y = (ym >= 0 && ym < p.oh && ym != y) ? ym : -1;
  }
  T.rY[hr][r] = y;
  int j0 = 0, j1 = 0;
  if (y >= 0) {
    const AxL ay = axis_l<C>(p.smp, __fadd_rn(__fmul_rn(p.A[5], __int2float_rn(p.oy + y)), p.A[7]), p.im.h);
    T.rT[hr][r] = make_float4(ay.a, ay.oma, __int_as_float(ay.i0), __int_as_float(ay.i1));
    lo = min(lo, min(ay.i0, ay.i1));
    hi = max(hi, max(ay.i0, ay.i1));
    j0 = ay.i0;
    j1 = ay.i1;
  }
  const int nj0 = __shfl_down_sync(0xffffffffu, j0, 1), nj1 = __shfl_down_sync(0xffffffffu, j1, 1);
  const bool last = (r & 7) == 7;
  const unsigned pres = __ballot_sync(0xffffffffu, y >= 0);
  const unsigned upm = __ballot_sync(0xffffffffu, last || j1 == nj0);
  const unsigned dnm = __ballot_sync(0xffffffffu, last || j0 == nj1);
  if ((r & 7) == 0) {
    const unsigned m = 0xffu << lane;
    T.rflag[hr][r >> 3] = ((pres & m) == m) ? (((upm & m) == m) ? 1 : (((dnm & m) == m) ? 2 : 0)) : 0;
  }
}

// a staged tile's rows (same lanes as fold_rows, after the box origin r0 is
// known): texel rows j0, j1 -> shared addresses of box rows j - r0; output
// row y -> its address in the output slice `out`
__device__ __forceinline__ void fold_rows_addr(const SampleParams& p, FoldTables& T, int idx, uint32_t box_s,
                                               int r0, const float4* out) {
  const int hr = idx / FOLD_TH, r = idx % FOLD_TH;
  const int y = T.rY[hr][r];
  if (y < 0) return;
  const float4 t = T.rT[hr][r];
  const uint32_t a0 = box_s + (uint32_t)(__float_as_int(t.z) - r0) * (FOLD_BW * 16u);
  const uint32_t a1 = box_s + (uint32_t)(__float_as_int(t.w) - r0) * (FOLD_BW * 16u);
  T.rT[hr][r] = make_float4(t.x, t.y, __uint_as_float(a0), __uint_as_float(a1));
  T.rO[hr][r] = reinterpret_cast<uint64_t>(out + (uint64_t)y * p.ow);
}

__device__ __forceinline__ float4 lds_f4(uint32_t a) {
  float4 v;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(a));
  return v;
}

// one warp's unit of a tile: column c (this lane) of column set hc, rows rb ..
// rb + 7 of row set hr; from the box (origin column c0) when staged, else
// the taps directly.  out = the output slice of the tile.
template <class C>
__device__ __forceinline__ void fold_unit(const SampleParams& p, const FoldTables& T, int c0, bool staged,
                                          float4* out, int c, int rb, int hc, int hr) {
  const Image& im = p.im;
  const int x = T.cX[hc][c];
  if (x < 0) return;  // (an absent column: nothing to store)
  const int i0 = T.cI0[hc][c], i1 = T.cI1[hc][c];
  const float a = T.cA[hc][c], oma = T.cOma[hc][c];
  if (!staged) {  // the taps directly
    const AxL ax{i0, i1, a, oma, true, true};
#pragma unroll 1
    for (int r = rb; r < rb + FOLD_TH / 2; ++r) {
      const int y = T.rY[hr][r];
      if (y < 0) continue;
      const float4 ry = T.rT[hr][r];
      const char* rows[4] = {row_ptr<C>(im, __float_as_int(ry.z), 0), row_ptr<C>(im, __float_as_int(ry.w), 0),
                             nullptr, nullptr};
      const bool rok[4] = {true, true, false, false};
      uint32_t res[4];
      linear_at<C>(p, rows, rok, ax, ry.x, ry.y, 0.f, 1.f, res, 4);
      __stcs(out + ((uint64_t)y * p.ow + x), make_float4(__uint_as_float(res[0]), __uint_as_float(res[1]),
                                                           __uint_as_float(res[2]), __uint_as_float(res[3])));
    }
    return;
  }
  // byte offsets of this column's two taps within a staged row, and of its
  // output within an output row
  const uint32_t o0 = (uint32_t)(i0 - c0) * 16u, o1 = (uint32_t)(i1 - c0) * 16u;
  const uint64_t xo = (uint64_t)(unsigned)x * 16u;
  auto xblend = [&](float rowaddr, float4& h) {
    const uint32_t ra = __float_as_uint(rowaddr);
    const float4 t0 = lds_f4(ra + o0);
    const float4 t1 = lds_f4(ra + o1);
    h = make_float4(lerp1(a, oma, t0.x, t1.x), lerp1(a, oma, t0.y, t1.y), lerp1(a, oma, t0.z, t1.z),
                    lerp1(a, oma, t0.w, t1.w));
  };
  auto emit = [&](int r, const float4& ry, const float4& n0, const float4& n1) {
    __stcs(reinterpret_cast<float4*>(T.rO[hr][r] + xo),
           make_float4(lerp1(ry.x, ry.y, n0.x, n1.x), lerp1(ry.x, ry.y, n0.y, n1.y), lerp1(ry.x, ry.y, n0.z, n1.z),
                       lerp1(ry.x, ry.y, n0.w, n1.w)));
  };
  // each 8-row block of the unit: all present and chained one way, so each
  // texel row is x-blended once; otherwise both taps per row
  auto walk = [&](int bk, auto upc) {
    constexpr bool UP = decltype(upc)::value;
    float4 hp;  // x-blend of the texel row shared with the previous output row
    {
      const float4 ry = T.rT[hr][bk];
      xblend(UP ? ry.z : ry.w, hp);
    }
#pragma unroll kFoldWalkUnroll
    for (int r = bk; r < bk + 8; ++r) {
      const float4 ry = T.rT[hr][r];
      float4 hn;
      xblend(UP ? ry.w : ry.z, hn);
      if (UP) emit(r, ry, hp, hn);
      else emit(r, ry, hn, hp);
      hp = hn;
    }
  };
#pragma unroll 1
  for (int bk = rb; bk < rb + FOLD_TH / 2; bk += 8) {
    const int flag = T.rflag[hr][bk >> 3];
    if (flag == 1) {
      walk(bk, std::true_type{});
    } else if (flag == 2) {
      walk(bk, std::false_type{});
    } else {
#pragma unroll 1
      for (int r = bk; r < bk + 8; ++r) {
        if (T.rY[hr][r] < 0) continue;  // (warp-uniform)
        const float4 ry = T.rT[hr][r];
        float4 n0, n1;
        xblend(ry.z, n0);
        xblend(ry.w, n1);
        emit(r, ry, n0, n1);
      }
    }
  }
}

// an estimate of the union box of tile (fx, fy) from the taps of the ends of
// its primary column / row segments, widened by one texel (for the L2
// prefetch of a later tile): called by a full warp, lanes 0-3 columns and 4-7
// rows; {c_lo, c_hi, r_lo, r_hi} clipped to the image, in every lane
template <class C>
__device__ __forceinline__ int4 fold_predict_box(const SampleParams& p, const FoldMap& fm, int fx, int fy, int lane) {
  const bool rowax = lane >= 4;
  const int k = lane & 3;
  const int base = rowax ? fy * FOLD_TH : fx * FOLD_TW, len = rowax ? FOLD_TH : FOLD_TW, P = rowax ? fm.Py : fm.Px;
  const int Aseg = rowax ? fm.Ay : fm.Ax, M = rowax ? fm.My : fm.Mx;
  int pi = k == 0 ? base : (k == 1 ? base + len - 1 : (k == 2 ? Aseg - 1 : Aseg));
  pi = min(max(pi, base), min(base + len, P) - 1);
  int lo = 0x7fffffff, hi = -1;
  if (lane < 8 && pi >= 0) {
    const int o = fold_prim(pi, M, Aseg);
    const float cc = rowax ? __fadd_rn(__fmul_rn(p.A[5], __int2float_rn(p.oy + o)), p.A[7])
                           : __fadd_rn(__fmul_rn(p.A[0], __int2float_rn(p.ox + o)), p.A[3]);
    const AxL a = axis_l<C>(p.smp, cc, rowax ? p.im.h : p.im.w);
    lo = min(a.i0, a.i1);
    hi = max(a.i0, a.i1);
  }
#pragma unroll
  for (int o = 1; o < 4; o <<= 1) {
    lo = min(lo, __shfl_xor_sync(0xffffffffu, lo, o));
    hi = max(hi, __shfl_xor_sync(0xffffffffu, hi, o));
  }
  const int clo = __shfl_sync(0xffffffffu, lo, 0) - 1, chi = __shfl_sync(0xffffffffu, hi, 0) + 1;
  const int rlo = __shfl_sync(0xffffffffu, lo, 4) - 1, rhi = __shfl_sync(0xffffffffu, hi, 4) + 1;
  return make_int4(max(clo, 0), min(chi, p.im.w - 1), max(rlo, 0), min(rhi, p.im.h - 1));
}

template <class C>
__global__ void __launch_bounds__(128, B2CL_FOLD_MINB)
    k_sample_grid_fold(const SampleParams p, const FoldMap fm, const __grid_constant__ CUtensorMap tmap) {
  static_assert(C::type == T_FLOAT && C::order == O_RGBA && C::dims == 2, "2D RGBA32F");
  static_assert(C::addr == A_REPEAT || C::addr == A_MIRROR, "taps always in range");
  constexpr int TW = FOLD_TW, TH = FOLD_TH, BW = FOLD_BW, BH = FOLD_BH;
  __shared__ __align__(128) float4 box[BH][BW];
  __shared__ FoldTables T;
  __shared__ int bb[4];         // column min, max, row min, max of the staged box
  __shared__ uint64_t fbar;     // the TMA box's completion
  const Image& im = p.im;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  // tiles (x fastest): one per CTA, or a grid-stride loop when the launch is
  // persistent (B2CL_FOLD_CTAS: a fixed number of CTAs per SM that run beside
  // the concurrent REPEAT read of the step)
  const long long ntiles = (long long)fm.gx * fm.gy * fm.gz;
  for (long long tile = blockIdx.x + (long long)gridDim.x * (blockIdx.y + (long long)gridDim.y * blockIdx.z);
       tile < ntiles; tile += (long long)gridDim.x * gridDim.y * gridDim.z) {
  const int BX = (int)(tile % fm.gx), BY = (int)((tile / fm.gx) % fm.gy), BZ = (int)(tile / ((long long)fm.gx * fm.gy));
  const int xp0 = BX * TW, yp0 = BY * TH;
  if (tid == 0) { bb[0] = 0x7fffffff; bb[1] = -1; bb[2] = 0x7fffffff; bb[3] = -1; }
  __syncthreads();
  {
    // 128 threads: 64 columns x {primary, partner}; warp 0 also the rows
    int lo = 0x7fffffff, hi = -1;
    fold_col<C>(p, fm, T, tid >> 6, tid & 63, xp0, lo, hi);
    if (hi >= 0) {
      atomicMin(&bb[0], lo);
      atomicMax(&bb[1], hi);
    }
    if (tid < 2 * TH) {
      int rlo = 0x7fffffff, rhi = -1;
      fold_rows<C>(p, fm, T, tid, yp0, rlo, rhi);
      if (rhi >= 0) {
        atomicMin(&bb[2], rlo);
        atomicMax(&bb[3], rhi);
      }
    }
  }
#if B2CL_FOLD_PF
  // warm L2 with the box of the tile B2CL_FOLD_PF launch positions ahead
  // (an estimate: a prefetch only; the tile's own box is computed exactly
  // when it runs)
  if (warp == 3 && !C::shard) {
    const long long t = tile + B2CL_FOLD_PF;
    if (t < ntiles) {
      const int4 e = fold_predict_box<C>(p, fm, (int)(t % fm.gx), (int)((t / fm.gx) % fm.gy), lane);
      if (e.y >= e.x && e.w >= e.z && e.y - e.x < BW + 8 && e.w - e.z < BH + 8 && e.z + lane <= e.w)
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(
                         row_ptr<C>(im, e.z + lane, 0) + (uint64_t)(unsigned)e.x * 16u),
                     "r"((uint32_t)(e.y - e.x + 1) * 16u)
                     : "memory");
    }
  }
#endif
  __syncthreads();
  const int c0 = bb[0], r0 = bb[2];
  const bool staged = bb[1] >= c0 && bb[1] - c0 < BW && bb[3] >= r0 && bb[3] - r0 < BH;
  const uint64_t zoff = (uint64_t)BZ * p.oh;
  float4* out = reinterpret_cast<float4*>(p.out) + zoff * p.ow;
  constexpr bool kTma = B2CL_FOLD_TMA && !C::shard;  // (shard rows may wrap in storage)
  if (staged && kTma) {  // the union box: ONE tensor copy (TMA) of BH rows x BW texels
    if (tid == 0) {
      mbar_init(&fbar, 1);
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      mbar_expect_tx(&fbar, (uint32_t)(BW * BH * 16));
      tma_load_3d(&box[0][0], &tmap, 0, c0, r0, &fbar);
    }
  } else if (staged) {  // warp w copies box rows w, w + 4, ...; 16-byte async copies
    const int nc = bb[1] - c0 + 1, nr = bb[3] - r0 + 1;
    for (int rr = warp; rr < nr; rr += 4) {
      const char* src = row_ptr<C>(im, r0 + rr, 0) + (uint64_t)(unsigned)c0 * 16u;
      const uint32_t dst = smem_u32(&box[rr][0]);
      for (int cc = lane; cc < nc; cc += 32)
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst + cc * 16), "l"(src + cc * 16)
                     : "memory");
    }
  }
  if (staged && tid < 2 * TH) fold_rows_addr(p, T, tid, smem_u32(&box[0][0]), r0, out);
  if (staged && !kTma) asm volatile("cp.async.wait_all;" ::: "memory");
  __syncthreads();
  if (staged && kTma) mbar_wait(&fbar, 0);
  // warp w: columns (w & 1)*32 + lane, rows (w >> 1)*8 .. +8, for each of the
  // four (column set, row set) combinations
  const int c = (warp & 1) * 32 + lane, rb = (warp >> 1) * (TH / 2);
#pragma unroll kFoldUnroll
  for (int combo = 0; combo < 4; ++combo)
    fold_unit<C>(p, T, c0, staged, out, c, rb, combo & 1, combo >> 1);
  __syncthreads();  // (the next tile of a persistent CTA reuses the tables and the box)
  }
}

#ifndef B2CL_LIST_SPT
#define B2CL_LIST_SPT 2  // samples per thread of k_sample_list, strided by the grid (C2 map A list: 1 / 2 / 4 = 116.9 / 106.8 / 109.9 us)
#endif
#ifndef B2CL_LIST_CS
#define B2CL_LIST_CS 0  // 1: coordinates loaded with evict-first (streaming) loads
#endif
template <class C, bool INT_COORD>
__global__ void __launch_bounds__(256) k_sample_list(const SampleParams p) {
  constexpr int stride = C::cdims == 1 ? 1 : (C::cdims == 2 ? 2 : 4);
  constexpr int SPT = B2CL_LIST_SPT;
  const uint64_t nthreads = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t s0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  float c[SPT][3];
  int ic[SPT][3];
  // every coordinate first (SPT loads in flight), then the reads
#pragma unroll
  for (int k = 0; k < SPT; ++k) {
    const uint64_t s = s0 + k * nthreads;
    c[k][0] = c[k][1] = c[k][2] = 0.f;
    ic[k][0] = ic[k][1] = ic[k][2] = 0;
    if (s >= p.n) continue;
    if (INT_COORD) {
      const int32_t* q = reinterpret_cast<const int32_t*>(p.coords) + s * stride;
#pragma unroll
      for (int d = 0; d < C::cdims; ++d) ic[k][d] = q[d];
    } else {
      const float* q = reinterpret_cast<const float*>(p.coords) + s * stride;
      if (stride == 4) {
        const float4 v = B2CL_LIST_CS ? __ldcs(reinterpret_cast<const float4*>(q)) : *reinterpret_cast<const float4*>(q);
        c[k][0] = v.x; c[k][1] = v.y; c[k][2] = v.z;
      } else if (stride == 2) {
        const float2 v = B2CL_LIST_CS ? __ldcs(reinterpret_cast<const float2*>(q)) : *reinterpret_cast<const float2*>(q);
        c[k][0] = v.x; c[k][1] = v.y;
      } else {
        c[k][0] = q[0];
      }
    }
  }
#pragma unroll
  for (int k = 0; k < SPT; ++k) {
    const uint64_t s = s0 + k * nthreads;
    if (s >= p.n) break;
    uint32_t r[4];
    if (INT_COORD) read_image_int<C>(p, ic[k], r);  // the coordinate is the texel index (A30)
    else read_image<C>(p, c[k], r);
    __stcs(reinterpret_cast<uint4*>(p.out) + s, make_uint4(r[0], r[1], r[2], r[3]));
  }
}

// ---------------------------------------------------------------- dispatch
// a shard stores a window of the outer axis (b2clCreateImageShard)
static bool is_shard(const SampleParams& p) {
  if (p.dims < 2 || p.arr) return false;
  return p.im.ob != 0 || p.im.os != (p.dims == 3 ? p.im.d : p.im.h);
}

template <class C, int OUTC>
static cudaError_t go_grid(const SampleParams& p, cudaStream_t st) {
  dim3 blk(32, 8, 1);
  dim3 grd((p.ow + 31) / 32, (p.oh + 7) / 8, p.od);
  if (is_shard(p)) k_sample_grid<WithShard<C, true>, OUTC><<<grd, blk, 0, st>>>(p);
  else k_sample_grid<WithShard<C, false>, OUTC><<<grd, blk, 0, st>>>(p);
  count_launch("k_sample_grid");
  return cudaGetLastError();
}

template <class C, int OUTC, int XPT, int WALK>
static cudaError_t go_walk(const SampleParams& p, cudaStream_t st) {
  dim3 blk(32, 4, 1);
  dim3 grd;
  if (C::dims == 3)
    grd = dim3((p.ow + 128 * XPT - 1) / (128 * XPT), p.oh, (p.od + WALK - 1) / WALK);
  else
    grd = dim3((p.ow + 32 * XPT - 1) / (32 * XPT), (p.oh + 4 * WALK - 1) / (4 * WALK), p.od);
  if (is_shard(p)) k_sample_grid_walk<WithShard<C, true>, OUTC, XPT, WALK><<<grd, blk, 0, st>>>(p);
  else k_sample_grid_walk<WithShard<C, false>, OUTC, XPT, WALK><<<grd, blk, 0, st>>>(p);
  count_launch("k_sample_grid_walk");
  return cudaGetLastError();
}

template <class C, int WALK>
static cudaError_t go_walk4(const SampleParams& p, cudaStream_t st) {
  dim3 blk(32, 4, 1);
  dim3 grd((p.ow + 511) / 512, p.oh, (p.od + WALK - 1) / WALK);
  if (is_shard(p)) k_sample_grid_walk4<WithShard<C, true>, WALK><<<grd, blk, 0, st>>>(p);
  else k_sample_grid_walk4<WithShard<C, false>, WALK><<<grd, blk, 0, st>>>(p);
  count_launch("k_sample_grid_walk4");
  return cudaGetLastError();
}

#ifndef B2CL_C2M_XPT
#define B2CL_C2M_XPT 2
#endif
#ifndef B2CL_C2M_RPW
#define B2CL_C2M_RPW 4
#endif
#ifndef B2CL_TILE_TH
#define B2CL_TILE_TH 16
#endif
template <class C, int TH>
static cudaError_t go_tile(const SampleParams& p, cudaStream_t st) {
  dim3 blk(128, 1, 1);
  dim3 grd((p.ow + 63) / 64, (p.oh + TH - 1) / TH, p.od);
  if (is_shard(p)) k_sample_grid_tile<WithShard<C, true>, 64, TH><<<grd, blk, 0, st>>>(p);
  else k_sample_grid_tile<WithShard<C, false>, 64, TH><<<grd, blk, 0, st>>>(p);
  count_launch("k_sample_grid_tile");
  return cudaGetLastError();
}

// the mirror pairing of one output axis under MIRRORED_REPEAT: the fold point
// (an integer of the coordinate) inside the region, and the index sum M with
// s(x) + s(M - x) = 2 * fold (double arithmetic: a guess the kernel checks)
static bool fold_axis(double a, double c, int o, int n, int* M, int* A, int* P) {
  if (!(a != 0.0) || !std::isfinite(a) || !std::isfinite(c) || n < 64) return false;
  const double s0 = a * o + c, s1 = a * (o + n - 1) + c;
  const double lo = std::min(s0, s1), hi = std::max(s0, s1);
  const double f = std::ceil(lo);
  if (!(f < hi) || f + 1.0 < hi) return false;  // exactly one fold point inside
  const double m = (2.0 * f - 2.0 * c) / a - 2.0 * o;
  if (!(std::fabs(m) < 1e9)) return false;
  const long long Mi = std::llround(m);
  // primary indices: [0, Mi/2] and (Mi, n)
  const long long A1 = std::min<long long>(n, std::max<long long>(0, Mi / 2 + 1));
  const long long A2 = std::max<long long>(0, n - 1 - std::max<long long>(Mi, -1));
  *M = (int)Mi;
  *A = (int)A1;
  *P = (int)(A1 + A2);
  return *P > 0 && *P < n;  // a real fold pairs something
}

template <class C>
static bool go_fold(const SampleParams& p, cudaStream_t st, cudaError_t* err) {
  FoldMap fm;
  if (!p.smp.norm) return false;
  if (!fold_axis((double)p.A[0], (double)p.A[3], p.ox, p.ow, &fm.Mx, &fm.Ax, &fm.Px)) return false;
  if (!fold_axis((double)p.A[5], (double)p.A[7], p.oy, p.oh, &fm.My, &fm.Ay, &fm.Py)) return false;
  fm.gx = (fm.Px + 63) / 64;
  fm.gy = (fm.Py + FOLD_TH - 1) / FOLD_TH;
  fm.gz = p.od;
  dim3 grd(fm.gx, fm.gy, fm.gz);
  static const char* ctas_env = getenv("B2CL_FOLD_CTAS");  // A/B: persistent CTAs per SM (0: one per tile)
  const int ctas = ctas_env ? atoi(ctas_env) : B2CL_FOLD_CTAS;
  if (ctas > 0) {
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const long long nt = (long long)fm.gx * fm.gy * fm.gz;
    grd = dim3((unsigned)std::min<long long>(nt, (long long)sms * ctas), 1, 1);
  }
  // the image as a (4 channels, width, height) fp32 tensor for the box copy
  // (a 70-texel row is 280 floats: over one dimension's 256-element box limit)
  CUtensorMap tm;
  memset(&tm, 0, sizeof(tm));
  bool tma = B2CL_FOLD_TMA && !is_shard(p);
  if (tma) {
    auto enc = tma_encode_fn();
    const cuuint64_t dims[3] = {4, (cuuint64_t)p.im.w, (cuuint64_t)p.im.h};
    const cuuint64_t strides[2] = {16, p.im.rp};
    const cuuint32_t box[3] = {4, (cuuint32_t)FOLD_BW, (cuuint32_t)FOLD_BH};
    const cuuint32_t es[3] = {1, 1, 1};
    tma = enc && !(reinterpret_cast<uintptr_t>(p.im.ptr) & 15) && !(p.im.rp & 15) &&
          enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, p.im.ptr, dims, strides, box, es,
              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
  }
  if (!tma && B2CL_FOLD_TMA && !is_shard(p)) return false;  // (no encoder: the separable path)
  if (is_shard(p)) k_sample_grid_fold<WithShard<C, true>><<<grd, 128, 0, st>>>(p, fm, tm);
  else k_sample_grid_fold<WithShard<C, false>><<<grd, 128, 0, st>>>(p, fm, tm);
  count_launch("k_sample_grid_fold");
  *err = cudaGetLastError();
  return true;
}

template <class C, int OUTC, int XPT, int RPW>
static cudaError_t go_sep(const SampleParams& p, cudaStream_t st) {
  dim3 blk(32, 4, 1);
  dim3 grd((p.ow + 32 * XPT - 1) / (32 * XPT), (p.oh + 4 * RPW - 1) / (4 * RPW), p.od);
  if (is_shard(p)) k_sample_grid_sep<WithShard<C, true>, OUTC, XPT, RPW><<<grd, blk, 0, st>>>(p);
  else k_sample_grid_sep<WithShard<C, false>, OUTC, XPT, RPW><<<grd, blk, 0, st>>>(p);
  count_launch("k_sample_grid_sep");
  return cudaGetLastError();
}

// MIRRORED_REPEAT: one fold per axis inside the region -> the fold kernel;
// otherwise (e.g. a shard's band of output rows that does not reach the
// mirror axis: config 5 at N > 1) the taps chain one way per axis and each
// texel is read about once, like REPEAT -> the staged tile kernel, which
// checks the chaining and reads unchained tiles directly
template <class C>
static cudaError_t fold_or_tile(const SampleParams& p, cudaStream_t st) {
  cudaError_t e = cudaSuccess;
  if (go_fold<C>(p, st, &e)) return e;
  return go_tile<C, B2CL_TILE_TH>(p, st);
}

template <class C>
static cudaError_t go_list(const SampleParams& p, bool int_coord, cudaStream_t st) {
  const uint64_t blocks = (p.n + 256 * B2CL_LIST_SPT - 1) / (256 * B2CL_LIST_SPT);
  using Cs = WithShard<C, true>;
  using Cp = WithShard<C, false>;
  const bool sh = is_shard(p);
  if (int_coord) {
    if (sh) k_sample_list<Cs, true><<<(unsigned)blocks, 256, 0, st>>>(p);
    else k_sample_list<Cp, true><<<(unsigned)blocks, 256, 0, st>>>(p);
  } else {
    if (sh) k_sample_list<Cs, false><<<(unsigned)blocks, 256, 0, st>>>(p);
    else k_sample_list<Cp, false><<<(unsigned)blocks, 256, 0, st>>>(p);
  }
  count_launch("k_sample_list");
  return cudaGetLastError();
}

template <int DIMS>
using Generic = Cfg<DIMS, RT, RT, RT, RT, RT, RT>;

// tile shapes of the hot instances (overridable at build time for A/B
// variants, tools/build_variant.py)
#ifndef B2CL_C3_XPT
#define B2CL_C3_XPT 4
#endif
#ifndef B2CL_C3_WALK
#define B2CL_C3_WALK 32
#endif

// hot configurations (BASELINE.json configs 1-3)
using C2Repeat = Cfg<2, T_FLOAT, O_RGBA, 1, A_REPEAT, F_LINEAR, R_F>;
using C2Mirror = Cfg<2, T_FLOAT, O_RGBA, 1, A_MIRROR, F_LINEAR, R_F>;
using C3Cte = Cfg<3, T_FLOAT, O_R, 1, A_CTE, F_LINEAR, R_F>;
using C1Clamp = Cfg<2, T_UNORM8, O_RGBA, 0, A_CLAMP, F_NEAREST, R_F>;

template <int DIMS>
static bool matches(const SampleParams& p, int type, int order, int norm, int addr, int filt) {
  return p.dims == DIMS && p.im.type == type && p.im.order == order && p.smp.norm == norm &&
         p.smp.addr == addr && p.smp.filt == filt && p.rclass == ret_class(type);
}

// every coefficient that couples an output axis into another coordinate is 0
static bool separable(const SampleParams& p) {
  const float* A = p.A;
  bool ok = A[1] == 0.0f && A[2] == 0.0f;
  if (p.dims > 1) ok = ok && A[4] == 0.0f && A[6] == 0.0f;
  if (p.dims > 2) ok = ok && A[8] == 0.0f && A[9] == 0.0f;
  return ok;
}

cudaError_t launch_sample(const SampleParams& p, int coord_mode, cudaStream_t st) {
  if (p.im.tiled) {  // tiled storage (2D): the one-thread-per-sample kernels with tiled addressing
    if (coord_mode == COORD_GRID) {
      if ((uint64_t)p.ow * p.oh * p.od == 0) return cudaSuccess;
      if (p.outc == 4 && matches<2>(p, T_FLOAT, O_RGBA, 1, A_REPEAT, F_LINEAR))
        return go_grid<TiledStore<C2Repeat>, 4>(p, st);
      if (p.outc == 4 && matches<2>(p, T_FLOAT, O_RGBA, 1, A_MIRROR, F_LINEAR))
        return go_grid<TiledStore<C2Mirror>, 4>(p, st);
      return go_grid<Generic<2>, RT>(p, st);
    }
    return p.n == 0 ? cudaSuccess : go_list<Generic<2>>(p, coord_mode == COORD_LIST_I, st);
  }
  if (coord_mode == COORD_GRID) {
    if ((uint64_t)p.ow * p.oh * p.od == 0) return cudaSuccess;
    // B2CL_GRID_KERNEL=general|sep|walk|4|tile|box forces a kernel family (A/B runs under ncu);
    // the default picks the variant measured fastest on B200 for each hot config
    static const char* force = getenv("B2CL_GRID_KERNEL");
    const int fk = !force ? 0 : (force[0] == 'g' ? 1 : (force[0] == 's' ? 2 : (force[0] == 'w' ? 3 : (force[0] == '4' ? 4 : (force[0] == 't' ? 5 : (force[0] == 'b' ? 6 : 0))))));
    if (fk == 6 && !is_shard(p)) {  // b: the footprint-box kernel for any map it accepts
      bool used = false;
      const cudaError_t e = launch_sample_box(p, st, &used);
      if (used || e != cudaSuccess) return e;
    }
    if (p.arr)  // image arrays: the general kernel, fully run-time format and sampler
      return p.dims == 1 ? go_grid<Layered<Generic<1>>, RT>(p, st) : go_grid<Layered<Generic<2>>, RT>(p, st);
    if (separable(p) && fk != 1) {
      if (p.outc == 4 && matches<2>(p, T_FLOAT, O_RGBA, 1, A_REPEAT, F_LINEAR))
        return fk == 3   ? go_walk<C2Repeat, 4, 2, 8>(p, st)
               : fk == 2 ? go_sep<C2Repeat, 4, 2, 4>(p, st)
                         : go_tile<C2Repeat, B2CL_TILE_TH>(p, st);
      if (p.outc == 4 && matches<2>(p, T_FLOAT, O_RGBA, 1, A_MIRROR, F_LINEAR))
        return fk == 3   ? go_walk<C2Mirror, 4, 2, 8>(p, st)
               : fk == 5 ? go_tile<C2Mirror, B2CL_TILE_TH>(p, st)
               : fk == 2 ? go_sep<C2Mirror, 4, B2CL_C2M_XPT, B2CL_C2M_RPW>(p, st)
               : fold_or_tile<C2Mirror>(p, st);
      if (p.outc == 1 && matches<3>(p, T_FLOAT, O_R, 1, A_CTE, F_LINEAR)) {
        if (fk == 0 && !is_shard(p)) {
          bool used = false;
          const cudaError_t e = launch_sample_vol(p, st, &used);
          if (used || e != cudaSuccess) return e;
        }
        return fk == 2   ? go_sep<C3Cte, 1, 4, 4>(p, st)
               : fk == 3 ? go_walk<C3Cte, 1, B2CL_C3_XPT, B2CL_C3_WALK>(p, st)
                         : go_walk4<C3Cte, B2CL_C3_WALK>(p, st);
      }
      if (p.outc == 4 && matches<2>(p, T_UNORM8, O_RGBA, 0, A_CLAMP, F_NEAREST)) return go_sep<C1Clamp, 4, 2, 4>(p, st);
      switch (p.dims) {
        case 1: return go_sep<Generic<1>, RT, 2, 2>(p, st);
        case 2: return go_sep<Generic<2>, RT, 2, 2>(p, st);
        default: return go_sep<Generic<3>, RT, 2, 2>(p, st);
      }
    }
    // any other affine map of a 2D RGBA32F image (rotations): the TMA-staged
    // footprint box (sample_box.cu), else one thread per sample
    if (fk == 0 && !is_shard(p)) {
      bool used = false;
      const cudaError_t e = launch_sample_box(p, st, &used);
      if (used || e != cudaSuccess) return e;
    }
    if (p.outc == 4 && matches<2>(p, T_FLOAT, O_RGBA, 1, A_REPEAT, F_LINEAR)) return go_grid<C2Repeat, 4>(p, st);
    if (p.outc == 4 && matches<2>(p, T_FLOAT, O_RGBA, 1, A_MIRROR, F_LINEAR)) return go_grid<C2Mirror, 4>(p, st);
    if (p.outc == 1 && matches<3>(p, T_FLOAT, O_R, 1, A_CTE, F_LINEAR)) {
      if (fk == 0 && !is_shard(p)) {
        bool used = false;
        const cudaError_t e = launch_sample_volr(p, st, &used);
        if (used || e != cudaSuccess) return e;
      }
      return go_grid<C3Cte, 1>(p, st);
    }
    switch (p.dims) {
      case 1: return go_grid<Generic<1>, RT>(p, st);
      case 2: return go_grid<Generic<2>, RT>(p, st);
      default: return go_grid<Generic<3>, RT>(p, st);
    }
  }
  if (p.n == 0) return cudaSuccess;
  const bool ic = coord_mode == COORD_LIST_I;
  if (p.arr)
    return p.dims == 1 ? go_list<Layered<Generic<1>>>(p, ic, st) : go_list<Layered<Generic<2>>>(p, ic, st);
  if (!ic && matches<2>(p, T_FLOAT, O_RGBA, 1, A_REPEAT, F_LINEAR)) return go_list<C2Repeat>(p, false, st);
  if (!ic && matches<2>(p, T_FLOAT, O_RGBA, 1, A_MIRROR, F_LINEAR)) return go_list<C2Mirror>(p, false, st);
  if (!ic && matches<2>(p, T_UNORM8, O_RGBA, 0, A_CLAMP, F_NEAREST)) return go_list<C1Clamp>(p, false, st);
  switch (p.dims) {
    case 1: return go_list<Generic<1>>(p, ic, st);
    case 2: return go_list<Generic<2>>(p, ic, st);
    default: return go_list<Generic<3>>(p, ic, st);
  }
}

static std::atomic<uint64_t> g_launches{0};
static thread_local const char* g_last_kernel = "";
void count_launch(const char* kernel) {
  g_launches.fetch_add(1, std::memory_order_relaxed);
  g_last_kernel = kernel ? kernel : "";
}
uint64_t launch_count() { return g_launches.load(std::memory_order_relaxed); }
const char* last_kernel() { return g_last_kernel; }

}  // namespace b2cl
