// read.cuh -- the read built-in (read_imagef / read_imagei / read_imageui)
// for one coordinate, shared by the library's kernels (csrc/kernels/sample.cu)
// and by user kernels through include/b2cl_device.cuh.
//
// Everything is templated on a configuration C (Cfg: dims, format, sampler,
// each possibly decided at run time) and on a parameter block P providing
// `im` (dev::Image), `smp` (dev::Sampler) and `rclass` (dev::RetCode).
// Rules: [CL1.2 §8.1-8.3] as implemented in image.cuh.
#pragma once
#include "image.cuh"

namespace b2cl {
using namespace dev;

template <int DIMS, int TYPE, int ORDER, int NORM, int ADDR, int FILT, int RC>
struct Cfg {
  static constexpr int dims = DIMS, type = TYPE, order = ORDER, norm = NORM, addr = ADDR,
                       filt = FILT, rc = RC;
  static constexpr int nch = ORDER == RT ? RT : order_channels(ORDER);
  static constexpr bool arr = false;   // image array (see Layered)
  static constexpr int cdims = DIMS;   // coordinates per sample
  static constexpr bool tiled = false; // compile-time tiled storage (see TiledStore)
};

// C reading a TILED image (B2CL_MEM_TILED_IMAGE) with its format compiled in
template <class C>
struct TiledStore : C {
  static constexpr bool tiled = true;
};

// C with the image-shard row mapping compiled in (SH) or out (plain images)
template <class C, bool SH>
struct WithShard : C {
  static constexpr bool shard = SH;
};

// C read from an image array: coordinate dims selects the layer, stored on
// the axis after the sampled ones (rows of a 1D array, slices of a 2D array)
template <class C>
struct Layered : C {
  static constexpr bool arr = true;
  static constexpr int cdims = C::dims + 1;
};

// [CL1.2 §8.4]: layer = clamp(rint(c), 0, n - 1).  cvt.rni rounds half to
// even, saturates, and gives 0 for NaN (reading A35).
__device__ __forceinline__ int layer_of(float c, int n) {
  return min(max(__float2int_rn(c), 0), n - 1);
}

// coordinate of output (x,y,z) under the affine map: ((A0*x + A1*y) + A2*z) + A3
__device__ __forceinline__ float affine_coord(const float* A, float x, float y, float z) {
  float v = __fmul_rn(A[0], x);
  v = __fadd_rn(v, __fmul_rn(A[1], y));
  v = __fadd_rn(v, __fmul_rn(A[2], z));
  return __fadd_rn(v, A[3]);
}

struct AxN {  // NEAREST, one axis
  int i;
  bool ok;
};
struct AxL {  // LINEAR, one axis
  int i0, i1;
  float a, oma;
  bool ok0, ok1;
};

template <class C>
__device__ __forceinline__ bool may_border(const Sampler& s) {
  if constexpr (C::addr == RT) return s.addr == A_NONE || s.addr == A_CLAMP;
  else return C::addr == A_NONE || C::addr == A_CLAMP;
}

template <class C>
__device__ __forceinline__ AxN axis_n(const Sampler& s, float c, int n) {
  AxN r;
  if constexpr (C::addr == RT) r.i = axis_nearest_rt(s.addr, s.norm, c, n);
  else r.i = axis_nearest<C::addr, C::norm>(c, n);
  r.ok = !may_border<C>(s) || in_range(r.i, n);
  return r;
}

template <class C>
__device__ __forceinline__ AxL axis_l(const Sampler& s, float c, int n) {
  AxL r;
  if constexpr (C::addr == RT) axis_linear_rt(s.addr, s.norm, c, n, r.i0, r.i1, r.a);
  else axis_linear<C::addr, C::norm>(c, n, r.i0, r.i1, r.a);
  r.oma = __fsub_rn(1.0f, r.a);
  const bool b = may_border<C>(s);
  r.ok0 = !b || in_range(r.i0, n);
  r.ok1 = !b || in_range(r.i1, n);
  return r;
}

template <class C, class P>
__device__ __forceinline__ int filt_of(const P& p) {
  return C::filt == RT ? p.smp.filt : C::filt;
}

// start of texel row (j,k): ptr + k*slice_pitch + j*row_pitch (Fig. 6)
// The outer index o (j of a 2D image, k of a 3D image) is a global index; its
// storage row is (o - ob) mod extent, clamped into the stored rows (a tap
// outside a shard's band + halo reads the nearest stored row: the caller
// provides the halo; this only keeps the access in bounds).
__device__ __forceinline__ int storage_row(const Image& im, int o, int extent) {
  int l = o - im.ob;
  l += l < 0 ? extent : 0;
  l -= l >= extent ? extent : 0;
  return min(max(l, 0), im.os - 1);
}

// Tiled images (Image::tiled) reach only the run-time-format instances
// (C::type == RT: the library's dispatch routes them there, and the device
// header's built-ins are all run-time); the compile-time hot instances keep
// the plain pitched addressing with no extra test.
template <class C>
__device__ __forceinline__ bool tiled_of(const Image& im) {
  if constexpr (C::tiled) return true;
  else if constexpr (C::type == RT) return im.tiled != 0;
  else return false;
}

template <class C>
__device__ __forceinline__ const char* row_ptr(const Image& im, int j, int k) {
  if (tiled_of<C>(im)) return tiled_row(im, j);  // (2D only: k = 0)
  if constexpr (C::shard) {
    if (C::dims == 3) k = storage_row(im, k, im.d);
    else if (C::dims == 2) j = storage_row(im, j, im.h);
  }
  const char* r = im.ptr + (uint64_t)(unsigned)k * im.sp + (uint64_t)(unsigned)j * im.rp;
  // keep the absolute row pointer in registers: without this the compiler
  // re-associates ptr + (row + i*es) and pays two extra 64-bit adds per tap
  asm("" : "+l"(r));
  return r;
}

// does any output component come from a constant of the channel map (0 or 1)?
// Only those need the explicit NaN of reading A26; stored channels carry the
// NaN weight through the blend by themselves.
__device__ __forceinline__ bool const_in_output(int order, int outc) {
  switch (order) {
    case O_RGBA: case O_BGRA: case O_ARGB: case O_INTENSITY: case O_RGBX: return false;
    case O_RGB: return outc > 3;
    case O_R: return outc > 1;
    case O_RG: case O_RA: return outc > 1 + (order == O_RG);
    case O_LUMINANCE: return outc > 3;
    default: return true;  // O_A
  }
}

template <class C>
__device__ __forceinline__ int elem_size(const Image& im) {
  return (C::type == RT || C::nch == RT) ? im.es : texel_bytes(C::type, C::order);
}

// memory-order channels of the texel at row + i*elem_size (zero if !ok)
template <class C>
__device__ __forceinline__ void fetch(const Image& im, const char* row, int i, bool ok, int rc,
                                      uint32_t m[4]) {
  const int type = C::type == RT ? im.type : C::type;
  const int nch = C::nch == RT ? im.nch : C::nch;
  const int es = elem_size<C>(im);
  m[0] = m[1] = m[2] = m[3] = 0u;
  if (!ok) return;
  Raw r = load_raw(row + (tiled_of<C>(im) ? tiled_col(im, i) : (uint64_t)(unsigned)i * (unsigned)es), es);
  if (is_packed(type)) {  // normalized only (read_imagef)
    unpack_rgb(r.w[0], type, m);
    // CL_RGBx: the in-range alpha 1 is carried as a channel, so that a border
    // tap (alpha 0, [CL1.2 §6.12.14.1]) blends into it
    if ((C::order == RT ? im.order : C::order) == O_RGBX) m[3] = 0x3f800000u;
    return;
  }
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    if (c < nch) {
      uint32_t v = channel_code(r, c, type);
      m[c] = rc == R_F ? __float_as_uint(code_to_float(v, type)) : v;
    }
  }
}

// NEAREST: one texel, channel-mapped
template <class C, class P>
__device__ __forceinline__ void nearest_at(const P& p, const char* row, const AxN& x,
                                           bool row_ok, uint32_t res[4]) {
  const int rc = C::rc == RT ? p.rclass : C::rc;
  const int order = C::order == RT ? p.im.order : C::order;
  uint32_t m[4];
  fetch<C>(p.im, row, x.i, row_ok && x.ok, rc, m);
  map_order(order, m, rc == R_F ? 0x3f800000u : 1u, res);
}

// LINEAR from the texel rows: rows[0] = (j0,k0), [1] = (j1,k0), [2] = (j0,k1),
// [3] = (j1,k1); blend x, then y, then z ([CL1.2 §8.2] weights, separable form)
template <class C, class P>
__device__ __forceinline__ void linear_at(const P& p, const char* const rows[4],
                                          const bool rok[4], const AxL& x, float b, float omb,
                                          float g, float omg, uint32_t res[4], int outc = 4) {
  constexpr int NR = C::dims == 1 ? 1 : (C::dims == 2 ? 2 : 4);
  const int order = C::order == RT ? p.im.order : C::order;
  // channels blended: the stored ones (CL_RGBx: also its alpha, see fetch)
  const int nch = order == O_RGBX ? 4 : (C::nch == RT ? p.im.nch : C::nch);
  uint32_t t0[NR][4], t1[NR][4];
#pragma unroll
  for (int r = 0; r < NR; ++r) {
    fetch<C>(p.im, rows[r], x.i0, rok[r] && x.ok0, R_F, t0[r]);
    fetch<C>(p.im, rows[r], x.i1, rok[r] && x.ok1, R_F, t1[r]);
  }
  uint32_t m[4];
#pragma unroll
  for (int ch = 0; ch < 4; ++ch) {
    float v[NR];
#pragma unroll
    for (int r = 0; r < NR; ++r)
      v[r] = lerp1(x.a, x.oma, __uint_as_float(t0[r][ch]), __uint_as_float(t1[r][ch]));
    float o = v[0];
    if constexpr (C::dims >= 2) {
      const float s0 = lerp1(b, omb, v[0], v[1]);
      o = s0;
      if constexpr (C::dims == 3) o = lerp1(g, omg, s0, lerp1(b, omb, v[2], v[3]));
    }
    // channels the format does not store stay exactly 0 / 1 after the map
    m[ch] = ch < nch ? __float_as_uint(o) : 0u;
  }
  map_order(order, m, 0x3f800000u, res);
  // a NaN weight (non-finite coordinate) makes the spec's sum NaN in every
  // component, including the constant ones (reading A26)
  if (const_in_output(order, outc) && (x.a != x.a || b != b || g != g))
    res[0] = res[1] = res[2] = res[3] = 0x7fffffffu;
}

// The built-in on one coordinate: c[0..DIMS-1] -> res (x,y,z,w) as 32-bit patterns.
template <class C, class P>
__device__ __forceinline__ void read_image(const P& p, const float c[3],
                                           uint32_t res[4], int outc = 4) {
  const Image& im = p.im;
  // an array's layer: the row (1D array) or slice (2D array) index, always
  // in range, weight 1 -- the sampler never touches it
  int layer = 0;
  if constexpr (C::arr) layer = layer_of(c[C::dims], C::dims == 1 ? im.h : im.d);
  if (filt_of<C>(p) == F_NEAREST) {
    const AxN x = axis_n<C>(p.smp, c[0], im.w);
    AxN y{0, true}, z{0, true};
    if (C::dims > 1) y = axis_n<C>(p.smp, c[1], im.h);
    if (C::dims > 2) z = axis_n<C>(p.smp, c[2], im.d);
    if constexpr (C::arr) (C::dims == 1 ? y : z) = AxN{layer, true};
    nearest_at<C>(p, row_ptr<C>(im, y.i, z.i), x, y.ok && z.ok, res);
  } else {
    const AxL x = axis_l<C>(p.smp, c[0], im.w);
    AxL y{0, 0, 0.f, 1.f, true, true}, z{0, 0, 0.f, 1.f, true, true};
    if (C::dims > 1) y = axis_l<C>(p.smp, c[1], im.h);
    if (C::dims > 2) z = axis_l<C>(p.smp, c[2], im.d);
    if constexpr (C::arr) (C::dims == 1 ? y : z) = AxL{layer, layer, 0.f, 1.f, true, true};
    const char* rows[4] = {row_ptr<C>(im, y.i0, z.i0), row_ptr<C>(im, y.i1, z.i0),
                           row_ptr<C>(im, y.i0, z.i1), row_ptr<C>(im, y.i1, z.i1)};
    const bool rok[4] = {y.ok0 && z.ok0, y.ok1 && z.ok0, y.ok0 && z.ok1, y.ok1 && z.ok1};
    linear_at<C>(p, rows, rok, x, y.a, y.oma, z.a, z.oma, res, outc);
  }
}

// The built-in on integer coordinates (reading A30): NEAREST, unnormalized,
// non-wrapping; the coordinate IS the texel index, i = address_mode(coord)
// (CLAMP_TO_EDGE clamps into [0, n-1]; NONE and CLAMP give the border out of
// range), exact at any width.  An array's layer is clamp(coord, 0, n-1).
template <class C, class P>
__device__ __forceinline__ void read_image_int(const P& p, const int ic[3], uint32_t res[4]) {
  const Image& im = p.im;
  const int addr = C::addr == RT ? p.smp.addr : C::addr;
  const int n[3] = {im.w, im.h, im.d};
  AxN a[3] = {{0, true}, {0, true}, {0, true}};
#pragma unroll
  for (int d = 0; d < C::dims; ++d) {
    a[d].i = addr == A_CTE ? min(max(ic[d], 0), n[d] - 1) : ic[d];
    a[d].ok = in_range(a[d].i, n[d]);
  }
  if constexpr (C::arr) a[C::dims] = AxN{min(max(ic[C::dims], 0), n[C::dims] - 1), true};
  nearest_at<C>(p, row_ptr<C>(im, a[1].i, a[2].i), a[0], a[1].ok && a[2].ok, res);
}

}  // namespace b2cl
