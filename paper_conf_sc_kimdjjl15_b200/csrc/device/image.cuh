// image.cuh -- device-side OpenCL image built-ins for sm_100a.
//
// The paper implements read_imageX / write_imageX as CUDA device wrappers
// that read and write through the CLImage pointer (
// CLImage fields Fig. 6).  Here the image is a by-value POD
// descriptor (reading A27: "an object with type CLImage is used as a CUDA
// kernel argument") and every rule is [CL1.2 §8.1-8.3]:
//   - addressing / filtering: [CL1.2 §8.2], each fp32 op a separate RN op
//     (__fmul_rn / __fadd_rn / __fsub_rn never contract, reading A2);
//   - (int)floor(x) is cvt.rmi.s32.f32: saturating, NaN -> 0 (reading A3);
//   - conversions: [CL1.2 §8.3] (readings A11-A14);
//   - border colour: every in-scope channel order's border equals the
//     channel map of an all-zero texel (reading A8), so an out-of-range tap
//     fetches a zero texel and goes through the same map.
// This header shares no code with oracle/ (the CPU oracle).
#pragma once
#include <cuda_fp16.h>
#include <stdint.h>

#include "codes.h"

namespace b2cl {
namespace dev {

// ------------------------------------------------------------------------
// addressing, one axis ([CL1.2 §8.2])
// ------------------------------------------------------------------------
__device__ __forceinline__ int ifloor(float x) { return __float2int_rd(x); }

template <int ADDR>
__device__ __forceinline__ int am_nonwrap(int i, int n) {
  if (ADDR == A_CTE) return min(max(i, 0), n - 1);
  if (ADDR == A_CLAMP) return min(max(i, -1), n);
  return i;
}

// NEAREST index (may be out of range only for NONE / CLAMP).
template <int ADDR, int NORM>
__device__ __forceinline__ int axis_nearest(float s, int n) {
  const float fn = __int2float_rn(n);
  if (ADDR == A_REPEAT) {
    float u = __fmul_rn(__fsub_rn(s, floorf(s)), fn);
    int i = ifloor(u);
    return i > n - 1 ? i - n : i;
  } else if (ADDR == A_MIRROR) {
    float sp = __fmul_rn(2.0f, rintf(__fmul_rn(0.5f, s)));
    sp = fabsf(__fsub_rn(s, sp));
    int i = ifloor(__fmul_rn(sp, fn));
    return min(i, n - 1);
  } else {
    float u = NORM ? __fmul_rn(s, fn) : s;
    return am_nonwrap<ADDR>(ifloor(u), n);
  }
}

// LINEAR indices and weight.
template <int ADDR, int NORM>
__device__ __forceinline__ void axis_linear(float s, int n, int& i0, int& i1, float& a) {
  const float fn = __int2float_rn(n);
  float u;
  if (ADDR == A_REPEAT) {
    u = __fmul_rn(__fsub_rn(s, floorf(s)), fn);
  } else if (ADDR == A_MIRROR) {
    float sp = __fmul_rn(2.0f, rintf(__fmul_rn(0.5f, s)));
    sp = fabsf(__fsub_rn(s, sp));
    u = __fmul_rn(sp, fn);
  } else {
    u = NORM ? __fmul_rn(s, fn) : s;
  }
  const float t = __fsub_rn(u, 0.5f);
  const float ft = floorf(t);
  const int b = ifloor(t);
  a = __fsub_rn(t, ft);
  if (ADDR == A_REPEAT) {
    i0 = b < 0 ? b + n : b;
    i1 = b + 1 > n - 1 ? b + 1 - n : b + 1;
  } else if (ADDR == A_MIRROR) {
    i0 = max(b, 0);
    i1 = min(b + 1, n - 1);
  } else {
    i0 = am_nonwrap<ADDR>(b, n);
    i1 = am_nonwrap<ADDR>(min(b, 0x7ffffffe) + 1, n);  // b+1 without int32 overflow
  }
}

// run-time dispatch of the addressing mode (generic kernels)
__device__ __forceinline__ int axis_nearest_rt(int addr, int norm, float s, int n) {
  switch (addr) {
    case A_REPEAT: return axis_nearest<A_REPEAT, 1>(s, n);
    case A_MIRROR: return axis_nearest<A_MIRROR, 1>(s, n);
    case A_CTE: return norm ? axis_nearest<A_CTE, 1>(s, n) : axis_nearest<A_CTE, 0>(s, n);
    case A_CLAMP: return norm ? axis_nearest<A_CLAMP, 1>(s, n) : axis_nearest<A_CLAMP, 0>(s, n);
    default: return norm ? axis_nearest<A_NONE, 1>(s, n) : axis_nearest<A_NONE, 0>(s, n);
  }
}
__device__ __forceinline__ void axis_linear_rt(int addr, int norm, float s, int n, int& i0,
                                               int& i1, float& a) {
  switch (addr) {
    case A_REPEAT: axis_linear<A_REPEAT, 1>(s, n, i0, i1, a); break;
    case A_MIRROR: axis_linear<A_MIRROR, 1>(s, n, i0, i1, a); break;
    case A_CTE:
      if (norm) axis_linear<A_CTE, 1>(s, n, i0, i1, a); else axis_linear<A_CTE, 0>(s, n, i0, i1, a);
      break;
    case A_CLAMP:
      if (norm) axis_linear<A_CLAMP, 1>(s, n, i0, i1, a); else axis_linear<A_CLAMP, 0>(s, n, i0, i1, a);
      break;
    default:
      if (norm) axis_linear<A_NONE, 1>(s, n, i0, i1, a); else axis_linear<A_NONE, 0>(s, n, i0, i1, a);
      break;
  }
}

__device__ __forceinline__ bool in_range(int i, int n) { return (unsigned)i < (unsigned)n; }

// ------------------------------------------------------------------------
// texel load and conversion ([CL1.2 §8.3])
// ------------------------------------------------------------------------
// Raw texel: up to 16 bytes as four 32-bit words, loaded with one vector
// access of the element size (rows are 128-B aligned, so every texel is
// naturally aligned).
struct Raw {
  uint32_t w[4];
};

__device__ __forceinline__ Raw load_raw(const char* p, int es) {
  Raw r;
  r.w[0] = r.w[1] = r.w[2] = r.w[3] = 0u;
  switch (es) {
    case 16: { uint4 v = __ldg(reinterpret_cast<const uint4*>(p)); r.w[0] = v.x; r.w[1] = v.y; r.w[2] = v.z; r.w[3] = v.w; break; }
    case 8: { uint2 v = __ldg(reinterpret_cast<const uint2*>(p)); r.w[0] = v.x; r.w[1] = v.y; break; }
    case 4: r.w[0] = __ldg(reinterpret_cast<const unsigned int*>(p)); break;
    case 2: r.w[0] = __ldg(reinterpret_cast<const unsigned short*>(p)); break;
    default: r.w[0] = __ldg(reinterpret_cast<const unsigned char*>(p)); break;
  }
  return r;
}

// stored code of channel c (memory order), zero/sign extended to 32 bits
__device__ __forceinline__ uint32_t channel_code(const Raw& r, int c, int type) {
  const int tb = type_bytes(type);
  uint32_t v;
  if (tb == 4) {
    v = r.w[c];
  } else if (tb == 2) {
    v = (r.w[c >> 1] >> ((c & 1) * 16)) & 0xffffu;
    if (type == T_SNORM16 || type == T_SINT16) v = (uint32_t)(int32_t)(int16_t)v;
  } else {
    v = (r.w[0] >> (c * 8)) & 0xffu;
    if (type == T_SNORM8 || type == T_SINT8) v = (uint32_t)(int32_t)(int8_t)v;
  }
  return v;
}

// read conversion to float (read_imagef), correctly rounded c/d (reading A11)
__device__ __forceinline__ float code_to_float(uint32_t v, int type) {
  switch (type) {
    case T_UNORM8: return __fdiv_rn(__uint2float_rn(v), 255.0f);
    case T_UNORM16: return __fdiv_rn(__uint2float_rn(v), 65535.0f);
    case T_SNORM8: return fmaxf(-1.0f, __fdiv_rn(__int2float_rn((int)v), 127.0f));
    case T_SNORM16: return fmaxf(-1.0f, __fdiv_rn(__int2float_rn((int)v), 32767.0f));
    case T_HALF: return __half2float(__ushort_as_half((unsigned short)v));
    default: return __uint_as_float(v);  // CL_FLOAT: bit copy (A14)
  }
}

// Packed word ([CL1.2 §5.3.1.1]: 565 = R 15:11, G 10:5, B 4:0; 555 = x 15,
// R 14:10, G 9:5, B 4:0; 101010 = x 31:30, R 29:20, G 19:10, B 9:0) ->
// R, G, B as floats c / (2^bits - 1), correctly rounded (reading A11)
__device__ __forceinline__ void unpack_rgb(uint32_t w, int type, uint32_t m[3]) {
  uint32_t c[3];
  float d[3];
  if (type == T_U565) {
    c[0] = (w >> 11) & 31u; c[1] = (w >> 5) & 63u; c[2] = w & 31u;
    d[0] = 31.0f; d[1] = 63.0f; d[2] = 31.0f;
  } else if (type == T_U555) {
    c[0] = (w >> 10) & 31u; c[1] = (w >> 5) & 31u; c[2] = w & 31u;
    d[0] = d[1] = d[2] = 31.0f;
  } else {
    c[0] = (w >> 20) & 1023u; c[1] = (w >> 10) & 1023u; c[2] = w & 1023u;
    d[0] = d[1] = d[2] = 1023.0f;
  }
#pragma unroll
  for (int k = 0; k < 3; ++k) m[k] = __float_as_uint(__fdiv_rn(__uint2float_rn(c[k]), d[k]));
}

// memory-order channel slots -> (x,y,z,w); one = 1.0f bits or integer 1
// (CL_RGBx: the fetch supplies slot 3 -- 1 in range, 0 for the border)
__device__ __forceinline__ void map_order(int order, const uint32_t m[4], uint32_t one,
                                          uint32_t out[4]) {
  switch (order) {
    case O_R: out[0] = m[0]; out[1] = 0; out[2] = 0; out[3] = one; break;
    case O_A: out[0] = 0; out[1] = 0; out[2] = 0; out[3] = m[0]; break;
    case O_RG: out[0] = m[0]; out[1] = m[1]; out[2] = 0; out[3] = one; break;
    case O_RA: out[0] = m[0]; out[1] = 0; out[2] = 0; out[3] = m[1]; break;
    case O_BGRA: out[0] = m[2]; out[1] = m[1]; out[2] = m[0]; out[3] = m[3]; break;
    case O_ARGB: out[0] = m[1]; out[1] = m[2]; out[2] = m[3]; out[3] = m[0]; break;
    case O_INTENSITY: out[0] = m[0]; out[1] = m[0]; out[2] = m[0]; out[3] = m[0]; break;
    case O_LUMINANCE: out[0] = m[0]; out[1] = m[0]; out[2] = m[0]; out[3] = one; break;
    case O_RGB: out[0] = m[0]; out[1] = m[1]; out[2] = m[2]; out[3] = one; break;
    default: out[0] = m[0]; out[1] = m[1]; out[2] = m[2]; out[3] = m[3]; break;
  }
}

// byte offset of column i inside a tiled row (see Image::tiled)
__device__ __forceinline__ uint64_t tiled_col(const Image& im, int i) {
  return ((uint64_t)((unsigned)i >> im.tshift) << 10) +
         (uint64_t)((unsigned)i & ((1u << im.tshift) - 1u)) * (unsigned)im.es;
}
// start of texel row j of a tiled image (its 128-byte row inside the band)
__device__ __forceinline__ const char* tiled_row(const Image& im, int j) {
  return im.ptr + (uint64_t)((unsigned)j >> 3) * im.rp + (uint64_t)((unsigned)j & 7u) * 128u;
}

// texel address (Fig. 6: ptr + k*slice_pitch + j*row_pitch + i*elem_size;
// tiled storage: the tile's address, see Image::tiled)
__device__ __forceinline__ const char* texel_ptr(const Image& im, int i, int j, int k) {
  if (im.tiled) return tiled_row(im, j) + tiled_col(im, i);
  return im.ptr + (uint64_t)(unsigned)k * im.sp + (uint64_t)(unsigned)j * im.rp +
         (uint64_t)(unsigned)i * (unsigned)im.es;
}

// ------------------------------------------------------------------------
// write conversion ([CL1.2 §8.3], readings A12, A13, A16)
// ------------------------------------------------------------------------
__device__ __forceinline__ uint32_t float_to_code(float f, int type) {
  switch (type) {
    case T_UNORM8: return (uint32_t)min(max(__float2int_rn(__fmul_rn(f, 255.0f)), 0), 255);
    case T_UNORM16: return (uint32_t)min(max(__float2int_rn(__fmul_rn(f, 65535.0f)), 0), 65535);
    case T_SNORM8: return (uint32_t)min(max(__float2int_rn(__fmul_rn(f, 127.0f)), -128), 127);
    case T_SNORM16: return (uint32_t)min(max(__float2int_rn(__fmul_rn(f, 32767.0f)), -32768), 32767);
    case T_HALF: return (uint32_t)__half_as_ushort(__float2half_rn(f));
    default: return __float_as_uint(f);
  }
}
__device__ __forceinline__ uint32_t int_to_code(uint32_t v, int type) {
  switch (type) {
    case T_SINT8: return (uint32_t)min(max((int)v, -128), 127);
    case T_SINT16: return (uint32_t)min(max((int)v, -32768), 32767);
    case T_UINT8: return min(v, 255u);
    case T_UINT16: return min(v, 65535u);
    default: return v;
  }
}

// (x,y,z,w) color -> packed word: convert_sat_rte(component * (2^bits - 1))
// (reading A12); the unused x bits are written 0 (reading A38)
__device__ __forceinline__ uint32_t pack_rgb(const uint32_t col[4], int type) {
  const float f[3] = {__uint_as_float(col[0]), __uint_as_float(col[1]), __uint_as_float(col[2])};
  auto q = [](float v, int hi) {
    return (uint32_t)min(max(__float2int_rn(__fmul_rn(v, (float)hi)), 0), hi);
  };
  if (type == T_U565) return (q(f[0], 31) << 11) | (q(f[1], 63) << 5) | q(f[2], 31);
  if (type == T_U555) return (q(f[0], 31) << 10) | (q(f[1], 31) << 5) | q(f[2], 31);
  return (q(f[0], 1023) << 20) | (q(f[1], 1023) << 10) | q(f[2], 1023);
}

// (x,y,z,w) color -> stored texel bytes in 4 words (little endian)
__device__ __forceinline__ Raw encode_texel(const uint32_t col[4], int type, int order) {
  if (is_packed(type)) {
    Raw r;
    r.w[0] = pack_rgb(col, type);
    r.w[1] = r.w[2] = r.w[3] = 0u;
    return r;
  }
  int slot[4] = {0, 1, 2, 3};
  if (order == O_A) slot[0] = 3;
  else if (order == O_RA) slot[1] = 3;
  else if (order == O_BGRA) { slot[0] = 2; slot[2] = 0; }
  else if (order == O_ARGB) { slot[0] = 3; slot[1] = 0; slot[2] = 1; slot[3] = 2; }
  const int nch = order_channels(order), tb = type_bytes(type);
  const int rc = ret_class(type);
  Raw r;
  r.w[0] = r.w[1] = r.w[2] = r.w[3] = 0u;
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    if (c < nch) {
      uint32_t v = col[slot[c]];
      uint32_t code = rc == R_F ? float_to_code(__uint_as_float(v), type) : int_to_code(v, type);
      if (tb == 4) r.w[c] = code;
      else if (tb == 2) r.w[c >> 1] |= (code & 0xffffu) << ((c & 1) * 16);
      else r.w[0] |= (code & 0xffu) << (c * 8);
    }
  }
  return r;
}

__device__ __forceinline__ void store_raw(char* p, int es, const Raw& r) {
  switch (es) {
    case 16: *reinterpret_cast<uint4*>(p) = make_uint4(r.w[0], r.w[1], r.w[2], r.w[3]); break;
    case 8: *reinterpret_cast<uint2*>(p) = make_uint2(r.w[0], r.w[1]); break;
    case 4: *reinterpret_cast<uint32_t*>(p) = r.w[0]; break;
    case 2: *reinterpret_cast<unsigned short*>(p) = (unsigned short)r.w[0]; break;
    default: *reinterpret_cast<unsigned char*>(p) = (unsigned char)r.w[0]; break;
  }
}

// separable LINEAR weight form: (1-a)*x0 + a*x1 as fma(a, x1, (1-a)*x0)
__device__ __forceinline__ float lerp1(float a, float oma, float x0, float x1) {
  return __fmaf_rn(a, x1, __fmul_rn(oma, x0));
}

}  // namespace dev
}  // namespace b2cl
