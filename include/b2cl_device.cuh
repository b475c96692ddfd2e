// b2cl_device.cuh -- OpenCL C built-ins for translated kernels (CUDA C, sm_100a).
//
// The paper translates an OpenCL kernel to CUDA C and implements the OpenCL
// built-ins it calls as CUDA device wrappers (read_imageX /
// write_imageX "handle the CLImage object to read or to write image data
// through pointer ptr"; §3.5 kernel launch; Fig. 5 dynamic __local carving).
// A kernel written against this header is compiled by nvcc to a cubin and
// run through clCreateProgramWithBinary / clBuildProgram / clCreateKernel /
// clSetKernelArg / clEnqueueNDRangeKernel of libb2cl.
//
// Argument conventions (what clSetKernelArg passes for each OpenCL argument):
//   __global / __constant buffer (cl_mem)  -> a device pointer
//   image1d_t / image2d_t / image3d_t /    -> the image descriptor by value
//   image1d_array_t / image2d_array_t /
//   image1d_buffer_t
//                                             (the paper's CLImage, Fig. 6;
//                                             reading A27)
//   sampler_t (cl_sampler)                 -> 32-bit CLK_* bits below
//   __local pointer (arg_value == NULL)    -> size_t size of that local
//                                             object; the kernel carves
//                                             __OC2CU_shared_mem by the
//                                             running sum of the sizes, in
//                                             argument order (Fig. 5(b))
//   anything else                          -> the bytes given
// The read / write built-ins are the library's own (csrc/device/read.cuh):
// same arithmetic, same readings as the enqueue extensions.
#pragma once
#include <stddef.h>

#include <type_traits>

#include "../paper_conf_sc_kimdjjl15_b200/csrc/device/read.cuh"

// ---- image and sampler types ----
struct image1d_t { b2cl::dev::Image im; };
struct image2d_t { b2cl::dev::Image im; };
struct image3d_t { b2cl::dev::Image im; };
// arrays: layers on the storage axis after the sampled ones (h of a 1D array,
// d of a 2D array); a 1D image buffer is a 1D image over a buffer's bytes
struct image1d_array_t { b2cl::dev::Image im; };
struct image2d_array_t { b2cl::dev::Image im; };
struct image1d_buffer_t { b2cl::dev::Image im; };
typedef unsigned int sampler_t;

// sampler bits (clang's CLK_* encoding)
#define CLK_NORMALIZED_COORDS_FALSE 0x0u
#define CLK_NORMALIZED_COORDS_TRUE 0x1u
#define CLK_ADDRESS_NONE 0x0u
#define CLK_ADDRESS_CLAMP_TO_EDGE 0x2u
#define CLK_ADDRESS_CLAMP 0x4u
#define CLK_ADDRESS_REPEAT 0x6u
#define CLK_ADDRESS_MIRRORED_REPEAT 0x8u
#define CLK_FILTER_NEAREST 0x10u
#define CLK_FILTER_LINEAR 0x20u

#define CLK_LOCAL_MEM_FENCE 0x1u
#define CLK_GLOBAL_MEM_FENCE 0x2u

// one dynamic shared array for every __local argument (Fig. 5(b))
extern __shared__ __align__(16) char __OC2CU_shared_mem[];

// global work offset of clEnqueueNDRangeKernel, written by the runtime before
// each launch when the module defines it (this header does)
__device__ size_t __b2cl_global_offset[3];

// Dynamic __constant arguments (Fig. 5(b) line 2): one constant
// array; each __constant argument becomes its size (size_t) and the kernel
// carves the array by the running sum, in argument order.  The buffer stays
// in global memory until the launch, which copies it here (the paper's
// deferred placement).  A kernel declares which arguments are
// __constant with B2CL_KERNEL_CONSTANT_ARGS(name, bitmask of argument indices).
#ifndef B2CL_MAX_CONST_SIZE
#define B2CL_MAX_CONST_SIZE 32768
#endif
__constant__ __align__(16) char __OC2CU_const_mem[B2CL_MAX_CONST_SIZE];
#define B2CL_KERNEL_CONSTANT_ARGS(kernel_name, mask) \
  extern "C" __device__ const unsigned int __b2cl_const_args_##kernel_name = (mask)

// ---- work-item functions ----
__device__ __forceinline__ size_t get_local_id(unsigned d) {
  return d == 0 ? threadIdx.x : (d == 1 ? threadIdx.y : (d == 2 ? threadIdx.z : 0));
}
__device__ __forceinline__ size_t get_local_size(unsigned d) {
  return d == 0 ? blockDim.x : (d == 1 ? blockDim.y : (d == 2 ? blockDim.z : 1));
}
__device__ __forceinline__ size_t get_group_id(unsigned d) {
  return d == 0 ? blockIdx.x : (d == 1 ? blockIdx.y : (d == 2 ? blockIdx.z : 0));
}
__device__ __forceinline__ size_t get_num_groups(unsigned d) {
  return d == 0 ? gridDim.x : (d == 1 ? gridDim.y : (d == 2 ? gridDim.z : 1));
}
__device__ __forceinline__ size_t get_global_offset(unsigned d) {
  return d < 3 ? __b2cl_global_offset[d] : 0;
}
__device__ __forceinline__ size_t get_global_id(unsigned d) {
  return get_group_id(d) * get_local_size(d) + get_local_id(d) + get_global_offset(d);
}
__device__ __forceinline__ size_t get_global_size(unsigned d) {
  return get_num_groups(d) * get_local_size(d);
}
__device__ __forceinline__ void barrier(unsigned) { __syncthreads(); }

// ---- read built-ins ([CL1.2 §6.12.14.2]) ----
namespace b2cl {
namespace cl_builtin {

struct ReadParams {  // the P of read.cuh
  dev::Image im;
  dev::Sampler smp;
  int rclass;
};

__device__ __forceinline__ dev::Sampler decode(sampler_t s) {
  dev::Sampler r;
  r.norm = (int)(s & 1u);
  r.addr = (int)((s & 0xEu) >> 1);  // NONE, CTE, CLAMP, REPEAT, MIRRORED -> 0..4
  r.filt = (s & CLK_FILTER_LINEAR) ? dev::F_LINEAR : dev::F_NEAREST;
  return r;
}

template <int DIMS>
__device__ __forceinline__ uint4 read(const dev::Image& im, sampler_t s, int rclass, float c0,
                                      float c1, float c2) {
  using C = WithShard<Cfg<DIMS, RT, RT, RT, RT, RT, RT>, true>;
  ReadParams p{im, decode(s), rclass};
  // LINEAR with read_imagei/ui is undefined; NEAREST is used (reading A6)
  if (rclass != dev::R_F) p.smp.filt = dev::F_NEAREST;
  const float c[3] = {c0, c1, c2};
  uint32_t r[4];
  read_image<C>(p, c, r, 4);
  return make_uint4(r[0], r[1], r[2], r[3]);
}

// image arrays ([CL1.2 §8.4]): coordinate DIMS is the layer, selected as
// clamp(rint(c), 0, layers - 1); arrays are never shards
template <int DIMS>
__device__ __forceinline__ uint4 read_array(const dev::Image& im, sampler_t s, int rclass, float c0,
                                            float c1, float c2) {
  using C = WithShard<Layered<Cfg<DIMS, RT, RT, RT, RT, RT, RT>>, false>;
  ReadParams p{im, decode(s), rclass};
  if (rclass != dev::R_F) p.smp.filt = dev::F_NEAREST;
  const float c[3] = {c0, c1, c2};
  uint32_t r[4];
  read_image<C>(p, c, r, 4);
  return make_uint4(r[0], r[1], r[2], r[3]);
}

// integer coordinates (reading A30): the coordinate is the texel index,
// exact at any width (a 1D image buffer reaches 2^31 - 1 texels)
template <int DIMS, bool ARR>
__device__ __forceinline__ uint4 read_int(const dev::Image& im, sampler_t s, int rclass, int c0,
                                          int c1, int c2) {
  using Base = Cfg<DIMS, RT, RT, RT, RT, RT, RT>;
  using C = std::conditional_t<ARR, WithShard<Layered<Base>, false>, WithShard<Base, true>>;
  ReadParams p{im, decode(s), rclass};
  const int ic[3] = {c0, c1, c2};
  uint32_t r[4];
  read_image_int<C>(p, ic, r);
  return make_uint4(r[0], r[1], r[2], r[3]);
}

__device__ __forceinline__ float4 as_f4(uint4 v) {
  return make_float4(__uint_as_float(v.x), __uint_as_float(v.y), __uint_as_float(v.z),
                     __uint_as_float(v.w));
}
__device__ __forceinline__ uint4 as_u4(uint4 v) { return v; }
__device__ __forceinline__ int4 as_i4(uint4 v) {
  return make_int4((int)v.x, (int)v.y, (int)v.z, (int)v.w);
}

// samplerless reads use NEAREST, unnormalized, CLK_ADDRESS_NONE (reading A31)
constexpr sampler_t kSamplerless = CLK_NORMALIZED_COORDS_FALSE | CLK_ADDRESS_NONE | CLK_FILTER_NEAREST;

template <int DIMS>
__device__ __forceinline__ void write(const dev::Image& im, int i, int j, int k, uint4 col) {
  if (!dev::in_range(i, im.w) || !dev::in_range(j, im.h) || !dev::in_range(k, im.d)) return;  // A15
  // global outer index -> stored row of a shard; rows the shard does not hold: no-op
  int& o = DIMS == 3 ? k : j;
  const int extent = DIMS == 3 ? im.d : im.h;
  if (DIMS > 1) {
    int l = o - im.ob;
    l += l < 0 ? extent : 0;
    l -= l >= extent ? extent : 0;
    if (l >= im.os) return;
    o = l;
  }
  const uint32_t cc[4] = {col.x, col.y, col.z, col.w};
  dev::Raw t = dev::encode_texel(cc, im.type, im.order);
  dev::store_raw(const_cast<char*>(dev::texel_ptr(im, i, j, k)), im.es, t);
}

}  // namespace cl_builtin
}  // namespace b2cl

#define B2CL_READ_OVERLOADS(RET, NAME, RC, CONV)                                                 \
  __device__ __forceinline__ RET NAME(image1d_t im, sampler_t s, float c) {                      \
    return CONV(b2cl::cl_builtin::read<1>(im.im, s, RC, c, 0.f, 0.f));                           \
  }                                                                                              \
  __device__ __forceinline__ RET NAME(image1d_t im, sampler_t s, int c) {                        \
    return CONV(b2cl::cl_builtin::read_int<1, false>(im.im, s, RC, c, 0, 0));           \
  }                                                                                              \
  __device__ __forceinline__ RET NAME(image2d_t im, sampler_t s, float2 c) {                     \
    return CONV(b2cl::cl_builtin::read<2>(im.im, s, RC, c.x, c.y, 0.f));                         \
  }                                                                                              \
  __device__ __forceinline__ RET NAME(image2d_t im, sampler_t s, int2 c) {                       \
    return CONV(b2cl::cl_builtin::read_int<2, false>(im.im, s, RC, c.x, c.y, 0));                                                 \
  }                                                                                              \
  __device__ __forceinline__ RET NAME(image3d_t im, sampler_t s, float4 c) {                     \
    return CONV(b2cl::cl_builtin::read<3>(im.im, s, RC, c.x, c.y, c.z));                         \
  }                                                                                              \
  __device__ __forceinline__ RET NAME(image3d_t im, sampler_t s, int4 c) {                       \
    return CONV(b2cl::cl_builtin::read_int<3, false>(im.im, s, RC, c.x, c.y, c.z));                                 \
  }                                                                                              \
  __device__ __forceinline__ RET NAME(image2d_t im, int2 c) {                                    \
    return NAME(im, b2cl::cl_builtin::kSamplerless, c);                                          \
  }                                                                                              \
  __device__ __forceinline__ RET NAME(image3d_t im, int4 c) {                                    \
    return NAME(im, b2cl::cl_builtin::kSamplerless, c);                                          \
  }                                                                                              \
  __device__ __forceinline__ RET NAME(image1d_t im, int c) {                                     \
    return NAME(im, b2cl::cl_builtin::kSamplerless, c);                                          \
  }                                                                                              \
  __device__ __forceinline__ RET NAME(image1d_array_t im, sampler_t s, float2 c) {               \
    return CONV(b2cl::cl_builtin::read_array<1>(im.im, s, RC, c.x, c.y, 0.f));                   \
  }                                                                                              \
  __device__ __forceinline__ RET NAME(image1d_array_t im, sampler_t s, int2 c) {                 \
    return CONV(b2cl::cl_builtin::read_int<1, true>(im.im, s, RC, c.x, c.y, 0));                      \
  }                                                                                              \
  __device__ __forceinline__ RET NAME(image2d_array_t im, sampler_t s, float4 c) {               \
    return CONV(b2cl::cl_builtin::read_array<2>(im.im, s, RC, c.x, c.y, c.z));                   \
  }                                                                                              \
  __device__ __forceinline__ RET NAME(image2d_array_t im, sampler_t s, int4 c) {                 \
    return CONV(b2cl::cl_builtin::read_int<2, true>(im.im, s, RC, c.x, c.y, c.z));      \
  }                                                                                              \
  __device__ __forceinline__ RET NAME(image1d_array_t im, int2 c) {                              \
    return NAME(im, b2cl::cl_builtin::kSamplerless, c);                                          \
  }                                                                                              \
  __device__ __forceinline__ RET NAME(image2d_array_t im, int4 c) {                              \
    return NAME(im, b2cl::cl_builtin::kSamplerless, c);                                          \
  }                                                                                              \
  /* image1d_buffer_t: samplerless reads only ([CL1.2 §6.12.14.2]) */                            \
  __device__ __forceinline__ RET NAME(image1d_buffer_t im, int c) {                              \
    return CONV(b2cl::cl_builtin::read_int<1, false>(im.im, b2cl::cl_builtin::kSamplerless, RC, c, 0, 0));                         \
  }

B2CL_READ_OVERLOADS(float4, read_imagef, b2cl::dev::R_F, b2cl::cl_builtin::as_f4)
B2CL_READ_OVERLOADS(int4, read_imagei, b2cl::dev::R_I, b2cl::cl_builtin::as_i4)
B2CL_READ_OVERLOADS(uint4, read_imageui, b2cl::dev::R_UI, b2cl::cl_builtin::as_u4)

// ---- write built-ins ([CL1.2 §6.12.14.4]); 3D writes as cl_khr_3d_image_writes ----
// Arrays write as the storage image they are (layer = the last coordinate,
// out of range -> no-op like every other out-of-range write, reading A15).
namespace b2cl {
namespace cl_builtin {
__device__ __forceinline__ uint4 bits(float4 v) {
  return make_uint4(__float_as_uint(v.x), __float_as_uint(v.y), __float_as_uint(v.z),
                    __float_as_uint(v.w));
}
__device__ __forceinline__ uint4 bits(int4 v) { return make_uint4(v.x, v.y, v.z, v.w); }
__device__ __forceinline__ uint4 bits(uint4 v) { return v; }
}  // namespace cl_builtin
}  // namespace b2cl

#define B2CL_WRITE_OVERLOADS(NAME, VT)                                                           \
  __device__ __forceinline__ void NAME(image1d_t im, int c, VT v) {                              \
    b2cl::cl_builtin::write<1>(im.im, c, 0, 0, b2cl::cl_builtin::bits(v));                       \
  }                                                                                              \
  __device__ __forceinline__ void NAME(image1d_buffer_t im, int c, VT v) {                       \
    b2cl::cl_builtin::write<1>(im.im, c, 0, 0, b2cl::cl_builtin::bits(v));                       \
  }                                                                                              \
  __device__ __forceinline__ void NAME(image2d_t im, int2 c, VT v) {                             \
    b2cl::cl_builtin::write<2>(im.im, c.x, c.y, 0, b2cl::cl_builtin::bits(v));                   \
  }                                                                                              \
  __device__ __forceinline__ void NAME(image1d_array_t im, int2 c, VT v) {                       \
    b2cl::cl_builtin::write<2>(im.im, c.x, c.y, 0, b2cl::cl_builtin::bits(v));                   \
  }                                                                                              \
  __device__ __forceinline__ void NAME(image3d_t im, int4 c, VT v) {                             \
    b2cl::cl_builtin::write<3>(im.im, c.x, c.y, c.z, b2cl::cl_builtin::bits(v));                 \
  }                                                                                              \
  __device__ __forceinline__ void NAME(image2d_array_t im, int4 c, VT v) {                       \
    b2cl::cl_builtin::write<3>(im.im, c.x, c.y, c.z, b2cl::cl_builtin::bits(v));                 \
  }
B2CL_WRITE_OVERLOADS(write_imagef, float4)
B2CL_WRITE_OVERLOADS(write_imagei, int4)
B2CL_WRITE_OVERLOADS(write_imageui, uint4)

// ---- image queries ([CL1.2 §6.12.14.5]) ----
__device__ __forceinline__ int get_image_width(image1d_t im) { return im.im.w; }
__device__ __forceinline__ int get_image_width(image2d_t im) { return im.im.w; }
__device__ __forceinline__ int get_image_width(image3d_t im) { return im.im.w; }
__device__ __forceinline__ int get_image_height(image2d_t im) { return im.im.h; }
__device__ __forceinline__ int get_image_height(image3d_t im) { return im.im.h; }
__device__ __forceinline__ int get_image_depth(image3d_t im) { return im.im.d; }
__device__ __forceinline__ int get_image_width(image1d_buffer_t im) { return im.im.w; }
__device__ __forceinline__ int get_image_width(image1d_array_t im) { return im.im.w; }
__device__ __forceinline__ int get_image_width(image2d_array_t im) { return im.im.w; }
__device__ __forceinline__ int get_image_height(image2d_array_t im) { return im.im.h; }
__device__ __forceinline__ size_t get_image_array_size(image1d_array_t im) { return im.im.h; }
__device__ __forceinline__ size_t get_image_array_size(image2d_array_t im) { return im.im.d; }

// ---- CUDA texture fetches, as the paper translates them ----
// A CUDA texture reference becomes an image argument plus a sampler
// argument (b2clCreateTextureObject makes both from a CUDA-style texture
// description), and tex1Dfetch / tex1D / tex2D / tex3D become read_imageX;
// the return type T picks X (f for float T, i for signed, ui for unsigned)
// and keeps T's components, converted as CUDA returns them (8/16-bit element
// types narrowed from the int4 / uint4 read).  The fetch is read_imageX
// exactly: the OpenCL sampler arithmetic of [CL1.2 §8.2] (readings A40, A41
// and A43 of DESIGN.md record where that differs from a CUDA texture unit).
namespace b2cl {
namespace tex {
template <class T> struct Ret;  // return class and components of T
#define B2CL_TEX_RET(T, RC, N)                              \
  template <> struct Ret<T> {                               \
    static constexpr int rc = RC, n = N;                    \
  };
B2CL_TEX_RET(float, dev::R_F, 1) B2CL_TEX_RET(float1, dev::R_F, 1) B2CL_TEX_RET(float2, dev::R_F, 2)
B2CL_TEX_RET(float4, dev::R_F, 4)
B2CL_TEX_RET(int, dev::R_I, 1) B2CL_TEX_RET(int1, dev::R_I, 1) B2CL_TEX_RET(int2, dev::R_I, 2)
B2CL_TEX_RET(int4, dev::R_I, 4)
B2CL_TEX_RET(unsigned int, dev::R_UI, 1) B2CL_TEX_RET(uint1, dev::R_UI, 1)
B2CL_TEX_RET(uint2, dev::R_UI, 2) B2CL_TEX_RET(uint4, dev::R_UI, 4)
B2CL_TEX_RET(signed char, dev::R_I, 1) B2CL_TEX_RET(char1, dev::R_I, 1) B2CL_TEX_RET(char2, dev::R_I, 2)
B2CL_TEX_RET(char4, dev::R_I, 4)
B2CL_TEX_RET(unsigned char, dev::R_UI, 1) B2CL_TEX_RET(uchar1, dev::R_UI, 1)
B2CL_TEX_RET(uchar2, dev::R_UI, 2) B2CL_TEX_RET(uchar4, dev::R_UI, 4)
B2CL_TEX_RET(short, dev::R_I, 1) B2CL_TEX_RET(short1, dev::R_I, 1) B2CL_TEX_RET(short2, dev::R_I, 2)
B2CL_TEX_RET(short4, dev::R_I, 4)
B2CL_TEX_RET(unsigned short, dev::R_UI, 1) B2CL_TEX_RET(ushort1, dev::R_UI, 1)
B2CL_TEX_RET(ushort2, dev::R_UI, 2) B2CL_TEX_RET(ushort4, dev::R_UI, 4)
#undef B2CL_TEX_RET

// the first components of the read's 32-bit result v, as T
template <class T>
__device__ __forceinline__ T take(uint4 v) {
  T r;
  if constexpr (std::is_arithmetic_v<T>) {
    if constexpr (std::is_same_v<T, float>) r = __uint_as_float(v.x);
    else r = (T)v.x;
  } else {
    using C = decltype(r.x);
    auto conv = [](uint32_t u) -> C {
      if constexpr (std::is_same_v<C, float>) return __uint_as_float(u);
      else return (C)u;
    };
    r.x = conv(v.x);
    if constexpr (Ret<T>::n > 1) r.y = conv(v.y);
    if constexpr (Ret<T>::n > 2) {
      r.z = conv(v.z);
      r.w = conv(v.w);
    }
  }
  return r;
}
}  // namespace tex
}  // namespace b2cl

template <class T>
__device__ __forceinline__ T tex1Dfetch(image1d_buffer_t im, int x) {
  return b2cl::tex::take<T>(b2cl::cl_builtin::read_int<1, false>(
      im.im, b2cl::cl_builtin::kSamplerless, b2cl::tex::Ret<T>::rc, x, 0, 0));
}
template <class T>
__device__ __forceinline__ T tex1D(image1d_t im, sampler_t s, float x) {
  return b2cl::tex::take<T>(b2cl::cl_builtin::read<1>(im.im, s, b2cl::tex::Ret<T>::rc, x, 0.f, 0.f));
}
template <class T>
__device__ __forceinline__ T tex2D(image2d_t im, sampler_t s, float x, float y) {
  return b2cl::tex::take<T>(b2cl::cl_builtin::read<2>(im.im, s, b2cl::tex::Ret<T>::rc, x, y, 0.f));
}
template <class T>
__device__ __forceinline__ T tex3D(image3d_t im, sampler_t s, float x, float y, float z) {
  return b2cl::tex::take<T>(b2cl::cl_builtin::read<3>(im.im, s, b2cl::tex::Ret<T>::rc, x, y, z));
}
// layered: the integer layer is the array coordinate (exact as a float below 2^24)
template <class T>
__device__ __forceinline__ T tex1DLayered(image1d_array_t im, sampler_t s, float x, int layer) {
  return b2cl::tex::take<T>(
      b2cl::cl_builtin::read_array<1>(im.im, s, b2cl::tex::Ret<T>::rc, x, (float)layer, 0.f));
}
template <class T>
__device__ __forceinline__ T tex2DLayered(image2d_array_t im, sampler_t s, float x, float y, int layer) {
  return b2cl::tex::take<T>(
      b2cl::cl_builtin::read_array<2>(im.im, s, b2cl::tex::Ret<T>::rc, x, y, (float)layer));
}
