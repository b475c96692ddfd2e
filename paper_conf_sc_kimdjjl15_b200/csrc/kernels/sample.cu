// sample.cu -- read_imagef / read_imagei / read_imageui kernels (steps a3-a7).
//
// One thread evaluates one sample: coordinates (affine grid or list) ->
// per-axis addressing ([CL1.2 §8.2]) -> texel fetch through the CLImage
// pointer with 16-byte vector loads for RGBA32F -> conversion and
// channel map ([CL1.2 §8.3]) -> LINEAR blend in the separable FMA form.
// Every template argument may be `RT` (decided from the parameters at run
// time): the fully run-time instance covers every format x sampler; the
// compile-time instances are the hot configurations of BASELINE.json
// (bit-identical arithmetic, fewer instructions).
#include <atomic>

#include "../device/image.cuh"
#include "launch.h"

namespace b2cl {
using namespace dev;

template <int DIMS, int TYPE, int ORDER, int NORM, int ADDR, int FILT, int RC>
struct Cfg {
  static constexpr int dims = DIMS, type = TYPE, order = ORDER, norm = NORM, addr = ADDR,
                       filt = FILT, rc = RC;
  static constexpr int nch = ORDER == RT ? RT : order_channels(ORDER);
};

template <class C>
__device__ __forceinline__ int near_idx(const Sampler& s, float c, int n) {
  if constexpr (C::addr == RT) return axis_nearest_rt(s.addr, s.norm, c, n);
  else return axis_nearest<C::addr, C::norm>(c, n);
}
template <class C>
__device__ __forceinline__ void lin_idx(const Sampler& s, float c, int n, int& i0, int& i1,
                                        float& a) {
  if constexpr (C::addr == RT) axis_linear_rt(s.addr, s.norm, c, n, i0, i1, a);
  else axis_linear<C::addr, C::norm>(c, n, i0, i1, a);
}
template <class C>
__device__ __forceinline__ bool may_border(const Sampler& s) {
  if constexpr (C::addr == RT) return s.addr == A_NONE || s.addr == A_CLAMP;
  else return C::addr == A_NONE || C::addr == A_CLAMP;
}

// The built-in: c[0..DIMS-1] -> res (x,y,z,w) as 32-bit patterns.
template <class C>
__device__ __forceinline__ void read_image(const SampleParams& p, const float c[3],
                                           uint32_t res[4]) {
  const Image& im = p.im;
  const int rc = C::rc == RT ? p.rclass : C::rc;
  const int order = C::order == RT ? im.order : C::order;
  const int nch = C::nch == RT ? im.nch : C::nch;
  const int filt = C::filt == RT ? p.smp.filt : C::filt;
  const uint32_t one = rc == R_F ? 0x3f800000u : 1u;
  const bool bord = may_border<C>(p.smp);
  uint32_t m[4];
  if (filt == F_NEAREST) {
    int i = near_idx<C>(p.smp, c[0], im.w);
    int j = C::dims > 1 ? near_idx<C>(p.smp, c[1], im.h) : 0;
    int k = C::dims > 2 ? near_idx<C>(p.smp, c[2], im.d) : 0;
    bool ok = !bord || (in_range(i, im.w) && (C::dims < 2 || in_range(j, im.h)) &&
                        (C::dims < 3 || in_range(k, im.d)));
    fetch_mem<C::type, C::nch>(im, i, j, k, ok, rc, m);
  } else {
    int i0, i1, j0 = 0, j1 = 0, k0 = 0, k1 = 0;
    float a, b = 0.f, g = 0.f;
    lin_idx<C>(p.smp, c[0], im.w, i0, i1, a);
    if (C::dims > 1) lin_idx<C>(p.smp, c[1], im.h, j0, j1, b);
    if (C::dims > 2) lin_idx<C>(p.smp, c[2], im.d, k0, k1, g);
    const bool oi0 = !bord || in_range(i0, im.w), oi1 = !bord || in_range(i1, im.w);
    const bool oj0 = C::dims < 2 || !bord || in_range(j0, im.h);
    const bool oj1 = C::dims < 2 || !bord || in_range(j1, im.h);
    const bool ok0 = C::dims < 3 || !bord || in_range(k0, im.d);
    const bool ok1 = C::dims < 3 || !bord || in_range(k1, im.d);
    const float oma = __fsub_rn(1.0f, a), omb = __fsub_rn(1.0f, b), omg = __fsub_rn(1.0f, g);
    uint32_t t000[4], t100[4];
    fetch_mem<C::type, C::nch>(im, i0, j0, k0, oi0 && oj0 && ok0, R_F, t000);
    fetch_mem<C::type, C::nch>(im, i1, j0, k0, oi1 && oj0 && ok0, R_F, t100);
    if (C::dims == 1) {
#pragma unroll
      for (int ch = 0; ch < 4; ++ch)
        m[ch] = __float_as_uint(lerp1(a, oma, __uint_as_float(t000[ch]), __uint_as_float(t100[ch])));
    } else {
      uint32_t t010[4], t110[4];
      fetch_mem<C::type, C::nch>(im, i0, j1, k0, oi0 && oj1 && ok0, R_F, t010);
      fetch_mem<C::type, C::nch>(im, i1, j1, k0, oi1 && oj1 && ok0, R_F, t110);
      float s0[4];
#pragma unroll
      for (int ch = 0; ch < 4; ++ch) {
        float r0 = lerp1(a, oma, __uint_as_float(t000[ch]), __uint_as_float(t100[ch]));
        float r1 = lerp1(a, oma, __uint_as_float(t010[ch]), __uint_as_float(t110[ch]));
        s0[ch] = lerp1(b, omb, r0, r1);
      }
      if (C::dims == 2) {
#pragma unroll
        for (int ch = 0; ch < 4; ++ch) m[ch] = __float_as_uint(s0[ch]);
      } else {
        uint32_t t001[4], t101[4], t011[4], t111[4];
        fetch_mem<C::type, C::nch>(im, i0, j0, k1, oi0 && oj0 && ok1, R_F, t001);
        fetch_mem<C::type, C::nch>(im, i1, j0, k1, oi1 && oj0 && ok1, R_F, t101);
        fetch_mem<C::type, C::nch>(im, i0, j1, k1, oi0 && oj1 && ok1, R_F, t011);
        fetch_mem<C::type, C::nch>(im, i1, j1, k1, oi1 && oj1 && ok1, R_F, t111);
#pragma unroll
        for (int ch = 0; ch < 4; ++ch) {
          float r0 = lerp1(a, oma, __uint_as_float(t001[ch]), __uint_as_float(t101[ch]));
          float r1 = lerp1(a, oma, __uint_as_float(t011[ch]), __uint_as_float(t111[ch]));
          float s1 = lerp1(b, omb, r0, r1);
          m[ch] = __float_as_uint(lerp1(g, omg, s0[ch], s1));
        }
      }
    }
    // channels the format does not store stay exactly 0 / 1 after the map
#pragma unroll
    for (int ch = 0; ch < 4; ++ch)
      if (ch >= nch) m[ch] = 0u;
  }
  map_order(order, m, one, res);
}

// coordinate of output (x,y,z) under the affine map: ((A0*x + A1*y) + A2*z) + A3
__device__ __forceinline__ float affine_coord(const float* A, float x, float y, float z) {
  float v = __fmul_rn(A[0], x);
  v = __fadd_rn(v, __fmul_rn(A[1], y));
  v = __fadd_rn(v, __fmul_rn(A[2], z));
  return __fadd_rn(v, A[3]);
}

template <class C, int OUTC>
__global__ void __launch_bounds__(256) k_sample_grid(const SampleParams p) {
  const int x = blockIdx.x * blockDim.x + threadIdx.x;
  const int y = blockIdx.y * blockDim.y + threadIdx.y;
  const int z = blockIdx.z;
  if (x >= p.ow || y >= p.oh) return;
  const float xf = __int2float_rn(x), yf = __int2float_rn(y), zf = __int2float_rn(z);
  float c[3];
  c[0] = affine_coord(p.A, xf, yf, zf);
  c[1] = C::dims > 1 ? affine_coord(p.A + 4, xf, yf, zf) : 0.f;
  c[2] = C::dims > 2 ? affine_coord(p.A + 8, xf, yf, zf) : 0.f;
  uint32_t r[4];
  read_image<C>(p, c, r);
  const int outc = OUTC == RT ? p.outc : OUTC;
  const uint64_t idx = ((uint64_t)z * p.oh + y) * p.ow + x;
  if (outc == 4) {
    reinterpret_cast<uint4*>(p.out)[idx] = make_uint4(r[0], r[1], r[2], r[3]);
  } else if (outc == 1) {
    reinterpret_cast<uint32_t*>(p.out)[idx] = r[0];
  } else if (outc == 2) {
    reinterpret_cast<uint2*>(p.out)[idx] = make_uint2(r[0], r[1]);
  } else {
    uint32_t* o = reinterpret_cast<uint32_t*>(p.out) + idx * 3;
    o[0] = r[0]; o[1] = r[1]; o[2] = r[2];
  }
}

template <class C, bool INT_COORD>
__global__ void __launch_bounds__(256) k_sample_list(const SampleParams p) {
  const uint64_t s = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (s >= p.n) return;
  float c[3] = {0.f, 0.f, 0.f};
  constexpr int stride = C::dims == 1 ? 1 : (C::dims == 2 ? 2 : 4);
  if (INT_COORD) {
    const int32_t* q = reinterpret_cast<const int32_t*>(p.coords) + s * stride;
#pragma unroll
    for (int d = 0; d < C::dims; ++d) c[d] = __int2float_rn(q[d]);  // u = (float)i (A30)
  } else {
    const float* q = reinterpret_cast<const float*>(p.coords) + s * stride;
    if (stride == 4) {
      float4 v = *reinterpret_cast<const float4*>(q);
      c[0] = v.x; c[1] = v.y; c[2] = v.z;
    } else if (stride == 2) {
      float2 v = *reinterpret_cast<const float2*>(q);
      c[0] = v.x; c[1] = v.y;
    } else {
      c[0] = q[0];
    }
  }
  uint32_t r[4];
  read_image<C>(p, c, r);
  reinterpret_cast<uint4*>(p.out)[s] = make_uint4(r[0], r[1], r[2], r[3]);
}

// ---------------------------------------------------------------- dispatch
template <class C, int OUTC>
static cudaError_t go_grid(const SampleParams& p, cudaStream_t st) {
  dim3 blk(32, 8, 1);
  dim3 grd((p.ow + 31) / 32, (p.oh + 7) / 8, p.od);
  k_sample_grid<C, OUTC><<<grd, blk, 0, st>>>(p);
  count_launch();
  return cudaGetLastError();
}

template <class C>
static cudaError_t go_list(const SampleParams& p, bool int_coord, cudaStream_t st) {
  const uint64_t blocks = (p.n + 255) / 256;
  if (int_coord) k_sample_list<C, true><<<(unsigned)blocks, 256, 0, st>>>(p);
  else k_sample_list<C, false><<<(unsigned)blocks, 256, 0, st>>>(p);
  count_launch();
  return cudaGetLastError();
}

template <int DIMS>
using Generic = Cfg<DIMS, RT, RT, RT, RT, RT, RT>;

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

cudaError_t launch_sample(const SampleParams& p, int coord_mode, cudaStream_t st) {
  if (coord_mode == COORD_GRID) {
    if ((uint64_t)p.ow * p.oh * p.od == 0) return cudaSuccess;
    if (p.outc == 4 && matches<2>(p, T_FLOAT, O_RGBA, 1, A_REPEAT, F_LINEAR)) return go_grid<C2Repeat, 4>(p, st);
    if (p.outc == 4 && matches<2>(p, T_FLOAT, O_RGBA, 1, A_MIRROR, F_LINEAR)) return go_grid<C2Mirror, 4>(p, st);
    if (p.outc == 1 && matches<3>(p, T_FLOAT, O_R, 1, A_CTE, F_LINEAR)) return go_grid<C3Cte, 1>(p, st);
    if (p.outc == 4 && matches<2>(p, T_UNORM8, O_RGBA, 0, A_CLAMP, F_NEAREST)) return go_grid<C1Clamp, 4>(p, st);
    switch (p.dims) {
      case 1: return go_grid<Generic<1>, RT>(p, st);
      case 2: return go_grid<Generic<2>, RT>(p, st);
      default: return go_grid<Generic<3>, RT>(p, st);
    }
  }
  if (p.n == 0) return cudaSuccess;
  const bool ic = coord_mode == COORD_LIST_I;
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
void count_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }
uint64_t launch_count() { return g_launches.load(std::memory_order_relaxed); }

}  // namespace b2cl
