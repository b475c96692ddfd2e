// rect.cu -- pitched 3D byte-box copy and fill (steps a9, a11-a14, a16).
//
// One kernel serves CopyBuffer / CopyBufferRect / CopyImage /
// CopyImageToBuffer / CopyBufferToImage / peer migration (RECT_COPY),
// FillBuffer (RECT_FILL) and FillImage (RECT_FILL_IMAGE).  The box is
// region[0] bytes x region[1] rows x region[2] slices ([CL1.2 §5.2.2]).
//
// Layout of the work: a block is TX x TY threads (TX*TY = 256); TY rows per
// block, TX threads across a row, each thread owns U 16-byte destination
// vectors spaced TX apart (coalesced).  Destination stores are always
// 16-byte aligned vectors; the ragged head/tail of a row is stored byte by
// byte.  A source that is misaligned relative to the destination (odd
// origins or pitches) is read as aligned 16-byte words -- one load per lane,
// the next word by warp shuffle -- and funnel-shifted (the shift is constant
// along a row and a warp covers one row, so the branch is warp-uniform).
// Misaligned copies of rows of 2 KiB or more take k_rect_staged instead
// (bulk-async staging through shared memory, below).  Sources are always
// local to the launching device except for migration, whose source and
// destination offsets are both 0 (the aligned instance).
#include <algorithm>
#include <atomic>

#include "../device/image.cuh"
#include "launch.h"

namespace b2cl {
using namespace dev;

__device__ __forceinline__ uint4 ld16(const char* p) {
  return __ldg(reinterpret_cast<const uint4*>(p));
}

// The 16 bytes starting sh bytes into the 32-byte pair (a, b) of consecutive
// aligned source words (0 < sh < 16).
__device__ __forceinline__ uint4 funnel16(const uint4& a, const uint4& b, int sh) {
  uint32_t w[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
  const int r = (sh & 3) * 8;
  uint4 o;
  switch (sh >> 2) {
    case 0:
      o.x = __funnelshift_r(w[0], w[1], r); o.y = __funnelshift_r(w[1], w[2], r);
      o.z = __funnelshift_r(w[2], w[3], r); o.w = __funnelshift_r(w[3], w[4], r); break;
    case 1:
      o.x = __funnelshift_r(w[1], w[2], r); o.y = __funnelshift_r(w[2], w[3], r);
      o.z = __funnelshift_r(w[3], w[4], r); o.w = __funnelshift_r(w[4], w[5], r); break;
    case 2:
      o.x = __funnelshift_r(w[2], w[3], r); o.y = __funnelshift_r(w[3], w[4], r);
      o.z = __funnelshift_r(w[4], w[5], r); o.w = __funnelshift_r(w[5], w[6], r); break;
    default:
      o.x = __funnelshift_r(w[3], w[4], r); o.y = __funnelshift_r(w[4], w[5], r);
      o.z = __funnelshift_r(w[5], w[6], r); o.w = __funnelshift_r(w[6], w[7], r); break;
  }
  return o;
}

template <int MODE, int U>
__global__ void __launch_bounds__(256) k_rect(const RectParams p) {
  __shared__ uint4 tile[8];  // FILL modes: 128-byte pattern tile
  constexpr bool COPY = MODE == RECT_COPY || MODE == RECT_COPY_ALIGNED;
  if (!COPY) {
    if (MODE == RECT_FILL_IMAGE) {
      if (threadIdx.x == 0 && threadIdx.y == 0) {
        // convert the fill colour once with the write_image rules (A23) ...
        Raw t = encode_texel(p.color, p.type, p.order);
        // ... and replicate the texel over 128 bytes (elem_size divides 16)
        uint32_t* tw = reinterpret_cast<uint32_t*>(tile);
        const unsigned char* tb = reinterpret_cast<const unsigned char*>(t.w);
        for (int b = 0; b < 128; b += 4) {
          uint32_t v = 0;
          for (int q = 0; q < 4; ++q) v |= (uint32_t)tb[(b + q) % p.es] << (8 * q);
          tw[b / 4] = v;
        }
      }
    } else {
      const int t = threadIdx.y * blockDim.x + threadIdx.x;
      if (t < 8)
        tile[t] = make_uint4(p.ptile[4 * t], p.ptile[4 * t + 1], p.ptile[4 * t + 2], p.ptile[4 * t + 3]);
    }
    __syncthreads();
  }
  // Grid: x = chunk of a row (TX*U vectors), y = group of TY rows; when there
  // are more groups than the grid allows, a thread walks rows with stride
  // gridDim.y*TY, stepping its (z, y) coordinates without divisions.
  const uint64_t v0 = (uint64_t)blockIdx.x * blockDim.x * U + threadIdx.x;
  uint64_t row = (uint64_t)blockIdx.y * blockDim.y + threadIdx.y;
  if (row >= p.rows) return;
  uint32_t z = (uint32_t)(row / p.R1), y = (uint32_t)(row - (uint64_t)z * p.R1);
  for (; row < p.rows; row += p.row_step) {
    char* drow = p.dst + z * p.dsp + y * p.drp;
    const char* srow = COPY ? p.src + z * p.ssp + y * p.srp : nullptr;
    const uintptr_t dlo = reinterpret_cast<uintptr_t>(drow), dhi = dlo + p.R0;
    const uintptr_t abase = dlo & ~uintptr_t(15);
    const uint64_t nvec = ((dhi + 15) >> 4) - (abase >> 4);
    // full 16-byte destination vectors are v in [vf0, vf1)
    const uint64_t vf0 = (dlo & 15) ? 1 : 0;
    const uint64_t vf1 = (dhi >> 4) - (abase >> 4);
    const int sh = MODE == RECT_COPY ? (int)((reinterpret_cast<uintptr_t>(srow) - dlo) & 15) : 0;
    uint4 val[U];
    if (MODE != RECT_COPY || sh == 0) {  // fills, aligned copies
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const uint64_t v = v0 + (uint64_t)u * blockDim.x;
        if (v >= vf0 && v < vf1) {
          const uintptr_t D = abase + 16 * v;
          if (COPY) val[u] = ld16(srow + (D - dlo));
          else val[u] = tile[(D >> 4) & 7];
        }
      }
    } else if (MODE == RECT_COPY) {
      // Misaligned source (warp-uniform: a warp covers one row): every lane
      // loads the aligned source word under its own vector once; the word
      // above comes from lane+1 by shuffle (lane 31, or a lane whose
      // neighbour has no vector, loads it itself).  The head vector's word
      // may lie before the row, so it is never loaded; every other word
      // contains a byte of the row.
      const unsigned lane = threadIdx.x & 31u;
      uint4 w0[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const uint64_t v = v0 + (uint64_t)u * blockDim.x;
        if (v >= vf0 && v < nvec) w0[u] = ld16(srow + (abase + 16 * v - dlo) - sh);
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const uint64_t v = v0 + (uint64_t)u * blockDim.x;
        uint4 w1;
        w1.x = __shfl_down_sync(0xffffffffu, w0[u].x, 1);
        w1.y = __shfl_down_sync(0xffffffffu, w0[u].y, 1);
        w1.z = __shfl_down_sync(0xffffffffu, w0[u].z, 1);
        w1.w = __shfl_down_sync(0xffffffffu, w0[u].w, 1);
        if (v >= vf0 && v < vf1) {
          if (lane == 31u || v + 1 >= nvec) w1 = ld16(srow + (abase + 16 * v - dlo) - sh + 16);
          val[u] = funnel16(w0[u], w1, sh);
        }
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t v = v0 + (uint64_t)u * blockDim.x;
      const uintptr_t D = abase + 16 * v;
      if (v >= vf0 && v < vf1) {
        *reinterpret_cast<uint4*>(D) = val[u];
      } else if (v < nvec) {  // ragged head / tail of the row
        const uintptr_t lo = D > dlo ? D : dlo, hi = D + 16 < dhi ? D + 16 : dhi;
        for (uintptr_t X = lo; X < hi; ++X) {
          unsigned char b;
          if (COPY) b = static_cast<unsigned char>(srow[X - dlo]);
          else b = reinterpret_cast<const unsigned char*>(tile)[X & 127];
          *reinterpret_cast<unsigned char*>(X) = b;
        }
      }
    }
    y += p.step_dy;
    z += p.step_dz;
    if (y >= p.R1) {
      y -= p.R1;
      ++z;
    }
  }
}

// ------------------------------------------------- staged misaligned copy
// A copy whose source is misaligned against its destination, with rows long
// enough to amortize a stage: each unit (up to ST_CH destination bytes of one
// row) has the 16-byte-aligned cover of its source bytes brought into shared
// memory by one bulk async copy (cp.async.bulk, the TMA engine) completing on
// an mbarrier; with ST_NS stages a block keeps ST_NS-1 units in flight while
// its threads funnel-shift the current one out of shared memory into aligned
// 16-byte global stores (at ST_NS = 1 the overlap comes from the other blocks
// of the SM).  The loads need no registers and no shuffles, so the bytes in
// flight do not depend on occupancy.  A persistent grid of ST_BPS blocks per
// SM strides over the units.
#ifndef B2CL_ST_CH
#define B2CL_ST_CH 16384
#endif
// (one stage per block measured best on B200: 0.94 of HBM on both misaligned
// configurations at 6 blocks per SM, against 0.90 / 0.87 for 3 stages x 3
// blocks -- fewer bulk copies in flight per block, more blocks to overlap;
// 12 blocks per SM with streaming stores 0.955 / 0.956, 8 / 10 blocks and
// 8 or 32 KiB units uneven across the two configurations)
#ifndef B2CL_ST_NS
#define B2CL_ST_NS 1
#endif
#ifndef B2CL_ST_BPS
#define B2CL_ST_BPS 12
#endif
constexpr int ST_CH = B2CL_ST_CH;   // destination bytes per unit (chunk 0: up to 15 more)
constexpr int ST_BUF = ST_CH + 48;  // aligned cover of its source bytes
constexpr int ST_NS = B2CL_ST_NS;   // stages per block
constexpr int ST_BPS = B2CL_ST_BPS; // blocks per SM
#ifndef B2CL_ST_CS
#define B2CL_ST_CS 1  // 1: streaming (evict-first) stores (0.940 -> 0.950 at 6 blocks per SM)
#endif
#ifndef B2CL_ST_THREADS
#define B2CL_ST_THREADS 256
#endif
constexpr int ST_THREADS = B2CL_ST_THREADS;
constexpr uint64_t ST_MIN_ROW = 2048;  // shorter rows: the register/shuffle kernel

__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

struct StUnit {
  const char* srow;
  uintptr_t dlo, dhi, abase;
  uintptr_t u0, u1;  // destination bytes of the unit: [u0, u1)
  const char* sa;    // aligned source cover: [sa, sa + bytes)
  uint32_t bytes;
};

__device__ __forceinline__ StUnit st_unit(const RectParams& p, uint64_t u, uint64_t cpr) {
  StUnit w;
  const uint64_t row = u / cpr, c = u - row * cpr;
  const uint64_t z = row / p.R1, y = row - z * p.R1;
  w.srow = p.src + z * p.ssp + y * p.srp;
  w.dlo = reinterpret_cast<uintptr_t>(p.dst + z * p.dsp + y * p.drp);
  w.dhi = w.dlo + p.R0;
  w.abase = w.dlo & ~uintptr_t(15);
  // chunk boundaries at h + c*ST_CH, h = the first 16-byte boundary at or
  // after the row start; chunk 0 also takes the partial head vector
  const uintptr_t h = (w.dlo + 15) & ~uintptr_t(15);
  const uintptr_t c1 = h + (c + 1) * ST_CH;
  w.u0 = c == 0 ? w.dlo : h + c * ST_CH;
  w.u1 = c1 < w.dhi ? c1 : w.dhi;
  if (w.u1 <= w.u0) {  // a row with fewer chunks than the grid's maximum
    w.u1 = w.u0;
    w.sa = w.srow;
    w.bytes = 0;
    return w;
  }
  const uintptr_t s0 = reinterpret_cast<uintptr_t>(w.srow) + (w.u0 - w.dlo);
  const uintptr_t s1 = reinterpret_cast<uintptr_t>(w.srow) + (w.u1 - w.dlo);
  const uintptr_t a0 = s0 & ~uintptr_t(15), a1 = (s1 + 15) & ~uintptr_t(15);
  w.sa = reinterpret_cast<const char*>(a0);
  w.bytes = static_cast<uint32_t>(a1 - a0);
  return w;
}

__device__ __forceinline__ void st_issue(const StUnit& w, char* buf, uint64_t* bar) {
  const uint32_t b = smem_addr(bar);
  // (an empty unit arrives with no transaction bytes: the phase completes at once)
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(w.bytes)
               : "memory");
  if (w.bytes == 0) return;
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_addr(buf)),
      "l"(w.sa), "r"(w.bytes), "r"(b)
      : "memory");
}

__device__ __forceinline__ void st_wait(uint64_t* bar, uint32_t parity) {
  const uint32_t b = smem_addr(bar);
  uint32_t done;
  do {
    asm volatile(
        "{ .reg .pred P; mbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2; selp.u32 %0, 1, 0, P; }"
        : "=r"(done)
        : "r"(b), "r"(parity)
        : "memory");
  } while (!done);
}

__global__ void __launch_bounds__(ST_THREADS, ST_BPS)
    k_rect_staged(const RectParams p, const uint64_t cpr, const uint64_t units) {
  extern __shared__ __align__(128) char sbuf[];
  __shared__ uint64_t full[ST_NS];
  if (threadIdx.x == 0) {
    for (int s = 0; s < ST_NS; ++s)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_addr(&full[s])) : "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  __syncthreads();
  const uint64_t u_first = blockIdx.x, u_step = gridDim.x;
  if (threadIdx.x == 0)
    for (int s = 0; s < ST_NS; ++s) {
      const uint64_t u = u_first + s * u_step;
      if (u < units) st_issue(st_unit(p, u, cpr), sbuf + s * ST_BUF, &full[s]);
    }
  uint64_t i = 0;
  for (uint64_t u = u_first; u < units; u += u_step, ++i) {
    const int s = (int)(i % ST_NS);
    const char* buf = sbuf + s * ST_BUF;
    const StUnit w = st_unit(p, u, cpr);
    st_wait(&full[s], (uint32_t)((i / ST_NS) & 1));
    // destination vectors of the unit, 16-byte aligned: [v0, v1) counted from abase
    const uint64_t va = (w.u0 - w.abase) >> 4, vb = (w.u1 - w.abase + 15) >> 4;
    const uintptr_t sbase = reinterpret_cast<uintptr_t>(w.sa);
    for (uint64_t v = va + threadIdx.x; v < vb; v += ST_THREADS) {
      const uintptr_t D = w.abase + 16 * v;
      // source byte of D, as an offset into the staged cover
      const uint32_t o = (uint32_t)(reinterpret_cast<uintptr_t>(w.srow) + (D - w.dlo) - sbase);
      if (D >= w.dlo && D + 16 <= w.dhi) {
        const uint4* q = reinterpret_cast<const uint4*>(buf + (o & ~15u));
        const int sh = (int)(o & 15u);
        const uint4 val = sh ? funnel16(q[0], q[1], sh) : q[0];
        if (B2CL_ST_CS) __stcs(reinterpret_cast<uint4*>(D), val);  // (evict-first: never re-read)
        else *reinterpret_cast<uint4*>(D) = val;
      } else {  // ragged head / tail of the row
        const uintptr_t lo = D > w.dlo ? D : w.dlo, hi = D + 16 < w.dhi ? D + 16 : w.dhi;
        for (uintptr_t X = lo; X < hi; ++X)
          *reinterpret_cast<char*>(X) = buf[o + (uint32_t)(X - D)];
      }
    }
    __syncthreads();  // every thread is done with stage s
    if (threadIdx.x == 0) {
      const uint64_t un = u + ST_NS * u_step;
      if (un < units) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        st_issue(st_unit(p, un, cpr), sbuf + s * ST_BUF, &full[s]);
      }
    }
  }
}

static cudaError_t launch_rect_staged(const RectParams& p, cudaStream_t st) {
  int dev = 0, sms = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (e != cudaSuccess) return e;
  const int smem = ST_NS * ST_BUF;
  static std::atomic<uint64_t> attr_set{0};  // per-device bit: opt-in to > 48 KiB
  if (!((attr_set.load() >> (dev & 63)) & 1)) {
    e = cudaFuncSetAttribute(k_rect_staged, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    attr_set.fetch_or(1ull << (dev & 63));
  }
  // chunks per row (a row's bytes past its first 16-byte boundary number at most R0)
  const uint64_t cpr = (p.R0 + ST_CH - 1) / ST_CH;
  const uint64_t units = cpr * p.R1 * p.R2;
  const uint64_t blocks = units < (uint64_t)sms * ST_BPS ? units : (uint64_t)sms * ST_BPS;
  k_rect_staged<<<(unsigned)blocks, ST_THREADS, smem, st>>>(p, cpr, units);
  count_launch("k_rect_staged");
  return cudaGetLastError();
}

cudaError_t launch_rect(RectParams& p, int mode, cudaStream_t st) {
  const uint64_t rows = (uint64_t)p.R1 * p.R2;
  if (p.R0 == 0 || rows == 0) return cudaSuccess;
  constexpr int U = 4;
  const uint64_t nvec_max = (p.R0 + 15) / 16 + 1;
  unsigned tx = 32;
  while (tx < 256 && (uint64_t)tx * U < nvec_max) tx *= 2;
  const unsigned ty = 256 / tx;
  const uint64_t cpr = (nvec_max + (uint64_t)tx * U - 1) / ((uint64_t)tx * U);
  const uint64_t groups = (rows + ty - 1) / ty;
  // one block per (row group, chunk) up to the grid limit; beyond it rows are
  // walked in-kernel (measured: short-lived blocks keep HBM busier than a
  // persistent grid for plain copies)
  const uint64_t gy = groups < 65535 ? groups : 65535;
  if (cpr > 0x7fffffffull) return cudaErrorInvalidValue;
  p.rows = rows;
  p.row_step = gy * ty;
  p.step_dz = (uint32_t)(p.row_step / p.R1);
  p.step_dy = (uint32_t)(p.row_step % p.R1);
  dim3 blk(tx, ty, 1), grd((unsigned)cpr, (unsigned)gy, 1);
  // a copy whose source/destination misalignment is the same on every row
  // and zero takes the shuffle-free instance
  const bool aligned = mode == RECT_COPY && ((uintptr_t)p.src - (uintptr_t)p.dst) % 16 == 0 &&
                       (p.srp - p.drp) % 16 == 0 && (p.ssp - p.dsp) % 16 == 0;
  if (aligned) mode = RECT_COPY_ALIGNED;
  // misaligned copies of rows long enough to fill a stage: bulk-async staged
  if (mode == RECT_COPY && p.R0 >= ST_MIN_ROW) return launch_rect_staged(p, st);
  switch (mode) {
    case RECT_COPY_ALIGNED: k_rect<RECT_COPY_ALIGNED, U><<<grd, blk, 0, st>>>(p); break;
    case RECT_COPY: k_rect<RECT_COPY, U><<<grd, blk, 0, st>>>(p); break;
    case RECT_FILL: k_rect<RECT_FILL, U><<<grd, blk, 0, st>>>(p); break;
    default: k_rect<RECT_FILL_IMAGE, U><<<grd, blk, 0, st>>>(p); break;
  }
  count_launch(mode == RECT_COPY_ALIGNED ? "k_rect<COPY_ALIGNED>"
               : mode == RECT_COPY       ? "k_rect<COPY>"
               : mode == RECT_FILL       ? "k_rect<FILL>"
                                         : "k_rect<FILL_IMAGE>");
  return cudaGetLastError();
}

// ---------------------------------------------------------------- tiled images
__device__ __forceinline__ char* tex_addr(const TexSide& s, uint32_t x, uint32_t y, uint32_t z, int es) {
  if (s.tiled) {
    const uint32_t i = (uint32_t)s.ox + x, j = (uint32_t)s.oy + y;
    return s.ptr + (uint64_t)(j >> 3) * s.rp + ((uint64_t)(i >> s.tshift) << 10) + (uint64_t)(j & 7u) * 128u +
           (uint64_t)(i & ((1u << s.tshift) - 1u)) * (unsigned)es;
  }
  return s.ptr + (uint64_t)z * s.sp + (uint64_t)y * s.rp + (uint64_t)x * (unsigned)es;
}

__global__ void __launch_bounds__(256) k_texcopy(const TexCopyParams p) {
  const uint64_t n = (uint64_t)p.w * p.h * p.d;
  Raw fill;
  if (p.fill) fill = encode_texel(p.color, p.type, p.order);  // (A23: converted once per thread)
  for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < n; t += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t x = (uint32_t)(t % p.w), y = (uint32_t)((t / p.w) % p.h), z = (uint32_t)(t / ((uint64_t)p.w * p.h));
    char* d = tex_addr(p.dst, x, y, z, p.es);
    if (p.fill) {
      store_raw(d, p.es, fill);
    } else {
      const char* s = tex_addr(p.src, x, y, z, p.es);
      store_raw(d, p.es, load_raw(s, p.es));
    }
  }
}

cudaError_t launch_texcopy(const TexCopyParams& p, cudaStream_t st) {
  const uint64_t n = (uint64_t)p.w * p.h * p.d;
  if (n == 0) return cudaSuccess;
  const uint64_t blocks = std::min<uint64_t>((n + 255) / 256, 148ull * 16);
  k_texcopy<<<(unsigned)blocks, 256, 0, st>>>(p);
  count_launch(p.fill ? "k_texcopy<FILL>" : "k_texcopy");
  return cudaGetLastError();
}

// ---------------------------------------------------------------- write_image
__global__ void __launch_bounds__(256) k_write(const WriteParams p) {
  const uint64_t s = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (s >= p.n) return;
  const int stride = p.dims == 1 ? 1 : (p.dims == 2 ? 2 : 4);
  const int32_t* q = p.coords + s * stride;
  const int i = q[0], j = p.dims > 1 ? q[1] : 0, k = p.dims > 2 ? q[2] : 0;
  const Image& im = p.im;
  if (!in_range(i, im.w) || !in_range(j, im.h) || !in_range(k, im.d)) return;  // A15
  const uint4 c = reinterpret_cast<const uint4*>(p.colors)[s];
  const uint32_t col[4] = {c.x, c.y, c.z, c.w};
  Raw t = encode_texel(col, im.type, im.order);
  store_raw(const_cast<char*>(texel_ptr(im, i, j, k)), im.es, t);
}

cudaError_t launch_write(const WriteParams& p, cudaStream_t st) {
  if (p.n == 0) return cudaSuccess;
  k_write<<<(unsigned)((p.n + 255) / 256), 256, 0, st>>>(p);
  count_launch("k_write");
  return cudaGetLastError();
}

}  // namespace b2cl
