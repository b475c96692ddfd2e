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
  switch (mode) {
    case RECT_COPY_ALIGNED: k_rect<RECT_COPY_ALIGNED, U><<<grd, blk, 0, st>>>(p); break;
    case RECT_COPY: k_rect<RECT_COPY, U><<<grd, blk, 0, st>>>(p); break;
    case RECT_FILL: k_rect<RECT_FILL, U><<<grd, blk, 0, st>>>(p); break;
    default: k_rect<RECT_FILL_IMAGE, U><<<grd, blk, 0, st>>>(p); break;
  }
  count_launch();
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
  count_launch();
  return cudaGetLastError();
}

}  // namespace b2cl
